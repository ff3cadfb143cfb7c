"""Galerkin product R A P of smoothed-aggregation AMG on the
n x n 5-point Poisson grid, as two chained SpGEMMs through the library, plus numeric-only re-runs
(new values, same structure: the AMG setup's repeated Galerkin products).

    python scripts/galerkin.py [--n 2048] [--dtype f64] [--reps 5]   -> one JSON line
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def timed(fn, stream, reps):
    ts = []
    for i in range(reps + 2):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        out = fn()
        e1.record(stream)
        torch.cuda.synchronize()
        if i >= 2:
            ts.append(e0.elapsed_time(e1))
    return statistics.median(ts), out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=2048)
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    A = synth.poisson2d(a.n)
    Pm = synth.aggregation_prolongator(a.n, seed=3)
    R = synth.transpose(Pm)
    dA, dP, dR = (P.CsrMatrix.from_host(M, "cuda", dt) for M in (A, Pm, R))
    h1, h2 = P.Handle(), P.Handle()
    t_ap, AP = timed(lambda: h1.multiply(dA, dP), h1.stream, a.reps)
    np_ap = h1.nprod
    t_rap, RAP = timed(lambda: h2.multiply(dR, AP), h2.stream, a.reps)
    np_rap = h2.nprod
    # numeric-only re-runs (structure fixed, values new)
    A2v = torch.rand_like(dA.val)
    P2v = torch.rand_like(dP.val)
    AP2 = P.CsrMatrix(AP.m, AP.n, AP.rpt, AP.col, torch.empty_like(AP.val))
    t_ap_num, _ = timed(lambda: h1.numeric(A2v, P2v, AP2.col, AP2.val), h1.stream, a.reps)
    RAP2v = torch.empty_like(RAP.val)
    RAP2c = torch.empty_like(RAP.col)
    t_rap_num, _ = timed(lambda: h2.numeric(dR.val, AP2.val, RAP2c, RAP2v), h2.stream, a.reps)
    line = {"workload": f"Galerkin R A P, smoothed aggregation 2x2, Poisson {a.n}x{a.n}", "dtype": a.dtype,
            "A": [A.m, A.nnz], "P": [Pm.m, Pm.n, Pm.nnz], "AP_nnz": AP.nnz, "RAP": [RAP.m, RAP.nnz],
            "AP": {"ms": t_ap, "gflops": 2 * np_ap / t_ap / 1e6, "nprod": int(np_ap),
                   "numeric_only_ms": t_ap_num, "numeric_only_gflops": 2 * np_ap / t_ap_num / 1e6},
            "R_AP": {"ms": t_rap, "gflops": 2 * np_rap / t_rap / 1e6, "nprod": int(np_rap),
                     "numeric_only_ms": t_rap_num, "numeric_only_gflops": 2 * np_rap / t_rap_num / 1e6},
            "total_ms": t_ap + t_rap, "total_numeric_only_ms": t_ap_num + t_rap_num}
    print(json.dumps(line), flush=True)
    h1.close()
    h2.close()


if __name__ == "__main__":
    main()
