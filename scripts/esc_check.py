"""Quick parity + timing check of the batched kernels (kernels_esc.cu) on graph configs.

    python scripts/esc_check.py [--scale 22] [--skip-big]
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import oracle
import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def run(A, dtype, opts):
    tdt = torch.float32 if dtype == np.float32 else torch.float64
    dA = P.CsrMatrix.from_host(A, "cuda", tdt)
    with P.Handle() as h:
        h.set_option("timing", 2)
        for k, v in opts.items():
            h.set_option(k, v)
        for _ in range(3):
            C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        st = h.stats()
        return C, st


def parity(A, dtype, opts, name):
    C, st = run(A, dtype, opts)
    rpt, col, val = C.numpy()
    r = oracle.spgemm(A, A, dtype, parallel=True)
    ok_r = np.array_equal(rpt, r[0])
    ok_c = ok_r and np.array_equal(col, r[1])
    rt = 1e-5 if dtype == np.float32 else 1e-12
    bad = int((np.abs(val.astype(np.float64) - r[2]) > rt * r[3]).sum()) if ok_c else -1
    ks = {g: st["num_kernel"][g] for g in range(len(st["num_kernel"])) if st["num_rows"][g]}
    print(f"{name:28s} {str(opts):32s} rpt {ok_r} col {ok_c} badval {bad}  sym {st['symbolic_ms']:.3f} "
          f"num {st['numeric_ms']:.3f} kernels {ks}", flush=True)
    return ok_c and bad == 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--skip-big", action="store_true")
    a = ap.parse_args()
    allok = True
    cases = [("rmat14", synth.rmat(14).with_values("uniform", 9), np.float32),
             ("rmat14 f64", synth.rmat(14).with_values("uniform", 9), np.float64),
             ("rmat14 int", synth.rmat(14).with_values("int", 2), np.float32),
             ("rmat16", synth.rmat(16).with_values("uniform", 3), np.float32),
             ("webbase", synth.config("webbase"), np.float32),
             ("economics", synth.config("mixed:economics"), np.float64),
             ("circuit", synth.config("mixed:circuit"), np.float64),
             ("qcd", synth.config("mixed:qcd"), np.float32)]
    for name, A, dt in cases:
        A = A.astype(dt)
        for opts in ({}, {"batch": 0}):
            allok &= parity(A, dt, opts, name)
    print("ALL OK" if allok else "FAILURES", flush=True)
    if a.skip_big:
        return
    for name in ["webbase", "rmat18", "rmat20", f"rmat{a.scale}"]:
        timing(name)


def timing(name):
    t0 = time.time()
    A = synth.config(name, "uniform", 7).astype(np.float32)
    print(f"{name} gen {time.time() - t0:.1f}s nnz {A.nnz}", flush=True)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
    for opts in ({"streams": 0}, {"streams": 0, "batch": 0}, {}):
        with P.Handle() as h:
            h.set_option("timing", 2)
            for k, v in opts.items():
                h.set_option(k, v)
            ms = []
            for i in range(4):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(h.stream)
                C = h.multiply(dA, dA)
                e1.record(h.stream)
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
                st = h.stats()
                del C
            best = min(ms[1:])
            print(f"{name} {opts}: {best:.2f} ms = {2 * st['nprod'] / best / 1e6:.1f} GFLOPS  sym {st['symbolic_ms']:.2f} "
                  f"num {st['numeric_ms']:.2f}", flush=True)
            for g in range(st["n_sym_groups"]):
                if st["sym_rows"][g]:
                    print(f"   sym g{g:2d} rows {st['sym_rows'][g]:9d} k{st['sym_kernel'][g]} ms {st['sym_group_ms'][g]:8.3f}")
            for g in range(st["n_num_groups"]):
                if st["num_rows"][g]:
                    print(f"   num g{g:2d} rows {st['num_rows'][g]:9d} k{st['num_kernel'][g]} ms {st['num_group_ms'][g]:8.3f}")


if __name__ == "__main__":
    main()
