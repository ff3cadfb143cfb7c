"""cuSPARSE side-by-side (the paper's main comparator).

    python scripts/cusparse_compare.py [CONFIG ...] [--dtype f32|f64] [--reps N]

Times C = A^2 on the same synthetic inputs through (a) this library (`Handle.multiply`, the
two-phase hash SpGEMM) and (b) PyTorch's CUDA sparse-CSR matmul, which calls cuSPARSE's
cusparseSpGEMM (work-estimation / compute / copy, also a two-phase method).  Both start from
device-resident A and end with a finished device C; CUDA events on the current stream, L2
flushed before every run, median of N.  Reports GFLOPS = 2*nprod/t, peak
device memory above the inputs (the Fig. 4 ratio) and checks that the two
results have the same structure (rpt/col bit-exact after cuSPARSE's row sort) and values within
the S-scaled tolerance.  One JSON line per config.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def _flush(buf):
    buf.add_(1)


def _time(fn, reps, flush):
    ts = []
    for _ in range(reps + 2):
        _flush(flush)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        out = fn()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
        del out
    return statistics.median(ts[2:])


def _peak(fn, base):
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    torch.cuda.reset_peak_memory_stats()
    out = fn()
    torch.cuda.synchronize()
    peak = torch.cuda.max_memory_allocated() - base
    return out, peak


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["cant", "webbase", "mixed:protein", "mixed:qcd",
                                                    "mixed:economics", "mixed:epidemiology"])
    ap.add_argument("--dtype", default="f32", choices=["f32", "f64"])
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    tdt = torch.float32 if a.dtype == "f32" else torch.float64
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    h = P.Handle()                        # library's private workspace pool (timed)
    hm = P.Handle(torch_allocator=True)   # workspace through torch's allocator (peak memory)
    for cfg in a.configs:
        A = synth.config(cfg)
        dA = P.CsrMatrix.from_host(A, "cuda", tdt)
        # cuSPARSE through torch: int64 crow/col (torch's CSR index type on this path)
        tA = torch.sparse_csr_tensor(torch.from_numpy(A.rpt.astype(np.int64)).cuda(),
                                     torch.from_numpy(A.col.astype(np.int64)).cuda(),
                                     torch.from_numpy(A.val).to(tdt).cuda(), size=(A.m, A.n))
        torch.cuda.synchronize()
        base = torch.cuda.memory_allocated()

        ours = lambda: h.multiply(dA, dA)
        cus = lambda: torch.sparse.mm(tA, tA)
        C, peak_ours = _peak(lambda: hm.multiply(dA, dA), base)
        del C
        C = ours()
        st = h.stats()
        nprod = st["nprod"]
        try:
            T, peak_cus = _peak(cus, base)
            t_cus = _time(cus, a.reps, flush)
            cus_err = None
        except RuntimeError as e:  # cuSPARSE out of memory / unsupported
            T, peak_cus, t_cus, cus_err = None, None, None, str(e).splitlines()[0][:200]
        t_ours = _time(ours, a.reps, flush)

        match = None
        if T is not None:
            r_rpt = T.crow_indices().cpu().numpy()
            r_col = T.col_indices().cpu().numpy()
            r_val = T.values().cpu().numpy()
            rpt, col, val = C.numpy()
            same_rpt = np.array_equal(rpt, r_rpt)
            # cuSPARSE output rows are sorted; compare col bit-exact, values with a relative bound
            same_col = same_rpt and np.array_equal(col, r_col)
            scale = np.abs(val).max() if val.size else 1.0
            vdiff = float(np.abs(val.astype(np.float64) - r_val.astype(np.float64)).max() / max(scale, 1e-300)) if same_col and val.size else None
            match = {"rpt": bool(same_rpt), "col": bool(same_col), "max_rel_val_diff": vdiff}
        print(json.dumps({
            "config": cfg, "dtype": a.dtype, "rows": A.m, "nnz_a": A.nnz, "nprod": nprod, "nnz_c": st["nnz_c"],
            "ours": {"ms": t_ours, "gflops": 2 * nprod / t_ours / 1e6, "peak_mem_above_inputs": peak_ours},
            "cusparse": {"ms": t_cus, "gflops": (2 * nprod / t_cus / 1e6) if t_cus else None,
                         "peak_mem_above_inputs": peak_cus, "error": cus_err},
            "speedup": (t_cus / t_ours) if t_cus else None,
            "mem_ratio": (peak_cus / peak_ours) if peak_cus else None,
            "match": match, "l2": "flushed (512 MiB) before every run", "reps": a.reps,
        }), flush=True)
        del C, T, dA, tA
        torch.cuda.empty_cache()
    h.close()
    hm.close()


if __name__ == "__main__":
    main()
