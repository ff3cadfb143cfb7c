"""Phase breakdown (Fig. 5/6 analogue) and peak memory (Fig. 4,
PAPER.md:256-260) of this library vs cuSPARSE's generic SpGEMM, fp32 and fp64, same inputs, same
box.

    python scripts/cusparse_phases.py [CONFIG:DTYPE ...] > profiles/cusparse_phases_r02.jsonl

Ours (per-phase CUDA events, kernels eager): setup (n_prod + grouping), count (symbolic hash
kernels + the rpt scan), malloc of C (warm: PyTorch caching allocator; cold: after empty_cache,
a cudaMalloc), calc (numeric).  cuSPARSE (scripts/cusparse_phases.cu): work estimation (+ its
buffer), compute (+ its buffer), cudaMalloc of C, copy.  GFLOPS = 2 n_prod / total.  Peak memory =
device memory above the resident inputs during one multiply.
"""
import ctypes
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

SRC = os.path.join(ROOT, "scripts", "cusparse_phases.cu")
SO = os.path.join(ROOT, "scripts", "_build", "libcusp_phases.so")
DEFAULT = ["cant:f32", "cant:f64", "mixed:protein:f64", "mixed:qcd:f64", "webbase:f32", "webbase:f64",
           "mixed:economics:f64", "rmat18:f32", "rmat20:f32", "rmat20:f64", "rmat22:f32"]


def lib():
    if not os.path.exists(SO) or os.path.getmtime(SO) < os.path.getmtime(SRC):
        os.makedirs(os.path.dirname(SO), exist_ok=True)
        subprocess.check_call(["nvcc", "-O2", "-shared", "-Xcompiler", "-fPIC", "-gencode",
                               "arch=compute_100a,code=sm_100a", "-o", SO, SRC, "-lcusparse"])
    L = ctypes.CDLL(SO)
    L.cusp_spgemm.restype = ctypes.c_int
    L.cusp_spgemm.argtypes = [ctypes.c_int64] * 5 + [ctypes.c_int] * 2 + [ctypes.c_void_p] * 7
    return L


def ours(dA, reps=3):
    """Per-phase times (median of reps) and peak memory of one multiply through the library."""
    rows = []
    with P.Handle() as h:
        h.set_option("timing", 2)
        for i in range(reps + 1):
            torch.cuda.synchronize()
            c_rpt, nnz, nprod = h.symbolic(dA, dA)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(h.stream)
            with torch.cuda.stream(h.stream):
                c_col = torch.empty(nnz, dtype=torch.int32, device="cuda")
                c_val = torch.empty(nnz, dtype=dA.val.dtype, device="cuda")
            e1.record(h.stream)
            h.numeric(dA.val, dA.val, c_col, c_val)
            torch.cuda.synchronize()
            st = h.stats()
            if i:
                rows.append((st["setup_ms"], st["symbolic_ms"] + st["scan_ms"], e0.elapsed_time(e1), st["numeric_ms"]))
            del c_col, c_val, c_rpt
        # cold allocation of C: the caching allocator emptied, so C comes from cudaMalloc
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        c_col = torch.empty(nnz, dtype=torch.int32, device="cuda")
        c_val = torch.empty(nnz, dtype=dA.val.dtype, device="cuda")
        e1.record()
        torch.cuda.synchronize()
        cold = e0.elapsed_time(e1)
        del c_col, c_val
    med = [statistics.median(r[i] for r in rows) for i in range(4)]
    # peak device memory with every library buffer through the torch allocator
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    base = torch.cuda.memory_allocated()
    torch.cuda.reset_peak_memory_stats()
    with P.Handle(torch_allocator=True) as hp:
        C = hp.multiply(dA, dA)
        torch.cuda.synchronize()
        peak = torch.cuda.max_memory_allocated() - base
        del C
    return {"setup": med[0], "count": med[1], "malloc_warm": med[2], "malloc_cold": cold, "calc": med[3],
            "total_warm": sum(med), "total_cold": med[0] + med[1] + cold + med[3], "nnz_c": int(nnz),
            "nprod": int(nprod), "peak_bytes": int(peak)}


def cusparse(L, A, dt, nprod):
    idx64 = A.nnz >= 2**31 - 1 or nprod >= 2**31 - 1
    it = torch.int64 if idx64 else torch.int32
    tdt = torch.float32 if dt == np.float32 else torch.float64
    rpt = torch.from_numpy(A.rpt).to("cuda", it)
    col = torch.from_numpy(A.col).to("cuda", it)
    val = torch.from_numpy(A.val.astype(dt)).to("cuda")
    out = (ctypes.c_double * 8)()
    runs = []
    for i in range(3):
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        L.cusp_spgemm(A.m, A.n, A.n, A.nnz, A.nnz, int(idx64), int(dt == np.float64), rpt.data_ptr(),
                      col.data_ptr(), val.data_ptr(), rpt.data_ptr(), col.data_ptr(), val.data_ptr(), out)
        r = list(out)
        if r[7] != 0:
            return {"status": int(r[7]), "index": "64I" if idx64 else "32I"}
        if i:
            runs.append(r)
    med = [statistics.median(x[i] for x in runs) for i in range(7)]
    return {"work_estimation": med[0], "compute": med[1], "malloc_c": med[2], "copy": med[3], "total": med[4],
            "nnz_c": int(med[5]), "peak_bytes": int(med[6]), "index": "64I" if idx64 else "32I", "status": 0}


def main():
    L = lib()
    todo = sys.argv[1:] or DEFAULT
    for item in todo:
        name, dty = item.rsplit(":", 1)
        dt = np.float32 if dty == "f32" else np.float64
        A = synth.config(name, "uniform", 7).astype(dt)
        dA = P.CsrMatrix.from_host(A, "cuda", torch.float32 if dt == np.float32 else torch.float64)
        o = ours(dA)
        del dA
        torch.cuda.empty_cache()
        c = cusparse(L, A, dt, o["nprod"])
        line = {"config": name, "dtype": dty, "nprod": o["nprod"], "ours": o, "cusparse": c,
                "gflops_ours_warm": 2 * o["nprod"] / o["total_warm"] / 1e6,
                "gflops_ours_cold": 2 * o["nprod"] / o["total_cold"] / 1e6,
                "gflops_cusparse": 2 * o["nprod"] / c["total"] / 1e6 if c.get("status") == 0 else None,
                "same_nnz": c.get("nnz_c") == o["nnz_c"] if c.get("status") == 0 else None,
                "peak_ratio_ours_over_cusparse": o["peak_bytes"] / c["peak_bytes"] if c.get("peak_bytes") else None}
        print(json.dumps(line), flush=True)
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
