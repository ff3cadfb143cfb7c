"""Config 5 on one B200: R-MAT s22/s23 ef16 C = A^2 (fp32), per-phase timing + group stats.

    python scripts/rmat_run.py [--scale 22] [--reps 3]
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--opt", action="append", default=[])
    a = ap.parse_args()
    t0 = time.time()
    A = synth.rmat(a.scale).with_values("uniform", 7).astype(np.float32)
    print(f"rmat{a.scale}: m={A.m} nnz={A.nnz} gen {time.time() - t0:.1f}s", flush=True)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
    h = P.Handle()
    h.set_option("timing", 2)
    for o in a.opt:
        k, v = o.split("=")
        h.set_option(k, int(v))
    for i in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(h.stream)
        C = h.multiply(dA, dA)
        e1.record(h.stream)
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1)
        st = h.stats()
        print(f"rep {i}: {ms:.2f} ms  {2 * st['nprod'] / ms / 1e6:.1f} GFLOPS  nprod {st['nprod']} nnzC {st['nnz_c']} "
              f"ws {st['workspace_peak_bytes'] / 2**30:.2f} GiB  sym {st['symbolic_ms']:.2f} num {st['numeric_ms']:.2f}",
              flush=True)
        del C
    for g in range(st["n_sym_groups"]):
        if st["sym_rows"][g]:
            print(f"  sym g{g:2d} rows {st['sym_rows'][g]:9d} ms {st['sym_group_ms'][g]:8.3f}")
    for g in range(st["n_num_groups"]):
        if st["num_rows"][g]:
            print(f"  num g{g:2d} rows {st['num_rows'][g]:9d} nnzC {st['num_nnzc'][g]:11d} ms {st['num_group_ms'][g]:8.3f}")
    print("overflow rows", st["sym_overflow_rows"], st["sym_overflow2_rows"], "max row nprod", st["max_row_nprod"],
          "nnz", st["max_row_nnz"], "torch peak", torch.cuda.max_memory_allocated() / 2**30)
    h.close()


if __name__ == "__main__":
    main()
