"""Per-group diagnostic: rows / n_prod / nnz / time of every group kernel for one config.

    python scripts/diag.py CONFIG [--dtype f32|f64] [--lanes L] [--opt name=value ...]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--opt", action="append", default=[])
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    A = synth.config(a.config)
    tdt = torch.float32 if a.dtype == "f32" else torch.float64
    dA = P.CsrMatrix.from_host(A, "cuda", tdt)
    h = P.Handle()
    h.set_option("timing", 2)  # per-group kernel events (eager launches)
    for o in a.opt:
        k, v = o.split("=")
        h.set_option(k, int(v))
    for _ in range(a.reps):
        C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        st = h.stats()
    print(f"{a.config}: m={A.m} nnzA={A.nnz} nprod={st['nprod']} nnzC={st['nnz_c']} maxrow nprod={st['max_row_nprod']} "
          f"nnz={st['max_row_nnz']} overflow={st['sym_overflow_rows']}")
    print(f"phases ms: setup {st['setup_ms']:.3f} sym {st['symbolic_ms']:.3f} scan {st['scan_ms']:.3f} num {st['numeric_ms']:.3f}")
    for g in range(st["n_sym_groups"]):
        if st["sym_rows"][g]:
            print(f"  sym g{g:2d} rows {st['sym_rows'][g]:9d} nprod {st['sym_nprod'][g]:12d} nnzA {st['sym_nnza'][g]:10d} "
                  f"ms {st['sym_group_ms'][g]:8.3f}")
    for g in range(st["n_num_groups"]):
        if st["num_rows"][g]:
            print(f"  num g{g:2d} rows {st['num_rows'][g]:9d} nprod {st['num_nprod'][g]:12d} nnzC {st['num_nnzc'][g]:10d} "
                  f"ms {st['num_group_ms'][g]:8.3f}")
    print("sym ms by group", [round(x, 3) for x in st["sym_group_ms"][:12]])
    h.close()


if __name__ == "__main__":
    main()
