"""Per symbolic group A/B of the numeric ESC kernels (ESC_GROUPS = one group at a time) vs the
rank/hash kernels, serial streams: python scripts/esc_groups.py CONFIG..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P


def num_ms(dA, opts):
    with P.Handle() as h:
        h.set_option("timing", 2).set_option("streams", 0)
        for k, v in opts.items():
            h.set_option(k, v)
        best = 1e9
        for i in range(4):
            C = h.multiply(dA, dA)
            torch.cuda.synchronize()
            st = h.stats()
            if i:
                best = min(best, st["numeric_ms"])
            del C
        return best, st


for name in sys.argv[1:]:
    A = synth.config(name, "uniform", 7).astype(np.float32)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
    base, st = num_ms(dA, {"esc_groups": 0})
    print(f"{name}: n {A.n} l1w {A.n // 1024 + 1} numeric without ESC {base:.3f} ms", flush=True)
    for g in range(2, 9):
        if not st["sym_rows"][g]:
            continue
        t, st2 = num_ms(dA, {"esc_groups": 1 << g})
        print(f"   sym g{g} rows {st['sym_rows'][g]:9d} nprod {st['sym_nprod'][g]:12d}: ESC delta {t - base:+8.3f} ms", flush=True)
    t, _ = num_ms(dA, {})
    print(f"   all ESC: {t:.3f} ms", flush=True)
