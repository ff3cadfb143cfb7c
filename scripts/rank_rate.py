"""Products per second of the numeric rank groups (ESC off), serial: python scripts/rank_rate.py CONFIG..."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

for name in sys.argv[1:]:
    A = synth.config(name, "uniform", 7).astype(np.float32)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
    with P.Handle() as h:
        h.set_option("timing", 2).set_option("streams", 0).set_option("esc_groups", 0).set_option("rank_l1_pct", 0)
        for i in range(3):
            C = h.multiply(dA, dA)
            torch.cuda.synchronize()
            st = h.stats()
            del C
        out = [f"g{g}[{st['num_kernel'][g]}]: {st['num_nprod'][g] / st['num_group_ms'][g] / 1e6:6.1f}"
               for g in range(3, 13) if st["num_rows"][g] and st["num_group_ms"][g] > 0]
        print(f"{name} B {A.nnz * 8 / 1e6:.0f} MB: " + "  ".join(out), flush=True)
