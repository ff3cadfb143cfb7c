"""Products per second of each ESC group (forced on all groups 2-7), serial: python scripts/esc_rate.py CONFIG..."""
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
        h.set_option("timing", 2).set_option("streams", 0).set_option("esc_groups", sum(1 << g for g in range(2, 8)))
        for i in range(3):
            C = h.multiply(dA, dA)
            torch.cuda.synchronize()
            st = h.stats()
            del C
        out = []
        for g in range(15, 21):
            if st["num_rows"][g]:
                sg = g - 13
                out.append(f"g{sg}: {st['num_nprod'][g] / st['num_group_ms'][g] / 1e6:6.1f} Gprod/s ({st['num_group_ms'][g]:.2f} ms)")
        for g in range(2, 8):
            if st["sym_rows"][g]:
                out.append(f"sym g{g}: {st['sym_nprod'][g] / st['sym_group_ms'][g] / 1e6:6.1f}")
        print(f"{name} B {A.nnz * 8 / 1e6:.0f} MB: " + "  ".join(out), flush=True)
