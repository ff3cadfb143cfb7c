"""One C = A^2 on R-MAT (for ncu captures): python scripts/rmat_once.py SCALE [name=value ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

scale = int(sys.argv[1])
cfg = synth.config(f"rmat{scale}" if scale > 0 else "webbase", "uniform", 7).astype(np.float32)
dA = P.CsrMatrix.from_host(cfg, "cuda", torch.float32)
with P.Handle() as h:
    h.set_option("timing", 2).set_option("streams", 0)
    for kv in sys.argv[2:]:
        k, v = kv.split("=")
        h.set_option(k, int(v))
    C = h.multiply(dA, dA)
    torch.cuda.synchronize()
    print("nnz", C.nnz, h.stats()["numeric_ms"])
