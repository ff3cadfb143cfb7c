"""A/B of option sets on configs (serial groups, best of 3): python scripts/ab.py CONFIGS -- OPTSETS
e.g. python scripts/ab.py rmat18,webbase -- wsort=0 wsort=3"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

cfgs = sys.argv[1].split(",")
sets = sys.argv[3:] if len(sys.argv) > 3 else [""]
for name in cfgs:
    A = synth.config(name, "uniform", 7).astype(np.float32)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
    for os_ in sets:
        opts = [kv.split("=") for kv in os_.split(",") if kv]
        with P.Handle() as h:
            h.set_option("timing", 2).set_option("streams", 0)
            for k, v in opts:
                h.set_option(k, int(v))
            best = None
            for i in range(4):
                C = h.multiply(dA, dA)
                torch.cuda.synchronize()
                st = h.stats()
                tot = st["setup_ms"] + st["symbolic_ms"] + st["scan_ms"] + st["numeric_ms"]
                if i and (best is None or tot < best[0]):
                    best = (tot, st)
                del C
            tot, st = best
            print(f"{name:10s} {os_:24s} total {tot:8.3f} ms {2 * st['nprod'] / tot / 1e6:7.1f} GFLOPS  sym {st['symbolic_ms']:7.3f} "
                  f"num {st['numeric_ms']:7.3f}  | sym " + " ".join(f"g{g}:{st['sym_group_ms'][g]:.2f}" for g in range(2, 8) if st['sym_group_ms'][g] > 0)
                  + " | num " + " ".join(f"g{g}:{st['num_group_ms'][g]:.2f}" for g in range(24) if st['num_group_ms'][g] > 0.05), flush=True)
