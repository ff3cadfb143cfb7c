"""Serial per-group kernel times (ms) of one config: python scripts/group_times.py CONFIG [name=value ...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

F64 = os.environ.get("GT_DTYPE") == "f64"
A = synth.config(sys.argv[1], "uniform", 7).astype(np.float64 if F64 else np.float32)
dA = P.CsrMatrix.from_host(A, "cuda", torch.float64 if F64 else torch.float32)
with P.Handle() as h:
    h.set_option("timing", 2).set_option("streams", 0)
    for kv in sys.argv[2:]:
        k, v = kv.split("=")
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
    print(f"{sys.argv[1]} {os.environ.get('SPGEMM_LIB', 'default')} {sys.argv[2:]}: total {tot:.2f} ms "
          f"({2 * st['nprod'] / tot / 1e6:.1f} GFLOPS) setup {st['setup_ms']:.2f} sym {st['symbolic_ms']:.2f} "
          f"num {st['numeric_ms']:.2f}")
    print("   sym " + " ".join(f"g{g}:{st['sym_group_ms'][g]:.2f}" for g in range(24) if st["sym_group_ms"][g] > 0))
    print("   num " + " ".join(f"g{g}:{st['num_group_ms'][g]:.2f}" for g in range(24) if st["num_group_ms"][g] > 0))
    if os.environ.get("GT_DETAIL"):
        for ph in ("sym", "num"):
            for g in range(24):
                ms = st[f"{ph}_group_ms"][g]
                if ms > 0:
                    rows, npr = st[f"{ph}_rows"][g], st[f"{ph}_nprod"][g]
                    nnzc = st["num_nnzc"][g] if ph == "num" else 0
                    print(f"   {ph} g{g:2d} kind {st[f'{ph}_kernel'][g] if f'{ph}_kernel' in st else '?'} rows {rows:9d} "
                          f"nprod {npr:12d} nnzc {nnzc:12d} ms {ms:7.3f} Gprod/s {npr / ms / 1e6:7.1f}")
