import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth, oracle
import paper_conf_icpp_nagasakanm17_b200 as P
name = sys.argv[1]; mask = int(sys.argv[2])
A = synth.config(name, "uniform", 7).astype(np.float32)
dA = P.CsrMatrix.from_host(A, "cuda", torch.float32)
with P.Handle() as h:
    h.set_option("timing", 2).set_option("streams", 0).set_option("esc_groups", mask)
    C = h.multiply(dA, dA); torch.cuda.synchronize()
    st = h.stats()
    print({g: (st["num_rows"][g], st["num_kernel"][g]) for g in range(22) if st["num_rows"][g]})
    rpt, col, val = C.numpy()
r = oracle.spgemm(A, A, np.float32, parallel=True)
print("rpt", np.array_equal(rpt, r[0]), "col", np.array_equal(col, r[1]), "val", bool(np.all(np.abs(val - r[2]) <= 1e-5 * r[3])))
