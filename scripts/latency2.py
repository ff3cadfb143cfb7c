import os, statistics, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_icpp_nagasakanm17_b200 as P
A = synth.config("poisson64")
dA = P.CsrMatrix.from_host(A, "cuda", torch.float64)
h = P.Handle()
for _ in range(20):
    h.multiply(dA, dA)
torch.cuda.synchronize()
ts = {"symbolic": [], "alloc": [], "numeric": [], "sync": []}
for _ in range(300):
    t0 = time.perf_counter()
    c_rpt, nnz, _ = h.symbolic(dA, dA)
    t1 = time.perf_counter()
    c_col = h._empty(nnz, torch.int32)
    c_val = h._empty(nnz, torch.float64)
    t2 = time.perf_counter()
    h.numeric(dA.val, dA.val, c_col, c_val)
    t3 = time.perf_counter()
    torch.cuda.synchronize()
    t4 = time.perf_counter()
    for k, a, b in (("symbolic", t0, t1), ("alloc", t1, t2), ("numeric", t2, t3), ("sync", t3, t4)):
        ts[k].append(1e6 * (b - a))
print({k: round(statistics.median(v), 1) for k, v in ts.items()})
h.set_option("timing", 0)
for _ in range(20):
    h.multiply(dA, dA)
t0 = time.perf_counter()
for _ in range(300):
    h.multiply(dA, dA)
torch.cuda.synchronize()
print("timing=0 per multiply us", 1e6 * (time.perf_counter() - t0) / 300)
