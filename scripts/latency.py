"""Per-multiply latency of small inputs (config 1 and friends): python scripts/latency.py [name=value ...]"""
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
import paper_conf_icpp_nagasakanm17_b200 as P

for name, dt in (("poisson64", torch.float64), ("mixed:economics", torch.float64), ("mixed:epidemiology", torch.float64)):
    A = synth.config(name)
    dA = P.CsrMatrix.from_host(A, "cuda", dt)
    with P.Handle() as h:
        for kv in sys.argv[1:]:
            k, v = kv.split("=")
            h.set_option(k, int(v))
        for _ in range(20):
            C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        ev, wall = [], []
        for _ in range(200):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            t0 = time.perf_counter()
            e0.record(h.stream)
            C = h.multiply(dA, dA)
            e1.record(h.stream)
            e1.synchronize()
            wall.append(1e6 * (time.perf_counter() - t0))
            ev.append(1e3 * e0.elapsed_time(e1))
        st = h.stats()
        print(f"{name:20s} {sys.argv[1:]}: device {statistics.median(ev):7.1f} us  wall {statistics.median(wall):7.1f} us  "
              f"GFLOPS {2 * st['nprod'] / statistics.median(ev) / 1e3:6.2f}  launches "
              f"{st['kernel_launches_symbolic'] + st['kernel_launches_numeric']}")
