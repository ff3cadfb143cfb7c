"""bench.py — SpGEMM GFLOPS (2*n_prod/s) of C = A^2 on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config cant] [--dtype f32|f64]

One step = the whole hot path of SURVEY.md §8(a) on one synthetic input already resident in
HBM: symbolic (n_prod, grouping, hash count, scan) -> exact allocation of C -> numeric
(grouping, hash accumulate, gather, sort, write).  N=1 workload: BASELINE.json configs[1],
the cant-like FEM matrix (62,451 rows, ~4.0M nnz), fp32.  N>1 (torchrun): weak scaling —
rank p computes row block p of diag(A_0..A_{N-1})^2 with A_p a cant-like instance of seed p
(the n_prod-balanced row split puts block p on rank p; no data-path collective).

Timing: W untimed warm-ups; K timed steps, each bracketed by CUDA events on the handle's
stream, the L2 flushed (512 MiB write) before every step outside the events; barrier +
synchronize on both sides; max over ranks.  `e2e` re-times the step through the public
Python API from pinned HOST buffers: H2D of A, the step, and D2H of all of C.

`--impl reference`: the CPU oracle (oracle/, plain C Gustavson, 1 core) on the same
config, rank 0 only — the reference arm of this tier (there is no reference library).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpGEMM GFLOPS (2*nprod/s) C=A^2"
UNIT = "GFLOPS"
REASON_BITS = {  # nvidia-smi clocks_event_reasons bitmask
    0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
    0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
    0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
}


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="cant")
    p.add_argument("--dtype", default="f32", choices=["f32", "f64"])
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--cpu-runs", type=int, default=5)
    p.add_argument("--lanes", type=int, default=0, help="lanes per B row (0 = library auto)")
    p.add_argument("--streams", type=int, default=1)
    p.add_argument("--opt", action="append", default=[],
                   help="library option name=value (ablations, e.g. rank_acc=0; see _lib.OPTIONS)")
    return p.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def workload(args, rank):
    import synth
    A = synth.config(args.config, "uniform", seed=rank)
    dt = np.float32 if args.dtype == "f32" else np.float64
    return A.astype(dt), dt


def config_dict(args, A, world):
    return {"workload": f"{args.config}-like A^2" if args.config != "poisson64" else "poisson64 A^2",
            "matrix": A.name, "rows": A.m, "nnz_a": A.nnz, "dtype": args.dtype,
            "per_rank": "row block p of diag(A_0..A_{N-1})^2 (weak scaling)" if world > 1 else "single GPU",
            "l2": "flushed (512 MiB write) before every timed step", "inputs": "device-resident (value)",
            **({"options": dict(o.split("=") for o in args.opt)} if getattr(args, "opt", None) else {})}


# ----------------------------------------------------------------------------- clocks
class ClockSampler:
    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        q = "clocks.sm,clocks.max.sm,clocks_event_reasons.active"
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 3:
                self.rows.append(parts)

    def __exit__(self, *exc):
        if self.proc:
            time.sleep(0.25)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        for c, m, r in self.rows:
            try:
                sm.append(float(c)); mx.append(float(m))
                bits = int(r, 16)
                for b, name in REASON_BITS.items():
                    if bits & b and name != "gpu_idle":
                        reasons.add(name)
            except ValueError:
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ----------------------------------------------------------------------------- roofline model
def algorithmic_bytes(st: dict, phase: str, g: int, vbytes: int) -> int:
    """SURVEY.md §8(d) / DESIGN.md §6 streaming model (no reuse), per group launch:
    symbolic: 4 B/product (col_B) + 20 B/nnz(A) (col_A + rpt_B pair) + 28 B/row;
    numeric: (4+s) B/product (col_B,val_B) + (20+s) B/nnz(A) + (4+s) B/nnz(C) write + 36 B/row."""
    if phase == "sym":
        return 4 * st["sym_nprod"][g] + 20 * st["sym_nnza"][g] + 28 * st["sym_rows"][g]
    return ((4 + vbytes) * st["num_nprod"][g] + (20 + vbytes) * st["num_nnza"][g]
            + (4 + vbytes) * st["num_nnzc"][g] + 36 * st["num_rows"][g])


def kernel_name(phase: str, g: int, kind: int = 0) -> str:
    """Group -> kernel template as it appears in ncu / cuobjdump (spgemm_internal.cuh group ids;
    kind = spgemm_kernel_t the library reports for the group)."""
    if phase == "sym":
        k = {2: "k_sym_rankcnt<TPR,UPPER,KP,MC>", 3: "k_sym_range", 5: "k_sym_global"}.get(kind, "k_sym_smem<T,TPR,BS,OPT>")
        return f"{k} (group {g})"
    k = {2: "k_num_rankacc<VT,TPR,UPPER,KP,MC>", 3: "k_num_range<VT>", 4: "k_num_cluster<VT,CS>",
         5: "k_num_global<VT>", 6: "k_num_rankbig<VT>"}.get(kind, "k_num_smem<VT,T,TPR,BS,UPPER>")
    return f"{k} (group {g})"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic(phase, g, dtype):
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if not os.path.exists(p):
        return None
    d = json.load(open(p))
    return d.get(f"{phase}_g{g}_{dtype}")


# ----------------------------------------------------------------------------- reference arm
def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    A, dt = workload(args, 0)
    _, total = oracle.nprod(A, A)
    oracle.build()
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.spgemm(A, A, dt)
        t = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(t)
    tot = sum(times)
    val = 2 * total * len(times) / tot / 1e9
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * tot / len(times), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": config_dict(args, A, 1), "impl": "reference",
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"full {A.name} A^2 per step (nprod {total})"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    import paper_conf_icpp_nagasakanm17_b200 as P

    A, dt = workload(args, rank)
    tdt = torch.float32 if dt == np.float32 else torch.float64
    vbytes = 4 if dt == np.float32 else 8
    h = P.Handle(dev)
    # per-group kernel events over the timed region (timing=2 runs the group kernels eagerly; the
    # CUDA-graph replay mode is timed separately below and reported as `graph_replay`)
    h.set_option("lanes", args.lanes).set_option("streams", args.streams).set_option("timing", 2)
    for o in args.opt:
        k, v = o.split("=")
        h.set_option(k, int(v))
    dA = P.CsrMatrix.from_host(A, dev, tdt)
    stream = h.stream
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def step():
        return h.multiply(dA, dA)

    for _ in range(max(3, args.warmup)):
        step()
    barrier()

    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    per_step_stats = []
    launches = 0
    with ClockSampler(local) as clk:
        barrier()
        t_wall = time.perf_counter()
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(i & 0xFF)
            ev[i][0].record(stream)
            C = step()
            ev[i][1].record(stream)
            st = h.stats()  # waits for this step's events (per-group kernel timings)
            per_step_stats.append(st)
            launches += st["kernel_launches_symbolic"] + st["kernel_launches_numeric"]
            del C
        barrier()
        t_wall = time.perf_counter() - t_wall
    step_ms = [a.elapsed_time(b) for a, b in ev]
    tot_ms = sum(step_ms)
    st = per_step_stats[-1]
    nprod = st["nprod"]
    tot_t = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(tot_t, op=dist.ReduceOp.MAX)
        np_t = torch.tensor([nprod], dtype=torch.float64, device=dev)
        dist.all_reduce(np_t, op=dist.ReduceOp.SUM)
        total_nprod = float(np_t.item())
    else:
        total_nprod = float(nprod)
    max_ms = float(tot_t.item())
    value = 2 * total_nprod * args.steps / (max_ms / 1e3) / 1e9

    # dominant kernel: group launch with the largest mean time across the timed steps
    cand = {}
    for s in per_step_stats:
        for ph, key in (("sym", "sym_group_ms"), ("num", "num_group_ms")):
            for g, ms in enumerate(s[key]):
                if ms > 0:
                    cand.setdefault((ph, g), []).append(ms)
    (ph, g), mss = max(cand.items(), key=lambda kv: statistics.mean(kv[1]))
    k_ms = statistics.mean(mss)
    bytes_alg = algorithmic_bytes(st, ph, g, vbytes)
    peak, peak_src = load_peaks()
    achieved = bytes_alg / (k_ms / 1e3) / 1e9
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": load_traffic(ph, g, args.dtype),
                "kernel": kernel_name(ph, g, st["sym_kernel" if ph == "sym" else "num_kernel"][g]), "phase": ph, "group": g,
                "launch_ms": k_ms, "share_of_step": k_ms / (tot_ms / args.steps),
                "algorithmic_bytes_per_launch": bytes_alg, "peak_source": peak_src}

    # the same step with the captured phase segments replayed as CUDA graphs (timing=1)
    h.set_option("timing", 1)
    for _ in range(max(3, args.warmup)):
        step()
    barrier()
    gev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    replays = 0
    for i in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(i & 0xFF)
        gev[i][0].record(stream)
        C = step()
        gev[i][1].record(stream)
        replays += h.stats()["graph_replays"]
        del C
    barrier()
    g_ms = sum(a.elapsed_time(b) for a, b in gev)
    gt = torch.tensor([g_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(gt, op=dist.ReduceOp.MAX)
    graph_replay = {"value": 2 * total_nprod * args.steps / (float(gt.item()) / 1e3) / 1e9, "unit": UNIT,
                    "ms_per_step": float(gt.item()) / args.steps, "segments_replayed": int(replays)}

    # end to end through the public API from pinned host buffers
    e2e = None
    if not args.no_e2e:
        hA = P.CsrMatrix.from_host(A, None, tdt, pin=True)
        bi = hA.rpt.numel() * 8 + hA.col.numel() * 4 + hA.val.numel() * vbytes
        e_ms, bo = [], 0
        for i in range(args.warmup + args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(i & 0xFF)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            with torch.cuda.stream(stream):
                dA2 = hA.to(dev, non_blocking=True)
            C = h.multiply(dA2, dA2)
            with torch.cuda.stream(stream):
                out = (torch.empty(C.rpt.shape, dtype=C.rpt.dtype, pin_memory=True),
                       torch.empty(C.col.shape, dtype=C.col.dtype, pin_memory=True),
                       torch.empty(C.val.shape, dtype=C.val.dtype, pin_memory=True))
                out[0].copy_(C.rpt, non_blocking=True)
                out[1].copy_(C.col, non_blocking=True)
                out[2].copy_(C.val, non_blocking=True)
            e1.record(stream)
            e1.synchronize()
            if i >= args.warmup:
                e_ms.append(e0.elapsed_time(e1))
                bo = sum(x.numel() * x.element_size() for x in out)
            del C, dA2, out
        et = torch.tensor([sum(e_ms)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e = {"value": 2 * total_nprod * len(e_ms) / (float(et.item()) / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(bi), "d2h_bytes_per_step": int(bo),
               "ms_per_step": float(et.item()) / len(e_ms)}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        ts = []
        for _ in range(args.cpu_runs):
            t0 = time.perf_counter()
            oracle.spgemm(A, A, dt)
            ts.append(time.perf_counter() - t0)
        cpu = {"value": 2 * nprod * len(ts) / sum(ts) / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"full {A.name} A^2 ({args.dtype}) x {len(ts)} runs, {sum(ts):.1f} s"}

    a_bytes = (A.m + 1) * 8 + A.nnz * (4 + vbytes)  # B = A shares these buffers
    c_bytes = (A.m + 1) * 8 + int(st["nnz_c"]) * (4 + vbytes)
    phases = {k: statistics.median([s[k] for s in per_step_stats]) for k in ("setup_ms", "symbolic_ms", "scan_ms", "numeric_ms")}
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": max_ms / args.steps, "higher_is_better": True,
                "scaling": "weak", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
                "config": config_dict(args, A, world), "impl": "ours",
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "graph_replay": graph_replay,
                "gpu_launches": int(launches), "clocks": clk.summary(),
                "nprod": int(total_nprod), "nnz_c": int(st["nnz_c"]), "phase_ms_median": phases,
                "step_ms": step_ms, "wall_s": t_wall,
                "peak_mem_bytes": int(a_bytes + c_bytes + max(s["workspace_peak_bytes"] for s in per_step_stats)),
                "workspace_peak_bytes": int(max(s["workspace_peak_bytes"] for s in per_step_stats))}
        print(json.dumps(line), flush=True)
    h.close()
    if world > 1:
        dist.destroy_process_group()


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
