"""bench.py — SpGEMM GFLOPS (2*nprod/s) of C = A^2 on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config rmat22] [--dtype f32|f64]

Workload: BASELINE.json configs[4] (config 5), the R-MAT(0.45, 0.15, 0.15, 0.25) graph at scale 22,
edge factor 16 (4.19 M rows, 67 M nnz, 2.5e9 intermediate products, nnz(C) 2.5e9 > 2^31),
fp32 — the largest configuration quoted at 1/2/4/8 GPUs that fits one B200 with room for the
bench's own buffers (scale 23: 40.5 GB peak, 0.3 s per step).  One step = the whole
hot path of SURVEY.md §8(a) on one input already resident in HBM: symbolic (n_prod, grouping,
hash count, scan) -> exact allocation of C -> numeric (grouping, accumulate, gather, sort, write).

N GPUs (torchrun, one rank per GPU, NCCL): the rows of C are independent, so the
SAME matrix is split into n_prod-balanced row blocks (strong scaling): rank 0
holds A, B = A is broadcast in chunks (NCCL) while rank 0 computes the split points on its GPU
(then broadcast), every rank multiplies its zero-copy row block, and the nnz counts are all-gathered
(dist.py).  `value` times
the per-rank step (the local two-phase SpGEMM), max over ranks; `e2e` adds the host->device copy,
the broadcast, the partition, the all-gather and the device->host copy of every rank's C block.

Timing: W untimed warm-ups; K timed steps, CUDA events on the handle's stream, L2 flushed (512 MiB
write) before every step outside the events (A is 0.54 GB, C 20 GB: larger than L2 anyway);
barrier + synchronize on both sides; max over ranks; nvidia-smi clocks sampled during the steps.
Attribution (roofline): one more step with the per-group kernels serialised on one stream and
timed per group (CUDA events): the dominant kernel is the group with the largest time; its
algorithmic bytes (SURVEY.md §8(d) streaming model) / its time = `roofline.achieved`.

`--impl reference`: the CPU oracle (oracle/, plain C Gustavson, row-parallel over the host's
cores) on a bounded sample of the same workload, rank 0 only.
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
PER_CONFIG = [("cant", "f32"), ("cant", "f64"), ("webbase", "f32")]


def parse():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", default="ours", choices=["ours", "reference"])
    p.add_argument("--config", default="rmat22")
    p.add_argument("--dtype", default="f32", choices=["f32", "f64"])
    p.add_argument("--no-e2e", action="store_true")
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--no-per-config", action="store_true")
    p.add_argument("--opt", action="append", default=[],
                   help="library option name=value (ablations, e.g. rank_acc=0; see _lib.OPTIONS)")
    return p.parse_args()


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def workload(config, dtype):
    import synth
    A = synth.config(config, "uniform", 7)
    dt = np.float32 if dtype == "f32" else np.float64
    return A.astype(dt), dt


def config_dict(args, A, world):
    return {"workload": f"{args.config} A^2", "matrix": A.name, "rows": A.m, "nnz_a": A.nnz,
            "dtype": args.dtype, "baseline_config": "BASELINE.json configs[4] (config 5)" if args.config.startswith("rmat")
            else "BASELINE.json configs[1..3]",
            "partition": "n_prod-balanced row blocks of one matrix (strong scaling)" if world > 1 else "single GPU",
            "l2": "flushed (512 MiB write) before every timed step; inputs larger than L2",
            "inputs": "device-resident (value)",
            **({"options": dict(o.split("=") for o in args.opt)} if args.opt else {})}


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
    """SURVEY.md §8(d) streaming model (no reuse), per group launch:
    symbolic: 4 B/product (col_B) + 20 B/nnz(A) (col_A + rpt_B pair) + 28 B/row;
    numeric: (4+s) B/product (col_B,val_B) + (20+s) B/nnz(A) + (4+s) B/nnz(C) write + 36 B/row."""
    if phase == "sym":
        return 4 * st["sym_nprod"][g] + 20 * st["sym_nnza"][g] + 28 * st["sym_rows"][g]
    return ((4 + vbytes) * st["num_nprod"][g] + (20 + vbytes) * st["num_nnza"][g]
            + (4 + vbytes) * st["num_nnzc"][g] + 36 * st["num_rows"][g])


FAMILY = {1: "hash", 2: "rank", 3: "range", 4: "cluster", 5: "global", 6: "rank_big", 7: "tiny", 8: "batch", 9: "esc"}
SYM_KERNEL = {1: "k_sym_smem", 2: "k_sym_rankcnt", 3: "k_sym_range_bits", 5: "k_sym_global", 7: "k_sym_tiny",
              8: "k_sym_batch"}
NUM_KERNEL = {1: "k_num_smem", 2: "k_num_rankacc", 3: "k_num_range", 4: "k_num_cluster", 5: "k_num_global",
              6: "k_num_rankbig", 7: "k_num_tiny", 9: "k_num_esc"}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy bandwidth)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def load_traffic(config, dtype, phase, g):
    """DRAM bytes of this group's launch from the committed ncu capture of the same config
    (profiles/traffic_r02.json, written by scripts/traffic.py), or None."""
    p = os.path.join(ROOT, "profiles", "traffic_r02.json")
    if not os.path.exists(p):
        return None, None
    d = json.load(open(p))
    e = d.get(f"{config}|{dtype}|{phase}|g{g}")
    return (e["dram_bytes"], e["source"]) if e else (None, None)


def load_inst(config, dtype, phase, g):
    """Executed warp instructions and issue-active % of this group's launch (same ncu capture)."""
    p = os.path.join(ROOT, "profiles", "traffic_r02.json")
    e = json.load(open(p)).get(f"{config}|{dtype}|{phase}|g{g}") if os.path.exists(p) else None
    return (e.get("warp_inst"), e.get("issue_active_pct")) if e else (None, None)


# ----------------------------------------------------------------------------- reference arm
def reference_sample(A, nprod_rows, frac):
    """Rows [0, r) of A holding about `frac` of the intermediate products (hubs included)."""
    import oracle
    cum = np.cumsum(nprod_rows)
    r = int(np.searchsorted(cum, frac * cum[-1])) + 1
    return oracle.row_slice(A, 0, min(r, A.m)), int(cum[min(r, A.m) - 1])


def run_reference(args):
    rank, world, _ = dist_env()
    if rank != 0:
        return
    import oracle
    A, dt = workload(args.config, args.dtype)
    nprod_rows, total = oracle.nprod(A, A)
    S, s_nprod = reference_sample(A, nprod_rows, 1.0 / 8)
    oracle.build()
    times = []
    for i in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        oracle.spgemm(S, A, dt, parallel=True, with_abs=False)
        t = time.perf_counter() - t0
        if i >= args.warmup:
            times.append(t)
    tot = sum(times)
    val = 2 * s_nprod * len(times) / tot / 1e9
    sample = (f"rows [0, {S.m}) of {A.name} (1/8 of its {total} products: {s_nprod}) times A, "
              f"row-parallel oracle on {oracle.threads()} threads, per step")
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1e3 * tot / len(times), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": config_dict(args, A, 1), "impl": "reference",
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": oracle.threads(), "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- our arm
def csr_bytes(M, vbytes):
    return M.rpt.numel() * 8 + M.col.numel() * 4 + (M.val.numel() * vbytes if M.val is not None else 0)


def quick_value(P, torch, dev, config, dtype, steps, flush, opts):
    """GFLOPS of `config` on this GPU (graphs on, L2 flushed), for the per_config block."""
    A, dt = workload(config, dtype)
    tdt = torch.float32 if dt == np.float32 else torch.float64
    dA = P.CsrMatrix.from_host(A, dev, tdt)
    h = P.Handle(dev)
    for k, v in opts:
        h.set_option(k, v)
    for _ in range(3):
        h.multiply(dA, dA)
    torch.cuda.synchronize()
    ms = []
    for _ in range(steps):
        with torch.cuda.stream(h.stream):
            flush.add_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(h.stream)
        C = h.multiply(dA, dA)
        e1.record(h.stream)
        e1.synchronize()
        ms.append(e0.elapsed_time(e1))
        del C
    nprod = h.nprod
    h.close()
    t = statistics.median(ms)
    return {"value": 2 * nprod / t / 1e6, "unit": UNIT, "ms_per_step": t, "steps": steps, "nprod": int(nprod)}


def run_ours(args):
    import torch
    import torch.distributed as dist

    rank, world, local = dist_env()
    if world > 1:
        backend = os.environ.get("BENCH_BACKEND", "nccl")  # gloo: multi-rank test on one GPU
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    torch.cuda.set_device(local if torch.cuda.device_count() > local else 0)
    dev = torch.device("cuda", torch.cuda.current_device())
    import paper_conf_icpp_nagasakanm17_b200 as P
    from paper_conf_icpp_nagasakanm17_b200 import dist as D

    opts = [(k, int(v)) for k, v in (o.split("=") for o in args.opt)]
    A, dt = workload(args.config, args.dtype)  # every rank builds the seeded host copy (for e2e)
    tdt = torch.float32 if dt == np.float32 else torch.float64
    vbytes = 4 if dt == np.float32 else 8
    h = P.Handle(dev)
    for k, v in opts:
        h.set_option(k, v)
    stream = h.stream
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def maxr(x):
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sumr(x):
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
        if world > 1:
            dist.all_reduce(t, op=dist.ReduceOp.SUM)
        return float(t.item())

    # setup (untimed): A on rank 0's GPU, chunked broadcast of B = A, n_prod-balanced split
    dA0 = P.CsrMatrix.from_host(A, dev, tdt) if rank == 0 else None
    barrier()
    t0 = time.perf_counter()
    if world > 1:  # chunked broadcast with the n_prod split computed on rank 0 meanwhile
        _, Bd, splits = D.broadcast_and_partition(dA0, None, src=0, device=dev, dtype=tdt, world=world,
                                                  partition=D.cuda_partition(h), square=True)
    else:
        Bd, splits = dA0, D.cuda_partition(h)(dA0, dA0, 1)
    barrier()
    bcast_s = time.perf_counter() - t0
    r0, r1 = splits[rank], splits[rank + 1]
    mine = D.row_slice(Bd, r0, r1)

    def step():
        return h.multiply(mine, Bd)

    for _ in range(max(3, args.warmup)):
        step()
    barrier()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches = 0
    with ClockSampler(dev.index) as clk:
        barrier()
        t_wall = time.perf_counter()
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                flush.add_(1)
            ev[i][0].record(stream)
            C = step()
            ev[i][1].record(stream)
            st = h.stats()
            launches += st["kernel_launches_symbolic"] + st["kernel_launches_numeric"]
            del C
        barrier()
        t_wall = time.perf_counter() - t_wall
    step_ms = [a.elapsed_time(b) for a, b in ev]
    my_ms = sum(step_ms)
    my_nprod = h.nprod
    max_ms = maxr(my_ms)
    total_nprod = sumr(my_nprod)
    value = 2 * total_nprod * args.steps / (max_ms / 1e3) / 1e9
    imbalance = {"nprod_max_over_mean": maxr(my_nprod) / (total_nprod / world),
                 "time_max_over_mean": max_ms / (sumr(my_ms) / world)}

    # attribution: one step with the group kernels serialised and timed per group
    h.set_option("streams", 0).set_option("timing", 2)
    with torch.cuda.stream(stream):
        flush.add_(1)
    C = step()
    torch.cuda.synchronize()
    sa = h.stats()
    del C
    h.set_option("streams", 1).set_option("timing", 1)
    serial_ms = sa["setup_ms"] + sa["symbolic_ms"] + sa["scan_ms"] + sa["numeric_ms"]
    groups = []
    for ph, key, kk in (("sym", "sym_group_ms", "sym_kernel"), ("num", "num_group_ms", "num_kernel")):
        for g, ms in enumerate(sa[key]):
            if ms > 0:
                groups.append((ms, ph, g, sa[kk][g]))
    groups.sort(reverse=True)
    k_ms, ph, g, kind = groups[0]
    bytes_alg = algorithmic_bytes(sa, ph, g, vbytes)
    peak, peak_src = load_peaks()
    achieved = bytes_alg / (k_ms / 1e3) / 1e9
    traffic, traffic_src = load_traffic(args.config, args.dtype, ph, g)
    kname = (SYM_KERNEL if ph == "sym" else NUM_KERNEL).get(kind, "?")
    roofline = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                "traffic": traffic, "traffic_source": traffic_src,
                "achieved_model": "algorithmic bytes (SURVEY.md §8(d) streaming model, no reuse: B-row re-reads "
                                  "that hit L2 count as HBM bytes) / kernel time",
                "frac_dram": (traffic / (k_ms / 1e3) / 1e9 / peak) if traffic else None,
                "kernel": f"{kname} ({FAMILY.get(kind, '?')}, {ph} group {g})", "phase": ph, "group": g,
                "launch_ms": k_ms, "share_of_serial_step": k_ms / serial_ms,
                "algorithmic_bytes_per_launch": int(bytes_alg), "peak_source": peak_src,
                "attribution": "per-group CUDA events, group kernels serialised on one stream (one extra step)",
                "top_groups": [{"phase": p, "group": q, "kernel": (SYM_KERNEL if p == "sym" else NUM_KERNEL).get(k, "?"),
                                "ms": m} for m, p, q, k in groups[:6]]}
    # the roof that binds the graph kernels: instruction issue — executed warp
    # instructions of the same launch (ncu) / kernel time against 4 issue slots per SM per cycle
    winst, issue_pct = load_inst(args.config, args.dtype, ph, g)
    if winst:
        sms = torch.cuda.get_device_properties(dev).multi_processor_count
        peak_issue = sms * 4 * 1965e6 / 1e9  # G warp-instructions/s at the B200's max SM clock
        ach_issue = winst / (k_ms / 1e3) / 1e9
        roofline["issue"] = {"bound": "issue", "achieved": ach_issue, "peak": peak_issue,
                             "unit": "G warp-instr/s", "frac": ach_issue / peak_issue,
                             "ncu_issue_active_pct": issue_pct, "warp_inst_per_launch": int(winst),
                             "peak_source": f"{sms} SMs x 4 schedulers x 1965 MHz (max SM clock, nvidia-smi)",
                             "source": "ncu smsp__inst_executed.sum of the same launch (scripts/traffic.py)"}

    # measured peak device memory of one step (all library workspace through torch's allocator)
    peak_mem = None
    if world == 1:
        hp = P.Handle(dev, torch_allocator=True)
        for k, v in opts:
            hp.set_option(k, v)
        del flush
        torch.cuda.synchronize()
        torch.cuda.empty_cache()
        free0 = torch.cuda.mem_get_info(dev)[0]
        torch.cuda.reset_peak_memory_stats(dev)
        base = torch.cuda.memory_allocated(dev)
        C = hp.multiply(mine, Bd)
        torch.cuda.synchronize()
        peak_alloc = torch.cuda.max_memory_allocated(dev)
        a_bytes = csr_bytes(Bd, vbytes)
        c_bytes = csr_bytes(C, vbytes)
        peak_mem = {"peak_device_bytes": int(peak_alloc), "inputs_bytes": int(a_bytes), "c_bytes": int(c_bytes),
                    "overhead_bytes": int(peak_alloc - a_bytes - c_bytes),
                    "step_increase_bytes": int(peak_alloc - base),
                    "cudaMemGetInfo_free_drop_bytes": int(free0 - torch.cuda.mem_get_info(dev)[0]),
                    "how": "torch.cuda.max_memory_allocated over one step, library workspace through the torch "
                           "allocator callbacks (include/spgemm.h spgemm_allocator_t); inputs resident, "
                           "no other buffers"}
        del C
        hp.close()
        # allocation of C (reading R18): warm (caching allocator) and cold (the
        # cache emptied first: cudaMalloc of nnz(C) entries)
        nnz_c = h.nnz_c
        def alloc_ms():
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            cc = torch.empty(nnz_c, dtype=torch.int32, device=dev)
            cv = torch.empty(nnz_c, dtype=tdt, device=dev)
            e1.record()
            torch.cuda.synchronize()
            del cc, cv
            return e0.elapsed_time(e1)
        alloc_ms()
        warm = statistics.median(alloc_ms() for _ in range(5))
        torch.cuda.empty_cache()
        cold = alloc_ms()
        peak_mem["c_alloc_ms"] = {"warm": warm, "cold": cold, "bytes": int(nnz_c * (4 + vbytes))}
        flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    # end to end through the public API: pinned host A -> device, (broadcast, split,) multiply,
    # device -> pinned host C block
    e2e = None
    if not args.no_e2e:
        hA = P.CsrMatrix.from_host(A, None, tdt, pin=True) if rank == 0 else None
        bi = csr_bytes(hA, vbytes) if rank == 0 else 0
        nnz_mine = h.nnz_c
        out = (torch.empty(r1 - r0 + 1, dtype=torch.int64, pin_memory=True),
               torch.empty(nnz_mine, dtype=torch.int32, pin_memory=True),
               torch.empty(nnz_mine, dtype=tdt, pin_memory=True))
        bo = sum(x.numel() * x.element_size() for x in out)
        e_ms = []
        for i in range(args.warmup + args.steps):
            with torch.cuda.stream(stream):
                flush.add_(1)
            barrier()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            with torch.cuda.stream(stream):
                dA2 = hA.to(dev, non_blocking=True) if rank == 0 else None
            if world > 1:
                with torch.cuda.stream(stream):
                    _, B2, sp = D.broadcast_and_partition(dA2, None, src=0, device=dev, dtype=tdt, world=world,
                                                          partition=D.cuda_partition(h), square=True)
            else:
                B2, sp = dA2, [0, A.m]
            C = h.multiply(D.row_slice(B2, sp[rank], sp[rank + 1]), B2)
            with torch.cuda.stream(stream):
                if world > 1:
                    cnt = torch.tensor([C.nnz], dtype=torch.int64, device=dev)
                    dist.all_gather([torch.zeros_like(cnt) for _ in range(world)], cnt)
                out[0].copy_(C.rpt, non_blocking=True)
                out[1].copy_(C.col, non_blocking=True)
                out[2].copy_(C.val, non_blocking=True)
            e1.record(stream)
            e1.synchronize()
            if i >= args.warmup:
                e_ms.append(e0.elapsed_time(e1))
            del C, dA2, B2
        et = maxr(sum(e_ms))
        e2e = {"value": 2 * total_nprod * len(e_ms) / (et / 1e3) / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": int(bi), "d2h_bytes_per_step": int(bo), "ms_per_step": et / len(e_ms),
               "includes": "H2D of A (rank 0), " + ("NCCL broadcast, partition, all-gather of nnz, " if world > 1 else "")
                           + "the step, D2H of the rank's C block (max over ranks)"}
        del out

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        oracle.build()
        t0 = time.perf_counter()
        oracle.spgemm(A, A, dt, parallel=True, with_abs=False)
        t_all = time.perf_counter() - t0
        nprod_rows, _ = oracle.nprod(A, A)
        S, s_nprod = reference_sample(A, nprod_rows, 1.0 / 64)
        t0 = time.perf_counter()
        oracle.spgemm(S, A, dt)
        t_one = time.perf_counter() - t0
        cpu = {"value": 2 * my_nprod / t_all / 1e9, "unit": UNIT, "cores": oracle.threads(), "kind": "oracle",
               "sample": f"full {A.name} A^2 ({args.dtype}), 1 run of the row-parallel oracle "
                         f"({oracle.threads()} threads of {oracle.cores()} host cores), {t_all:.1f} s",
               "single_thread": {"value": 2 * s_nprod / t_one / 1e9, "unit": UNIT, "cores": 1,
                                 "sample": f"rows [0, {S.m}) (1/64 of the products) x A, {t_one:.1f} s"}}

    per_config = None
    if rank == 0 and world == 1 and not args.no_per_config:
        per_config = {}
        for cfg, dty in PER_CONFIG:
            if (cfg, dty) != (args.config, args.dtype):
                per_config[f"{cfg}_{dty}"] = quick_value(P, torch, dev, cfg, dty, 10, flush, opts)

    phases = {k: sa[k] for k in ("setup_ms", "symbolic_ms", "scan_ms", "numeric_ms")}
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": max_ms / args.steps, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
                "config": config_dict(args, A, world), "impl": "ours",
                "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": int(launches), "clocks": clk.summary(),
                "nprod": int(total_nprod), "nnz_c": int(sumr(h.nnz_c)),
                "phase_ms_serial_step": phases, "step_ms": step_ms, "wall_s": t_wall,
                "peak_mem": peak_mem, "workspace_peak_bytes": int(st["workspace_peak_bytes"]),
                "multi_gpu": {"ranks": world, "splits": [int(x) for x in splits], "broadcast_s": bcast_s,
                              "imbalance": imbalance} if world > 1 else None,
                "per_config": per_config}
        print(json.dumps(line), flush=True)
    else:
        sumr(h.nnz_c)
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
