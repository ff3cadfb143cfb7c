"""Summarise a round's ncu outputs into profiles/ (tracked).

    python scripts/summarize_profile.py TAG
reads gpurun_out/launches_TAG.csv (gpu__time_duration launch list of a bench command) and
gpurun_out/prof_TAG.ncu-rep (--set full capture of the group kernels of one bench step), writes
profiles/launches_TAG.md, profiles/ncu_TAG.md and profiles/traffic.json (DRAM bytes per launch of
each captured group kernel, read by bench.py for roofline.traffic).
"""
import csv
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TAG = sys.argv[1] if len(sys.argv) > 1 else "r01"
OUT = os.path.join(ROOT, "profiles")
os.makedirs(OUT, exist_ok=True)

SYM = {}  # template signature -> group id, from the group tables in csrc/spgemm_internal.cuh
NUM = {}


def _tables():
    src = open(os.path.join(ROOT, "paper_conf_icpp_nagasakanm17_b200/csrc/spgemm_internal.cuh")).read()
    for name, dst in (("kSymGroups", SYM), ("kNumGroups", NUM)):
        body = src[src.index(f"constexpr GroupSpec {name}[] = {{"):]
        body = body[:body.index("};")]
        for g, m in enumerate(re.finditer(r"\{(-?\d+),\s*(\d+),\s*(\d+),\s*(\d+)\}", body)):
            upper, T, TPR, BS = m.groups()
            dst[(int(T), int(TPR), int(BS), int(upper))] = g


def group_of(kname: str):
    m = re.search(r"k_sym_smem<(?:\(int\))?(\d+), (?:\(int\))?(\d+), (?:\(int\))?(\d+), (?:\(bool\))?(\w+)>", kname)
    if m:
        T, TPR, BS, opt = int(m.group(1)), int(m.group(2)), int(m.group(3)), m.group(4)
        for (t, tpr, bs, up), g in SYM.items():
            if (t, tpr, bs) == (T, TPR, BS) and ((up == -1) == (opt in ("1", "true"))):
                return "sym", g
    m = re.search(r"k_num_smem<(\w+), (?:\(int\))?(\d+), (?:\(int\))?(\d+), (?:\(int\))?(\d+), (?:\(long long\))?(\d+)L?L?>", kname)
    if m:
        T, TPR, BS, up = int(m.group(2)), int(m.group(3)), int(m.group(4)), int(m.group(5))
        return "num", NUM.get((T, TPR, BS, up))
    m = re.search(r"k_num_rankacc<\w+, (?:\(int\))?(\d+), (?:\(long long\))?(\d+)", kname)
    if m:
        up = int(m.group(2))
        return "num", next((g for (t, tpr, bs, u), g in NUM.items() if u == up), None)
    m = re.search(r"k_sym_rankcnt<(?:\(int\))?(\d+), (?:\(long long\))?(\d+)", kname)
    if m:
        up = int(m.group(2))
        return "sym", next((g for (t, tpr, bs, u), g in SYM.items() if u == up), None)
    if "k_num_rankbig" in kname:
        return "num", 10
    if re.search(r"k_sym_range(_bits)?\b", kname):
        return "sym", 12  # kSymRange
    if "k_num_range" in kname:
        return "num", 14  # kNumRange
    if "k_sym_cluster" in kname:
        return "sym", 10
    if "k_num_cluster" in kname:
        return "num", 10
    return None, None


def launches():
    path = os.path.join(ROOT, "gpurun_out", f"launches_{TAG}.csv")
    rows = list(csv.reader(open(path)))
    hdr, out = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            out.append((int(d["ID"]), d["Kernel Name"], float(d["Metric Value"]) / 1e3))
    # one bench step = the launches between two k_brow_minmax (first kernel of a step)
    starts = [i for i, (_, k, _) in enumerate(out) if "k_brow_minmax" in k or "k_nprod_group" in k and "k_brow" not in k]
    starts = [i for i, (_, k, _) in enumerate(out) if re.search(r"k_brow_minmax(?!_)", k)] or starts
    step = out[starts[-2]:starts[-1]] if len(starts) >= 2 else out
    tot = sum(t for _, k, t in step if k.startswith(("void spg", "spg")))
    lines = [f"# ncu launch list ({TAG}) — one bench step of `python bench.py` (cant-like A^2, fp32)", "",
             "`ncu --metrics gpu__time_duration.sum --clock-control none` (serialised, cold L2 per launch: compare",
             "shares, not absolutes; the bench times the step with CUDA events).", "",
             "| # | kernel | µs | share |", "|---|---|---:|---:|"]
    for i, (lid, k, t) in enumerate(step):
        short = re.sub(r"\(.*", "", k).replace("spg::<unnamed>::", "").replace("void ", "")
        ph, g = group_of(k)
        tag = f" [{ph} group {g}]" if ph else ("" if "spg" in k else " (bench L2 flush, outside the timed events)")
        lines.append(f"| {i} | `{short}`{tag} | {t:.1f} | {t / tot:.1%} |")
    lines += ["", f"Library kernels in the step: {sum(1 for _, k, _ in step if 'spg' in k)}; total {tot:.1f} µs "
              "(serialised)."]
    open(os.path.join(OUT, f"launches_{TAG}.md"), "w").write("\n".join(lines) + "\n")
    return step


METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
           "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
           "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
           "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "launch__registers_per_thread",
           "launch__occupancy_limit_shared_mem", "launch__grid_size", "launch__block_size"]


def full():
    rep = os.path.join(ROOT, "gpurun_out", f"prof_{TAG}.ncu-rep")
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units = rows[0], rows[1]
    uni = dict(zip(hdr, units))
    traffic = {}
    lines = [f"# ncu --set full ({TAG}) — group kernels of one bench step (cant-like A^2, fp32)", "",
             "`ncu --set full --clock-control none --import-source on -k regex:<group kernels> -c 6` "
             "(scripts/gpu_round.sh)", ""]
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        k = d["Kernel Name"]
        ph, g = group_of(k)
        lines.append(f"## `{re.sub(r'[(].*', '', k).replace('spg::<unnamed>::', '')}` — {ph} group {g}")
        for mname in METRICS:
            if mname in d:
                lines.append(f"- {mname} = {d[mname]} {uni.get(mname, '')}")
        stalls = sorted(((float(d[h].replace(",", "") or 0), h) for h in hdr
                         if h.startswith("smsp__pcsamp_warps_issue_stalled") and not h.endswith("not_issued")
                         and d.get(h)), reverse=True)[:6]
        lines.append("- top stall reasons (pc samples): " + ", ".join(
            f"{h.replace('smsp__pcsamp_warps_issue_stalled_', '')} {v:.0f}" for v, h in stalls))
        lines.append("")

        def tobytes(v, u):
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            return float(v.replace(",", "")) * scale
        if ph:
            b = tobytes(d["dram__bytes_read.sum"], uni["dram__bytes_read.sum"]) + \
                tobytes(d["dram__bytes_write.sum"], uni["dram__bytes_write.sum"])
            traffic[f"{ph}_g{g}_f32"] = int(b)  # the captured bench step is fp32
    open(os.path.join(OUT, f"ncu_{TAG}.md"), "w").write("\n".join(lines) + "\n")
    tj = os.path.join(OUT, "traffic.json")
    old = json.load(open(tj)) if os.path.exists(tj) else {}
    old.update(traffic)
    old["_source"] = f"profiles/ncu_{TAG}.md: dram__bytes_read.sum + dram__bytes_write.sum per launch"
    json.dump(old, open(tj, "w"), indent=1)
    return traffic


if __name__ == "__main__":
    _tables()
    launches()
    print(full())
