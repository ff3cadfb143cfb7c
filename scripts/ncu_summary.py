"""Markdown summary of an ncu --set full report: key metrics per captured kernel and the top source
lines by stall samples (with their stall reasons and shared-memory wavefronts).

    python scripts/ncu_summary.py REPORT.ncu-rep "title" > profiles/ncu_TAG.md
"""
import csv
import io
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
METRICS = [
    ("gpu__time_duration.sum", "time (ns)"),
    ("dram__bytes_read.sum", "DRAM read (B)"),
    ("dram__bytes_write.sum", "DRAM write (B)"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_active", "L1TEX % of peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads / instruction"),
    ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "shared wavefronts"),
    ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "shared bank conflicts"),
    ("launch__registers_per_thread", "registers"),
    ("launch__block_size", "block"),
    ("launch__grid_size", "grid"),
]


def ncu(args):
    return subprocess.run(["ncu", "-i", *args], capture_output=True, text=True).stdout


def main():
    rep, title = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    raw = list(csv.reader(io.StringIO(ncu([rep, "--page", "raw", "--csv", "--print-units", "base", "--metrics",
                                           ",".join(m for m, _ in METRICS)]))))
    hi = next(i for i, r in enumerate(raw) if r and r[0] == "ID")
    hdr = raw[hi]
    rows = [dict(zip(hdr, r)) for r in raw[hi + 1:] if len(r) == len(hdr) and r[0].isdigit()]
    print(f"# ncu --set full — {title}\n")
    print(f"Report `{os.path.basename(rep)}` (`--clock-control none --import-source on`, kernel replay: "
          "cold caches, serialised; compare shares, not absolute times).\n")
    print("| metric | " + " | ".join(f"#{r['ID']}" for r in rows) + " |")
    print("|---|" + "---:|" * len(rows))
    print("| kernel | " + " | ".join(r["Kernel Name"].replace("(unnamed namespace)::", "").split("(")[0][:48]
                                      for r in rows) + " |")
    for m, name in METRICS:
        vals = []
        for r in rows:
            v = r.get(m, "")
            try:
                x = float(v.replace(",", ""))
                vals.append(f"{x:,.0f}" if x >= 100 else f"{x:.3g}")
            except ValueError:
                vals.append(v)
        print(f"| {name} | " + " | ".join(vals) + " |")
    for i, r in enumerate(rows):
        src = ncu([rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "--launch-skip", str(i),
                   "--launch-count", "1"])
        path = f"/tmp/ncu_src_{i}.csv"
        open(path, "w").write(src)
        out = subprocess.run([sys.executable, os.path.join(HERE, "src_stalls.py"), path, "12"],
                             capture_output=True, text=True).stdout
        print(f"\n### #{r['ID']} top source lines by stall samples\n\n```\n{out.strip()}\n```")


if __name__ == "__main__":
    main()
