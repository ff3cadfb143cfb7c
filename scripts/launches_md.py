"""ncu launch list (gpu__time_duration.sum per launch) of one bench step -> markdown table.

    python scripts/launches_md.py gpurun_out/launches_TAG_CONFIG.csv "title" > profiles/launches_TAG_CONFIG.md

The csv comes from scripts/gpu_launches.sh (`ncu --metrics gpu__time_duration.sum --clock-control
none` around `bench.py --steps 1 --streams 0`): launches are serialised and cold-cache, so compare
shares, not absolute times, with the bench's CUDA-event numbers.
"""
import csv
import re
import sys


def main():
    path, title = sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""
    rows = list(csv.reader(open(path)))
    hdr, out = None, []
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            out.append((d["Kernel Name"], float(d["Metric Value"]) / 1e3))
    starts = [i for i, (k, _) in enumerate(out) if "k_brow_minmax" in k or "k_nprod_group" in k]
    starts = [i for i in starts if i == 0 or "k_brow_minmax" not in out[i - 1][0]]
    step = out[starts[-1]:] if starts else out
    lib = [(k, t) for k, t in step if "spg" in k or "k_" in k]
    tot = sum(t for _, t in lib)
    print(f"# ncu launch list — {title}\n")
    print("`ncu --metrics gpu__time_duration.sum --clock-control none`, one `bench.py` step with one stream "
          "(serialised, cold cache per launch: compare shares).\n")
    print("| # | kernel | µs | share |\n|---|---|---:|---:|")
    for i, (k, t) in enumerate(lib):
        short = re.sub(r"\(.*", "", k).replace("spg::<unnamed>::", "").replace("void ", "")
        short = re.sub(r"^unnamed>::", "", short)
        print(f"| {i} | `{short}` | {t:.1f} | {t / tot:.1%} |")
    print(f"\nLibrary kernels: {len(lib)}; total {tot:.1f} µs.")


if __name__ == "__main__":
    main()
