"""Top CUDA source lines by warp-stall samples from `ncu -i R --page source --csv --print-source cuda,sass`.
usage: python scripts/src_hot.py file.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
path, hdr, out = None, None, []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        path = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = {h: i for i, h in enumerate(r)}
        continue
    if hdr and r[0]:
        try:
            s = int(r[hdr["Warp Stall Sampling (All Samples)"]] or 0)
            ins = int(r[hdr["Instructions Executed"]] or 0)
        except (ValueError, IndexError):
            continue
        out.append((s, ins, path, r[0], r[1].strip()))
tot = sum(o[0] for o in out)
toti = sum(o[1] for o in out)
print(f"samples {tot:,} warp-instructions {toti:,}")
for s, ins, p, ln, src in sorted(out, reverse=True)[:N]:
    print(f"{100 * s / max(tot, 1):5.1f}% {ins:12,d} {p}:{ln} {src[:90]}")
