"""Per CUDA source line: stall samples, warp-instructions, shared-memory wavefronts (and the excess
over ideal = bank conflicts), from `ncu -i R --page source --csv --print-source cuda,sass`.
usage: python scripts/src_lines.py file.csv [N] [sort: samples|wf]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
key = sys.argv[3] if len(sys.argv) > 3 else "samples"
hdr = None
agg = collections.defaultdict(lambda: [0, 0, 0, 0, ""])
cur = None
for r in rows:
    if len(r) > 1 and r[0] == "Line No":
        hdr = {h: i for i, h in enumerate(r)}
        continue
    if not hdr or len(r) < 5:
        continue
    if not r[0]:
        continue  # SASS rows repeat their line's totals: count the CUDA row only
    cur = (int(r[0]), r[1].strip())
    def g(name):
        try:
            return int(float(r[hdr[name]] or 0))
        except (KeyError, ValueError):
            return 0
    a = agg[cur[0]]
    a[0] += g("Warp Stall Sampling (All Samples)")
    a[1] += g("Instructions Executed")
    a[2] += g("L1 Wavefronts Shared")
    a[3] += g("L1 Wavefronts Shared Excessive")
    a[4] = cur[1]
tot = [sum(v[i] for v in agg.values()) for i in range(4)]
print(f"samples {tot[0]:,}  warp-inst {tot[1]:,}  smem wavefronts {tot[2]:,} (excess {tot[3]:,})")
idx = 0 if key == "samples" else 2
for ln, v in sorted(agg.items(), key=lambda kv: -kv[1][idx])[:N]:
    print(f"{100*v[0]/max(tot[0],1):5.1f}% {v[1]:12,d} wf {v[2]:12,d} ex {v[3]:12,d}  :{ln} {v[4][:80]}")
