"""Summarise an ncu --page source --print-source sass CSV: top instructions by stall samples
and executed warp-instructions.  usage: python scripts/sass_hot.py file.csv [N]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
sec = int(sys.argv[3]) if len(sys.argv) > 3 else 0
starts = [i for i, r in enumerate(rows) if r and r[0] == "Kernel Name"]
print("sections:", [rows[i][1][:80] for i in starts])
s0 = starts[sec]
s1 = starts[sec + 1] if sec + 1 < len(starts) else len(rows)
hdr = rows[s0 + 1]
ix = {h: i for i, h in enumerate(hdr)}
data = rows[s0 + 2:s1]
tot_s = sum(int(r[ix["Warp Stall Sampling (All Samples)"]] or 0) for r in data)
tot_i = sum(int(r[ix["Instructions Executed"]] or 0) for r in data)
print(f"instructions executed (warp) {tot_i:,}  samples {tot_s:,}  sass lines {len(data)}")
N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
order = sorted(range(len(data)), key=lambda i: -int(data[i][ix["Warp Stall Sampling (All Samples)"]] or 0))
for i in sorted(order[:N]):
    r = data[i]
    print(f"{i:5d} {int(r[ix['Warp Stall Sampling (All Samples)']] or 0):7d} {int(r[ix['Instructions Executed']] or 0):11,d} "
          f"{r[ix['L1 Conflicts Shared N-Way']]:>4} {r[ix['Source']].strip()[:70]}")
