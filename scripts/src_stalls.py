"""Top source lines by stall samples with their dominant stall reasons.
usage: python scripts/src_stalls.py file.csv [N]   (csv from ncu --page source --csv --print-source cuda,sass)"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
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
    if hdr and r[0] and r[0].isdigit():
        try:
            s = int(r[hdr["Warp Stall Sampling (All Samples)"]] or 0)
            ins = int(r[hdr["Instructions Executed"]] or 0)
        except (ValueError, IndexError):
            continue
        st = {}
        for h, i in hdr.items():
            if h.startswith("stall_") and "Not Issued" not in h:
                try:
                    v = int(r[i] or 0)
                except ValueError:
                    v = 0
                if v:
                    st[h[6:]] = v
        top = sorted(st.items(), key=lambda kv: -kv[1])[:3]
        out.append((s, ins, path, r[0], r[1].strip(), top))
tot = sum(o[0] for o in out)
print(f"samples {tot:,}")
for s, ins, p, ln, src, top in sorted(out, key=lambda o: -o[0])[:N]:
    t = " ".join(f"{k}:{100 * v / max(s, 1):.0f}%" for k, v in top)
    print(f"{100 * s / max(tot, 1):5.1f}% {ins:11,d} {p}:{ln} {src[:70]:70s} | {t}")
