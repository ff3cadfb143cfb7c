"""DRAM traffic per group kernel of one serialised multiply, from ncu, for bench.py's
roofline.traffic (profiles/traffic_r02.json; run on the GPU box).

    python scripts/traffic.py CONFIG [DTYPE] [--top N]

(round 2: also executed warp instructions and issue-active %, for the issue roofline)

1. runs one serialised multiply (streams 0, per-group events) and lists the groups with their
   kernel family and time (same as bench.py's attribution step);
2. for each of the N slowest groups runs ncu on one more serialised multiply restricted to the
   group's kernel family (`--metrics dram__bytes_read.sum,dram__bytes_write.sum,
   gpu__time_duration.sum`): within one serialised multiply a family's launches come in ascending
   group order, so the i-th captured launch is the i-th group of that family;
3. merges {"CONFIG|DTYPE|phase|gG": {dram_bytes, ncu_time_ns, source}} into
   profiles/traffic_r02.json.
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
OUT = os.path.join(ROOT, "profiles", "traffic_r02.json")
SYM = {1: "k_sym_smem", 2: "k_sym_rankcnt", 3: "k_sym_range_bits", 5: "k_sym_global", 7: "k_sym_tiny", 8: "k_sym_batch"}
NUM = {1: "k_num_smem", 2: "k_num_rankacc", 3: "k_num_range", 4: "k_num_cluster", 5: "k_num_global",
       6: "k_num_rankbig", 7: "k_num_tiny", 9: "k_num_esc"}


def one_multiply(config, dtype):
    import numpy as np
    import torch
    import synth
    import paper_conf_icpp_nagasakanm17_b200 as P
    A = synth.config(config, "uniform", 7).astype(np.float32 if dtype == "f32" else np.float64)
    dA = P.CsrMatrix.from_host(A, "cuda", torch.float32 if dtype == "f32" else torch.float64)
    with P.Handle() as h:
        h.set_option("streams", 0).set_option("timing", 2)
        C = h.multiply(dA, dA)
        torch.cuda.synchronize()
        st = h.stats()
        del C
    return st


def main():
    if sys.argv[1] == "--child":
        st = one_multiply(sys.argv[2], sys.argv[3])
        print("STATS " + json.dumps({k: st[k] for k in ("sym_kernel", "num_kernel", "sym_group_ms", "num_group_ms")}))
        return
    config = sys.argv[1]
    dtype = sys.argv[2] if len(sys.argv) > 2 and not sys.argv[2].startswith("--") else "f32"
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 3
    st = one_multiply(config, dtype)
    groups = []
    for ph, key, kk, fam in (("sym", "sym_group_ms", "sym_kernel", SYM), ("num", "num_group_ms", "num_kernel", NUM)):
        for g, ms in enumerate(st[key]):
            if ms > 0 and st[kk][g] in fam:
                groups.append((ms, ph, g, fam[st[kk][g]]))
    groups.sort(reverse=True)
    db = json.load(open(OUT)) if os.path.exists(OUT) else {}
    done = set()
    for ms, ph, g, kname in groups[:top]:
        if kname in done:
            continue
        done.add(kname)
        # all groups of this family, in launch order
        fam_groups = sorted(q for _, p, q, k in groups if k == kname and p == ph)
        r = subprocess.run(["ncu", "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,"
                            "smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active",
                            "--clock-control", "none", "--csv", "--print-units", "base", "-k", f"regex:{kname}",
                            sys.executable, __file__, "--child", config, dtype], capture_output=True, text=True)
        rows = list(csv.reader(io.StringIO(r.stdout)))
        hi = next(i for i, x in enumerate(rows) if x and x[0] == "ID")
        hdr = rows[hi]
        launches = {}
        for x in rows[hi + 1:]:
            if len(x) != len(hdr) or not x[0].isdigit():
                continue
            d = dict(zip(hdr, x))
            launches.setdefault(int(d["ID"]), {})[d["Metric Name"]] = float(d["Metric Value"])
        ids = sorted(launches)
        if len(ids) != len(fam_groups):
            print(f"{kname}: {len(ids)} launches for groups {fam_groups}; skipped", flush=True)
            continue
        for i, q in zip(ids, fam_groups):
            m = launches[i]
            byts = int(m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0))
            db[f"{config}|{dtype}|{ph}|g{q}"] = {"dram_bytes": byts, "ncu_time_ns": m.get("gpu__time_duration.sum"),
                                                 "warp_inst": int(m.get("smsp__inst_executed.sum", 0)),
                                                 "issue_active_pct": m.get(
                                                     "smsp__issue_active.avg.pct_of_peak_sustained_active"),
                                                 "kernel": kname,
                                                 "source": f"ncu --metrics dram__bytes_read/write.sum, serialised "
                                                           f"multiply of {config} {dtype} (scripts/traffic.py)"}
            print(f"{config} {dtype} {ph} g{q} {kname}: {byts / 1e9:.3f} GB", flush=True)
    os.makedirs(os.path.dirname(OUT), exist_ok=True)
    json.dump(db, open(OUT, "w"), indent=1, sort_keys=True)


if __name__ == "__main__":
    main()
