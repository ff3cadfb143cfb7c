#!/bin/bash
# Paper-style ablations on B200:
#   streams (concurrent per-group kernels) on/off, rank-indexed tables on/off, range rows on/off,
#   paper hash only (no column spans), partial-warp groups off (every row in a CTA group),
#   cluster tables off (overflow rows straight to global memory), lanes per B row.
#   bash scripts/gpu_ablation.sh TAG [configs...]
TAG=${1:-abl}; shift
CFGS=${@:-"cant webbase rmat18 mixed:qcd"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
OUT=gpurun_out/ablation_$TAG.jsonl; : > $OUT
run() {  # config label args...
  local c=$1 lab=$2; shift 2
  timeout 300 python bench.py --config $c --no-cpu-baseline --no-e2e --steps 5 "$@" > /tmp/abl.json 2>/dev/null || return
  python - "$c" "$lab" >> $OUT <<'PY'
import json, sys
d = json.load(open("/tmp/abl.json"))
print(json.dumps({"config": sys.argv[1], "variant": sys.argv[2], "gflops": d["value"], "ms": d["ms_per_step"],
                  "phases": d["phase_ms_median"], "graph_ms": d["graph_replay"]["ms_per_step"]}))
PY
  tail -1 $OUT | cut -c1-200
}
for c in $CFGS; do
  run $c default
  run $c streams_off --streams 0
  run $c rank_off --opt rank_acc=0
  run $c range_rows_off --opt range_warp=0
  run $c paper_hash_only --opt range_hash=0
  run $c no_partial_warp --opt sym_min_group=5 --opt num_min_group=4
  run $c cluster_off --opt cluster=0
  for l in 1 4 32; do run $c lanes_$l --lanes $l; done
done
