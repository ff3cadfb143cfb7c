#!/bin/bash
# bench lines of every single-GPU config (no CPU baseline):  bash scripts/gpu_benchset.sh TAG [configs...]
TAG=${1:-bs}; shift
CFGS=${@:-"cant webbase rmat20 mixed:protein mixed:qcd mixed:economics mixed:epidemiology poisson64"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for c in $CFGS; do
  for dt in f32 f64; do
    timeout 300 python bench.py --config $c --dtype $dt --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_${TAG}_${c#mixed:}_$dt.json 2>/dev/null
    python -c "
import json,sys; d=json.load(open('gpurun_out/bench_${TAG}_${c#mixed:}_$dt.json')); print('$c $dt', round(d['value'],1), 'GFLOPS', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['phase_ms_median'].items()}, 'graph', round(d['graph_replay']['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), d['roofline']['kernel'])" 2>&1 | tail -1
  done
done
