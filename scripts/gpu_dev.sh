#!/bin/bash
# dev cycle: build, selected GPU tests (-k EXPR), serial per-group diag of configs, bench line
#   TESTS="rank_acc" DIAG="rmat20 webbase" bash scripts/gpu_dev.sh TAG
TAG=${1:-dev}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
if [ -n "$TESTS" ]; then timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "$TESTS" > gpurun_out/t_$TAG.log 2>&1; tail -5 gpurun_out/t_$TAG.log; fi
for c in $DIAG; do timeout 300 python scripts/diag.py $c --opt streams=0 $DIAGOPT > gpurun_out/diag_${TAG}_${c#mixed:}.log 2>&1; grep -A30 phases gpurun_out/diag_${TAG}_${c#mixed:}.log | grep "phases\|num g"; done
if [ -n "$BENCH" ]; then timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_$TAG.json 2>gpurun_out/bench_$TAG.err; python -c "
import json; d=json.load(open('gpurun_out/bench_$TAG.json')); print(d['value'], d['ms_per_step'], d['phase_ms_median'], d['roofline']['frac'], d['graph_replay']['ms_per_step'])"; fi
