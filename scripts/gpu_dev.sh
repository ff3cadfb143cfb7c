#!/bin/bash
# Dev cycle: build, selected GPU tests (-k expr), diag on configs ($DIAG), bench line.
#   DIAG="cant webbase" bash scripts/gpu_dev.sh TAG "pytest -k expr"
TAG=${1:-dev}; KEXPR=${2:-"not slow"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "$KEXPR" > gpurun_out/tests_$TAG.log 2>&1; tail -15 gpurun_out/tests_$TAG.log
for c in $DIAG; do timeout 300 python scripts/diag.py $c --opt streams=0 > gpurun_out/diag_${TAG}_$c.log 2>&1; cat gpurun_out/diag_${TAG}_$c.log | head -30; done
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_$TAG.json 2>gpurun_out/bench_$TAG.err; tail -2 gpurun_out/bench_$TAG.err
python -c "
import json; d=json.load(open('gpurun_out/bench_$TAG.json')); print(d['value'], d['ms_per_step'], d['phase_ms_median'], d['roofline']['frac'], d['roofline']['kernel'], d['graph_replay']['ms_per_step'])"
