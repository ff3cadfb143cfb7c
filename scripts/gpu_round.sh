#!/bin/bash
# Round evidence: build, GPU parity tests, smoke, bench (default config + f64 + reference arm),
# per-group diag of the other configs, ncu launch list of the bench command, one ncu --set full
# capture of the hot group kernels of one bench step.
#   bash scripts/gpu_round.sh TAG [KREGEX]
TAG=${1:-r01}
KRE=${2:-'k_(num|sym)_(smem|range|range_bits|cluster|rankacc|rankcnt)'}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1500 python -m pytest tests/ -q -m gpu > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; head -c 400 gpurun_out/bench_$TAG.json; echo
timeout 600 python bench.py --dtype f64 --no-cpu-baseline > gpurun_out/bench_${TAG}_f64.json 2>&1
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_${TAG}_ref.json 2>&1
for c in webbase mixed:protein mixed:qcd mixed:epidemiology rmat20; do timeout 300 python scripts/diag.py $c > gpurun_out/diag_${TAG}_${c#mixed:}.log 2>&1; grep phases gpurun_out/diag_${TAG}_${c#mixed:}.log; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$KRE" -c 6 \
  -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
tail -1 gpurun_out/ncu_$TAG.log
