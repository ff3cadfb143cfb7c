#!/bin/bash
# One GPU iteration: build, parity tests, bench, launch list (+ optional ncu full capture).
#   bash scripts/gpu_cycle.sh TAG [tests|notests] [full|nofull] [pytest -k expr]
TAG=${1:-dev}; TESTS=${2:-tests}; FULL=${3:-nofull}; KEXPR=${4:-"not slow"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
if [ "$TESTS" = tests ]; then
  timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "$KEXPR" > gpurun_out/tests_$TAG.log 2>&1
  tail -5 gpurun_out/tests_$TAG.log
fi
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
cat gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
if [ "$FULL" = full ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_(num|sym)_smem" -c 8 \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$TAG.log 2>&1
  tail -2 gpurun_out/ncu_$TAG.log
fi
