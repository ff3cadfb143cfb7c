#!/bin/bash
# Round-2 evidence (final): build, DRAM traffic per group (before the bench reads it), all GPU
# tests, smoke, bench (config 5 headline, fp64, reference arm), config-1 latency, ncu launch list
# of one serialised R-MAT s22 multiply, ncu --set full of the top kernels.
#   bash scripts/gpu_round2c.sh TAG
TAG=${1:-r02c}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python scripts/traffic.py rmat22 f32 --top 6 > gpurun_out/traffic_$TAG.log 2>&1
cp profiles/traffic_r02.json gpurun_out/traffic_r02.json
timeout 3000 python -m pytest tests/ -q -m gpu --durations=10 > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; head -c 300 gpurun_out/bench_$TAG.json; echo
timeout 900 python bench.py --dtype f64 --no-cpu-baseline --no-per-config --no-e2e > gpurun_out/bench_${TAG}_f64.json 2>&1
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_${TAG}_ref.json 2>&1
timeout 300 python scripts/latency2.py > gpurun_out/latency_$TAG.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --print-units base \
  --log-file gpurun_out/launches_${TAG}_rmat22.csv python scripts/rmat_once.py 22 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_num_esc --launch-skip 4 -c 2 \
  -o gpurun_out/prof_${TAG}_esc python scripts/rmat_once.py 22 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_num_rankacc|k_num_rankbig" -c 3 \
  -o gpurun_out/prof_${TAG}_rank python scripts/rmat_once.py 22 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sym_smem|k_sym_rankcnt" --launch-skip 5 -c 3 \
  -o gpurun_out/prof_${TAG}_sym python scripts/rmat_once.py 22 > /dev/null 2>&1
ls gpurun_out | grep $TAG
