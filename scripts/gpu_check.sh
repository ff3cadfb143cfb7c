#!/bin/bash
# Build, full GPU parity suite, then config 5 (R-MAT s22) and the graph configs' per-group times.
#   bash scripts/gpu_check.sh TAG
TAG=${1:-chk}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1500 python -m pytest tests/ -q -m gpu -x > gpurun_out/tests_$TAG.log 2>&1; tail -3 gpurun_out/tests_$TAG.log
timeout 600 python scripts/rmat_run.py --scale 22 --reps 3 > gpurun_out/rmat22_$TAG.log 2>&1; grep "^rep" gpurun_out/rmat22_$TAG.log
for c in rmat20 webbase; do timeout 300 python scripts/diag.py $c > gpurun_out/diag_${TAG}_$c.log 2>&1; grep phases gpurun_out/diag_${TAG}_$c.log; done
for c in rmat20 webbase; do timeout 300 python bench.py --config $c --steps 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_${TAG}_$c.json 2>&1; head -c 200 gpurun_out/bench_${TAG}_$c.json; echo; done
