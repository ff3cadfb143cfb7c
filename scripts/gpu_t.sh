#!/bin/bash
# build, selected GPU tests (-k EXPR), group times on CONFIGS
#   bash scripts/gpu_t.sh "pytest -k expr" "rmat22 webbase"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/ -x -q -m gpu -k "$1" > gpurun_out/t.log 2>&1; tail -5 gpurun_out/t.log
for c in $2; do timeout 300 python scripts/group_times.py $c; done
