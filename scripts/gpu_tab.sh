#!/bin/bash
# build, selected GPU tests (-k EXPR), A/B group times (default vs variants) on CONFIGS
#   bash scripts/gpu_tab.sh "expr" "rmat22 webbase" NAME...
K=$1; CFGS=$2; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/ -x -q -m gpu -k "$K" > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for c in $CFGS; do
  timeout 300 python scripts/group_times.py $c
  for v in "$@"; do SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c; done
done
