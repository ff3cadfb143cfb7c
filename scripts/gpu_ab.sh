#!/bin/bash
# A/B of per-group serial times: default build vs variants/NAME.so on CONFIGS
#   bash scripts/gpu_ab.sh "rmat22 webbase" NAME...
CFGS=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in $CFGS; do
  timeout 300 python scripts/group_times.py $c
  for v in "$@"; do SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c; done
done
