#!/bin/bash
# ncu --set full of the range kernels on one config: bash scripts/gpu_ncu_range.sh TAG CONFIG
TAG=${1:-rng}; CFG=${2:-cant}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_(num|sym)_range" -c 2 \
  -o gpurun_out/prof_$TAG python scripts/diag.py $CFG --reps 1 --opt streams=0 > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
