#!/bin/bash
# ncu --set full of kernels matching REGEX while running diag on CONFIG:
#   bash scripts/gpu_ncu_cfg.sh TAG CONFIG REGEX COUNT [diag opts...]
TAG=$1; CFG=$2; RX=$3; CNT=${4:-6}; shift 4
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$RX" -c $CNT \
  -o gpurun_out/prof_$TAG python scripts/diag.py $CFG --reps 1 --opt streams=0 "$@" > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
