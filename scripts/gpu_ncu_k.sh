#!/bin/bash
# ncu --set full of launches of kernel REGEX (after SKIP matches) while running diag on CONFIG (serial groups)
#   bash scripts/gpu_ncu_k.sh TAG CONFIG REGEX SKIP COUNT [diag opts...]
TAG=$1; CFG=$2; RX=$3; SKIP=$4; CNT=$5; shift 5
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$RX" --launch-skip $SKIP -c $CNT \
  -o gpurun_out/prof_$TAG python scripts/diag.py $CFG --reps 1 --opt streams=0 "$@" > gpurun_out/ncu_$TAG.log 2>&1
tail -2 gpurun_out/ncu_$TAG.log
