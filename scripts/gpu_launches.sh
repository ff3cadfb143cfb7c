#!/bin/bash
# ncu launch list (gpu__time_duration per kernel) of one bench step per config:
#   bash scripts/gpu_launches.sh TAG config...
TAG=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for c in "$@"; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_${c#mixed:}.csv \
    python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --streams 0 > /dev/null 2>&1
done
