#!/bin/bash
# ncu --set full (source) of the top ESC numeric launch and the top symbolic hash launch at R-MAT s22
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_num_esc --launch-skip 4 -c 1 \
  -o gpurun_out/prof_${TAG}_esc python scripts/rmat_once.py 22 > gpurun_out/ncu_${TAG}_esc.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sym_smem --launch-skip 5 -c 2 \
  -o gpurun_out/prof_${TAG}_sym python scripts/rmat_once.py 22 > gpurun_out/ncu_${TAG}_sym.log 2>&1
tail -2 gpurun_out/ncu_${TAG}_*.log
