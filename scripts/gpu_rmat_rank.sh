#!/bin/bash
# Config 5 (R-MAT s22 fp32, one GPU): per-group times with the rank kernels on / off and the
# level-1 bitmap ordering on / off, to place the rank kernels by level-1 width vs group bound.
#   bash scripts/gpu_rmat_rank.sh TAG [SCALE] [extra --opt ...]
TAG=${1:-rk}; SC=${2:-22}; shift 2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for v in "" "--opt rank_acc=0" "--opt rank_acc=0 --opt bitmap_rank=0" "--opt rank_l1_pct=100" "--opt rank_l1_pct=400" "--opt rank_l1_pct=1600" "$@"; do
  echo "== $v"; timeout 600 python scripts/rmat_run.py --scale $SC --reps 3 $v 2>&1 | grep -v "^rmat"
done > gpurun_out/rmat_rank_$TAG.log
cat gpurun_out/rmat_rank_$TAG.log
