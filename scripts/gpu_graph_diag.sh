#!/bin/bash
# Graph-shaped configs: serial per-group timings, cuSPARSE side-by-side, ncu of the heaviest
# numeric/symbolic CTA-per-row groups of R-MAT s20.   bash scripts/gpu_graph_diag.sh TAG
TAG=${1:-g1}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" || exit 1
for c in rmat20 webbase; do timeout 300 python scripts/diag.py $c --opt streams=0 > gpurun_out/diag_${TAG}_${c}_serial.log 2>&1; grep phases gpurun_out/diag_${TAG}_${c}_serial.log; done
timeout 900 python scripts/cusparse_compare.py cant webbase mixed:protein mixed:economics rmat18 --reps 3 > gpurun_out/cusparse_${TAG}.jsonl 2> gpurun_out/cusparse_${TAG}.err; cut -c1-400 gpurun_out/cusparse_${TAG}.jsonl; tail -3 gpurun_out/cusparse_${TAG}.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_num_smem --launch-skip 6 -c 2 \
  -o gpurun_out/prof_${TAG}_num python scripts/diag.py rmat20 --reps 1 --opt streams=0 > gpurun_out/ncu_${TAG}_num.log 2>&1; tail -1 gpurun_out/ncu_${TAG}_num.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sym_smem --launch-skip 6 -c 1 \
  -o gpurun_out/prof_${TAG}_sym python scripts/diag.py rmat20 --reps 1 --opt streams=0 > gpurun_out/ncu_${TAG}_sym.log 2>&1; tail -1 gpurun_out/ncu_${TAG}_sym.log
