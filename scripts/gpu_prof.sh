# full ncu of the numeric + symbolic kernels for one config: CFG=webbase KREGEX='k_num_(smem|cluster)' TAG=x
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"${KREGEX:-k_num_(smem|cluster)}" -c ${COUNT:-16} -o gpurun_out/prof_${TAG:-$CFG} python scripts/diag.py $CFG --reps 1 --opt streams=0 $OPTS > gpurun_out/ncu_${TAG:-$CFG}.log 2>&1
tail -2 gpurun_out/ncu_${TAG:-$CFG}.log
