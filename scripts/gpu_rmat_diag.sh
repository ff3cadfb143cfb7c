# R-MAT s20 numeric diagnosis: option sweep + full ncu of the numeric group kernels
set -x
python -c "import __graft_entry__ as g; g.build()"
for o in "" "--opt range_hash=0" "--opt long_row=-1" "--opt flat=1" "--opt flat=0" "--opt lanes=4" "--opt lanes=16" "--opt cluster=0"; do
  timeout 300 python scripts/diag.py rmat20 --opt streams=0 $o > gpurun_out/diag_rmat20_$(echo $o | tr -c 'a-z0-9' _).log 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_num_(smem|cluster)" -c 12 -o gpurun_out/prof_rmat20 python scripts/diag.py rmat20 --reps 1 --opt streams=0 > gpurun_out/ncu_rmat20.log 2>&1
tail -3 gpurun_out/ncu_rmat20.log
