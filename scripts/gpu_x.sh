mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in rmat22; do
  timeout 300 python scripts/group_times.py $c | sed -n '3p'
  for v in sk16 sk24 sk48 sk64; do echo -n "$v "; SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c | sed -n '3p'; done
done
