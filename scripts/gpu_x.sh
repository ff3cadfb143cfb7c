mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
export GT_DTYPE=f64
for c in rmat22 rmat20; do
  timeout 300 python scripts/group_times.py $c | sed -n '1p;3p'
  for v in e64d e64e e64f e64g; do echo -n "$v "; SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c | sed -n '1p;3p'; done
done
