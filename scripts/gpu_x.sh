mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in $CFGS; do
  timeout 300 python scripts/group_times.py $c | sed -n "$LINES"
  for v in $VARS; do echo -n "$v "; SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c | sed -n "$LINES"; done
done
