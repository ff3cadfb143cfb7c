mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in $CFGS; do for r in 1 2 3; do
  timeout 300 python scripts/group_times.py $c | sed -n '1p'
  for v in $VARS; do echo -n "$v "; SPGEMM_LIB=variants/$v.so timeout 300 python scripts/group_times.py $c | sed -n '1p'; done
done; done
for v in "" $VARS; do if [ -n "$v" ]; then export SPGEMM_LIB=variants/$v.so; fi; echo "bench $v"; timeout 300 python bench.py --config webbase --no-cpu-baseline --no-per-config --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])"; done
