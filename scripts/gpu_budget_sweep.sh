python -c "import __graft_entry__ as g; g.build()" >/dev/null
for b in 98304 131072 163840 196608; do for c in cant mixed:protein; do for dt in f32 f64; do
  SPGEMM_RANGE_BUDGET=$b timeout 300 python bench.py --config $c --dtype $dt --no-cpu-baseline --no-e2e --steps 5 > /tmp/b.json 2>/dev/null
  python -c "import json; d=json.load(open('/tmp/b.json')); print('$b $c $dt', round(d['value'],1), round(d['phase_ms_median']['numeric_ms'],3))"
done; done; done
