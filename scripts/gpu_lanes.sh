#!/bin/bash
# Lanes-per-B-row ablation (PAPER.md:124 threads-per-row sweep, B200 analogue).
python -c "import __graft_entry__ as g; g.build()" || exit 1
for cfg in cant webbase; do for L in 1 2 4 8 16 32; do
  echo -n "$cfg lanes=$L "; timeout 300 python bench.py --config $cfg --lanes $L --steps 5 --no-e2e --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), 'GFLOPS', {k: round(v,3) for k,v in d['phase_ms_median'].items()})"
done; done
