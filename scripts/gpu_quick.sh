# quick cycle: build, gpu tests (not slow), diag on the given configs, bench line
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu -k "not slow" > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
for c in $DIAG; do timeout 300 python scripts/diag.py $c --opt streams=0 > gpurun_out/diag_$c.log 2>&1; grep phases gpurun_out/diag_$c.log; done
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench.json 2>gpurun_out/bench.err; tail -2 gpurun_out/bench.err
python -c "
import json; d=json.load(open('gpurun_out/bench.json')); print(d['value'], d['ms_per_step'], d['phase_ms_median'], d['roofline']['frac'], d['roofline']['kernel'], d['graph_replay']['ms_per_step'], d['e2e']['ms_per_step'])"
