mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python scripts/traffic.py rmat22 f32 --top 6 > gpurun_out/traffic_x.log 2>&1; tail -8 gpurun_out/traffic_x.log
timeout 900 python scripts/traffic.py rmat22 f64 --top 3 >> gpurun_out/traffic_x.log 2>&1; tail -3 gpurun_out/traffic_x.log
cp profiles/traffic_r02.json gpurun_out/traffic_r02.json
timeout 600 python bench.py --no-cpu-baseline --no-per-config --no-e2e --steps 3 > gpurun_out/bx.json 2>gpurun_out/bx.err
python -c "import json; d=json.load(open('gpurun_out/bx.json')); print(d['value'], json.dumps(d['roofline'].get('issue')))"
