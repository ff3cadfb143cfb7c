mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
GT_DETAIL=1 timeout 300 python scripts/group_times.py rmat22 > gpurun_out/gt22.log 2>&1
GT_DETAIL=1 timeout 300 python scripts/group_times.py webbase > gpurun_out/gtweb.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-per-config > gpurun_out/bench0.json 2>gpurun_out/bench0.err
cat gpurun_out/gt22.log gpurun_out/gtweb.log; head -c 400 gpurun_out/bench0.json
