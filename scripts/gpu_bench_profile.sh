set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python bench.py > gpurun_out/bench_r01.json 2> gpurun_out/bench_r01.err
tail -3 gpurun_out/bench_r01.err
cat gpurun_out/bench_r01.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.json 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_(num|sym)_smem" -c 8 -o gpurun_out/prof_r01 python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1
tail -5 gpurun_out/ncu_full.log
ls -la gpurun_out
