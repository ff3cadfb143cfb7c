mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/ -x -q -m gpu -k "group9 or big_rows" 2>&1 | tail -2
for o in "rank_mid=1" "rank_mid=2" "rank_mid=0"; do timeout 300 python scripts/group_times.py rmat22 $o | head -3 | tail -1; done
for o in "rank_mid=1" "rank_mid=2"; do timeout 300 python scripts/group_times.py rmat20 $o | head -3 | tail -1; done
