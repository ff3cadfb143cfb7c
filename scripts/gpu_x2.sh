mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/ -x -q -m gpu -k "big_rows or cluster or overflow" 2>&1 | tail -2
for c in rmat22 webbase rmat20; do for o in rank_big_max=3 rank_big_max=2 rank_big_max=1; do timeout 300 python scripts/group_times.py $c $o | sed -n '1p;3p'; done; done
