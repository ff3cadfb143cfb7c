mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in rmat22 rmat20 webbase; do for o in "rank_gout=0" "rank_gout=1"; do timeout 300 python scripts/group_times.py $c $o | head -3 | sed -n '1p;3p'; done; done
