mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
for c in rmat20 webbase rmat18 mixed:economics mixed:circuit; do for o in "rank_l1_pct_sym=150" "rank_l1_pct_sym=100" "rank_l1_pct_sym=50"; do
  timeout 300 python scripts/group_times.py $c $o | sed -n "1,2p"
done; done
