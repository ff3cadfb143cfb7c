mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/ -x -q -m gpu -k "esc or rmat_s20 or rmat_s16" 2>&1 | tail -2
for c in rmat22 rmat20; do for o in esc_cdf=0 esc_cdf=1; do timeout 300 python scripts/group_times.py $c $o | sed -n '1p;3p'; done; done
