mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests/ -x -q -m gpu -k "nprod or rmat_s16 or rmat_s20 or webbase or config or range or mixed or paper_hash or duplicates" 2>&1 | tail -2
for c in rmat22 webbase cant; do timeout 300 python scripts/group_times.py $c | sed -n '1p'; done
