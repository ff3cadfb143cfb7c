#!/bin/bash
# Key metrics of every kernel in an ncu report matching a regex: bash scripts/ncu_metrics.sh REP [REGEX]
ncu -i "$1" --page raw --csv -k regex:"${2:-.}" --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,l1tex__t_sector_hit_rate.pct,l1tex__throughput.avg.pct_of_peak_sustained_active,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,launch__registers_per_thread,launch__grid_size,launch__block_size 2>/dev/null | python3 -c "
import csv,sys
r=list(csv.reader(sys.stdin))
h=r[0]
for row in r[2:]:
    print(row[h.index('Kernel Name')][:80])
    for i,x in enumerate(h):
        if '__' in x: print('   %-60s %s' % (x,row[i]))
"
