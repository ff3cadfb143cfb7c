#!/bin/bash
# key metrics of every kernel in an ncu report:  bash scripts/ncu_brief.sh REPORT
ncu -i "$1" --page raw --csv --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,l1tex__t_sector_hit_rate.pct,lts__t_sector_hit_rate.pct,dram__bytes_read.sum,dram__bytes_write.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,launch__grid_size,launch__block_size,launch__occupancy_limit_shared_mem,launch__occupancy_limit_registers,launch__registers_per_thread,dram__throughput.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,l1tex__throughput.avg.pct_of_peak_sustained_active 2>/dev/null | python3 -c "
import csv,sys
r=list(csv.reader(sys.stdin))
for row in r[2:]:
    d=dict(zip(r[0],row)); u=dict(zip(r[0],r[1]))
    print(d['Kernel Name'][:90])
    print('  '+'  '.join(f'{h.split(\"__\")[1][:40]}={v} {u[h]}' for h,v in d.items() if '__' in h))
"
