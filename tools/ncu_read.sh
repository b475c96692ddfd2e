#!/bin/bash
# usage: ncu_read.sh report.ncu-rep
ncu -i "$1" --page raw --csv 2>/dev/null | python3 -c "
import csv,sys
rows=list(csv.reader(sys.stdin))
h=rows[0]; units=rows[1]
for r in rows[2:]:
    d=dict(zip(h,r))
    print('KERNEL', d.get('Kernel Name','')[:100])
    keys=['gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','smsp__issue_active.avg.pct_of_peak_sustained_active','sm__warps_active.avg.pct_of_peak_sustained_active','smsp__inst_executed.sum','launch__registers_per_thread','l1tex__t_sector_hit_rate.pct','lts__t_sector_hit_rate.pct','gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed','sm__cycles_elapsed.avg.per_second']
    for k in keys:
        if k in d: print('  ',k,d[k])
    st=[(float(d[k].replace(',','')),k) for k in h if 'smsp__average_warps_issue_stalled_' in k and k.endswith('_per_issue_active.ratio') and d[k] not in ('','n/a')]
    st.sort(reverse=True)
    for v,k in st[:10]: print('   stall',k.replace('smsp__average_warps_issue_stalled_','').replace('_per_issue_active.ratio',''),round(v,3))
"
