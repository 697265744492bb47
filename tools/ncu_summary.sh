#!/bin/bash
# summarise an ncu --set full capture into the per-kernel metric table kept under profiles/
ncu -i "$1" --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct,launch__grid_size,launch__block_size 2>/dev/null | python3 -c "
import csv,sys
r=list(csv.reader(sys.stdin)); h=r[0]
keep=['Kernel Name','launch__grid_size','launch__block_size','gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed','sm__throughput.avg.pct_of_peak_sustained_elapsed','sm__warps_active.avg.pct_of_peak_sustained_active','launch__registers_per_thread','sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed','lts__t_sector_hit_rate.pct']
idx=[h.index(k) for k in keep]
w=csv.writer(sys.stdout)
for x in r: w.writerow([x[i] for i in idx])
"
