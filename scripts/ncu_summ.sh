#!/bin/bash
# summarize an ncu report: key metrics (raw page)
for f in "$@"; do echo "== $f"; ncu -i $f --page raw --csv 2>/dev/null | python -c "
import csv,sys
rows=list(csv.reader(sys.stdin)); h=rows[0]
want=['Kernel Name','gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','lts__t_sector_hit_rate.pct','sm__warps_active.avg.pct_of_peak_sustained_active','smsp__inst_executed.sum','dram__throughput.avg.pct_of_peak_sustained_elapsed','lts__throughput.avg.pct_of_peak_sustained_elapsed','l1tex__t_sector_hit_rate.pct','smsp__issue_active.avg.pct_of_peak_sustained_active','launch__registers_per_thread','launch__occupancy_limit_registers','sm__cycles_elapsed.avg.per_second']
for r in rows[2:]:
  for w in want:
    if w in h: i=h.index(w); print('  ',w, r[i], rows[1][i])
"; done
