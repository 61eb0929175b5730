#!/bin/bash
mkdir -p gpurun_out
for pk in . ab_m16; do
GALLATIN_PKG_ROOT=$PWD/$pk timeout 600 ncu --clock-control none --csv --metrics gpu__time_duration.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__cycles_active.avg,dram__throughput.avg.pct_of_peak_sustained_elapsed -k regex:k_bulk_malloc -s 1 -c 1 python tools/prof_cells.py 16 > gpurun_out/occ_$pk.log 2>&1
echo "== $pk"; grep -E "duration|warps_active|inst_executed|cycles_active|dram__throughput" gpurun_out/occ_$pk.log | awk -F'","' '{print $(NF-2), $NF}'
done
