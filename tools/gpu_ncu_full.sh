#!/bin/bash
# ncu --set full capture of the bulk kernels on the C2 cells given as $1
mkdir -p gpurun_out
CELLS=${1:-16,512}; SKIP=$(( $(echo $CELLS | tr , "\n" | wc -l) * 2 ))
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_bulk -s $SKIP -c $SKIP \
  -o gpurun_out/prof -f python tools/prof_cells.py $CELLS > gpurun_out/ncu_full.log 2>&1
echo "ncu rc=$?"; tail -5 gpurun_out/ncu_full.log
