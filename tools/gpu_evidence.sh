#!/bin/bash
# Full evidence pass on the current build: smoke, GPU tests, sanitizers, the
# bench line, the launch list of the bench command, ncu --set full captures
# (C2 cells, vEB, C3 mixed, graph) with the atomic counters.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
# compute-sanitizer is closed on this pool
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-extras --no-cpu > gpurun_out/ncu_bench.log 2>&1; echo "ncu launches rc=$?"
M=lts__t_requests_op_atom.sum,lts__t_requests_op_red.sum,lts__t_requests_op_atom.sum.per_second,l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_atom.sum,smsp__inst_executed_op_global_atom.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,lts__t_sectors_srcunit_tex_op_read.sum
timeout 1200 ncu --set full --metrics $M --clock-control none --import-source on -k regex:k_bulk -s 4 -c 4 \
    -o gpurun_out/prof_c2 -f python tools/prof_extra.py c2 > gpurun_out/ncu_c2.log 2>&1; echo "ncu c2 rc=$?"
timeout 900 ncu --set full --metrics $M --clock-control none --import-source on -k regex:"k_update|k_query" -s 3 -c 3 \
    -o gpurun_out/prof_veb -f python tools/prof_extra.py veb > gpurun_out/ncu_veb.log 2>&1; echo "ncu veb rc=$?"
timeout 900 ncu --set full --metrics $M --clock-control none --import-source on -k regex:"k_bulk|k_big" -s 3 -c 3 \
    -o gpurun_out/prof_mixed -f python tools/prof_extra.py mixed > gpurun_out/ncu_mixed.log 2>&1; echo "ncu mixed rc=$?"
timeout 1500 ncu --set full --metrics $M --clock-control none --import-source on -k regex:"k_(count|grow|copy|scatter|hash|list|shrink|expand|edge|delete|free_all)" -c 60 \
    -o gpurun_out/prof_graph -f python tools/prof_extra.py graph > gpurun_out/ncu_graph.log 2>&1; echo "ncu graph rc=$?"
