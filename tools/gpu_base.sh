#!/bin/bash
# Baseline on a fresh box: build, smoke, short bench, refill phase traces per C2 cell, C3 breakdown.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py --no-extras --no-cpu > gpurun_out/bench_base.json 2> gpurun_out/bench_base.err; echo "bench rc=$?"
bash tools/build_trace.sh
timeout 600 python tools/trace_phases.py 16,32,64,128,256,512,1024,2048,4096 > gpurun_out/trace_base.jsonl 2>&1; echo "trace rc=$?"
timeout 600 python tools/mixed_probe.py > gpurun_out/mixed_base.jsonl 2>&1; echo "mixed rc=$?"
