#!/bin/bash
set -x
mkdir -p gpurun_out
bash tools/build_trace.sh 2>/dev/null
timeout 600 python tools/trace_phases.py 16,32,512,4096 > gpurun_out/trace_plan3.jsonl 2>&1; echo "trace rc=$?"
GALLATIN_CFG='{"launch_plan": 2}' timeout 600 python tools/trace_phases.py 16,32,512,4096 > gpurun_out/trace_noplan3.jsonl 2>&1; echo "trace rc=$?"
