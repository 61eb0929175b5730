#!/bin/bash
set -x
mkdir -p gpurun_out
./tools/smid_probe > gpurun_out/smid.txt 2>&1
bash tools/build_trace.sh 2>/dev/null
timeout 600 python tools/trace_phases.py 16,32,64,128,512,1024,4096 > gpurun_out/trace_plan.jsonl 2>&1; echo "trace rc=$?"
GALLATIN_CFG='{"launch_plan": 2}' timeout 600 python tools/trace_phases.py 32,4096 > gpurun_out/trace_noplan.jsonl 2>&1; echo "trace rc=$?"
