#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/trace_phases.py 512,4096 > gpurun_out/trace_plan4.jsonl 2>&1; echo "trace rc=$?"
