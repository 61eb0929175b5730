#!/bin/bash
mkdir -p gpurun_out
timeout 600 python tools/trace_mixed.py > gpurun_out/trace_mixed.jsonl 2>&1
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
bash tools/gpu_ab_head.sh
