#!/bin/bash
timeout 300 python tools/trace_mixed.py > gpurun_out/trace_mixed.jsonl 2>&1
timeout 1800 python -m pytest tests/test_gpu_alloc.py -x -q > gpurun_out/pytest_alloc.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_alloc.log
for r in 1 2 3; do
timeout 300 python tools/mixed_probe.py 2>/dev/null | head -1
GALLATIN_PKG_ROOT=$PWD/ab_head timeout 300 python tools/mixed_probe.py 2>/dev/null | head -1
done
