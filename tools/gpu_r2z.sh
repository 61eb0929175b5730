#!/bin/bash
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log
bash tools/gpu_abbench.sh . ab_head
timeout 300 python tools/mixed_probe.py | head -2
GALLATIN_PKG_ROOT=$PWD/ab_head timeout 300 python tools/mixed_probe.py | head -2
