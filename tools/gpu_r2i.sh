#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --no-extras --no-cpu > gpurun_out/bench_r2i.json 2> gpurun_out/bench_r2i.err; echo "bench rc=$?"
timeout 600 python tools/mixed_probe.py > gpurun_out/mixed_r2i.jsonl 2>&1
GALLATIN_CFG='{"launch_plan": 1}' timeout 600 python tools/mixed_probe.py > gpurun_out/mixed_r2i_plan.jsonl 2>&1
