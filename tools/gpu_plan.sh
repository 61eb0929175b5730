#!/bin/bash
# launch plan: correctness subset + A/B sweep + C3 breakdown
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_alloc.py -x -q -k "full_size or variants or oom or thread_scaling or mixed" > gpurun_out/pytest_plan.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_plan.log
timeout 900 python tools/knob_sweep.py --reps 7 --configs '[{}, {"launch_plan": 2}]' > gpurun_out/sweep_plan.jsonl 2>&1; echo "sweep rc=$?"
timeout 600 python tools/mixed_probe.py > gpurun_out/mixed_plan.jsonl 2>&1; echo "mixed rc=$?"
