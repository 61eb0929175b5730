#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
bash tools/build_trace.sh 2>/dev/null
timeout 600 python tools/trace_phases.py 16,32,512,4096 > gpurun_out/trace_plan5.jsonl 2>&1; echo "trace rc=$?"
GALLATIN_CFG='{"launch_plan": 2}' timeout 600 python tools/trace_phases.py 32,512,4096 > gpurun_out/trace_noplan5.jsonl 2>&1; echo "trace rc=$?"
timeout 900 python -m pytest tests/test_gpu_alloc.py -x -q -k "full_size or variants or oom or thread_scaling or mixed or zero" > gpurun_out/pytest_plan.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_plan.log
timeout 900 python tools/knob_sweep.py --reps 7 --configs '[{}, {"launch_plan": 2}]' > gpurun_out/sweep_plan5.jsonl 2>&1; echo "sweep rc=$?"
timeout 600 python tools/mixed_probe.py > gpurun_out/mixed_plan5.jsonl 2>&1; echo "mixed rc=$?"
