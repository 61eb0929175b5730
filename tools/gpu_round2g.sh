#!/bin/bash
set -x
mkdir -p gpurun_out; rm -f gpurun_out/ab_*.jsonl
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
for r in 1 2; do
  GALLATIN_PKG_ROOT=ab_r1 timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"ab_r1\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_cold.jsonl
  timeout 900 python tools/knob_sweep.py --reps 7 --configs '[{}, {"prefill": 2}]' | sed "s|^|{\"pkg\": \".\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_cold.jsonl
done
timeout 600 python tools/warm_cold.py 16,32,64,512,1024,2048,4096 > gpurun_out/ab_warm.jsonl
timeout 600 python tools/frag_probe.py > gpurun_out/ab_frag.jsonl
timeout 900 python tools/mixed_probe.py > gpurun_out/mixed_probe.jsonl 2>&1; echo "mixed rc=$?"
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/bench.err
