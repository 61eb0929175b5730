#!/bin/bash
set -x
mkdir -p gpurun_out; rm -f gpurun_out/ab_*.jsonl gpurun_out/veb_ab.jsonl
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
for r in 1 2; do for p in ab_claim ab_comb .; do GALLATIN_PKG_ROOT=$p timeout 300 python tools/veb_probe.py >> gpurun_out/veb_ab.jsonl; done; done
bash tools/gpu_ab.sh ab_r1 ab_comb . > gpurun_out/ab.log 2>&1; echo "ab rc=$?"
timeout 900 python tools/mixed_probe.py > gpurun_out/mixed_probe.jsonl 2>&1; echo "mixed rc=$?"
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/bench.err
