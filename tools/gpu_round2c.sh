set -x
rm -f gpurun_out/ab_*.jsonl
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -5 gpurun_out/pytest_gpu.log
bash tools/gpu_ab.sh ab_r1 ab_claim . > gpurun_out/ab.log 2>&1; echo "ab rc=$?"
timeout 900 python tools/mixed_probe.py > gpurun_out/mixed_probe.jsonl 2>&1; echo "mixed rc=$?"
timeout 1200 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"; tail -3 gpurun_out/bench.err
