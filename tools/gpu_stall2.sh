#!/bin/bash
mkdir -p gpurun_out; rm -f gpurun_out/stall.jsonl
timeout 900 python tools/stall_probe.py 32,128,512,1024,2048,4096 150 >> gpurun_out/stall.jsonl 2>&1
for pdl in 1 0; do
GALLATIN_PDL=$pdl timeout 900 python bench.py --no-extras --no-cpu > gpurun_out/bench_pdl$pdl.json 2> gpurun_out/bench_pdl$pdl.err; echo "bench rc=$?"
GALLATIN_PDL=$pdl timeout 900 python bench.py --no-extras --no-cpu --no-graph > gpurun_out/bench_pdl${pdl}_ng.json 2> gpurun_out/bench_pdl${pdl}_ng.err; echo "bench rc=$?"
done
