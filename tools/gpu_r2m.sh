#!/bin/bash
mkdir -p gpurun_out
for pdl in 1 0; do
GALLATIN_PDL=$pdl timeout 900 python bench.py --no-extras --no-cpu > gpurun_out/bench_pdl$pdl.json 2> gpurun_out/bench_pdl$pdl.err; echo "bench rc=$?"
GALLATIN_PDL=$pdl timeout 900 python bench.py --no-extras --no-cpu --no-graph > gpurun_out/bench_pdl${pdl}_ng.json 2> gpurun_out/bench_pdl${pdl}_ng.err; echo "bench rc=$?"
done
