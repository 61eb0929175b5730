#!/bin/bash
mkdir -p gpurun_out
python -c "import oracle; oracle.build()" > /dev/null 2>&1
timeout 1800 python -m pytest tests/test_gpu_alloc.py -x -q > gpurun_out/pytest_alloc.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_alloc.log
for r in 1 2; do for pk in . ab_head; do GALLATIN_PKG_ROOT=$PWD/$pk timeout 900 python bench.py --no-cpu 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$pk', round(d['value']/1e9,2), round(d['ms_per_step'],4), 'mixed', round(d['mixed']['malloc_ms'],4), 'warm', [round(v['warm_over_cold_malloc'],2) for v in d['grid']['warm_vs_cold'].values()])"; done; done
