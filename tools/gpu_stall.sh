#!/bin/bash
mkdir -p gpurun_out; rm -f gpurun_out/stall.jsonl
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python tools/stall_probe.py 512,1024,2048,4096 100 >> gpurun_out/stall.jsonl 2>&1
GALLATIN_PKG_ROOT=$PWD/ab_head timeout 600 python tools/stall_probe.py 512,1024,2048,4096 100 >> gpurun_out/stall.jsonl 2>&1
GALLATIN_PKG_ROOT=$PWD/ab_r2start timeout 600 python tools/stall_probe.py 512,1024,2048,4096 100 >> gpurun_out/stall.jsonl 2>&1
