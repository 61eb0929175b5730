#!/bin/bash
mkdir -p gpurun_out; rm -f gpurun_out/warmabc.jsonl
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for pk in "$@"; do
  GALLATIN_PKG_ROOT=$PWD/$pk timeout 600 python tools/warm_cold.py 128,512,1024,2048,4096 >> gpurun_out/warmabc.jsonl 2>&1
done
