#!/bin/bash
# cold C2 sweep A/B over package builds + E7 fragmentation of each
set -x
mkdir -p gpurun_out; rm -f gpurun_out/ab_*.jsonl
python -c "import __graft_entry__ as g; g.build()"
for r in 1 2; do for p in "$@"; do
  GALLATIN_PKG_ROOT=$p timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"$p\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_cold.jsonl
done; done
for p in "$@"; do GALLATIN_PKG_ROOT=$p timeout 600 python tools/frag_probe.py >> gpurun_out/ab_frag.jsonl; done
timeout 600 python tools/warm_cold.py 16,32,64,512,1024,2048,4096 > gpurun_out/ab_warm.jsonl
