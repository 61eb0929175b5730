#!/bin/bash
mkdir -p gpurun_out; rm -f gpurun_out/ab_head.jsonl
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do
  timeout 600 python tools/knob_sweep.py --reps 7 --configs '[{"launch_plan": 2}, {}]' | sed "s|^|{\"pkg\": \"new\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_head.jsonl
  GALLATIN_PKG_ROOT=$PWD/ab_head timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"head\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_head.jsonl
done
