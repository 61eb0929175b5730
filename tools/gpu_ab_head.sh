#!/bin/bash
# same-session A/B: this tree vs ab_head/ (tools/ab_build.sh HEAD head), C2 cold sweep + C3 breakdown
mkdir -p gpurun_out; rm -f gpurun_out/ab_head.jsonl gpurun_out/ab_mixed.jsonl
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do
  timeout 600 python tools/knob_sweep.py --reps 7 ${AB_CFG:+--configs "$AB_CFG"} | sed "s|^|{\"pkg\": \"new\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_head.jsonl
  GALLATIN_PKG_ROOT=$PWD/ab_head timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"head\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/ab_head.jsonl
done
timeout 300 python tools/mixed_probe.py | sed 's|^|{"pkg": "new", "row": |; s|$|}|' >> gpurun_out/ab_mixed.jsonl
GALLATIN_PKG_ROOT=$PWD/ab_head timeout 300 python tools/mixed_probe.py | sed 's|^|{"pkg": "head", "row": |; s|$|}|' >> gpurun_out/ab_mixed.jsonl
