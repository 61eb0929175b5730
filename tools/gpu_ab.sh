#!/bin/bash
# Same-box A/B of package builds (ab_<name>/ from tools/ab_build.sh, "." = the
# working tree): cold C2 sweep (knob_sweep), warm vs cold rounds, E7
# fragmentation; two interleaved rounds.  Usage: tools/gpu_ab.sh ab_r1 ab_x .
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for round in 1 2; do
  for pkg in "$@"; do
    GALLATIN_PKG_ROOT=$pkg timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"$pkg\", \"round\": $round, \"row\": |; s|$|}|" >> gpurun_out/ab_cold.jsonl
    GALLATIN_PKG_ROOT=$pkg timeout 600 python tools/warm_cold.py 16,32,64,512,1024,2048,4096 >> gpurun_out/ab_warm.jsonl
  done
done
for pkg in "$@"; do GALLATIN_PKG_ROOT=$pkg timeout 600 python tools/frag_probe.py >> gpurun_out/ab_frag.jsonl; done
echo ab done
