#!/bin/bash
# same-session A/B/C of package builds given as arguments (dirs with the package), cold sweep
mkdir -p gpurun_out; rm -f gpurun_out/abc.jsonl
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for pk in "$@"; do
  GALLATIN_PKG_ROOT=$PWD/$pk timeout 600 python tools/knob_sweep.py --reps 7 | sed "s|^|{\"pkg\": \"$pk\", \"round\": $r, \"row\": |; s|$|}|" >> gpurun_out/abc.jsonl
done; done
