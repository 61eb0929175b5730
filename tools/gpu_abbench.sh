#!/bin/bash
# same-box bench (--no-extras) of package builds given as arguments, two rounds
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for pk in "$@"; do [ -d "$pk/paper_conf_ppopp_mccoyp24_b200" ] || { echo "$pk: no package"; continue; }; GALLATIN_PKG_ROOT=$PWD/$pk timeout 600 python bench.py --no-extras --no-cpu 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$pk', round(d['value']/1e9,2), round(d['ms_per_step'],4), {k:(v['malloc_ms'],v['free_ms']) for k,v in d['per_size'].items()})"; done; done
