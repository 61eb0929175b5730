#!/bin/bash
bash tools/gpu_abbench.sh . ab_nowin ab_free1
for pk in . ab_nowin; do for r in 1 2; do GALLATIN_PKG_ROOT=$PWD/$pk timeout 600 python bench.py --no-cpu 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$pk warm', [round(v['warm_over_cold_malloc'],2) for v in d['grid']['warm_vs_cold'].values()], 'mixed', round(d['mixed']['malloc_ms'],4))"; done; done
