"""ncu driver: one warm-up round, then one reset + malloc + free per C2 cell,
under the allocator knobs given as JSON (argv[2]).  Usage:
python tools/prof_knobs.py 16,512 '{"pipeline": 3}'"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402

sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16").split(",")]
knobs = json.loads(sys.argv[2]) if len(sys.argv) > 2 else {}
G.gallatin_init(16 << 30, **knobs)
for warm in (True, False):
    for sz in sizes:
        n = min(1 << 24, (8 << 30) // sz)
        st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
        p = torch.empty_like(st)
        G.gallatin_reset()
        G.gallatin_malloc(st, p)
        G.gallatin_free(p)
        torch.cuda.synchronize()
G.gallatin_destroy()
print("ok")
