"""Fast-path cost of the bulk kernels: a C2 cell launched twice without a
reset in between (the second malloc finds its slots' runs still holding
slices, so it takes no refills when the run outlasts one launch), next to a
plain 8 B-read / 8 B-write copy of the same element count."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402


def t(fn, reps=5):
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


cfg = json.loads(sys.argv[1]) if len(sys.argv) > 1 else {}
G.gallatin_init(16 << 30, **cfg)
for sz in [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "16,64,512").split(",")]:
    n = min(1 << 24, (8 << 30) // sz) // 2
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
    p = torch.empty_like(st)
    first, second = [], []
    for rep in range(5):
        G.gallatin_reset(); torch.cuda.synchronize()
        first.append(t(lambda: G.gallatin_malloc(st, p), 1)); G.gallatin_free(p)
        second.append(t(lambda: G.gallatin_malloc(st, p), 1)); G.gallatin_free(p)
    buf = torch.empty_like(st)
    copy = t(lambda: buf.copy_(st))
    print(json.dumps({"size": sz, "n": n, "first_ms": round(min(first), 4), "second_ms": round(min(second), 4),
                      "copy_ms": round(copy, 4), "stats_run_init": G.gallatin_stats()["run_init"]}), flush=True)
G.gallatin_destroy()
