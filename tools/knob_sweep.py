"""Time malloc/free kernels of the C2 sweep under different allocator knobs
(slot_base, slot_min, theta, fence_free).  Diagnostic tool, prints one JSON
line per configuration."""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402

SIZES = [16 << i for i in range(9)]


def run(cfg, sizes, reps=5, scale=1):
    G.gallatin_init(16 << 30, **cfg)
    out = {}
    s = torch.cuda.current_stream()
    for sz in sizes:
        n = min(1 << 24, (8 << 30) // sz) // scale
        st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
        p = torch.empty_like(st)
        mm, fm = [], []
        for r in range(reps + 2):
            G.gallatin_reset()
            a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            a.record(s)
            G.gallatin_malloc(st, p)
            b.record(s)
            G.gallatin_free(p)
            c.record(s)
            torch.cuda.synchronize()
            if r >= 2:
                mm.append(a.elapsed_time(b))
                fm.append(b.elapsed_time(c))
        nulls = int((p == 0).sum().item())
        out[sz] = (round(statistics.median(mm), 4), round(statistics.median(fm), 4), nulls)
    G.gallatin_destroy()
    return out


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default='[{}]')
    ap.add_argument("--sizes", default=",".join(map(str, SIZES)))
    ap.add_argument("--scale", type=int, default=1)
    a = ap.parse_args()
    sizes = [int(x) for x in a.sizes.split(",")]
    for cfg in json.loads(a.configs):
        print(json.dumps({"cfg": cfg, "ms(malloc,free,nulls)": run(cfg, sizes, scale=a.scale)}), flush=True)
