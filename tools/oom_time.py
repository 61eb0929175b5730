"""Exhaustion timing: a bulk malloc that asks for more than the heap holds.
Prints per case the malloc / free time, the NULL count, and whether the heap
is pristine after free-all + drain.  Usage: python tools/oom_time.py
[size:n:heap_segments,...]"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
from helpers import diff_images, pristine_image  # noqa: E402

SEG = 1 << 24
cases = sys.argv[1] if len(sys.argv) > 1 else "8192:65536:1024,8192:262144:1024,8192:1048576:1024,16:16777216:8,1024:262144:4"
for case in cases.split(","):
    size, n, nseg = (int(x) for x in case.split(":"))
    G.gallatin_init(nseg * SEG)
    st = torch.full((n,), size, dtype=torch.int64, device="cuda")
    p = torch.empty_like(st)
    G.gallatin_malloc(st[:1 << 12], p[:1 << 12])       # load the kernels (lazy module loading)
    G.gallatin_free(p[:1 << 12])
    G.gallatin_drain()
    torch.cuda.synchronize()
    a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    t0 = time.time()
    a.record()
    G.gallatin_malloc(st, p)
    b.record()
    torch.cuda.synchronize()
    t_malloc = a.elapsed_time(b)
    nulls = int((p == 0).sum().item())
    b.record()                                        # the free alone (not the host-side count above)
    G.gallatin_free(p)
    c.record()
    torch.cuda.synchronize()
    G.gallatin_drain()
    img = G.gallatin_snapshot()
    msg = diff_images(img, pristine_image(nseg, int(img[4])))
    print(json.dumps({"size": size, "n": n, "heap_segments": nseg, "malloc_ms": round(t_malloc, 3),
                      "free_ms": round(b.elapsed_time(c), 3), "wall_s": round(time.time() - t0, 2), "nulls": nulls,
                      "granted": n - nulls, "pristine": not msg}), flush=True)
    del st, p
    G.gallatin_destroy()
