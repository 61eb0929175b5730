"""Full-size C2 correctness check under a watchdog, printing per cell/rep."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
import workload_gen as wg  # noqa: E402
from helpers import SEG, diff_images, pristine_image  # noqa: E402

sizes = [int(x) for x in sys.argv[1].split(",")]
reps = int(sys.argv[2])
nseg = 1024
G.gallatin_init(nseg * SEG)
for size in sizes:
    n = min(1 << 24, (8 << 30) // size)
    st = torch.full((n,), size, dtype=torch.int64, device="cuda")
    for r in range(reps):
        t = time.time()
        p = G.gallatin_malloc(st)
        torch.cuda.synchronize()
        nulls = int((p == 0).sum())
        G.gallatin_stamp(p, st)
        bad = G.gallatin_verify(p, st)
        usum, ubad = G.gallatin_usable(p, st)
        srt = torch.sort(p).values
        dup = int((srt[1:] == srt[:-1]).sum())
        gap = int(((srt[1:] - srt[:-1]) < size).sum())
        t1 = time.time()
        G.gallatin_free(p)
        torch.cuda.synchronize()
        G.gallatin_drain()
        img = G.gallatin_snapshot()
        msg = diff_images(img, pristine_image(nseg, int(img[4])))
        print(f"size {size} rep {r}: nulls {nulls} stamp_bad {bad} usable_bad {ubad} usable {usum == n * max(16, size)} "
              f"dup {dup} gap {gap} pristine {'yes' if not msg else msg[:300]} t {t1 - t:.3f}s", flush=True)
print("done", flush=True)
