"""Near-OOM probe: where is the memory when the utilization loop (E8) sees its
first NULL?  Prints free segments, blocks available in rings, undrawn slot
blocks, and how many more allocations later batches still get."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
from paper_conf_ppopp_mccoyp24_b200 import experiments as X  # noqa: E402
from helpers import image_sections  # noqa: E402

for size in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16,32,64").split(",")]:
    for trial in range(3):
        G.gallatin_init(2 << 30)
        r = X.utilization(size)
        c = max(0, (size - 1).bit_length() - 4)
        d = image_sections(G.gallatin_snapshot())
        st = G.gallatin_stats()
        free_segs = st["free_segments"]
        sw = d["segword"]
        tree = (sw >> np.uint64(32)).astype(np.int64)
        avail = (sw & np.uint64(0xFFFFFFFF)).astype(np.int64)
        avail = np.where(avail >= 1 << 31, avail - (1 << 32), avail)
        ring_blocks = int(avail[tree == c].sum())
        off = sum(st["nslot"][:c])
        slots = d["slots"][off:off + st["nslot"][c]]
        issued = (slots >> np.uint64(32)).astype(np.int64)
        run = ((slots >> np.uint64(22)) & np.uint64(0x3FF)).astype(np.int64)
        undrawn = int(np.maximum(0, run * 4096 - issued).sum())
        more = 0
        for _ in range(5):
            p = G.gallatin_malloc(torch.full((100_000,), size, dtype=torch.int64, device="cuda"))
            more += int(torch.count_nonzero(p).item())
        print(json.dumps({"size": size, "trial": trial, "successes": r["successes"], "util": round(r["utilization"], 4),
                          "free_segments": free_segs, "ring_blocks_avail": ring_blocks,
                          "slot_undrawn_slices": undrawn, "slots_nonempty": int((run > 0).sum()),
                          "more_after": more, "tree_segments": st["tree_segments"]}), flush=True)
        del r
        G.gallatin_destroy()
