"""Small driver for ncu --set full captures: one reset + malloc + free per
requested C2 cell (bench's launch configuration), after one warm-up round."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])  # another build of the package
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402

sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16,128").split(",")]
G.gallatin_init(16 << 30)
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
