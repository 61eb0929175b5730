"""Cold (reset before the call: every slot refills at the launch's start)
vs warm (no reset: slots keep the runs of the previous round) bulk malloc on
C2 cells; median of 7.  Shows what the launch-start refill burst costs."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])  # A/B against another build of the package
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402

G.gallatin_init(16 << 30)
for sz in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16,128,512,4096").split(",")]:
    n = min(1 << 24, (8 << 30) // sz) // 2            # half the cell: warm rounds keep runs of the last one
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
    p = torch.empty_like(st)
    res = {}
    for mode in ("cold", "warm", "cold", "warm"):
        ts = []
        for it in range(9):
            if mode == "cold":
                G.gallatin_reset()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            G.gallatin_malloc(st, p)
            b.record()
            G.gallatin_free(p)
            torch.cuda.synchronize()
            if it >= 2:
                ts.append(a.elapsed_time(b))
        res.setdefault(mode, []).append(round(statistics.median(ts), 4))
    print(json.dumps({"pkg": os.environ.get("GALLATIN_PKG_ROOT", "."), "size": sz, "n": n, **res}), flush=True)
G.gallatin_destroy()
