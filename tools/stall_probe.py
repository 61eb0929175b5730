"""Repeat reset + malloc + free of C2 cells many times; report slow launches
(> 1 ms) and NULL results (a liveness / exhaustion-path probe)."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])
import torch  # noqa: E402
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "1024,2048,4096").split(",")]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 100
G.gallatin_init(16 << 30)
for sz in sizes:
    n = min(1 << 24, (8 << 30) // sz)
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda"); p = torch.empty_like(st)
    ms, nulls = [], 0
    for r in range(reps):
        G.gallatin_reset()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); G.gallatin_malloc(st, p); b.record(); torch.cuda.synchronize()
        ms.append(a.elapsed_time(b)); nulls += int((p == 0).sum().item())
        G.gallatin_free(p)
    ms.sort()
    print(json.dumps({"pkg": os.environ.get("GALLATIN_PKG_ROOT", "new")[-8:], "size": sz, "p50": round(ms[len(ms) // 2], 4),
                      "max": round(ms[-1], 3), "slow_gt_1ms": sum(x > 1 for x in ms), "nulls": nulls}), flush=True)
G.gallatin_destroy()
