"""Time one C2 cell's reset+malloc+free repeated R times as ONE CUDA graph
without event nodes (total / R), and the malloc alone the same way."""
import json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])
import torch  # noqa: E402
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16,512,4096").split(",")]
R = 20
G.gallatin_init(16 << 30)
for sz in sizes:
    n = min(1 << 24, (8 << 30) // sz)
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda"); p = torch.empty_like(st)
    res = {}
    for name, body in (("reset+malloc+free", lambda: (G.gallatin_reset(), G.gallatin_malloc(st, p), G.gallatin_free(p))),
                       ("reset+free(NULL)", lambda: (G.gallatin_reset(), p.zero_(), G.gallatin_free(p)))):
        g = torch.cuda.CUDAGraph(); cap = torch.cuda.Stream(); cap.wait_stream(torch.cuda.current_stream())
        with torch.cuda.graph(g, stream=cap):
            for _ in range(R):
                body()
        g.replay(); torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ts = []
        for _ in range(3):
            a.record(); g.replay(); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b) / R)
        res[name] = round(sorted(ts)[1], 4)
        del g
    print(json.dumps({"pkg": os.environ.get("GALLATIN_PKG_ROOT", ".")[-6:], "size": sz, **res}), flush=True)
G.gallatin_destroy()
