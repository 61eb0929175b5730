"""Time malloc/free kernels of the C2 sweep under different allocator knobs
(slot_base, slot_min, run_max, run_bytes, format_ahead, fence_free,
bulk_items).  Diagnostic tool: every (config, size) cell runs in its own
subprocess under a watchdog so a hang is reported instead of stalling the
sweep.  Prints one JSON line per cell."""
import argparse
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])  # A/B against another build of the package
SIZES = [16 << i for i in range(9)]


def one(cfg, sz, reps, scale, heap):
    import torch
    import paper_conf_ppopp_mccoyp24_b200 as G
    G.gallatin_init(heap, **cfg)
    s = torch.cuda.current_stream()
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
    G.gallatin_drain()
    st_ = G.gallatin_stats()
    G.gallatin_destroy()
    m, f = statistics.median(mm), statistics.median(fm)
    return {"malloc_ms": round(m, 4), "free_ms": round(f, 4), "malloc_Gops": round(n / m / 1e6, 2),
            "free_Gops": round(n / f / 1e6, 2), "nulls": nulls, "n": n, "free_segs_after_drain": st_["free_segments"]}


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default='[{}]')
    ap.add_argument("--sizes", default=",".join(map(str, SIZES)))
    ap.add_argument("--scale", type=int, default=1)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--heap", type=int, default=16 << 30)
    ap.add_argument("--timeout", type=int, default=60)
    ap.add_argument("--one", default=None)
    a = ap.parse_args()
    if a.one:
        cfg, sz = json.loads(a.one)
        print(json.dumps(one(cfg, sz, a.reps, a.scale, a.heap)))
        sys.exit(0)
    for cfg in json.loads(a.configs):
        for sz in [int(x) for x in a.sizes.split(",")]:
            cmd = [sys.executable, __file__, "--one", json.dumps([cfg, sz]), "--reps", str(a.reps),
                   "--scale", str(a.scale), "--heap", str(a.heap)]
            try:
                out = subprocess.run(cmd, capture_output=True, text=True, timeout=a.timeout)
                res = out.stdout.strip().splitlines()[-1] if out.returncode == 0 and out.stdout.strip() else \
                    json.dumps({"error": (out.stderr or "")[-400:]})
            except subprocess.TimeoutExpired:
                res = json.dumps({"error": f"TIMEOUT {a.timeout}s"})
            print(json.dumps({"cfg": cfg, "size": sz, **json.loads(res)}), flush=True)
