"""Refill latency trace (debug build with -DGALLATIN_TRACE): per C2 cell,
count, latency percentiles and the time span of refills in one malloc kernel."""
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ["GALLATIN_LIB"] = os.path.join(ROOT, "tools", "libgallatin_trace.so")
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402

cfg = json.loads(sys.argv[1]) if len(sys.argv) > 1 else {}
sizes = [int(x) for x in (sys.argv[2] if len(sys.argv) > 2 else "16,128,512,4096").split(",")]
L = G.lib()
L.gallatin_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
G.gallatin_init(16 << 30, **cfg)
cap = 1 << 20
buf = torch.zeros(3 * cap, dtype=torch.int64, device="cuda")
for sz in sizes:
    n = min(1 << 24, (8 << 30) // sz)
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
    p = torch.empty_like(st)
    for rep in range(3):
        G.gallatin_reset()
        torch.cuda.synchronize()
        L.gallatin_debug_trace(buf.data_ptr(), cap, None)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); G.gallatin_malloc(st, p); e1.record()
        cnt = ctypes.c_uint64()
        L.gallatin_debug_trace(None, 0, ctypes.byref(cnt))
        G.gallatin_free(p)
    k = min(cnt.value, cap)
    t = buf[: 3 * k].view(k, 3).cpu().numpy().view(np.uint64)
    lat = (t[:, 1] - t[:, 0]).astype(np.float64) / 1e3
    want = (t[:, 2] >> np.uint64(12)) & np.uint64(0xFFF)
    got = t[:, 2] & np.uint64(0xFFF)
    span = (t[:, 1].max() - t[:, 0].min()) / 1e3
    print(json.dumps({"size": sz, "kernel_ms": round(e0.elapsed_time(e1), 4), "refills": int(k),
                      "lat_us_p50": round(float(np.percentile(lat, 50)), 2), "p90": round(float(np.percentile(lat, 90)), 2),
                      "p99": round(float(np.percentile(lat, 99)), 2), "max": round(float(lat.max()), 2),
                      "sum_lat_us": round(float(lat.sum()), 1), "span_us": round(float(span), 1),
                      "want_hist": {int(w): int(c) for w, c in zip(*np.unique(want, return_counts=True))},
                      "short_runs": int((got < want).sum())}), flush=True)
