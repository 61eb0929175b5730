"""Refill phase trace (debug build with -DGALLATIN_TRACE, tools/libgallatin_trace.so):
per C2 cell, latency percentiles per traced phase (tag 0 whole refill_slot,
1 take_segments claim, 2 take_segments publish, 3 get_run), the time from the
first CTA's start to the last CTA's start, and the refill time span."""
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

sizes = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "16,512,4096").split(",")]
L = G.lib()
L.gallatin_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
G.gallatin_init(16 << 30, **(json.loads(os.environ.get('GALLATIN_CFG', '{}'))))
cap = 1 << 20
buf = torch.zeros(3 * cap, dtype=torch.int64, device="cuda")
for sz in sizes:
    n = min(1 << 24, (8 << 30) // sz)
    st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
    p = torch.empty_like(st)
    warm = os.environ.get("TRACE_WARM") == "1"
    for rep in range(3):
        if not (warm and rep > 0):
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
    tag = (t[:, 2] >> np.uint64(60)).astype(int)
    t0 = t[:, 0].astype(np.int64)
    base = t0[tag == 7].min() if (tag == 7).any() else t0.min()
    out = {"size": sz, "kernel_ms": round(e0.elapsed_time(e1), 4)}
    if (tag == 8).any():
        out["plan_segments"] = int(t[tag == 8, 2][0] & np.uint64(0xFFFFFFFF))
    if (tag == 7).sum() >= 2:
        m7 = tag == 7
        out["cta_start_span_us"] = round((t0[m7].max() - t0[m7].min()) / 1e3, 1)
        end7 = (t[m7, 1].astype(np.int64) - base) / 1e3
        dur7 = (t[m7, 1] - t[m7, 0]).astype(np.float64) / 1e3
        bid = (t[m7, 2] & np.uint64(0xFFFFFFFF)).astype(np.int64)
        out["cta_end_us_p50_p90_p99_max"] = [round(float(np.percentile(end7, q)), 1) for q in (50, 90, 99, 100)]
        out["cta_dur_us_p50_p90_p99_max"] = [round(float(np.percentile(dur7, q)), 2) for q in (50, 90, 99, 100)]
        slow = np.argsort(-dur7)[:5]
        out["slowest_ctas"] = [[int(bid[i]), round(float((t0[m7][i] - base) / 1e3), 1), round(float(dur7[i]), 1)] for i in slow]
    for g_ in (0, 1, 2, 3, 8, 10, 11):
        m = tag == g_
        if not m.any():
            continue
        lat = (t[m, 1] - t[m, 0]).astype(np.float64) / 1e3
        st_ = (t0[m] - base) / 1e3
        out[f"tag{g_}"] = {"n": int(m.sum()), "p50": round(float(np.percentile(lat, 50)), 2),
                           "p90": round(float(np.percentile(lat, 90)), 2), "max": round(float(lat.max()), 2),
                           "first_start_us": round(float(st_.min()), 1), "last_end_us": round(float(((t[m, 1].astype(np.int64) - base) / 1e3).max()), 1)}
    m0 = tag == 0
    if m0.any():
        info = t[m0, 2]
        want = ((info >> np.uint64(12)) & np.uint64(0xFFF)).astype(int)
        got = (info & np.uint64(0xFFF)).astype(int)
        slot = ((info >> np.uint64(32)) & np.uint64(0xFFFFFFF)).astype(int)
        st0 = (t0[m0] - base) / 1e3
        pairs, cnts = np.unique(np.stack([want, got], 1), axis=0, return_counts=True)
        out["refill_want_got"] = {f"{a}->{b}": int(c) for (a, b), c in zip(pairs, cnts)}
        out["refills_per_slot_max"] = int(np.bincount(slot).max())
        out["late_refills"] = int((st0 > 20).sum())
    m1 = tag == 1
    if m1.any():
        att = ((t[m1, 2] >> np.uint64(32)) & np.uint64(0xFFFF)).astype(int)
        out["claim_attempts"] = {"mean": round(float(att.mean()), 2), "max": int(att.max()),
                                 "hist": np.bincount(att, minlength=1)[:12].tolist()}
    print(json.dumps(out), flush=True)
