"""C3 mixed launch traced (debug build, tools/libgallatin_trace.so): latency of
the whole-block and segment requests (tag 12) by size, refills (tag 0), and the
CTA timeline (tag 7)."""
import ctypes, json, os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ["GALLATIN_LIB"] = os.path.join(ROOT, "tools", "libgallatin_trace.so")
sys.path.insert(0, ROOT)
import numpy as np, torch  # noqa: E402
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
import workload_gen as wg  # noqa: E402
L = G.lib()
L.gallatin_debug_trace.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
G.gallatin_init(64 << 30)
cap = 1 << 20
buf = torch.zeros(3 * cap, dtype=torch.int64, device="cuda")
for case in ("mixed", "no_large"):
    s = wg.mixed_sizes(1 << 22, **({} if case == "mixed" else {"p_large": 0.0}))
    st = torch.from_numpy(s.astype(np.int64)).cuda(); p = torch.empty_like(st)
    for rep in range(3):
        G.gallatin_reset(); torch.cuda.synchronize()
        L.gallatin_debug_trace(buf.data_ptr(), cap, None)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); G.gallatin_malloc(st, p); e1.record()
        cnt = ctypes.c_uint64(); L.gallatin_debug_trace(None, 0, ctypes.byref(cnt))
        G.gallatin_free(p)
    k = min(cnt.value, cap)
    t = buf[: 3 * k].view(k, 3).cpu().numpy().view(np.uint64)
    tag = (t[:, 2] >> np.uint64(60)).astype(int)
    t0 = t[:, 0].astype(np.int64); base = t0[tag == 7].min()
    out = {"case": case, "kernel_ms": round(e0.elapsed_time(e1), 4)}
    m7 = tag == 7
    end7 = (t[m7, 1].astype(np.int64) - base) / 1e3; dur7 = (t[m7, 1] - t[m7, 0]).astype(float) / 1e3
    out["cta_start_span_us"] = round((t0[m7].max() - base) / 1e3, 1)
    out["cta_end_p50_p90_p99_max"] = [round(float(np.percentile(end7, q)), 1) for q in (50, 90, 99, 100)]
    out["cta_dur_p50_p90_p99_max"] = [round(float(np.percentile(dur7, q)), 2) for q in (50, 90, 99, 100)]
    m12 = tag == 12
    if m12.any():
        mb = (t[m12, 2] & np.uint64(0xFFFFFFFF)).astype(int)
        lat = (t[m12, 1] - t[m12, 0]).astype(float) / 1e3
        st12 = (t0[m12] - base) / 1e3
        for sz in sorted(set(mb.tolist())):
            m = mb == sz
            out[f"big_{sz}MB"] = {"n": int(m.sum()), "lat_p50": round(float(np.percentile(lat[m], 50)), 1),
                                  "p90": round(float(np.percentile(lat[m], 90)), 1), "max": round(float(lat[m].max()), 1),
                                  "last_end": round(float((st12[m] + lat[m]).max()), 1)}
    for g_ in (13, 15):
        m = tag == g_
        for j in np.nonzero(m)[0]:
            out.setdefault(f"tag{g_}", []).append([round(float((t0[j] - base) / 1e3), 1), round(float((t[j, 1] - t[j, 0]) / 1e3), 1),
                                                    int(t[j, 2] & np.uint64((1 << 60) - 1))])
    for g_ in (0, 1, 3):
        m = tag == g_
        if m.any():
            lat = (t[m, 1] - t[m, 0]).astype(float) / 1e3
            out[f"tag{g_}"] = {"n": int(m.sum()), "p50": round(float(np.percentile(lat, 50)), 1), "max": round(float(lat.max()), 1),
                               "last_end": round(float(((t[m, 1].astype(np.int64) - base) / 1e3).max()), 1)}
    print(json.dumps(out), flush=True)
