"""C3 mixed workload broken down: which requests make the malloc slow."""
import sys, os, json, statistics
sys.path.insert(0, os.getcwd())
if os.environ.get('GALLATIN_PKG_ROOT'):
    sys.path.insert(0, os.environ['GALLATIN_PKG_ROOT'])
import numpy as np, torch
import paper_conf_ppopp_mccoyp24_b200 as G
import workload_gen as wg
G.gallatin_init(64 << 30, **json.loads(os.environ.get('GALLATIN_CFG', '{}')))
for name, kw in [("mixed", {}), ("no_large", dict(p_large=0.0)), ("large_only", None), ("segment_only", 1),
                 ("block_only", 2)]:
    if kw is None or isinstance(kw, int):
        s = wg.mixed_sizes(1 << 22)
        s = s[s > 4096]
        if kw == 1:
            s = s[s >= (16 << 20)]
        elif kw == 2:
            s = s[s < (16 << 20)]
    else:
        s = wg.mixed_sizes(1 << 22, **kw)
    st = torch.from_numpy(s.astype(np.int64)).cuda(); p = torch.empty_like(st)
    mm, fm = [], []
    for it in range(7):
        G.gallatin_reset()
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record(); G.gallatin_malloc(st, p); b.record(); G.gallatin_free(p); c.record(); torch.cuda.synchronize()
        if it >= 2: mm.append(a.elapsed_time(b)); fm.append(b.elapsed_time(c))
    print(json.dumps({"case": name, "n": len(s), "large": int((s >= (16 << 20)).sum()), "block": int(((s > 4096) & (s < (16 << 20))).sum()),
                      "malloc_ms": round(statistics.median(mm), 4), "free_ms": round(statistics.median(fm), 4)}), flush=True)
