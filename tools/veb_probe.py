"""vEB bulk insert/delete timing (A/B helper; honors GALLATIN_PKG_ROOT):
median per-launch time over rounds of (clear, insert, delete) for the C1
batch (2^16 keys, u = 2^20), 4M random keys at u = 2^24, and the same 4M
keys sorted (warp-combinable)."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
import workload_gen as wg  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64).view(np.int64)).cuda()


def run(k, keys, dkeys, rounds=12):
    v = G.Veb(k)
    ins, dele = [], []
    for r in range(rounds):
        v.clear()
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record()
        v.insert(keys, want_out=False)
        b.record()
        v.delete(dkeys, want_out=False)
        c.record()
        torch.cuda.synchronize()
        if r >= 2:
            ins.append(a.elapsed_time(b))
            dele.append(b.elapsed_time(c))
    v.close()
    n = keys.numel()
    return {"insert_us": round(statistics.median(ins) * 1e3, 2), "delete_us": round(statistics.median(dele) * 1e3, 2),
            "insert_Gops": round(n / statistics.median(ins) / 1e6, 2), "delete_Gops": round(dkeys.numel() / statistics.median(dele) / 1e6, 2)}


w = wg.veb_workload(20, 1 << 16)
out = {"pkg": os.environ.get("GALLATIN_PKG_ROOT", "."), "c1": run(20, dev(w["insert"]), dev(w["delete"]))}
big = wg.distinct_below(wg.cell_seed(1, 424), 1 << 22, 1 << 24)
out["u24_random"] = run(24, dev(big), dev(big))
out["u24_sorted"] = run(24, dev(np.sort(big)), dev(np.sort(big)))
print(json.dumps(out), flush=True)
