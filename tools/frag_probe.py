"""E7 fragmentation (range of one bulk call of 2^20 requests / bytes
requested) under the default knobs and the paper's one-block policy, per size.
Honors GALLATIN_PKG_ROOT (A/B against another build)."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if os.environ.get("GALLATIN_PKG_ROOT"):
    sys.path.insert(0, os.environ["GALLATIN_PKG_ROOT"])
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
from paper_conf_ppopp_mccoyp24_b200 import experiments as X  # noqa: E402

for name, knobs in (("default", {}), ("paper_policy", dict(run_max=1, run_init=1, format_ahead=2, prefetch=2, prefill=2))):
    G.gallatin_init(16 << 30, **knobs)
    out = {}
    for sz in [16 << i for i in range(9)]:
        G.gallatin_reset()
        r = X.fragmentation(sz, 1 << 20)
        out[sz] = round(r["range_over_requested"], 2)
        G.gallatin_free(r["ptrs"])
    G.gallatin_destroy()
    print(json.dumps({"pkg": os.environ.get("GALLATIN_PKG_ROOT", "."), "knobs": name, "range_over_requested": out}),
          flush=True)
