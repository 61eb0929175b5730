"""Graph workload (bench.run_graph, BASELINE configs[4]) under allocator knobs:
  python tools/graph_probe.py '[{}, {"run_grow": 1}]'
prints G edges/s per phase for each knob set."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402


class Args:
    scale = 1


orig = G.gallatin_init
for cfg in json.loads(sys.argv[1] if len(sys.argv) > 1 else "[{}]"):
    G.gallatin_init = lambda heap, _c=cfg, **kw: orig(heap, **{**_c, **kw})
    G.gallatin_init(bench.HEAP_C2)
    for rep in range(2):
        r = bench.run_graph(Args, G, torch, torch.cuda.current_stream())
        print(json.dumps({"cfg": cfg, "rep": rep, "failed": r["failed_mallocs"],
                          **{k: round(v["edges_per_s"] / 1e9, 3) for k, v in r["phases"].items()}}), flush=True)
    G.gallatin_destroy()
