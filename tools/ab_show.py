"""Summarize gpurun_out/ab_head.jsonl / ab_mixed.jsonl (tools/gpu_ab_head.sh)."""
import json, os, statistics
R = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "gpurun_out")
rows = {}
for l in open(os.path.join(R, "ab_head.jsonl")):
    d = json.loads(l); r = d["row"]
    k = d["pkg"] + ("" if not r["cfg"] else json.dumps(r["cfg"]))
    rows.setdefault(r["size"], {}).setdefault(k, []).append((r.get("malloc_ms"), r.get("free_ms")))
tot = {}
for sz, v in rows.items():
    print(sz, {k: (round(statistics.median(x[0] for x in xs), 4), round(statistics.median(x[1] for x in xs), 4)) for k, xs in v.items()})
    for k, xs in v.items():
        tot[k] = tot.get(k, 0) + statistics.median(x[0] for x in xs) + statistics.median(x[1] for x in xs)
print("sum malloc+free ms:", {k: round(t, 4) for k, t in tot.items()})
p = os.path.join(R, "ab_mixed.jsonl")
if os.path.exists(p):
    for l in open(p):
        d = json.loads(l); print(d["pkg"], d["row"])
