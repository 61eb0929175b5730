"""Driver for ncu --set full captures of the non-headline kernels (VERDICT r1
"missing" 3): one warm-up of each, then the launches ncu captures.

  veb   -- configs[0] tree (u = 2^20): k_insert of the 2^16 keys, k_query<kSucc,4>
           over 2^24 queries, k_delete of the 2^16 delete keys
  mixed -- configs[2]: 2^22 mixed requests on the 64 GiB heap, malloc + free
  graph -- configs[4] phases at R-MAT scale 20 (2^24 edges): bulk insert, delete,
           one expansion round, single-edge inserts/deletes (device-API calls)
  c2    -- configs[1] cells 16 B and 4 KB (the bulk malloc/free kernels)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
import workload_gen as wg  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64).view(np.int64)).cuda()


def veb():
    w = wg.veb_workload(20, 1 << 16)
    q = dev(wg.uniform_below(wg.cell_seed(1, 7), 1 << 24, 1 << 20))
    res = torch.empty_like(q)
    keys, dk = dev(w["insert"]), dev(w["delete"])
    for _ in range(2):                      # warm-up round, then the captured one
        v = G.Veb(20)
        v.insert(keys, want_out=False)
        v.successor(q, res)
        v.delete(dk, want_out=False)
        torch.cuda.synchronize()
        v.close()


def mixed():
    G.gallatin_init(64 << 30)
    sizes = dev(wg.mixed_sizes(1 << 22))
    p = torch.empty_like(sizes)
    for _ in range(2):
        G.gallatin_reset()
        G.gallatin_malloc(sizes, p)
        G.gallatin_free(p)
        torch.cuda.synchronize()
    G.gallatin_destroy()


def graph():
    G.gallatin_init(16 << 30)
    w = wg.graph_workload(20, 1 << 24, device="cuda", n_expand=1 << 14)
    g = G.Graph(w["V"])
    s0, d0 = w["init"]
    g.insert(s0, d0)
    s1, d1 = w["insert"][0]
    g.insert(s1, d1)
    s2, d2 = w["delete"][0]
    g.delete(s2, d2)
    g.expand(w["expand"])
    es, ed = s1[:1 << 18].contiguous(), d1[:1 << 18].contiguous()
    g.insert_edges(es, ed)
    g.delete_edges(es, ed)
    torch.cuda.synchronize()
    g.destroy()
    G.gallatin_destroy()


def c2():
    G.gallatin_init(16 << 30)
    for warm in (True, False):
        for sz in (16, 4096):
            n = min(1 << 24, (8 << 30) // sz)
            st = torch.full((n,), sz, dtype=torch.int64, device="cuda")
            p = torch.empty_like(st)
            G.gallatin_reset()
            G.gallatin_malloc(st, p)
            G.gallatin_free(p)
            torch.cuda.synchronize()
    G.gallatin_destroy()


if __name__ == "__main__":
    for part in (sys.argv[1:] or ["veb", "mixed", "graph", "c2"]):
        globals()[part]()
    print("ok")
