"""Small workloads for compute-sanitizer (memcheck / racecheck / synccheck).

    compute-sanitizer --tool memcheck python tools/sanitize.py [veb|alloc|replay|graph|all]

Each part runs the hot path through the C-ABI on a small input and checks its
result (so a sanitizer run is also a correctness run):
  veb    -- configs[0] vEB: insert / successor / predecessor / member / delete
            on u = 2^20 vs O1 (the oracle), bit-exact image;
  alloc  -- configs[0] allocator (64 MB heap, 2^16 x 16 B) on the small-batch
            kernels, and 2^20 mixed 16 B-4 KB (+ 1-64 MB) requests on a 4 GB
            heap on the CTA-aggregated
            kernels (shared-memory ranking: the racecheck target), stamp +
            verify, free-all + drain -> pristine;
  replay -- serialized replay of a mixed op list vs O2 (offsets + image);
  graph  -- the streaming-graph workload at scale 10 (device-API malloc/free
            from user kernels) vs O3.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_mccoyp24_b200 as G  # noqa: E402
import workload_gen as wg  # noqa: E402
from helpers import SEG, diff_images, pristine_image  # noqa: E402


def dev(a, dt=np.uint64):
    a = np.ascontiguousarray(a, dtype=dt)
    return torch.from_numpy(a.view(np.int64) if a.dtype.itemsize == 8 else a).cuda()


def part_veb():
    w = wg.veb_workload(20, 1 << 16)
    g, o = G.Veb(20), oracle.Veb(20)
    assert np.array_equal(g.insert(dev(w["insert"])).cpu().numpy(), o.batch(oracle.OV_INSERT, w["insert"]).astype(np.uint8))
    for q in (w["succ1"], w["succ2"]):
        assert np.array_equal(g.successor(dev(q)).cpu().numpy().view(np.uint64), o.batch(oracle.OV_SUCC, q))
        assert np.array_equal(g.predecessor(dev(q)).cpu().numpy().view(np.uint64), o.batch(oracle.OV_PRED, q))
        assert np.array_equal(g.member(dev(q)).cpu().numpy(), o.batch(oracle.OV_MEMBER, q).astype(np.uint8))
    assert np.array_equal(g.delete(dev(w["delete"])).cpu().numpy(), o.batch(oracle.OV_DELETE, w["delete"]).astype(np.uint8))
    assert np.array_equal(g.snapshot(), o.image())
    g.close()
    print("veb ok")


def _round(nseg, sizes):
    d = dev(sizes)
    p = G.gallatin_malloc(d)
    G.gallatin_stamp(p, d)
    assert G.gallatin_verify(p, d) == 0
    assert int((p == 0).sum()) == 0
    G.gallatin_free(p)
    G.gallatin_drain()
    img = G.gallatin_snapshot()
    assert not diff_images(img, pristine_image(nseg, int(img[4])))


def part_alloc():
    G.gallatin_init(4 * SEG)
    try:
        _round(4, wg.single_sizes(16, 1 << 16))
    finally:
        G.gallatin_destroy()
    G.gallatin_init(256 * SEG)
    try:
        _round(256, wg.mixed_sizes(1 << 20, p_large=2.0 ** -14))
        _round(256, wg.single_sizes(64, 1 << 20))
    finally:
        G.gallatin_destroy()
    print("alloc ok")


def part_replay():
    nseg = 6
    kinds, args, keys = wg.replay_ops(1500, 3, p_free=0.45, p_drain=0.003, nkeys=64)
    G.gallatin_init(nseg * SEG, slot_base=16, slot_min=2, run_max=16, run_bytes=32 << 20, format_ahead=1,
                    prefetch=1, run_init=1, oom_record=2)
    try:
        out = G.gallatin_replay(dev(kinds, np.uint8), dev(args), dev(keys)).cpu().numpy().view(np.uint64)
        o2 = oracle.model(nseg, **G.oracle_params())
        assert np.array_equal(out, o2.replay(kinds, args, keys))
        assert not diff_images(G.gallatin_snapshot(), o2.image())
    finally:
        G.gallatin_destroy()
    print("replay ok")


def part_graph():
    from oracle.graph import GraphOracle
    G.gallatin_init(64 * SEG)
    try:
        w = wg.graph_workload(10, 1 << 14, device="cuda")
        V = w["V"]
        g = G.Graph(V)
        o = GraphOracle(V)
        s0, d0 = w["init"]
        g.insert(s0, d0)
        o.insert(s0.cpu().numpy().astype(np.int64), d0.cpu().numpy().astype(np.int64))
        for s, d in w["delete"][:2]:
            g.delete(s, d)
            o.delete(s.cpu().numpy().astype(np.int64), d.cpu().numpy().astype(np.int64))
        g.expand(w["expand"][:64])
        o.expand(w["expand"][:64].cpu().numpy().astype(np.int64))
        size, cap, _ = g.export()
        assert np.array_equal(size.cpu().numpy().astype(np.int64), o.size)
        assert np.array_equal(cap.cpu().numpy().astype(np.int64), o.cap)
        g.destroy()
    finally:
        G.gallatin_destroy()
    print("graph ok")


if __name__ == "__main__":
    parts = sys.argv[1:] or ["all"]
    if parts == ["all"]:
        parts = ["veb", "alloc", "replay", "graph"]
    for p in parts:
        globals()["part_" + p]()
    torch.cuda.synchronize()
    print("sanitize workload ok:", ",".join(parts))
