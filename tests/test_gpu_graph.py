"""GPU parity of the streaming-graph workload (BASELINE configs[4]) built on
the device-side allocator, against O3 (oracle/graph.py):
per-vertex sizes and capacities and the sorted adjacency multiset after every
phase, the bytes the lists hold (read from the allocator's memory table), and a
pristine heap after teardown."""
import numpy as np
import pytest
import torch

import workload_gen as wg
from helpers import SEG, class_size, diff_images, pristine_image
from oracle.graph import GraphOracle

pytestmark = pytest.mark.gpu


def _np(t):
    return t.cpu().numpy().astype(np.int64)


def _check(G, g, o, V, tag):
    size, cap, ptr = g.export()
    torch.cuda.synchronize()
    s, c = _np(size), _np(cap)
    bad = np.nonzero((s != o.size) | (c != o.cap))[0]
    assert len(bad) == 0, f"{tag}: {len(bad)} vertices differ, e.g. v={bad[:3]} gpu size/cap " \
                          f"{s[bad[:3]]}/{c[bad[:3]]} oracle {o.size[bad[:3]]}/{o.cap[bad[:3]]}"
    off = torch.cumsum(size.long(), 0) - size.long()
    total = int(s.sum())
    flat = g.gather(off, total)
    src = torch.repeat_interleave(torch.arange(V, device="cuda"), size.long())
    keys = (src.cpu().numpy().astype(np.uint64) << np.uint64(32)) | flat.cpu().numpy().astype(np.uint32).astype(np.uint64)
    assert np.array_equal(np.sort(keys), o.sorted_keys()), f"{tag}: adjacency multiset differs"
    # bytes held by the lists, read from the memory table, vs the closed form
    live = ptr != 0
    if int(live.sum()):
        req = (cap[live].long() * 4).contiguous()
        usum, ubad = G.gallatin_usable(ptr[live].contiguous(), req)
        assert ubad == 0, f"{tag}: {ubad} lists contradict their size class"
        assert usum == sum(class_size(int(b)) for b in req.cpu().numpy()), tag


@pytest.mark.parametrize("scale,n", [(12, 1 << 16), (16, 1 << 20)])
def test_graph_phases_match_o3(cuda_ok, scale, n):
    import paper_conf_ppopp_mccoyp24_b200 as G
    nseg = 512
    G.gallatin_init(nseg * SEG)
    try:
        w = wg.graph_workload(scale, n, device="cuda")
        V = w["V"]
        g = G.Graph(V)
        o = GraphOracle(V)
        s0, d0 = w["init"]
        g.insert(s0, d0)
        o.insert(_np(s0), _np(d0))
        _check(G, g, o, V, "init")
        for k, (s, d) in enumerate(w["insert"]):
            g.insert(s, d)
            o.insert(_np(s), _np(d))
        _check(G, g, o, V, "bulk insert")
        for k, (s, d) in enumerate(w["delete"]):
            g.delete(s, d)
            o.delete(_np(s), _np(d))
            if k == 0:
                _check(G, g, o, V, "first delete batch")
        _check(G, g, o, V, "bulk delete")
        for r in range(w["rounds"]):
            g.expand(w["expand"])
            o.expand(_np(w["expand"]))
        _check(G, g, o, V, "expansion")
        ctr = g.counters()
        assert ctr["failed"] == 0
        g.destroy()
        ctr = None
        G.gallatin_drain()
        img = G.gallatin_snapshot()
        msg = diff_images(img, pristine_image(nseg, int(img[4])))
        assert not msg, msg
        assert int(img[6]) == 0
    finally:
        G.gallatin_destroy()


@pytest.mark.parametrize("scale,n", [(12, 1 << 16), (16, 1 << 20)])
def test_graph_single_edge_ops_match_o3(cuda_ok, scale, n):
    """P:355's non-bulk edge updates and deletes (one thread per edge under a
    vertex lock, the allocator called per overflowing / shrinking edge),
    interleaved with bulk batches: sizes, capacities, adjacency multisets and
    list bytes equal O3's per-edge trajectory; the heap is pristine after
    teardown."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    nseg = 512
    G.gallatin_init(nseg * SEG)
    try:
        w = wg.graph_workload(scale, n, device="cuda", seed=scale + 11)
        V = w["V"]
        g = G.Graph(V)
        o = GraphOracle(V)
        steps = [("insert", w["init"]), ("insert_edges", w["insert"][0]), ("delete_edges", w["delete"][0]),
                 ("insert", w["insert"][1]), ("delete_edges", w["delete"][1]), ("delete", w["delete"][2]),
                 ("insert_edges", w["insert"][2]), ("delete_edges", w["delete"][3])]
        for kind, (s, d) in steps:
            getattr(g, kind)(s, d)
            getattr(o, kind)(_np(s), _np(d))
            _check(G, g, o, V, kind)
        assert g.counters()["failed"] == 0
        g.destroy()
        G.gallatin_drain()
        img = G.gallatin_snapshot()
        msg = diff_images(img, pristine_image(nseg, int(img[4])))
        assert not msg, msg
    finally:
        G.gallatin_destroy()


def test_graph_huge_lists_match_o3(cuda_ok):
    """Lists of >= 2^16 entries take the whole-grid paths (k_copy_huge when a
    batch grows them, k_expand_huge when an expansion round appends to them):
    a star whose hub receives 2^17 edges in two batches, three expansion
    rounds on the hub and a few small vertices, then a delete batch; sizes,
    capacities and multisets equal O3's after every phase; pristine after."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    nseg = 256
    G.gallatin_init(nseg * SEG)
    try:
        V = 1 << 12
        rng = np.random.Generator(np.random.PCG64(5))
        g, o = G.Graph(V), GraphOracle(V)

        def dev(a):
            return torch.from_numpy(np.ascontiguousarray(a, dtype=np.int32)).cuda()

        for half in range(2):
            src = np.where(rng.random(1 << 16) < 0.9, 0, rng.integers(1, V, 1 << 16))
            dst = rng.integers(0, V, 1 << 16)
            g.insert(dev(src), dev(dst))
            o.insert(src.astype(np.int64), dst.astype(np.int64))
            _check(G, g, o, V, f"insert {half}")
        vs = np.array([0, 1, 2, 3], dtype=np.int64)
        for r in range(3):
            g.expand(dev(vs))
            o.expand(vs)
            _check(G, g, o, V, f"expansion round {r}")
        keys = np.sort(o.sorted_keys())
        pick = keys[rng.choice(len(keys), 1 << 14, replace=False)]
        ds, dd = (pick >> np.uint64(32)).astype(np.int64), (pick & np.uint64(0xFFFFFFFF)).astype(np.int64)
        g.delete(dev(ds), dev(dd))
        o.delete(ds, dd)
        _check(G, g, o, V, "delete")
        assert g.counters()["failed"] == 0
        g.destroy()
        G.gallatin_drain()
        img = G.gallatin_snapshot()
        msg = diff_images(img, pristine_image(nseg, int(img[4])))
        assert not msg, msg
    finally:
        G.gallatin_destroy()
