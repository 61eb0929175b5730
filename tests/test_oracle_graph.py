"""Pins for O3 (oracle/graph.py): the vectorized numpy oracle against a
one-edge-at-a-time Python simulation of the same policy on small RMAT graphs,
plus closed forms of the capacity rule ("the next largest power of two")."""
import numpy as np
import pytest

import workload_gen as wg
from oracle.graph import BruteGraph, GraphOracle, list_cap


def _np(t):
    return t.numpy().astype(np.int64)


@pytest.mark.parametrize("scale,n", [(6, 1 << 10), (8, 1 << 12)])
def test_o3_matches_brute_force(scale, n):
    w = wg.graph_workload(scale, n, seed=scale, batches=4, n_expand=16, rounds=3)
    o, b = GraphOracle(w["V"]), BruteGraph(w["V"])
    steps = [("insert", w["init"])] + [("insert", x) for x in w["insert"]] + [("delete", x) for x in w["delete"]]
    for kind, (s, d) in steps:
        getattr(o, kind)(_np(s), _np(d))
        getattr(b, kind)(_np(s), _np(d))
        assert np.array_equal(o.sorted_keys(), b.sorted_keys()), kind
        assert np.array_equal(o.cap, np.array(b.cap)), kind
    for _ in range(w["rounds"]):
        o.expand(_np(w["expand"]))
        b.expand(_np(w["expand"]))
    assert np.array_equal(o.sorted_keys(), b.sorted_keys())
    assert np.array_equal(o.cap, np.array(b.cap))
    assert np.array_equal(o.size, np.array([len(b.lists[v]) for v in range(w["V"])]))


def test_capacity_closed_forms():
    """cap = next power of two >= max(size, 4): 0->4, 4->4, 5->8, 1000->1024, 1025->2048."""
    assert list(list_cap(np.array([0, 1, 4, 5, 1000, 1024, 1025]))) == [4, 4, 4, 8, 1024, 1024, 2048]
    o = GraphOracle(4)
    o.insert(np.array([1] * 5), np.array([2] * 5))
    assert o.size[1] == 5 and o.cap[1] == 8 and o.cap[0] == 0
    o.delete(np.array([1] * 4), np.array([2] * 4))      # 1 left: 1 <= 8/4 -> shrink to 4
    assert o.size[1] == 1 and o.cap[1] == 4
    o.delete(np.array([1, 1]), np.array([2, 3]))        # the absent edge (1,3) is ignored
    assert o.size[1] == 0 and o.cap[1] == 0             # empty list freed
    o.expand(np.array([2]))                              # 4 edges 2->3,0,1,2
    assert o.size[2] == 4 and o.cap[2] == 4
    assert sorted(int(k) & 0xFFFFFFFF for k in o.keys) == [0, 1, 2, 3]


@pytest.mark.parametrize("scale,n", [(6, 1 << 10), (8, 1 << 12)])
def test_o3_single_edge_ops_match_brute_force(scale, n):
    """P:355's non-bulk edge updates / deletes: O3's vectorized per-edge
    capacity trajectory against the one-edge-at-a-time simulation, starting
    from bulk-built lists and interleaved with bulk batches."""
    w = wg.graph_workload(scale, n, seed=scale + 7, batches=4, n_expand=16, rounds=2)
    o, b = GraphOracle(w["V"]), BruteGraph(w["V"])
    steps = [("insert", w["init"]), ("insert_edges", w["insert"][0]), ("delete_edges", w["delete"][0]),
             ("insert", w["insert"][1]), ("delete_edges", w["delete"][1]), ("delete", w["delete"][2]),
             ("insert_edges", w["insert"][2]), ("delete_edges", w["delete"][3]), ("delete_edges", w["init"])]
    for kind, (s, d) in steps:
        getattr(o, kind)(_np(s), _np(d))
        getattr(b, kind)(_np(s), _np(d))
        assert np.array_equal(o.sorted_keys(), b.sorted_keys()), kind
        assert np.array_equal(o.cap, np.array(b.cap)), kind
        assert np.array_equal(o.size, np.array([len(b.lists[v]) for v in range(w["V"])])), kind


def test_single_edge_capacity_closed_forms():
    """Doubling on a full list: 9 single inserts into an empty list go 0->4->8->16;
    deleting down from 16 entries shrinks at 4 (= 16/4) to 4 and frees at 0."""
    o = GraphOracle(2)
    o.insert_edges(np.array([1] * 9), np.arange(9))
    assert o.size[1] == 9 and o.cap[1] == 16
    o.insert_edges(np.array([1] * 7), np.arange(9, 16))
    assert o.size[1] == 16 and o.cap[1] == 16
    o.delete_edges(np.array([1] * 11), np.arange(11))        # 5 left: 5 > 16/4 -> keeps 16
    assert o.size[1] == 5 and o.cap[1] == 16
    o.delete_edges(np.array([1]), np.array([11]))             # 4 left: shrink to 4
    assert o.size[1] == 4 and o.cap[1] == 4
    o.delete_edges(np.array([1] * 5), np.array([12, 13, 14, 15, 99]))   # absent edge ignored
    assert o.size[1] == 0 and o.cap[1] == 0
