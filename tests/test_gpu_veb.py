"""GPU parity of the concurrent vEB bitmap tree (C-ABI veb_*) against O1.

BASELINE north_star: "vEB successor/insert/delete results for the same op
batches" bit-exact vs the CPU oracle; final level words bit-exact (SURVEY
8(c): leaf words = O1 membership, summaries = OR reduction at quiescence).
"""
import numpy as np
import pytest
import torch

import oracle
import workload_gen as wg
from oracle import NONE, OV_DELETE, OV_INSERT, OV_MEMBER, OV_PRED, OV_SUCC

pytestmark = pytest.mark.gpu


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64).view(np.int64)).cuda()


def _u64(t):
    return t.cpu().numpy().view(np.uint64)


def _run_batches(k, batches, concurrent=False):
    """Apply the same homogeneous batches to the GPU tree and to O1; compare
    every per-op output and the final image.  concurrent: the coherent query
    path (veb_set_concurrent) instead of the read-only one."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    g = G.Veb(k)
    if concurrent:
        g.set_concurrent(True)
    o = oracle.Veb(k)
    for op, keys in batches:
        d = _dev(keys)
        want = o.batch(op, keys)
        if op == OV_INSERT:
            got = g.insert(d).cpu().numpy().astype(np.uint64)
        elif op == OV_DELETE:
            got = g.delete(d).cpu().numpy().astype(np.uint64)
        elif op == OV_MEMBER:
            got = g.member(d).cpu().numpy().astype(np.uint64)
        elif op == OV_SUCC:
            got = _u64(g.successor(d))
        else:
            got = _u64(g.predecessor(d))
        bad = np.nonzero(got != want)[0]
        assert len(bad) == 0, f"op {op}: {len(bad)} mismatches, e.g. key {keys[bad[:3]]} got {got[bad[:3]]} want {want[bad[:3]]}"
    torch.cuda.synchronize()
    img_g, img_o = g.snapshot(), o.image()
    assert np.array_equal(img_g, img_o), f"image differs at words {np.nonzero(img_g != img_o)[0][:8]}"
    g.close()


@pytest.mark.parametrize("concurrent", [False, True])
def test_config1_veb_parity(cuda_ok, concurrent):
    """BASELINE configs[0]: 2^16 random insert / successor / delete on a 2^20
    universe, plus pred/member of the same queries -- on the
    read-only and on the coherent (concurrent-mode) query path."""
    w = wg.veb_workload(20, 1 << 16)
    _run_batches(20, [
        (OV_SUCC, w["succ1"]),                     # empty tree: all none
        (OV_INSERT, w["insert"]),
        (OV_SUCC, w["succ1"]),
        (OV_PRED, w["succ1"]),
        (OV_MEMBER, w["succ1"]),
        (OV_DELETE, w["delete"]),
        (OV_SUCC, w["succ2"]),
        (OV_PRED, w["succ2"]),
    ], concurrent=concurrent)


def test_bulk_queries_four_per_thread(cuda_ok):
    """Query batches of >= 2^20 keys run 4 queries per thread (keys loaded
    first); a ragged count exercises the clamped tail: successor, predecessor
    and member equal O1's bit-exactly."""
    k = 20
    seed = wg.cell_seed(1, 320)
    ins = wg.distinct_below(seed, 1 << 16, 1 << k)
    q = np.concatenate([wg.uniform_below(seed ^ 3, (1 << 20) + 1021, 1 << k),
                        np.array([0, (1 << k) - 1, 1 << k], dtype=np.uint64)])
    _run_batches(k, [(OV_INSERT, ins), (OV_SUCC, q), (OV_PRED, q), (OV_MEMBER, q)])


@pytest.mark.parametrize("concurrent", [False, True])
@pytest.mark.parametrize("k", [1, 3, 6, 7, 12, 13, 18, 19, 24])
def test_universe_sizes(cuda_ok, k, concurrent):
    """Every level count (1..5) incl. partial top words; dense and sparse sets."""
    u = 1 << k
    n = min(u, 1 << 15)
    seed = wg.cell_seed(1, 200 + k)
    ins = wg.distinct_below(seed, n, u)
    q = np.concatenate([wg.uniform_below(seed ^ 1, 4096, u), np.array([0, u - 1, u, u + 7], dtype=np.uint64)])
    dele = ins[: n // 2]
    _run_batches(k, [(OV_INSERT, ins), (OV_SUCC, q), (OV_PRED, q), (OV_DELETE, dele), (OV_SUCC, q),
                     (OV_PRED, q), (OV_MEMBER, q), (OV_DELETE, ins), (OV_SUCC, q)], concurrent=concurrent)


def test_universe_2_32_sampled(cuda_ok):
    k = 32
    seed = wg.cell_seed(1, 232)
    ins = np.unique(wg.uniform_below(seed, 1 << 14, 1 << 32))
    q = wg.uniform_below(seed ^ 9, 1 << 14, 1 << 32)
    _run_batches(k, [(OV_INSERT, ins), (OV_SUCC, q), (OV_PRED, q), (OV_DELETE, ins[::3]), (OV_SUCC, q)])


def test_duplicate_keys_exactly_one_reports(cuda_ok):
    """Reading A-23: with repeated keys in one batch, exactly one op per
    distinct key reports 'newly added' / 'was present'."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    k = 16
    rng = np.random.Generator(np.random.PCG64(3))
    keys = rng.integers(0, 1 << 12, size=1 << 16).astype(np.uint64)     # heavy duplication
    g = G.Veb(k)
    got = g.insert(_dev(keys)).cpu().numpy()
    uniq = np.unique(keys)
    per_key = np.bincount(keys.astype(np.int64), weights=got, minlength=1 << 12)
    assert got.sum() == len(uniq) and np.all(per_key[uniq.astype(np.int64)] == 1)
    o = oracle.Veb(k)
    o.batch(OV_INSERT, keys)
    assert np.array_equal(g.snapshot(), o.image())
    got = g.delete(_dev(keys)).cpu().numpy()
    per_key = np.bincount(keys.astype(np.int64), weights=got, minlength=1 << 12)
    assert got.sum() == len(uniq) and np.all(per_key[uniq.astype(np.int64)] == 1)
    assert not g.snapshot().any()


def test_concurrent_insert_delete_quiescent_exact(cuda_ok):
    """Inserts and deletes of disjoint key sets racing on different streams
    hammer the same leaf words; at quiescence every summary word must equal the
    OR of its children and the leaves must equal the set semantics."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    k = 14
    u = 1 << k
    g = G.Veb(k)
    evens = np.arange(0, u, 2, dtype=np.uint64)
    odds = np.arange(1, u, 2, dtype=np.uint64)
    g.insert(_dev(odds), want_out=False)
    torch.cuda.synchronize()
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    de, do = _dev(evens), _dev(odds)
    for _ in range(20):
        with torch.cuda.stream(s1):
            g.insert(de, want_out=False, stream=s1.cuda_stream)
        with torch.cuda.stream(s2):
            g.delete(do, want_out=False, stream=s2.cuda_stream)
        torch.cuda.synchronize()
        with torch.cuda.stream(s1):
            g.delete(de, want_out=False, stream=s1.cuda_stream)
        with torch.cuda.stream(s2):
            g.insert(do, want_out=False, stream=s2.cuda_stream)
        torch.cuda.synchronize()
    o = oracle.Veb(k)
    o.batch(OV_INSERT, odds)
    assert np.array_equal(g.snapshot(), o.image())


@pytest.mark.parametrize("k", [16, 24])
def test_concurrent_mixed_batches_linearizable(cuda_ok, k):
    """Concurrent mixed-batch mode (veb_set_concurrent):
    successor / predecessor / member queries race with inserts and deletes of
    VOLATILE keys on other streams.  Linearizability-style invariants, for every query x:
    succ(x) is NONE only if no STABLE key (present throughout) is >= x;
    otherwise x <= succ(x) <= the smallest stable key >= x and succ(x) is a
    stable or volatile key (never a key that was never present); pred
    mirrors it; member is 1 on stable keys and 0 on never-present keys.  At
    quiescence the image is exact."""
    import paper_conf_ppopp_mccoyp24_b200 as G
    u = 1 << k
    seed = wg.cell_seed(1, 300 + k)
    keys = wg.distinct_below(seed, min(u // 4, 1 << 20), u)
    third = len(keys) // 3
    stable, vol_in, vol_out = keys[:third], keys[third:2 * third], keys[2 * third:]
    q = wg.uniform_below(seed ^ 5, 1 << 20, u)
    g = G.Veb(k)
    g.set_concurrent(True)            # queries overlap updates: coherent loads (include/gallatin.h)
    g.insert(_dev(np.concatenate([stable, vol_out])), want_out=False)
    torch.cuda.synchronize()
    s1, s2, s3 = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
    dq = _dev(q)
    di, dd = _dev(vol_in), _dev(vol_out)
    outs = []
    for rep in range(4):
        with torch.cuda.stream(s1):
            (g.insert if rep % 2 == 0 else g.delete)(di, want_out=False, stream=s1.cuda_stream)
        with torch.cuda.stream(s2):
            (g.delete if rep % 2 == 0 else g.insert)(dd, want_out=False, stream=s2.cuda_stream)
        with torch.cuda.stream(s3):
            su = torch.empty_like(dq)
            pr = torch.empty_like(dq)
            g.successor(dq, su, stream=s3.cuda_stream)
            g.predecessor(dq, pr, stream=s3.cuda_stream)
            me = g.member(_dev(stable[:4096]), stream=s3.cuda_stream)
            outs.append((su, pr, me))
        torch.cuda.synchronize()
    st = np.sort(stable)
    allowed = np.sort(keys)
    NONE64 = np.uint64(NONE)
    i_ge = np.searchsorted(st, q, side="left")
    succ_stable = np.where(i_ge < len(st), st[np.minimum(i_ge, len(st) - 1)], NONE64)
    i_le = np.searchsorted(st, q, side="right") - 1
    pred_stable = np.where(i_le >= 0, st[np.maximum(i_le, 0)], NONE64)
    for su, pr, me in outs:
        s, p = _u64(su), _u64(pr)
        none_s = s == NONE64
        assert np.all(succ_stable[none_s] == NONE64)
        ok = ~none_s
        assert np.all(s[ok] >= q[ok]) and np.all(s[ok] <= succ_stable[ok])
        assert np.all(np.isin(s[ok], allowed))
        none_p = p == NONE64
        assert np.all(pred_stable[none_p] == NONE64)
        okp = ~none_p
        assert np.all(p[okp] <= q[okp]) and np.all((pred_stable[okp] == NONE64) | (p[okp] >= pred_stable[okp]))
        assert np.all(np.isin(p[okp], allowed))
        assert np.all(me.cpu().numpy() == 1)
    # quiescent: after 4 rounds vol_in was inserted then deleted twice, vol_out the reverse
    o = oracle.Veb(k)
    o.batch(OV_INSERT, np.concatenate([stable, vol_out]))
    assert np.array_equal(g.snapshot(), o.image())
    g.close()
