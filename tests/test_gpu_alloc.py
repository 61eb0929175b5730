"""GPU parity of the allocator (C-ABI gallatin_*) against O2 and the paper's invariants.

* Serialized replay (one GPU thread, slot key = the op's key): every pointer
  offset and the final metadata image equal O2's bit-exactly.
* Concurrent bulk runs (address assignment is nondeterministic, reading A-30):
  stamp-and-verify finds 0 overwritten words, the sorted pointers never
  overlap, every pointer is aligned and in the heap, the usable bytes read from
  the memory table equal the closed form and O2's accounting, and free-all +
  drain restores the pristine image bit-exactly (== O2's == analytic).
"""
import numpy as np
import pytest
import torch

import oracle
import workload_gen as wg
from helpers import SEG, check_live_invariants, class_size, diff_images, pristine_image

pytestmark = pytest.mark.gpu
NONE = (1 << 64) - 1


def _dev(a, dtype=np.uint64):
    a = np.ascontiguousarray(a, dtype=dtype)
    return torch.from_numpy(a.view(np.int64) if a.dtype.itemsize == 8 else a).cuda()


def _u64(t):
    return t.cpu().numpy().view(np.uint64)


@pytest.fixture()
def G():
    import paper_conf_ppopp_mccoyp24_b200 as G
    yield G
    if G.gallatin_is_initialized():
        G.gallatin_destroy()


def _replay_case(G, nseg, run_max, fa, kinds, args, keys, slot_base=16, slot_min=2, run_bytes=32 << 20, pf=None,
                 run_init=1, run_grow=0, record=None, prefill=False):
    """GPU serialized replay vs O2: O2-P at the paper's knobs without prefill
    (with the exhaustion record on, where it is state-neutral), O2-R otherwise
    (the GPU with the record off: O2-R does not model it)."""
    if pf is None:
        pf = run_max > 1                    # the paper's policy (run_max=1) has no prefetch
    paper = run_max == 1 and not fa and not pf and run_init == 1 and not prefill
    if record is None:
        record = paper
    G.gallatin_init(nseg * SEG, slot_base=slot_base, slot_min=slot_min, run_max=run_max, run_bytes=run_bytes,
                    format_ahead=1 if fa else 2, prefetch=1 if pf else 2, run_init=run_init, run_grow=run_grow,
                    oom_record=1 if record else 2, prefill=1 if prefill else 2)
    if prefill:
        assert G.gallatin_stats()["prefill_segments"] > 0, "the case must exercise a prefilled buffer"
    out = _u64(G.gallatin_replay(_dev(kinds, np.uint8), _dev(args), _dev(keys)))
    o2 = oracle.model(nseg, **G.oracle_params())
    assert isinstance(o2, oracle.RunsAllocator) != paper
    want = o2.replay(kinds, args, keys)
    bad = np.nonzero(out != want)[0]
    assert len(bad) == 0, f"{len(bad)} ops differ; first op {bad[0]} kind {kinds[bad[0]]} size {args[bad[0]]}: " \
                          f"gpu {out[bad[0]]:#x} oracle {want[bad[0]]:#x}"
    msg = diff_images(G.gallatin_snapshot(), o2.image())
    assert not msg, msg
    G.gallatin_destroy()
    return out


@pytest.mark.parametrize("seed,nseg,run_max,fa", [(1, 4, 1, 0), (2, 8, 1, 0), (3, 6, 16, 1), (4, 64, 8, 1),
                                                  (5, 5, 128, 0), (6, 16, 4, 1), (7, 3, 2, 1), (8, 32, 1, 1)])
def test_serialized_replay_matches_oracle(cuda_ok, G, seed, nseg, run_max, fa):
    """Mixed slices / blocks / multi-segment allocations, interleaved frees,
    drains and OOM on 3-64 segment heaps (SURVEY 8(c) "Scope of serialized
    replay"); run_max=1, fa=0 is the paper's policy."""
    kinds, args, keys = wg.replay_ops(6000, seed + 100, p_free=0.45, p_drain=0.003, nkeys=64)
    _replay_case(G, nseg, run_max, fa, kinds, args, keys)


@pytest.mark.parametrize("seed,nseg,run_max,fa,ri,rg", [(21, 96, 1, 0, 1, 1), (22, 128, 16, 1, 4, 1),
                                                        (23, 160, 256, 1, 16, 3), (24, 256, 512, 0, 64, 3)])
def test_serialized_replay_prefilled(cuda_ok, G, seed, nseg, run_max, fa, ri, rg):
    """A prefilled block buffer ("always populated", O2-R R7): init and
    the replay's drains leave the state O2-R reaches; at the paper's one-block
    knobs (first case) and with runs."""
    kinds, args, keys = wg.replay_ops(6000, seed + 100, p_free=0.45, p_drain=0.003, nkeys=64)
    _replay_case(G, nseg, run_max, fa, kinds, args, keys, pf=False, run_init=ri, run_grow=rg, prefill=True)


def test_reset_prefills_block_buffer(cuda_ok, G):
    """gallatin_reset with the prefill knob (default) leaves exactly O2-R's
    prefilled initial state (R7); drain turns it into the pristine image."""
    nseg = 4096                                    # 64 GB: the first runs fit in nseg / 8
    G.gallatin_init(nseg * SEG)
    st = G.gallatin_stats()
    assert st["prefill_segments"] > 0
    G.gallatin_malloc(_dev(wg.mixed_sizes(1 << 16, p_large=2.0 ** -8)))
    G.gallatin_reset()
    o2 = oracle.model(nseg, **G.oracle_params())
    msg = diff_images(G.gallatin_snapshot(), o2.image())
    assert not msg, msg
    _assert_pristine(G, nseg)


def test_serialized_replay_full_word_window(cuda_ok, G):
    """A run of 64 whole segments claimed at a leaf-word boundary (all 64 bits
    of the word in one window): 64 slots of the 4 KB class take segments
    0..63 with their first one-block runs, then slot 0 exhausts its block and
    refills with a 64-segment run (growth 2^6) -- segments 64..127.  (A round-1
    bug read such a window's consecutive prefix as 2^16 - 1 segments.)"""
    nseg = 256
    n1, n2 = 64, 4096 + 3
    kinds = np.zeros(n1 + n2 + 2, dtype=np.uint8)
    args = np.full(n1 + n2 + 2, 4096, dtype=np.uint64)
    keys = np.concatenate([np.arange(n1), np.zeros(n2 + 2, dtype=np.int64)]).astype(np.uint64)
    kinds[-2], args[-2] = 1, n1 + n2 - 1                   # free the first slice of the 64-segment run
    kinds[-1], args[-1] = 2, 0                             # drain
    out = _replay_case(G, nseg, 512, False, kinds, args, keys, slot_base=64, slot_min=64, run_bytes=64 << 24,
                       pf=False, run_init=1, run_grow=6)
    assert out[n1 + n2 - 1] == 64 * SEG + 3 * 4096         # the 4th slice of slot 0's run at segment 64


def test_serialized_replay_block_boundaries(cuda_ok, G):
    """Exactly-full blocks and runs, exhausted slots and refills with a single
    slot per class (every request hits the same slot)."""
    n = 7 * 4096 + 7
    kinds = np.zeros(n, dtype=np.uint8)
    args = np.full(n, 16, dtype=np.uint64)
    keys = np.zeros(n, dtype=np.uint64)
    kinds2 = np.concatenate([kinds, np.ones(4096, dtype=np.uint8), np.array([2], dtype=np.uint8)])
    args2 = np.concatenate([args, np.arange(4096, dtype=np.uint64), np.array([0], dtype=np.uint64)])
    keys2 = np.concatenate([keys, np.zeros(4097, dtype=np.uint64)])
    for run_max, fa, pf, ri, rg in ((1, 0, 0, 1, 1), (4, 1, 0, 1, 1), (128, 1, 1, 1, 3), (512, 1, 1, 8, 2),
                                    (16, 0, 1, 4, 8), (256, 1, 0, 256, 3)):
        _replay_case(G, 2, run_max, fa, kinds2, args2, keys2, slot_base=1, slot_min=1, pf=pf, run_init=ri,
                     run_grow=rg)


@pytest.mark.parametrize("seed,nseg,run_max,fa,pf,ri,rg", [(11, 8, 64, 1, 1, 4, 1), (12, 48, 512, 1, 1, 8, 3),
                                                           (13, 6, 16, 0, 1, 2, 2), (14, 12, 256, 1, 0, 1, 3),
                                                           (15, 4, 256, 1, 0, 256, 3), (16, 6, 256, 0, 1, 64, 8),
                                                           (17, 3, 512, 1, 1, 256, 4)])
def test_serialized_replay_runs_prefetch_matrix(cuda_ok, G, seed, nseg, run_max, fa, pf, ri, rg):
    """The run / prefetch / run_init / run_grow / format-ahead knobs (DESIGN.md
    Deviations 5) against O2 modelling the same policy, with OOM and drains;
    the whole-segment first runs on 3-6 segment heaps force slot trims."""
    kinds, args, keys = wg.replay_ops(6000, seed + 100, p_free=0.45, p_drain=0.003, nkeys=64)
    _replay_case(G, nseg, run_max, fa, kinds, args, keys, pf=pf, run_init=ri, run_grow=rg)


def test_serialized_replay_default_knobs(cuda_ok, G):
    """The production knobs gallatin_init picks for a 64-segment heap (148
    slots at 16 B, slot_min 4, runs up to 256 blocks / heap/64 bytes, x8
    growth, the derived first run, format-ahead) with the exhaustion record
    off, against O2-R; keys span every slot."""
    nseg = 64
    kinds, args, keys = wg.replay_ops(8000, 141, p_free=0.45, p_drain=0.002, nkeys=148 * 4)
    G.gallatin_init(nseg * SEG, oom_record=2)
    st = G.gallatin_stats()
    assert st["slot_base"] == 148 and st["run_max"] == 256 and st["format_ahead"] == 1 and st["run_grow"] == 3
    out = _u64(G.gallatin_replay(_dev(kinds, np.uint8), _dev(args), _dev(keys)))
    o2 = oracle.model(nseg, **G.oracle_params())
    want = o2.replay(kinds, args, keys)
    assert np.array_equal(out, want), f"{int((out != want).sum())} ops differ"
    msg = diff_images(G.gallatin_snapshot(), o2.image())
    assert not msg, msg


@pytest.mark.parametrize("seed,nseg", [(151, 3), (152, 6), (153, 16)])
def test_serialized_replay_record_on_invariants(cuda_ok, G, seed, nseg):
    """Run knobs with the exhaustion record ON (the production setting) under
    heavy OOM: the record is a concurrency device O2-R does not model, so the
    replay is checked by the invariants instead -- every pointer in the heap,
    aligned to its class, live allocations disjoint, the accounting of the
    live set equal to the closed form, and free-all + drain pristine."""
    kinds, args, keys = wg.replay_ops(6000, seed, p_free=0.4, p_drain=0.003, nkeys=64)
    G.gallatin_init(nseg * SEG, slot_base=16, slot_min=2, run_max=64, run_bytes=32 << 20, format_ahead=1,
                    prefetch=1, run_init=4, run_grow=2)
    out = _u64(G.gallatin_replay(_dev(kinds, np.uint8), _dev(args), _dev(keys)))
    live = {}
    for i, k in enumerate(kinds):
        if k == 0 and out[i] != np.uint64(NONE):
            live[i] = (int(out[i]), int(args[i]))
        elif k == 1:
            live.pop(int(args[i]), None)
        elif k == 2:
            pass
    assert (out[kinds == 0] == np.uint64(NONE)).sum() > 100          # OOM exercised
    offs = np.array([v[0] for v in live.values()], dtype=np.uint64)
    sizes = [v[1] for v in live.values()]
    check_live_invariants(nseg, offs, sizes)
    assert G.gallatin_stats()["errors"] == 0
    G.gallatin_free(_dev(offs + np.uint64(G.gallatin_stats()["heap_base"])))
    _assert_pristine(G, nseg)


def _bulk_round(G, nseg, sizes, check_accounting=True):
    """malloc -> stamp -> verify -> usable/overlap checks -> free; returns #NULL."""
    d_sizes = _dev(sizes)
    ptrs = G.gallatin_malloc(d_sizes)
    torch.cuda.synchronize()
    p = _u64(ptrs)
    null = p == 0
    st = G.gallatin_stats()
    base = st["heap_base"]
    G.gallatin_stamp(ptrs, d_sizes)
    assert G.gallatin_verify(ptrs, d_sizes) == 0, "stamp-verify found overwritten words"
    usable = torch.empty_like(ptrs)
    usum, ubad = G.gallatin_usable(ptrs, d_sizes, usable)
    assert ubad == 0, f"{ubad} pointers contradict their size class / alignment"
    if check_accounting:
        want = int(sum(class_size(int(s)) * int(c) for s, c in zip(*np.unique(sizes[~null], return_counts=True))))
        assert usum == want, f"usable {usum} != closed form {want}"
    # no overlap: sort live pointers, each ends before the next begins
    live = ~null
    order = np.argsort(p[live])
    sp, su = p[live][order], _u64(usable)[live][order]
    assert np.all(sp[:-1] + su[:-1] <= sp[1:]), "overlapping allocations"
    assert np.all((sp - np.uint64(base)) < np.uint64(nseg * SEG))
    G.gallatin_free(ptrs)
    torch.cuda.synchronize()
    return int(null.sum())


def _assert_pristine(G, nseg):
    G.gallatin_drain()
    img = G.gallatin_snapshot()
    S = int(img[4])
    msg = diff_images(img, pristine_image(nseg, S))
    assert not msg, msg


def test_config1_concurrent(cuda_ok, G):
    """BASELINE configs[0]: 64 MB heap, 2^16 threads malloc 16 B then free."""
    nseg = 4
    G.gallatin_init(nseg * SEG)
    sizes = wg.single_sizes(16, 1 << 16)
    assert _bulk_round(G, nseg, sizes) == 0
    _assert_pristine(G, nseg)
    # accounting equals O2's on the same sizes
    o2 = oracle.model(nseg, **G.oracle_params())
    o2.malloc_batch(sizes)
    assert o2.usable_live == (1 << 16) * 16


@pytest.mark.parametrize("size", wg.SLICE_SIZES)
def test_config2_single_size_reduced(cuda_ok, G, size):
    """BASELINE configs[1] shape at 2^20 threads on the 16 GB heap."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    for rep in range(2):                     # second round: warm (no reset)
        assert _bulk_round(G, nseg, wg.single_sizes(size, 1 << 20)) == 0
        _assert_pristine(G, nseg)


def test_config3_mixed_reduced(cuda_ok, G):
    """BASELINE configs[2] shape: random 16 B-4 KB plus 1-64 MB large
    allocations (p = 2^-12) at 2^20 threads on a 64 GB heap."""
    nseg = 4096
    G.gallatin_init(nseg * SEG)
    sizes = wg.mixed_sizes(1 << 20)
    assert (sizes > 4096).sum() > 100
    assert _bulk_round(G, nseg, sizes) == 0
    _assert_pristine(G, nseg)
    sizes_b = wg.mixed_sizes(1 << 20, seed=wg.cell_seed(3, 1), exact_pow2=False, p_large=2.0 ** -10)
    assert _bulk_round(G, nseg, sizes_b) == 0
    _assert_pristine(G, nseg)


def test_oom_capacity_and_recovery(cuda_ok, G):
    """A 4-segment heap asked for 4x its capacity: NULLs, no overlap, and after
    freeing everything the heap is pristine (P:274 nullptr on exhaustion)."""
    nseg = 4
    G.gallatin_init(nseg * SEG)
    sizes = wg.single_sizes(1024, 1 << 18)          # 256 MiB requested, 64 MiB heap
    nulls = _bulk_round(G, nseg, sizes, check_accounting=False)
    assert nulls >= (1 << 18) - nseg * SEG // 1024
    _assert_pristine(G, nseg)
    sizes = wg.mixed_sizes(1 << 16, p_large=2.0 ** -6)
    _bulk_round(G, nseg, sizes, check_accounting=False)
    _assert_pristine(G, nseg)


def test_bad_frees_counted(cuda_ok, G):
    G.gallatin_init(4 * SEG)
    base = G.gallatin_stats()["heap_base"]
    bad = np.array([base + 9 * SEG, base + 2 * SEG + 64, 0], dtype=np.uint64)   # outside; FREE segment; NULL
    G.gallatin_free(_dev(bad))
    torch.cuda.synchronize()
    assert G.gallatin_stats()["errors"] == 2


def test_host_buffer_api(cuda_ok, G):
    nseg = 16
    G.gallatin_init(nseg * SEG)
    sizes = wg.mixed_sizes(1 << 14, p_large=0.0)
    p = G.gallatin_malloc_host(sizes)
    assert np.all(p != 0)
    o = np.sort(p)
    assert len(np.unique(o)) == len(o)
    G.gallatin_free_host(p)
    _assert_pristine(G, nseg)


def test_host_buffer_api_chunked(cuda_ok, G):
    """Host-array calls cut into several copy/kernel/copy chunks (a ragged last
    chunk): every pointer distinct, aligned to its class, in the heap, and the
    usable bytes equal the closed form; free-all + drain is pristine."""
    nseg = 64
    G.gallatin_init(nseg * SEG)
    n = 3 * (1 << 20) + 12345
    sizes = wg.mixed_sizes(n, upper=256, p_large=0.0)
    p = G.gallatin_malloc_host(sizes)
    assert np.all(p != 0)
    base = G.gallatin_stats()["heap_base"]
    offs = p - np.uint64(base)
    cls = np.array([class_size(int(s)) for s in sizes[:4096]], dtype=np.uint64)
    assert np.all(offs[:4096] % cls == 0)
    assert len(np.unique(p)) == n and int(offs.max()) < nseg * SEG
    usable, bad = G.gallatin_usable(_dev(p), _dev(sizes))
    u, c = np.unique(sizes, return_counts=True)
    assert bad == 0 and usable == sum(class_size(int(a)) * int(b) for a, b in zip(u, c))
    G.gallatin_free_host(p)
    _assert_pristine(G, nseg)


def test_reset_restores_pristine(cuda_ok, G):
    nseg = 8
    G.gallatin_init(nseg * SEG, prefill=2)
    G.gallatin_malloc(_dev(wg.mixed_sizes(1 << 14, p_large=2.0 ** -8)))
    G.gallatin_reset()
    img = G.gallatin_snapshot()
    assert not diff_images(img, pristine_image(nseg, int(img[4])))


@pytest.mark.parametrize("size", wg.SLICE_SIZES)
def test_config2_full_size_bench_launch(cuda_ok, G, size):
    """BASELINE configs[1] at its full size, in the launch configuration
    bench.py times (default knobs, ITEMS=4 bulk kernels): two warm rounds and
    one after a reset, each stamp-verified, accounted, overlap-checked, and
    drained back to the pristine image."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    n = min(1 << 24, (8 << 30) // size)
    for rep in range(3):
        if rep == 2:
            G.gallatin_reset()
        assert _bulk_round(G, nseg, wg.single_sizes(size, n)) == 0
        _assert_pristine(G, nseg)


@pytest.mark.parametrize("n", [1, 31, 33, 255, 1000, 1 << 10, 4097, 1 << 16, 1 << 26])
def test_config4_thread_scaling_points(cuda_ok, G, n):
    """BASELINE configs[3]: 64 B at 2^10..2^26 threads, plus ragged counts
    (one thread, partial warps and CTAs, one slice past a block)."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    assert _bulk_round(G, nseg, wg.single_sizes(64, n)) == 0
    _assert_pristine(G, nseg)


def test_config3_full_size_bench_launch(cuda_ok, G):
    """BASELINE configs[2] at its full size (2^22 threads, 64 GB heap), as
    bench.py runs it: stamp-verified, accounted, overlap-checked, pristine."""
    nseg = 4096
    G.gallatin_init(nseg * SEG)
    sizes = wg.mixed_sizes(1 << 22)
    for rep in range(2):
        if rep:
            G.gallatin_reset()
        assert _bulk_round(G, nseg, sizes) == 0
        _assert_pristine(G, nseg)


@pytest.mark.parametrize("knobs", [dict(bulk_items=1), dict(bulk_items=4), dict(demand_hint=2), dict(oom_record=2),
                                   dict(prefetch=1), dict(fence_free=2), dict(run_max=1, format_ahead=2, run_init=1)])
@pytest.mark.parametrize("n", [(1 << 21) + 77, (1 << 23) + 5])
def test_bulk_kernel_variants(cuda_ok, G, knobs, n):
    """Both bulk-kernel pairs (one request per thread with warp teams; four
    per thread with one slot RMW per class per CTA tile) at both free CTA
    shapes (2^21 and 2^23+ pointers), and the policy knobs, on mixed sizes
    with a ragged tail: stamp-verified, accounted, overlap-checked, pristine
    after free-all + drain."""
    nseg = 1024 if n < (1 << 22) else 2048       # ~0.9 KB per small request + 1-64 MB every 2^14
    G.gallatin_init(nseg * SEG, **knobs)
    sizes = wg.mixed_sizes(n, p_large=2.0 ** -14)
    assert _bulk_round(G, nseg, sizes) == 0
    _assert_pristine(G, nseg)


@pytest.mark.parametrize("items", [1, 4])
def test_malloc_zero_and_nulls(cuda_ok, G, items):
    """malloc(0) is NULL (reading A-4) in both bulk kernels, next to real
    requests in the same warps and CTA tiles; freeing the NULLs is a no-op
    (P:241); non-power-of-two sizes round up to their class."""
    nseg = 512                                     # ~2.8 KB per request after rounding: 8 GB heap
    G.gallatin_init(nseg * SEG, bulk_items=items)
    n = (1 << 20) + 17
    rng = np.random.Generator(np.random.PCG64(5))
    sizes = rng.integers(0, 4097, n).astype(np.uint64)
    sizes[rng.random(n) < 0.25] = 0
    d = _dev(sizes)
    p = G.gallatin_malloc(d)
    torch.cuda.synchronize()
    pu = _u64(p)
    assert np.all((pu == 0) == (sizes == 0)), "malloc(0) must be NULL and every other request granted"
    G.gallatin_stamp(p, d)
    assert G.gallatin_verify(p, d) == 0
    usum, ubad = G.gallatin_usable(p, d)
    assert ubad == 0 and usum == sum(class_size(int(s)) for s in sizes)
    G.gallatin_free(p)
    assert G.gallatin_stats()["errors"] == 0
    _assert_pristine(G, nseg)


def test_bulk_kernels_unaligned_arrays(cuda_ok, G):
    """Size and pointer arrays that start 8 bytes past a 16-byte boundary,
    through both bulk-kernel pairs."""
    nseg = 256
    for knobs in (dict(bulk_items=1), {}):
        G.gallatin_init(nseg * SEG, **knobs)
        n = (1 << 20) + 3
        sizes = _dev(np.concatenate([[0], wg.mixed_sizes(n, upper=512, p_large=0.0)]))[1:]
        ptrs = torch.zeros(n + 1, dtype=torch.int64, device="cuda")[1:]
        assert sizes.data_ptr() % 16 == 8 and ptrs.data_ptr() % 16 == 8
        G.gallatin_malloc(sizes, ptrs)
        G.gallatin_stamp(ptrs, sizes)
        assert G.gallatin_verify(ptrs, sizes) == 0
        assert int((ptrs == 0).sum()) == 0
        G.gallatin_free(ptrs)
        _assert_pristine(G, nseg)
        G.gallatin_destroy()


@pytest.mark.parametrize("size,n", [(8192, 1 << 16), (65537, 1 << 12), (3 << 20, 1 << 10)])
def test_block_path_teams(cuda_ok, G, size, n):
    """Whole-block requests (A-2) from every lane of every warp: the lanes
    asking one block tree share GetBlock runs (P:190 coalescing applied to
    blocks).  Stamp-verified, accounted, overlap-checked, pristine after."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    assert _bulk_round(G, nseg, wg.single_sizes(size, n)) == 0
    _assert_pristine(G, nseg)


def test_block_path_mixed_tail(cuda_ok, G):
    """Block sizes mixed with slices in every warp, ragged count."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    rng = np.random.Generator(np.random.PCG64(11))
    n = (1 << 16) + 123
    sizes = np.where(rng.random(n) < 0.5, rng.integers(4097, 1 << 18, n), rng.integers(1, 4097, n)).astype(np.uint64)
    assert _bulk_round(G, nseg, sizes) == 0
    _assert_pristine(G, nseg)


@pytest.mark.parametrize("size,n,nseg", [(16, 1 << 24, 8), (1024, 1 << 18, 4), (8192, 1 << 20, 1024),
                                         (4096, 1 << 20, 64)])
def test_oom_fails_fast(cuda_ok, G, size, n, nseg):
    """A bulk call asking 2-4x the heap (DESIGN.md Deviations 11): it ends in
    well under a second (it took 0.5-112 s before the exhaustion record), it is
    granted the capacity up to one partly drawn block per slot, the grants are
    stamp-verified and disjoint, and free-all + drain is pristine."""
    import time
    G.gallatin_init(nseg * SEG)
    st = G.gallatin_stats()
    d_sizes = _dev(wg.single_sizes(size, n))
    torch.cuda.synchronize()
    t0 = time.time()
    nulls = _bulk_round(G, nseg, wg.single_sizes(size, n), check_accounting=False)
    assert time.time() - t0 < 10.0, "exhaustion took too long"
    granted = n - nulls
    c = class_size(size)
    if size > 4096:
        blocks = nseg * SEG // 65536                     # 64 KB blocks (A-2)
        assert 0.99 * blocks <= granted <= blocks
    else:
        cap = nseg * SEG // c
        slack = st["nslot"][max(0, (c.bit_length() - 1) - 4)] * 4096
        assert cap - slack <= granted <= cap
    _assert_pristine(G, nseg)
    # timed on its own: the malloc kernel alone
    G.gallatin_reset()
    p = torch.empty_like(d_sizes)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    G.gallatin_malloc(d_sizes, p)
    b.record()
    torch.cuda.synchronize()
    assert a.elapsed_time(b) < 1000.0, f"exhausting malloc took {a.elapsed_time(b):.1f} ms"
    G.gallatin_free(p)
    _assert_pristine(G, nseg)


def test_oom_record_cleared_by_frees(cuda_ok, G):
    """After a class was found exhausted, frees that return blocks make its
    memory allocatable again (the record's epoch moves), for the same class
    and for another one."""
    nseg = 4
    G.gallatin_init(nseg * SEG)
    cap16 = nseg * SEG // 16
    slack = G.gallatin_stats()["nslot"][0] * 4096
    sizes = _dev(wg.single_sizes(16, 2 * cap16))
    p = G.gallatin_malloc(sizes)
    torch.cuda.synchronize()
    got1 = int((p != 0).sum().item())
    assert cap16 - slack <= got1 <= cap16
    # free the first half of the array: whole blocks come back
    half = p[: cap16].clone()
    G.gallatin_free(half)
    q = G.gallatin_malloc(_dev(wg.single_sizes(16, cap16)))
    torch.cuda.synchronize()
    got2 = int((q != 0).sum().item())
    freed = int((half != 0).sum().item())
    assert got2 >= freed - 2 * slack, f"only {got2} of ~{freed} freed slices allocatable again"
    G.gallatin_free(p[cap16:].clone())
    G.gallatin_free(q)
    # exhausted by 16 B, everything freed: 1 KB requests get the heap
    G.gallatin_drain()
    r = G.gallatin_malloc(_dev(wg.single_sizes(1024, nseg * SEG // 1024)))
    torch.cuda.synchronize()
    got3 = int((r != 0).sum().item())
    assert got3 >= nseg * SEG // 1024 - G.gallatin_stats()["nslot"][6] * 4096
    G.gallatin_free(r)
    _assert_pristine(G, nseg)


# ---- the batch kernel of deferred big requests (k_big, DESIGN.md Deviations 21) ----
def _check_live(G, nseg, sizes_list, ptrs_list):
    """stamp / verify / usable / overlap over the union of several launches' pointers."""
    base = G.gallatin_stats()["heap_base"]
    ps, us = [], []
    for sizes, ptrs in zip(sizes_list, ptrs_list):
        d = _dev(sizes)
        G.gallatin_stamp(ptrs, d)
        assert G.gallatin_verify(ptrs, d) == 0, "stamp-verify found overwritten words"
        usable = torch.empty_like(ptrs)
        usum, ubad = G.gallatin_usable(ptrs, d, usable)
        assert ubad == 0
        p = _u64(ptrs)
        live = p != 0
        want = int(sum(class_size(int(s)) * int(c) for s, c in zip(*np.unique(sizes[live], return_counts=True))))
        assert usum == want
        ps.append(p[live])
        us.append(_u64(usable)[live])
    p, u = np.concatenate(ps), np.concatenate(us)
    order = np.argsort(p)
    assert np.all(p[order][:-1] + u[order][:-1] <= p[order][1:]), "overlapping allocations"
    assert np.all((p - np.uint64(base)) < np.uint64(nseg * SEG))


def test_deferred_big_requests_two_streams(cuda_ok, G):
    """Two bulk launches with whole-block and segment requests run at once on
    two streams: one claims the deferred-request queue, the other finds it
    taken and serves its big requests inline; every request is granted,
    disjoint, stamp-verified and accounted; free-all + drain is pristine."""
    nseg = 2048
    G.gallatin_init(nseg * SEG)
    n = (1 << 20) + 77                                   # the CTA kernel (>= 606,208 requests)
    sizes = [wg.mixed_sizes(n, seed=wg.cell_seed(3, 70 + k), p_large=2.0 ** -12) for k in range(2)]
    d = [_dev(s) for s in sizes]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    for s in streams:
        s.wait_stream(torch.cuda.current_stream())
    ptrs = []
    for k in range(2):
        with torch.cuda.stream(streams[k]):
            ptrs.append(G.gallatin_malloc(d[k], stream=streams[k].cuda_stream))
    torch.cuda.synchronize()
    assert all(int((p == 0).sum().item()) == 0 for p in ptrs)
    assert sum(int((s > 4096).sum()) for s in sizes) > 300   # both launches carry big requests
    _check_live(G, nseg, sizes, ptrs)
    for p in ptrs:
        G.gallatin_free(p)
    torch.cuda.synchronize()
    _assert_pristine(G, nseg)


def test_deferred_queue_overflow(cuda_ok, G):
    """More big requests than the queue holds (8192): the rest are served
    inline by their tiles; everything granted, disjoint, pristine after."""
    nseg = 1024
    G.gallatin_init(nseg * SEG)
    n = 1 << 20
    sizes = wg.single_sizes(64, n).copy()
    idx = wg.distinct_below(wg.cell_seed(3, 80), 12000, n).astype(np.int64)
    sizes[idx] = 65537                                   # 128 KB blocks of tree 1 (12000 x 128 KB = 1.5 GB)
    assert _bulk_round(G, nseg, sizes) == 0
    _assert_pristine(G, nseg)


def test_deferred_big_near_exhaustion(cuda_ok, G):
    """Segment and block requests that do not all fit (a 1 GB heap, 100 x 16 MB
    + 200 x 1 MB + 2^20 x 16 B): the batch claims fail, the per-request path
    grants what fits and returns NULL for the rest; the granted ones are
    disjoint and verified, and free-all + drain is pristine."""
    nseg = 64
    G.gallatin_init(nseg * SEG)
    n = 1 << 20
    sizes = wg.single_sizes(16, n).copy()
    idx = wg.distinct_below(wg.cell_seed(3, 81), 300, n).astype(np.int64)
    sizes[idx[:100]] = 16 << 20
    sizes[idx[100:]] = 1 << 20
    nulls = _bulk_round(G, nseg, sizes)
    assert 0 < nulls <= 300
    _assert_pristine(G, nseg)
