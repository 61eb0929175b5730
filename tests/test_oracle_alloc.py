"""Pins for O2, the sequential allocator oracle (oracle/alloc_oracle.c).

Each test checks O2 against something other than O2: numbers PAPER.md prints
(tests/golden/paper_geometry.txt), closed forms derived in the test from the
paper's rules, and invariants recomputed here in Python from the returned
offsets (in heap, aligned, non-overlapping, byte accounting, pristine image
after free-all + drain).
"""
import numpy as np
import pytest

import oracle
import workload_gen as wg
from oracle import NONE, TREE_CONT, TREE_FREE
from helpers import SEG, check_live_invariants, class_size, golden, image_sections, pristine_image


def test_block_buffer_slots_match_paper_a40():
    """on the A40 the 16 B buffer holds 128 blocks, halving per class,
    capped below at four."""
    g = golden()
    a = oracle.Allocator(4, slot_base=128, slot_min=4)
    assert [a.nslot(c) for c in range(9)] == g["block_buffer_a40"]
    b = oracle.Allocator(4, slot_base=148, slot_min=4)        # B200: 148 SMs
    assert [b.nslot(c) for c in range(9)] == [148, 74, 37, 18, 9, 4, 4, 4, 4]


@pytest.mark.parametrize("run_max,fa,pf", [(1, 0, 0), (16, 1, 1), (128, 0, 1)])
@pytest.mark.parametrize("size,blocks", [(16, "blocks_per_segment_16B"), (32, "blocks_per_segment_32B")])
def test_blocks_per_segment_and_in_order_slices(size, blocks, run_max, fa, pf):
    """256 blocks per segment at 16 B, 128 at 32 B; 4096 slices
    per block handed out in order; segments used front first.  With
    one slot, the k-th request lands at k*size exactly until the segment is
    full, then the next segment starts at 16 MB -- with one-block buffers
    (the paper) and with growing runs of consecutive blocks (ours)."""
    g = golden()
    nb = g[blocks]
    a = oracle.Allocator(4, slot_base=1, slot_min=1, run_max=run_max, format_ahead=fa, prefetch=pf)
    n = nb * g["slices_per_block"]
    offs = a.malloc_batch(np.full(n + 5, size, dtype=np.uint64), keydiv=0)
    assert np.array_equal(offs[:n], np.arange(n, dtype=np.uint64) * np.uint64(size))
    assert np.array_equal(offs[n:], np.uint64(SEG) + np.arange(5, dtype=np.uint64) * np.uint64(size))
    assert a.check() == 0


def test_free_returns_block_on_the_4096th_free():
    """the free whose counter was 4095 returns the block; the
    segment returns to the segment tree when all its blocks are back."""
    g = golden()
    a = oracle.Allocator(4, slot_base=1, slot_min=1)
    offs = a.malloc_batch(np.full(4096 + 1, 64, dtype=np.uint64), keydiv=0)   # block 0 full, block 1 started
    d = image_sections(a.image())
    assert d["segword"][0] >> 32 == 2                     # tree 2 (64 B slices)
    nb = 256 >> 2
    assert int(d["segword"][0]) & 0xFFFFFFFF == nb - 2      # two blocks out
    a.free_batch(offs[:4095])
    d = image_sections(a.image())
    assert d["block_free"][0] == g["free_return_old_value"]
    assert int(d["segword"][0]) & 0xFFFFFFFF == nb - 2
    a.free(int(offs[4095]))
    d = image_sections(a.image())
    assert d["block_free"][0] == 0
    assert int(d["segword"][0]) & 0xFFFFFFFF == nb - 1      # block 0 back in the ring
    assert list(d["qentries"][0][:2]) == [2, 3] and d["qentries"][0][nb - 2] == 0   # FIFO tail
    # free the last slice and drain: the segment goes back -> pristine
    a.free(int(offs[4096]))
    a.drain()
    assert np.array_equal(a.image(), pristine_image(4, 9))
    assert a.check() == 0


def test_large_allocations_come_from_the_back():
    """P:138 'pulled from the end ... first-fit ... predecessor'; P:235 tree id =
    numBlockTrees + numSegments; non-first segments marked CONT (A-18)."""
    a = oracle.Allocator(8)
    o1 = a.malloc(SEG, 0)                 # exactly 16 MB -> 1 segment (A-3)
    o2 = a.malloc(2 * SEG - 1, 0)         # 2 segments
    o3 = a.malloc(16, 0)                  # a slice: front segment 0
    o4 = a.malloc(3 * SEG, 0)
    assert (o1, o2, o3, o4) == (7 * SEG, 5 * SEG, 0, 2 * SEG)
    d = image_sections(a.image())
    tw = d["segword"] >> np.uint64(32)
    assert list(tw) == [0, TREE_FREE, 9 + 3, TREE_CONT, TREE_CONT, 9 + 2, TREE_CONT, 9 + 1]
    assert a.malloc(2 * SEG, 0) == NONE   # only segment 1 is free: no 2-run
    assert a.malloc(SEG, 0) == SEG
    a.free(o2)
    assert a.malloc(SEG + 1, 0) == 5 * SEG  # the freed run is reused, highest start
    assert a.check() == 0


def test_capacity_closed_form_single_class():
    """One slot, one class, empty heap: exactly nseg * (256 >> c) * 4096
    slices fit, then NULL."""
    for c, nseg in [(8, 4), (5, 2), (2, 1)]:
        size = 16 << c
        a = oracle.Allocator(nseg, slot_base=1, slot_min=1)
        cap = nseg * (256 >> c) * 4096
        offs = a.malloc_batch(np.full(cap + 3, size, dtype=np.uint64), keydiv=0)
        assert np.all(offs[:cap] != np.uint64(NONE))
        assert np.all(offs[cap:] == np.uint64(NONE))
        assert a.usable_live == cap * size == nseg * SEG


def test_accounting_matches_closed_form_mixed():
    sizes = wg.mixed_sizes(50_000, seed=5, p_large=2.0 ** -9)
    a = oracle.Allocator(256)
    offs = a.malloc_batch(sizes, keydiv=32)
    ok = offs != np.uint64(NONE)
    assert ok.all()
    total = check_live_invariants(256, offs, sizes)
    assert total == sum(class_size(int(s)) for s in sizes) == a.usable_live
    assert a.check() == 0
    a.free_batch(offs)
    a.drain()
    assert a.usable_live == 0 and a.live_count == 0
    assert np.array_equal(a.image(), pristine_image(256, 302))


@pytest.mark.parametrize("seed,nseg,run_max,fa,pf", [(1, 4, 1, 0, 0), (2, 8, 1, 0, 0), (3, 6, 16, 1, 1), (4, 64, 8, 1, 1),
                                                     (5, 5, 128, 0, 0), (6, 16, 4, 1, 0), (7, 32, 512, 1, 1)])
def test_random_sequences_tiny_heaps(seed, nseg, run_max, fa, pf):
    """Random malloc/free/drain sequences on 4-64 segment heaps, including OOM:
    live allocations re-checked in Python, structure checked, and free-all +
    drain restores the analytic pristine image bit-exactly."""
    kinds, args, keys = wg.replay_ops(20_000, seed, p_free=0.45, p_drain=0.002, nkeys=64)
    a = oracle.Allocator(nseg, slot_base=16, slot_min=2, run_max=run_max, run_bytes=32 << 20, format_ahead=fa,
                         prefetch=pf)
    out = a.replay(kinds, args, keys)
    live = {}
    for i, k in enumerate(kinds):
        if k == 0 and out[i] != np.uint64(NONE):
            live[i] = (int(out[i]), int(args[i]))
        elif k == 1:
            live.pop(int(args[i]), None)
    offs = [v[0] for v in live.values()]
    sizes = [v[1] for v in live.values()]
    if offs:
        assert check_live_invariants(nseg, offs, sizes) == a.usable_live
    assert a.check() == 0, oracle.violation_names(a.check())
    assert a.errors == 0
    nulls = sum(1 for i, k in enumerate(kinds) if k == 0 and out[i] == np.uint64(NONE))
    assert nulls > 0 or nseg >= 64   # the tiny heaps do hit OOM
    for o in offs:
        a.free(o)
    a.drain()
    S = sum(a.nslot(c) for c in range(9))
    assert np.array_equal(a.image(), pristine_image(nseg, S))


def test_errors_counted_for_foreign_frees():
    a = oracle.Allocator(2)
    a.free(5 * SEG)            # outside the heap
    a.free(SEG + 16)           # a FREE segment
    a.free(NONE)               # NULL: no-op
    assert a.errors == 2


def test_trim_gives_back_undrawn_blocks_before_oom():
    """DESIGN.md Deviations 5 (runs) + Alg.2's "no allocations left":
    a slot's whole-segment run must not starve another request.  On a
    one-segment heap the 16 B slot's first run takes all 256 blocks; a 64 KB
    block request then finds no segment, the slot keeps the ceil(1/4096) = 1
    block it has drawn from and gives back blocks 1..255 in order (FIFO ring,
    P:178), so the request gets block 1 at 64 KB, the next ones blocks 2..255,
    and only then NULL -- closed forms from the paper's layout."""
    a = oracle.Allocator(1, slot_base=1, slot_min=1, run_max=256, run_bytes=16 << 20, run_init=256, run_grow=3)
    assert a.malloc(16, 0) == 0
    d = image_sections(a.image())
    assert int(d["segword"][0]) & 0xFFFFFFFF == 0                 # all 256 blocks held by the run
    blocks = [a.malloc(65536, 0) for _ in range(255)]
    assert blocks == [j * 65536 for j in range(1, 256)]
    assert a.malloc(16, 0) == 16                                   # the kept block still serves the slot
    assert a.malloc(65536, 0) == NONE                              # nothing left to give back
    d = image_sections(a.image())
    assert int(d["slots"][0]) >> 32 == 2 and (int(d["slots"][0]) >> 22) & 0x3FF == 1
    for off in [0, 16] + blocks:
        a.free(off)
    a.drain()
    img = a.image()
    assert a.check() == 0
    assert np.array_equal(img, pristine_image(1, int(img[4])))


@pytest.mark.parametrize("run_grow", [1, 2, 3, 8])
def test_run_growth_factor(run_grow):
    """A refilled run is 2^run_grow times the last (capped): with one 16 B slot
    and first run 1 block, the k-th run starts right after the (k-1)-th, so the
    addresses stay consecutive and the slot's run length after
    r refills is min(2^(run_grow*r), cap) -- the closed form, read from the
    image's slot word."""
    cap = 64
    a = oracle.Allocator(4, slot_base=1, slot_min=1, run_max=cap, run_bytes=64 << 20, run_init=1, run_grow=run_grow)
    m, total = 1, 0
    for r in range(4):
        total += m * 4096
        offs = a.malloc_batch(np.full(m * 4096 if r else 4096, 16, dtype=np.uint64), keydiv=0)
        assert offs[-1] == (total - 1) * 16
        d = image_sections(a.image())
        assert (int(d["slots"][0]) >> 22) & 0x3FF == m
        m = min(m << run_grow, cap)
    assert a.check() == 0


def test_shared_run_keeps_longest_consecutive_blocks():
    """DESIGN.md Deviations 5: a run taken from a block-tree segment keeps the
    longest run of consecutive block indices among the ring entries it
    dequeues (lowest start on ties), not the FIFO prefix.  One segment, one
    64 B slot whose first run is the whole segment (64 blocks of 256 KB,
    P:174); its 64*4096 slices are drawn, then every block except 9 is
    freed in the order 30..63, 0..8, 10..29 (ring order).  The refill
    (want = cap = 64) dequeues those 63 entries and keeps 10..63 (54 blocks),
    re-enqueueing 0..8; the prefix rule would have kept 30..63."""
    bb = 64 * 4096                                            # 64 B slices: 256 KB blocks
    a = oracle.Allocator(1, slot_base=1, slot_min=1, run_max=64, run_bytes=16 << 20, run_init=256, run_grow=1)
    offs = a.malloc_batch(np.full(64 * 4096, 64, dtype=np.uint64), keydiv=0)
    assert np.array_equal(offs, np.arange(64 * 4096, dtype=np.uint64) * np.uint64(64))
    for b in list(range(30, 64)) + list(range(0, 9)) + list(range(10, 30)):
        a.free_batch(offs[b * 4096:(b + 1) * 4096])
    nxt = a.malloc_batch(np.full(54 * 4096 + 1, 64, dtype=np.uint64), keydiv=0)
    assert np.array_equal(nxt[:-1], np.uint64(10 * bb) + np.arange(54 * 4096, dtype=np.uint64) * np.uint64(64))
    assert nxt[-1] == 0                                       # then blocks 0..8: the next longest run
    d = image_sections(a.image())
    w = int(d["slots"][2])                                    # one slot per class: class 2's
    assert (w >> 22) & 0x3FF == 9 and w & 0x3FFFFF == 0 and w >> 32 == 1
    assert a.check() == 0


@pytest.mark.parametrize("size", [4, 16, 64, 256, 4096, 8192, 1 << 20, 1 << 24, 3 << 24])
def test_utilization_closed_form(size):
    """E8: batches of 100,000 allocations of one size until
    the first NULL.  Closed forms from the paper's geometry on an empty heap of
    nseg segments: a slice class has nseg * (256 >> c) * 4096 slices (P:188,
    P:264) of which at most one partly drawn block per block-buffer slot
     is left unissued; a whole-block request (reading A-2) gets exactly
    nseg * (256 >> t) blocks; a k-segment request exactly floor(nseg / k)
    (P:138)."""
    nseg = 8
    a = oracle.Allocator(nseg, slot_base=148, slot_min=4, run_max=256, run_init=64, run_grow=3,
                         run_bytes=256 << 20, format_ahead=1)
    succ = 0
    while True:
        o = a.malloc_batch(np.full(100_000, size, dtype=np.uint64), keydiv=32)
        ok = int((o != NONE).sum())
        succ += ok
        if ok < len(o):
            break
    assert a.check() == 0
    if size <= 4096:
        c = max(0, (size - 1).bit_length() - 4)
        total = nseg * (256 >> c) * 4096
        assert total - a.nslot(c) * 4096 <= succ <= total
    elif size < SEG:
        t = max(0, (size - 1).bit_length() - 16)
        assert succ == nseg * (256 >> t)
    else:
        assert succ == nseg // -(-size // SEG)


@pytest.mark.parametrize("seed,nseg,run_max,fa,pf", [(21, 2, 1, 0, 0), (22, 3, 16, 1, 1), (23, 4, 64, 1, 0),
                                                     (24, 2, 256, 0, 1), (25, 6, 8, 1, 1)])
def test_exhaustion_record_is_exact(seed, nseg, run_max, fa, pf):
    """DESIGN.md Deviations 11: a request failed by the exhaustion record is
    one the full search (trims + retry) would fail too.  O2 checks every
    record-failed request against a side-effect-free dry run of that search
    (violation bit 512); heavy pressure on 2-6 segment heaps makes records
    fire thousands of times; free-all + drain is still pristine."""
    kinds, args, keys = wg.replay_ops(30_000, seed, p_free=0.3, p_drain=0.001, nkeys=64)
    a = oracle.Allocator(nseg, slot_base=16, slot_min=2, run_max=run_max, run_bytes=32 << 20, format_ahead=fa,
                         prefetch=pf)
    out = a.replay(kinds, args, keys)
    assert a.oom_fast > 100, "the record never fired"
    assert a.check() == 0, oracle.violation_names(a.check())
    freed = {int(args[i]) for i, k in enumerate(kinds) if k == 1}
    for i, k in enumerate(kinds):
        if k == 0 and out[i] != np.uint64(NONE) and i not in freed:
            a.free(int(out[i]))
    a.drain()
    S = sum(a.nslot(c) for c in range(9))
    assert np.array_equal(a.image(), pristine_image(nseg, S))


def test_exhaustion_record_cleared_by_a_block_return():
    """Closed form on a one-segment heap with one slot per class (P:134,
    P:188): 2^20 16 B slices fill it; the next 16 B and 64 KB requests fail
    (the second by the record); freeing 4095 slices of block 0 returns
    nothing and the record stands; the 4096th free returns block 0,
    the record is cleared, and the next 16 B request gets it again."""
    a = oracle.Allocator(1, slot_base=1, slot_min=1, run_max=256, run_bytes=16 << 20, run_init=256, run_grow=3)
    offs = a.malloc_batch(np.full(1 << 20, 16, dtype=np.uint64))
    assert np.array_equal(offs, np.arange(1 << 20, dtype=np.uint64) * 16)
    assert a.malloc(16, 0) == NONE
    f0 = a.oom_fast
    assert a.malloc(65536, 0) == NONE and a.oom_fast == f0 + 1
    for o in offs[:4095]:
        a.free(int(o))
    assert a.malloc(16, 0) == NONE and a.oom_fast == f0 + 2
    a.free(int(offs[4095]))
    assert a.malloc(16, 0) == 0                    # block 0 again, slice 0
    assert a.check() == 0
