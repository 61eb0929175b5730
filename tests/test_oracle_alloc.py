"""Pins for O2, the sequential allocator oracle (oracle/alloc_*.c).

O2-P (``oracle.Allocator``, alloc_paper.c) is the paper's policy POL; O2-R
(``oracle.RunsAllocator``, alloc_runs.c) is the deviation model (DESIGN.md
Deviations 5, 8).  Each test checks O2 against something other than O2:
numbers PAPER.md prints (tests/golden/paper_geometry.txt), closed forms
derived in the test from the paper's rules, invariants recomputed here in
Python from the returned offsets, and a naive brute-force simulation written
from the policy text (tests/pol_sim.py).  DESIGN.md 11 lists which test pins
which O2 function.
"""
import numpy as np
import pytest

import oracle
import workload_gen as wg
from helpers import SEG, check_live_invariants, class_size, diff_images, golden, image_sections, pristine_image
from oracle import NONE, TREE_CONT, TREE_FREE
from pol_sim import PolSim


def runs(nseg, **kw):
    kw.setdefault("run_bytes", 32 << 20)
    return oracle.RunsAllocator(nseg, **kw)


# ------------------------------------------------------------ O2-P (POL) ---
def test_block_buffer_slots_match_paper_a40():
    """on the A40 the 16 B buffer holds 128 blocks, halving per class,
    capped below at four."""
    g = golden()
    a = oracle.Allocator(4, slot_base=128, slot_min=4)
    assert [a.nslot(c) for c in range(9)] == g["block_buffer_a40"]
    b = oracle.Allocator(4, slot_base=148, slot_min=4)        # B200: 148 SMs
    assert [b.nslot(c) for c in range(9)] == [148, 74, 37, 18, 9, 4, 4, 4, 4]


@pytest.mark.parametrize("knobs", [None, dict(run_max=16, format_ahead=1, prefetch=1),
                                   dict(run_max=64, prefetch=1)])
@pytest.mark.parametrize("size,blocks", [(16, "blocks_per_segment_16B"), (32, "blocks_per_segment_32B")])
def test_blocks_per_segment_and_in_order_slices(size, blocks, knobs):
    """256 blocks per segment at 16 B, 128 at 32 B; 4096 slices
    per block handed out in order; segments used front first.  With
    one slot, the k-th request lands at k*size exactly until the segment is
    full, then the next segment starts at 16 MB -- with one-block buffers
    (O2-P, the paper) and with growing runs of consecutive blocks (O2-R)."""
    g = golden()
    nb = g[blocks]
    a = oracle.Allocator(4, slot_base=1, slot_min=1) if knobs is None else runs(4, slot_base=1, slot_min=1, **knobs)
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


def test_size_classes_rounding_and_zero():
    """A-1..A-4 closed forms: malloc(0) is NULL; 1 and 16 B share the 16 B
    class, 17 B takes 32 B, 4095 B the 4 KB class; 4097 B a
    whole 64 KB block of the tree the 16 B slices use (A-1, A-2); exactly 16 MB one segment (A-3) from the back
    (P:138), 16 MB + 1 two segments."""
    a = oracle.Allocator(8, slot_base=1, slot_min=1)
    assert a.malloc(0, 0) == NONE and a.live_count == 0
    assert [a.malloc(s, 0) for s in (1, 16, 5)] == [0, 16, 32]               # one 16 B block, in order
    assert a.malloc(17, 0) == SEG                                             # 32 B class: next segment
    assert a.malloc(4095, 0) == 2 * SEG and a.malloc(4096, 0) == 2 * SEG + 4096
    assert a.malloc(4097, 0) == 65536          # a whole 64 KB block of tree 0: block 1 of segment 0 (A-2)
    assert a.malloc(SEG, 0) == 7 * SEG
    assert a.malloc(SEG + 1, 0) == 5 * SEG
    d = image_sections(a.image())
    assert list(d["segword"][5:8] >> np.uint64(32)) == [9 + 2, TREE_CONT, 9 + 1]
    assert a.usable_live == 3 * 16 + 32 + 2 * 4096 + 65536 + 3 * SEG
    assert [oracle.usable_size(s) for s in (0, 1, 17, 4095, 4097, SEG, SEG + 1)] == \
        [class_size(s) for s in (0, 1, 17, 4095, 4097, SEG, SEG + 1)]
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


@pytest.mark.parametrize("model", ["paper", "runs"])
def test_accounting_matches_closed_form_mixed(model):
    sizes = wg.mixed_sizes(50_000, seed=5, p_large=2.0 ** -9)
    a = oracle.Allocator(256) if model == "paper" else runs(256, run_max=256, format_ahead=1, run_init=8, run_grow=3)
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


@pytest.mark.parametrize("seed,nseg,knobs", [(1, 4, None), (2, 8, None), (3, 6, dict(run_max=16, format_ahead=1, prefetch=1)),
                                             (4, 64, dict(run_max=8, format_ahead=1, prefetch=1)),
                                             (5, 5, dict(run_max=128)), (6, 16, dict(run_max=4, format_ahead=1)),
                                             (7, 32, dict(run_max=512, format_ahead=1, prefetch=1))])
def test_random_sequences_tiny_heaps(seed, nseg, knobs):
    """Random malloc/free/drain sequences on 4-64 segment heaps, including OOM:
    live allocations re-checked in Python, structure checked, and free-all +
    drain restores the analytic pristine image bit-exactly."""
    kinds, args, keys = wg.replay_ops(20_000, seed, p_free=0.45, p_drain=0.002, nkeys=64)
    a = oracle.Allocator(nseg, 16, 2) if knobs is None else runs(nseg, slot_base=16, slot_min=2, **knobs)
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
    nulls = sum(1 for i, k in enumerate(kinds) if k == 0 and out[i] == np.uint64(NONE) and args[i] != 0)
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


# --------------------------------------------- brute-force simulation pin ---
SIM_CASES = [
    (11, 3, 16, 2, None), (12, 4, 16, 2, None), (13, 8, 16, 2, None), (14, 6, 4, 1, None), (15, 2, 148, 4, None),
    (16, 6, 16, 2, dict(run_max=16, format_ahead=1, prefetch=1)),
    (17, 5, 16, 2, dict(run_max=128)),
    (18, 16, 16, 2, dict(run_max=4, format_ahead=1)),
    (19, 3, 16, 2, dict(run_max=512, run_init=256, run_grow=4, format_ahead=1, prefetch=1)),
    (20, 6, 16, 2, dict(run_max=256, run_init=64, run_grow=8, prefetch=1)),
    (21, 4, 1, 1, dict(run_max=256, run_init=256, run_grow=3, format_ahead=1)),
    # production-shaped knobs (gallatin_init defaults at 64 segments): 148 slots at 16 B,
    # runs up to 256 blocks / 16 MB, format-ahead, x8 growth, first runs of 4 blocks
    (22, 64, 148, 4, dict(run_max=256, run_bytes=16 << 20, run_init=4, run_grow=3, format_ahead=1)),
    # prefilled block buffers (R7): the paper's one-block slots, and the production-shaped knobs
    (23, 96, 16, 2, dict(prefill=1)),
    (24, 256, 148, 4, dict(run_max=256, run_bytes=16 << 20, run_init=4, run_grow=3, format_ahead=1, prefill=1)),
    (25, 128, 16, 2, dict(run_max=512, run_init=16, run_grow=3, prefetch=1, prefill=1)),
]


@pytest.mark.parametrize("seed,nseg,sb,sm,knobs", SIM_CASES)
def test_o2_matches_brute_force_simulation(seed, nseg, sb, sm, knobs):
    """Every offset and the whole canonical image after a random op list
    (slices of every class, non-power-of-two sizes, malloc(0), whole blocks,
    1 and 2+ segments, frees, drains, OOM) equal a naive simulation written
    from the policy text (tests/pol_sim.py: set scans instead of vEB trees,
    deques for rings) -- for O2-P at the paper's knobs and O2-R at run /
    format-ahead / prefetch / trim settings."""
    kinds, args, keys = wg.replay_ops(4000 if nseg < 64 else 6000, seed, p_free=0.45, p_drain=0.003, nkeys=64)
    kw = dict(knobs or {})
    if knobs is not None:
        kw.setdefault("run_bytes", 32 << 20)
    sim = PolSim(nseg, sb, sm, **kw)
    a = oracle.model(nseg, slot_base=sb, slot_min=sm, **kw)
    assert isinstance(a, oracle.RunsAllocator) == (knobs is not None)
    if kw.get("prefill"):
        assert a.image()[8] != pristine_image(nseg, int(a.image()[4]))[8], "the prefill must apply"
    want = sim.replay(kinds, args, keys)
    got = a.replay(kinds, args, keys)
    bad = np.nonzero(got != want)[0]
    assert len(bad) == 0, f"op {bad[0]} (kind {kinds[bad[0]]}, arg {args[bad[0]]}): o2 {got[bad[0]]:#x} sim {want[bad[0]]:#x}"
    msg = diff_images(a.image(), sim.image())
    assert not msg, msg
    assert (got == NONE).sum() > (kinds == 0).sum() // 20 or nseg >= 64     # OOM exercised on the tiny heaps


@pytest.mark.parametrize("mutant", ["lifo_ring", "back_first_blocks", "tree_off_by_one"])
def test_brute_force_simulation_detects_mutants(mutant, monkeypatch):
    """The simulation pin has teeth: a plausible mistake in the policy -- a
    LIFO ring (A-15), block segments taken from the back, a block
    tree that drops segments with a single block available (off by one in
    A-16) -- makes the simulation disagree with O2-P on the same op list."""
    import pol_sim
    from collections import deque

    if mutant == "lifo_ring":
        def return_block(self, s, j):
            self.ring[s].appendleft(j)
            if len(self.ring[s]) == pol_sim.nb(self.tree[s]):
                self.tree[s] = pol_sim.FREE
                self.ring[s] = deque()
        monkeypatch.setattr(PolSim, "return_block", return_block)
    elif mutant == "back_first_blocks":
        monkeypatch.setattr(PolSim, "free_segs", lambda self: [s for s in range(self.nseg - 1, -1, -1)
                                                               if self.tree[s] == pol_sim.FREE])
    else:
        monkeypatch.setattr(PolSim, "tree_segs", lambda self, t: [s for s in range(self.nseg) if self.tree[s] == t
                                                                  and len(self.ring[s]) > 1])
    kinds, args, keys = wg.replay_ops(4000, 11, p_free=0.45, p_drain=0.003, nkeys=64)
    sim = PolSim(3, 16, 2)
    a = oracle.Allocator(3, 16, 2)
    same = np.array_equal(sim.replay(kinds, args, keys), a.replay(kinds, args, keys)) and \
        np.array_equal(sim.image(), a.image())
    assert not same, f"the {mutant} mutant went unnoticed"


@pytest.mark.parametrize("seed,nseg", [(31, 3), (32, 8), (33, 32)])
def test_runs_model_at_paper_knobs_equals_paper_core(seed, nseg):
    """O2-R with run_max = run_init = 1, no format-ahead, no prefetch is the
    paper's one-block buffer: offsets and images equal O2-P's (its trims
    give back nothing when every run is one partly drawn block)."""
    kinds, args, keys = wg.replay_ops(8000, seed, p_free=0.45, p_drain=0.003, nkeys=64)
    a, b = oracle.Allocator(nseg, 16, 2), runs(nseg, slot_base=16, slot_min=2, run_max=1, run_init=1)
    assert np.array_equal(a.replay(kinds, args, keys), b.replay(kinds, args, keys))
    assert np.array_equal(a.image(), b.image())


# --------------------------------------------------- O2-R closed forms ---
def test_trim_gives_back_undrawn_blocks_before_oom():
    """R5 (DESIGN.md Deviations 8) + Alg.2's "no allocations left":
    a slot's whole-segment run must not starve another request.  On a
    one-segment heap the 16 B slot's first run takes all 256 blocks; a 64 KB
    block request then finds no segment, the slot keeps the ceil(1/4096) = 1
    block it has drawn from and gives back blocks 1..255 in order (FIFO ring,
    P:178), so the request gets block 1 at 64 KB, the next ones blocks 2..255,
    and only then NULL -- closed forms from the paper's layout."""
    a = runs(1, slot_base=1, slot_min=1, run_max=256, run_bytes=16 << 20, run_init=256, run_grow=3)
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
    """R1: a refilled run is 2^run_grow times the last (capped): with one 16 B
    slot and first run 1 block, the k-th run starts right after the (k-1)-th,
    so the addresses stay consecutive and the slot's run length
    after r refills is min(2^(run_grow*r), cap) -- the closed form, read from
    the image's slot word."""
    cap = 64
    a = runs(4, slot_base=1, slot_min=1, run_max=cap, run_bytes=64 << 20, run_init=1, run_grow=run_grow)
    m, total = 1, 0
    for r in range(4):
        total += m * 4096
        offs = a.malloc_batch(np.full(m * 4096 if r else 4096, 16, dtype=np.uint64), keydiv=0)
        assert offs[-1] == (total - 1) * 16
        d = image_sections(a.image())
        assert (int(d["slots"][0]) >> 22) & 0x3FF == m
        m = min(m << run_grow, cap)
    assert a.check() == 0


@pytest.mark.parametrize("run_init,c,want", [(1, 0, 1), (4, 0, 4), (256, 0, 256), (256, 3, 32), (256, 8, 1),
                                             (64, 5, 8), (64, 4, 8), (2, 7, 2)])
def test_first_run_length(run_init, c, want):
    """R1 first run: min(max(run_init >> c, min(run_init, 8)), 256 >> c)
    blocks -- read from the slot word after one request of class c."""
    a = runs(8, slot_base=1, slot_min=1, run_max=512, run_bytes=1 << 30, run_init=run_init, run_grow=1)
    assert a.malloc(16 << c, 0) == 0
    w = int(image_sections(a.image())["slots"][c])
    assert (w >> 22) & 0x3FF == want and w >> 32 == 1 and w & 0x3FFFFF == 0


def test_shared_run_keeps_longest_consecutive_blocks():
    """R2: a run taken from a block-tree segment keeps the longest run of
    consecutive block indices among the ring entries it dequeues (lowest
    start on ties), not the FIFO prefix.  One segment, one 64 B slot whose
    first run is the whole segment (64 blocks of 256 KB); its
    64*4096 slices are drawn, then every block except 9 is freed in the order
    30..63, 0..8, 10..29 (ring order).  The refill (want = cap = 64)
    dequeues those 63 entries and keeps 10..63 (54 blocks), re-enqueueing
    0..8; the prefix rule would have kept 30..63."""
    bb = 64 * 4096                                            # 64 B slices: 256 KB blocks
    a = runs(1, slot_base=1, slot_min=1, run_max=64, run_bytes=16 << 20, run_init=256, run_grow=1)
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


def test_whole_segment_runs_taken_privately():
    """R2 (>= nb blocks): a run of whole segments takes the lowest free
    segment and the free ones right after it, with no ring and no block-tree
    entry.  4 segments; two 16 MB requests take 3 and 2 from the back
    (P:138); the 16 B slot's first run is segment 0 (256 blocks, 1 MB run
    cap 512 blocks), its refill wants 512 blocks = 2 segments but only
    segment 1 is free before the taken ones, so the run is 256 blocks at
    segment 1 -- and slices stay consecutive across the boundary."""
    a = runs(4, slot_base=1, slot_min=1, run_max=512, run_bytes=32 << 20, run_init=256, run_grow=1)
    assert [a.malloc(SEG, 0), a.malloc(SEG, 0)] == [3 * SEG, 2 * SEG]
    n = (1 << 20) + 3
    offs = a.malloc_batch(np.full(n, 16, dtype=np.uint64), keydiv=0)
    assert np.array_equal(offs, np.arange(n, dtype=np.uint64) * np.uint64(16))
    d = image_sections(a.image())
    assert list(d["segword"][:2]) == [0, 0]                   # tree 0, no block available, both
    assert not d["btrees"].any() and int(d["qcount"][:2].sum()) == 0
    w = int(d["slots"][0])
    assert (w >> 22) & 0x3FF == 256 and w & 0x3FFFFF == 256 and w >> 32 == 3   # second run: segment 1
    assert int(d["segtree"][0]) == 0                          # no segment free
    assert a.malloc(16, 0) == (1 << 20) * 16 + 3 * 16 and a.check() == 0


def test_whole_segment_runs_prefer_fresh_segments():
    """R2: a run of >= nb blocks is taken from fresh segments while any is
    free, not from a partly returned segment of the block tree (which would
    give a run as short as its available blocks -- the warm-state refills).
    One 2 KB slot (8 MB blocks, nb = 2), runs of 1 then 2 blocks: the first
    run is block 0 of segment 0 (block 1 published in the ring), the second
    run wants 2 >= nb: segment 1 whole, not block 1 of segment 0; a whole
    8 MB block request (tree 7, want 1 < nb) still takes segment 0's block 1."""
    a = runs(4, slot_base=1, slot_min=1, run_max=2, run_bytes=32 << 20, run_init=1, run_grow=1)
    bb = 8 << 20
    offs = a.malloc_batch(np.full(4096 + 1, 2048, dtype=np.uint64), keydiv=0)
    assert offs[4095] == 4095 * 2048 and offs[4096] == SEG          # second run: segment 1, not block 1
    w = int(image_sections(a.image())["slots"][7])
    assert (w >> 22) & 0x3FF == 2 and w & 0x3FFFFF == 2             # run of 2 from linear block 2
    assert a.malloc(bb, 0) == bb                                      # block path: segment 0's block 1
    assert a.check() == 0


def test_prefill_layout_closed_form():
    """R7 ("always populated"): with run_init 64 every class's slots
    start with runs of min(max(64 >> c, 8), nb(c)) blocks = 64, 32, 16, 8, 8,
    8, 4, 2, 1 (R1), laid out class by class from segment 0: 4 slots of 16 B
    fill segment 0; 2 slots x 32 of the 128 32-B blocks use half of segment 1,
    whose other 64 blocks stay in its ring (ascending) and block tree 1; ...;
    13 segments in all (<= 128 / 8), the rest free.  The first
    16 B request of slot 1 lands at block 64 of segment 0."""
    a = runs(128, slot_base=4, slot_min=2, run_max=512, run_bytes=1 << 30, run_init=64, prefill=1)
    d = image_sections(a.image())
    runs_ = [64, 32, 16, 8, 8, 8, 4, 2, 1]
    nslot = [4, 2, 2, 2, 2, 2, 2, 2, 2]
    segs = [-(-n * r // (256 >> c)) for c, (n, r) in enumerate(zip(nslot, runs_))]
    assert segs == [1, 1, 1, 1, 1, 2, 2, 2, 2]
    base = np.cumsum([0] + segs)
    slots = d["slots"]
    for c in range(9):
        for q in range(nslot[c]):
            w = int(slots[sum(nslot[:c]) + q])
            assert w == (runs_[c] << 22) | (int(base[c]) * (256 >> c) + q * runs_[c]), (c, q, hex(w))
    assert int(d["segtree"][0]) == ((1 << 64) - 1) & ~((1 << 13) - 1) and int(d["segtree"][1]) == (1 << 64) - 1
    assert int(d["segword"][1]) == (1 << 32) | 64 and int(d["btrees"][1][0]) == 1 << 1
    assert list(d["qentries"][1][:2]) == [64, 65] and int(d["qcount"][1]) == 64
    assert int(d["segword"][0]) == 0 and int(d["segword"][5]) == (5 << 32)   # full segments: avail 0
    assert a.malloc(16, 1) == 64 * 65536 and a.check() == 0
    a.free(64 * 65536)
    a.drain()
    assert np.array_equal(a.image(), pristine_image(128, 20))


def test_prefill_budget():
    """R7's budget nseg / 8.  Runs start at the largest power of two <= the
    first run: 256 blocks at 16 B (2 slots = 2 segments), one segment for
    each other class: 10 in all.  An 80-segment heap (budget 10) takes them
    as they are (16 B slot 1 at block 256 = segment 1).  On 72 segments
    (budget 9) the class with the most segments -- 16 B -- is halved once,
    to 128 >= 256 >> run_grow: both 16 B runs in segment 0.  With run_grow 1
    the floor is 128 too; on 64 segments (budget 8) nothing can be halved
    below the floors (each class still needs a segment): no prefill."""
    b = runs(80, slot_base=2, slot_min=1, run_max=512, run_bytes=1 << 30, run_init=256, run_grow=3, prefill=1)
    d = image_sections(b.image())
    assert [int(w) for w in d["slots"][:2]] == [256 << 22, (256 << 22) | 256]
    assert [int(w) >> 32 for w in d["segword"][:11]] == [0, 0] + list(range(1, 9)) + [TREE_FREE]
    h = runs(72, slot_base=2, slot_min=1, run_max=512, run_bytes=1 << 30, run_init=256, run_grow=3, prefill=1)
    d = image_sections(h.image())
    assert [int(w) for w in d["slots"][:2]] == [128 << 22, (128 << 22) | 128]
    assert [int(w) >> 32 for w in d["segword"][:10]] == list(range(9)) + [TREE_FREE]
    c = runs(64, slot_base=2, slot_min=1, run_max=512, run_bytes=1 << 30, run_init=256, run_grow=1, prefill=1)
    assert np.array_equal(c.image(), pristine_image(64, 10))
    e = runs(80, slot_base=2, slot_min=1, run_max=100, run_bytes=1 << 30, run_init=256, prefill=1)
    assert int(image_sections(e.image())["slots"][0]) >> 22 == 64                # 100 -> 64 (power of two)


def test_prefill_skipped_when_it_does_not_fit():
    """R7 / reading A-19: a buffer that does not fit in nseg / 8 segments is
    not prefilled (a 64 MB heap cannot hold one
    block of every class for every slot): the initial image is pristine."""
    a = runs(4, slot_base=148, slot_min=4, run_max=256, run_init=1, prefill=1)
    assert np.array_equal(a.image(), pristine_image(4, 302))


def test_format_ahead_closed_form():
    """R3: the reservation that takes a segment's available blocks from >= nb/4
    to < nb/4 formats the next segment of its tree.  One 16 B slot (nb = 256,
    nb/4 = 64), runs of 1, 2, 4, 8, then 16 blocks (run_max 16): the first
    comes from a fresh segment (no format-ahead there), the run that takes
    blocks 191..206 leaves 49 < 64 of 65: the refill at slice 191 * 4096
    formats segment 1 (tree 0, 256 available, in block tree 0)."""
    a = runs(4, slot_base=1, slot_min=1, run_max=16, run_bytes=32 << 20, format_ahead=1, run_init=1, run_grow=1)
    a.malloc_batch(np.full(191 * 4096, 16, dtype=np.uint64), keydiv=0)
    d = image_sections(a.image())
    assert int(d["segword"][1]) >> 32 == TREE_FREE and int(d["segword"][0]) & 0xFFFFFFFF == 256 - 191
    assert a.malloc(16, 0) == 191 * 65536
    d = image_sections(a.image())
    assert int(d["segword"][0]) & 0xFFFFFFFF == 256 - 207
    assert int(d["segword"][1]) == (0 << 32) | 256 and int(d["btrees"][0][0]) == 0b11
    assert list(d["qentries"][1][:3]) == [0, 1, 2] and int(d["qcount"][1]) == 256
    assert a.check() == 0


def test_prefetch_closed_form():
    """R4: the request drawing the middle of a run (index 2048 of a one-block
    run) fetches the next run -- 2^run_grow times as long -- into the slot's
    second word; the run's end swaps it in and the slices stay consecutive.
    One 16 B slot, runs of 1, 2, 4 blocks from segment 0's ring."""
    a = runs(4, slot_base=1, slot_min=1, run_max=16, run_bytes=32 << 20, prefetch=1, run_init=1, run_grow=1)
    a.malloc_batch(np.full(2048, 16, dtype=np.uint64), keydiv=0)
    assert int(image_sections(a.image())["next"][0]) == 0x3FFFFF              # not yet
    a.malloc(16, 0)                                                          # draws index 2048
    assert int(image_sections(a.image())["next"][0]) == (2 << 22) | 1        # blocks 1..2
    offs = a.malloc_batch(np.full(2047 + 1, 16, dtype=np.uint64), keydiv=0)  # to the run's end + 1
    assert offs[-1] == 4096 * 16
    d = image_sections(a.image())
    assert int(d["slots"][0]) == (1 << 32) | (2 << 22) | 1                 # one slice of blocks 1..2 drawn
    assert int(d["next"][0]) == 0x3FFFFF
    a.malloc_batch(np.full(4095, 16, dtype=np.uint64), keydiv=0)            # index 4096 of the 2-block run next
    a.malloc(16, 0)
    assert int(image_sections(a.image())["next"][0]) == (4 << 22) | 3        # blocks 3..6
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
    a = runs(nseg, slot_base=148, slot_min=4, run_max=256, run_init=64, run_grow=3, run_bytes=256 << 20,
             format_ahead=1)
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
