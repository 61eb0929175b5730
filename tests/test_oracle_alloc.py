"""Pins for O2, the sequential allocator oracle (oracle/alloc_oracle.c).

Each test checks O2 against something other than O2: numbers PAPER.md prints
(tests/golden/paper_geometry.txt), closed forms derived in the test from the
paper's rules, and invariants recomputed here in Python from the returned
offsets (in heap, aligned, non-overlapping, byte accounting, pristine image
after free-all + drain).
"""
import os

import numpy as np
import pytest

import oracle
import workload_gen as wg
from oracle import NONE, TREE_CONT, TREE_FREE, GID_NONE

SEG = 1 << 24
GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_geometry.txt")


def golden():
    out = {}
    for line in open(GOLDEN):
        line = line.split("#")[0].strip()
        if line:
            k, v = (s.strip() for s in line.split("="))
            out[k] = [int(x) for x in v.split(",")] if "," in v else int(v)
    return out


def class_size(size: int) -> int:
    """Usable bytes by the paper's carving, written out here independently:
    slices are powers of two >= 16 B, blocks are powers of two
    64 KB..16 MB (4096 slices; reading A-2), big requests take whole
    16 MB segments."""
    if size == 0:
        return 0
    if size <= 4096:
        return max(16, 1 << (size - 1).bit_length())
    if size < SEG:
        return max(1 << 16, 1 << (size - 1).bit_length())
    return -(-size // SEG) * SEG


def image_sections(img: np.ndarray) -> dict:
    """Split the canonical image (layout in include/gallatin.h)."""
    nseg, L, W, S = (int(x) for x in img[1:5])
    p = 8
    d = {"magic": int(img[0]), "nseg": nseg, "levels": L, "W": W, "nslots": S, "err": int(img[5])}
    d["segtree"] = img[p:p + W]; p += W
    d["btrees"] = img[p:p + 9 * W].reshape(9, W); p += 9 * W
    d["segword"] = img[p:p + nseg]; p += nseg
    q = img[p:p + nseg * 65].reshape(nseg, 65); p += nseg * 65
    d["qcount"] = q[:, 0]
    d["qentries"] = q[:, 1:].copy().view(np.uint16).reshape(nseg, 256)
    d["block_free"] = img[p:p + nseg * 128].copy().view(np.uint32); p += nseg * 128
    d["slots"] = img[p:p + S]; p += S
    d["next"] = img[p:p + S]; p += S
    assert p == len(img)
    return d


def pristine_image(nseg: int, nslots: int) -> np.ndarray:
    """The analytic pristine image: every segment free (bit 1 below nseg,
    summaries consistent), block trees empty, table FREE, rings empty,
    counters 0, slots empty (SURVEY 8(c) "Canonical image")."""
    W_levels = []
    w = (nseg + 63) // 64
    while True:
        W_levels.append(w)
        if w == 1:
            break
        w = (w + 63) // 64
    bits = np.zeros(W_levels[0] * 64, dtype=np.uint8)
    bits[:nseg] = 1
    levels = [np.packbits(bits, bitorder="little").view(np.uint64)]
    for wl in W_levels[1:]:
        nz = (levels[-1] != 0).astype(np.uint8)
        nz = np.concatenate([nz, np.zeros(wl * 64 - len(nz), dtype=np.uint8)])
        levels.append(np.packbits(nz, bitorder="little").view(np.uint64))
    W = sum(W_levels)
    out = [np.array([0x47414C4C494D4731, nseg, len(W_levels), W, nslots, 0, 0, 0], dtype=np.uint64)]
    out.append(np.concatenate(levels))
    out.append(np.zeros(9 * W, dtype=np.uint64))
    out.append(np.full(nseg, (TREE_FREE << 32), dtype=np.uint64))
    q = np.zeros((nseg, 65), dtype=np.uint64)
    q[:, 1:] = 0xFFFFFFFFFFFFFFFF
    out.append(q.reshape(-1))
    out.append(np.zeros(nseg * 128, dtype=np.uint64))
    out.append(np.full(nslots, (4096 << 32) | GID_NONE, dtype=np.uint64))
    out.append(np.full(nslots, GID_NONE, dtype=np.uint64))
    return np.concatenate(out)


def check_live_invariants(nseg, offs, sizes):
    """In heap, aligned to min(class size, 16 MB), non-overlapping; returns Σ usable."""
    offs = np.asarray(offs, dtype=np.uint64)
    use = np.array([class_size(int(s)) for s in sizes], dtype=np.uint64)
    assert np.all(offs + use <= np.uint64(nseg * SEG)), "outside heap"
    align = np.minimum(use, np.uint64(SEG))
    assert np.all(offs % align == 0), "misaligned"
    o = np.argsort(offs)
    so, su = offs[o], use[o]
    assert np.all(so[:-1] + su[:-1] <= so[1:]), "overlap"
    return int(use.sum())


def test_block_buffer_slots_match_paper_a40():
    """on the A40 the 16 B buffer holds 128 blocks, halving per class,
    capped below at four."""
    g = golden()
    a = oracle.Allocator(4, slot_base=128, slot_min=4)
    assert [a.nslot(c) for c in range(9)] == g["block_buffer_a40"]
    b = oracle.Allocator(4, slot_base=148, slot_min=4)        # B200: 148 SMs
    assert [b.nslot(c) for c in range(9)] == [148, 74, 37, 18, 9, 4, 4, 4, 4]


@pytest.mark.parametrize("size,blocks", [(16, "blocks_per_segment_16B"), (32, "blocks_per_segment_32B")])
def test_blocks_per_segment_and_in_order_slices(size, blocks):
    """256 blocks per segment at 16 B, 128 at 32 B; 4096 slices
    per block handed out in order; segments used front first.  With
    one slot, the k-th request lands at k*size exactly until the segment is
    full, then the next segment starts at 16 MB."""
    g = golden()
    nb = g[blocks]
    a = oracle.Allocator(4, slot_base=1, slot_min=1)
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


@pytest.mark.parametrize("seed,nseg,theta", [(1, 4, 0), (2, 8, 0), (3, 6, 2048), (4, 64, 0), (5, 5, 100)])
def test_random_sequences_tiny_heaps(seed, nseg, theta):
    """Random malloc/free/drain sequences on 4-64 segment heaps, including OOM:
    live allocations re-checked in Python, structure checked, and free-all +
    drain restores the analytic pristine image bit-exactly."""
    kinds, args, keys = wg.replay_ops(20_000, seed, p_free=0.45, p_drain=0.002, nkeys=64)
    a = oracle.Allocator(nseg, slot_base=16, slot_min=2, theta=theta)
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
