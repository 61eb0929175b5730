"""Pins for O1, the textbook vEB oracle (oracle/veb_oracle.c).

The oracle is checked against things other than itself (SURVEY 8(c) "What
pins each part"): brute force over every subset of a 2^4 universe, random
op sequences against a sorted Python list on 2^6..2^12 universes (BASELINE
north_star: "checked by brute force on universes up to 2^12"), closed forms
(empty / full / singleton sets), and the paper's level geometry.
"""
import bisect
import os

import numpy as np
import pytest

import oracle
from oracle import NONE, OV_DELETE, OV_INSERT, OV_MEMBER, OV_PRED, OV_SUCC

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "paper_geometry.txt")


def golden():
    out = {}
    for line in open(GOLDEN):
        line = line.split("#")[0].strip()
        if line:
            k, v = (s.strip() for s in line.split("="))
            out[k] = [int(x) for x in v.split(",")] if "," in v else int(v)
    return out


def _brute_tables(u):
    """succ_ge / pred_le / member of every (mask, x) for a 2^4 universe, by brute force."""
    masks = np.arange(1 << u, dtype=np.int64)
    xs = np.arange(u)
    bits = (masks[:, None] >> np.arange(u)[None, :]) & 1        # [mask, element]
    succ = np.full((1 << u, u), NONE, dtype=np.uint64)
    pred = np.full((1 << u, u), NONE, dtype=np.uint64)
    for x in xs:
        for y in range(u - 1, x - 1, -1):                         # smallest y >= x wins
            succ[bits[:, y] == 1, x] = y
        for y in range(0, x + 1):                                 # largest y <= x wins
            pred[bits[:, y] == 1, x] = y
    return bits.astype(np.uint64), succ, pred


def test_exhaustive_universe_16_gray_code():
    """Every subset of U={0..15} (2^16 of them), reached by a Gray-code walk of
    single inserts/deletes, then succ/pred/member of all 16 x."""
    u = 16
    bits, succ, pred = _brute_tables(u)
    ops, keys, exp = [], [], []
    mask = 0
    for g in range(1 << u):
        if g:
            flip = (g & -g).bit_length() - 1          # Gray code: flip the lowest set bit of g
            had = (mask >> flip) & 1
            ops.append(OV_DELETE if had else OV_INSERT)
            keys.append(flip)
            exp.append(1)
            mask ^= 1 << flip
        for x in range(u):
            ops += [OV_SUCC, OV_PRED, OV_MEMBER]
            keys += [x, x, x]
            exp += [int(succ[mask, x]), int(pred[mask, x]), int(bits[mask, x])]
    v = oracle.Veb(4)
    got = v.apply(np.array(ops, dtype=np.uint8), np.array(keys, dtype=np.uint64))
    exp = np.array(exp, dtype=np.uint64)
    bad = np.nonzero(got != exp)[0]
    assert len(bad) == 0, f"{len(bad)} mismatches, first at op {bad[:5]}"


@pytest.mark.parametrize("k", [6, 8, 10, 12])
def test_random_sequences_vs_sorted_list(k):
    """10^5 random mixed ops vs a sorted Python list (brute force)."""
    u = 1 << k
    rng = np.random.Generator(np.random.PCG64(1000 + k))
    n = 100_000
    ops = rng.integers(0, 5, size=n).astype(np.uint8)
    # bias inserts early so the set gets dense, then mixes
    keys = rng.integers(0, u + 8, size=n).astype(np.uint64)   # a few out-of-range keys too
    v = oracle.Veb(k)
    got = v.apply(ops, keys)
    s: list[int] = []
    for i in range(n):
        x = int(keys[i])
        o = ops[i]
        j = bisect.bisect_left(s, x)
        present = j < len(s) and s[j] == x
        if o == OV_INSERT:
            e = int(x < u and not present)
            if e:
                s.insert(j, x)
        elif o == OV_DELETE:
            e = int(present)
            if present:
                s.pop(j)
        elif o == OV_MEMBER:
            e = int(present)
        elif o == OV_SUCC:
            e = s[j] if (x < u and j < len(s)) else NONE
        else:
            jj = bisect.bisect_right(s, x)
            e = s[jj - 1] if jj > 0 else NONE
        assert int(got[i]) == e, f"op {i}: op={o} x={x} got {int(got[i])} want {e}"
    assert len(v) == len(s)


@pytest.mark.parametrize("k", [1, 5, 10, 20])
def test_closed_forms(k):
    u = 1 << k
    xs = np.unique(np.concatenate([np.arange(min(u, 64)), np.array([u - 1, u // 2, u // 3])])).astype(np.uint64)
    v = oracle.Veb(k)
    # empty set: no successor, no predecessor
    assert all(int(r) == NONE for r in v.batch(OV_SUCC, xs))
    assert all(int(r) == NONE for r in v.batch(OV_PRED, xs))
    # singleton {m}: succ(x) = m iff x <= m
    m = u // 3
    assert v.insert(m) == 1 and v.insert(m) == 0
    for x, r in zip(xs, v.batch(OV_SUCC, xs)):
        assert int(r) == (m if int(x) <= m else NONE)
    for x, r in zip(xs, v.batch(OV_PRED, xs)):
        assert int(r) == (m if int(x) >= m else NONE)
    assert v.delete(m) == 1 and v.delete(m) == 0
    if k <= 12:
        # full set: succ(x) = pred(x) = x
        v.batch(OV_INSERT, np.arange(u, dtype=np.uint64))
        assert len(v) == u
        assert np.array_equal(v.batch(OV_SUCC, xs), xs)
        assert np.array_equal(v.batch(OV_PRED, xs), xs)
    # out of range: successor none, insert refused
    assert v.successor(u) == NONE and v.insert(u) == 0


def test_image_is_bitmap_and_or_reduction():
    """The image format definition: level 0 = membership packed LSB-first,
    level l = "child word non-zero", computed here independently with numpy."""
    k = 14
    u = 1 << k
    rng = np.random.Generator(np.random.PCG64(7))
    keys = rng.choice(u, size=300, replace=False).astype(np.uint64)
    v = oracle.Veb(k)
    v.batch(OV_INSERT, keys)
    img = v.image()
    bits = np.zeros(u, dtype=np.uint8)
    bits[keys.astype(np.int64)] = 1
    leaf = np.packbits(bits, bitorder="little").view(np.uint64)
    levels = [leaf]
    while len(levels[-1]) > 1:
        nz = (levels[-1] != 0).astype(np.uint8)
        pad = (-len(nz)) % 64
        nz = np.concatenate([nz, np.zeros(pad, dtype=np.uint8)])
        levels.append(np.packbits(nz, bitorder="little").view(np.uint64))
    assert np.array_equal(img, np.concatenate(levels))


def test_level_geometry_matches_paper():
    """P:93 64-bit nodes; P:136 a leaf covers 64 segments and 3 levels cover
    4 TB of 16 MB segments."""
    g = golden()
    assert g["node_bits"] == 64
    assert g["segments_per_leaf"] * g["segment_bytes"] == g["leaf_bytes"]
    segs_4tb = g["three_level_bytes"] // g["segment_bytes"]
    assert segs_4tb == 1 << 18
    assert oracle.veb_image_levels(18) == [4096, 64, 1]            # 3 levels
    assert len(oracle.veb_image_levels(19)) == 4                   # one more segment bit needs a 4th
    assert oracle.veb_image_levels(20) == [16384, 256, 4, 1]       # the C1 standalone tree
