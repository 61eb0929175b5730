"""Test-side helpers: independent restatements of the paper's rules and of the
documented snapshot layout (include/gallatin.h).  Used by the oracle pins and
the GPU parity tests alike; no code of either implementation."""
import os

import numpy as np

from oracle import TREE_FREE

SEG = 1 << 24
SLOT_EMPTY = 0x3FFFFF            # issued 0, run length 0, no block (include/gallatin.h)
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
    out.append(np.full(nslots, SLOT_EMPTY, dtype=np.uint64))
    out.append(np.full(nslots, SLOT_EMPTY, dtype=np.uint64))
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


def diff_images(got: np.ndarray, want: np.ndarray) -> str:
    """'' if equal, else a readable description of the first differing section."""
    if len(got) == len(want) and np.array_equal(got, want):
        return ""
    if len(got) != len(want):
        return f"image lengths differ: {len(got)} vs {len(want)}"
    a, b = image_sections(got), image_sections(want)
    for k in ["magic", "nseg", "levels", "W", "nslots", "err", "segtree", "btrees", "segword", "qcount",
              "qentries", "block_free", "slots", "next"]:
        x, y = a[k], b[k]
        if isinstance(x, int):
            if x != y:
                return f"{k}: {x} != {y}"
        elif not np.array_equal(x, y):
            idx = np.argwhere(np.asarray(x) != np.asarray(y))[:5]
            return f"{k} differs at {idx.tolist()}: got {[x[tuple(i)] for i in idx]} want {[y[tuple(i)] for i in idx]}"
    return "equal?"
