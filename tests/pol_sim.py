"""Brute-force simulation of the allocator policy -- a pin for O2 (oracle/).

An independent, deliberately naive restatement of SURVEY.md 8(c) POL (the
paper's policy, Alg. 1-4) and of the deviation model R1-R6 of
DESIGN.md "Deviations" 5 and 8 (oracle/alloc_runs.c's header), written from
the text, not from the C code:

* no vEB trees: the segment tree is "every s with kind[s] is None", block tree
  t is "every s formatted for t with a non-empty ring" -- both recomputed by a
  scan whenever they are asked (successor(0) = min of the scan);
* rings are Python deques, the large-allocation search tries every start from
  the top.

It is O(nseg) per request and only meant for tiny heaps.  ``image()`` writes
the canonical snapshot layout (include/gallatin.h) so tests can compare it
with O2's image word for word.  Nothing here is imported by the oracle or the
CUDA path.
"""
from __future__ import annotations

from collections import deque

import numpy as np

SEG = 1 << 24
NB_MAX = 256
SLICES = 4096
TREES = 9
FREE, CONT = 0xFFFFFFFF, 0xFFFFFFFE
EMPTY = 0x3FFFFF                  # slot word with no run


def nb(t: int) -> int:
    return NB_MAX >> t                                   # P:264 (A-1)


def classify(size: int):
    """('slice', c) | ('block', t) | ('large', k) | None (A-1..A-4)."""
    if size == 0:
        return None
    if size <= 4096:
        return ("slice", max(0, (size - 1).bit_length() - 4))
    if size < SEG:
        return ("block", max(0, (size - 1).bit_length() - 16))       # A-2
    return ("large", -(-size // SEG))                                # P:138, A-3


class PolSim:
    def __init__(self, nseg, slot_base=148, slot_min=4, run_max=1, run_bytes=64 << 20, format_ahead=0, run_init=1,
                 prefetch=0, run_grow=1, prefill=0):
        self.nseg = nseg
        self.runs = not (run_max == 1 and run_init == 1 and format_ahead == 0 and prefetch == 0 and not prefill)
        self.nslot = [max(slot_base >> c, slot_min, 1) for c in range(TREES)]
        self.off = [sum(self.nslot[:c]) for c in range(TREES)]
        self.run_max, self.run_bytes, self.fa, self.run_init = run_max, run_bytes, format_ahead, run_init
        self.pf, self.grow = prefetch, run_grow
        self.tree = [FREE] * nseg            # FREE | 0..8 | 9 + k | CONT
        self.ring = [deque() for _ in range(nseg)]
        self.cnt = [0] * (nseg * NB_MAX)     # free counter per block
        S = sum(self.nslot)
        self.slot = [None] * S               # None or [issued, m, first]
        self.next = [None] * S
        self.err = 0
        if prefill:
            self.prefill()

    def first_run(self, c):
        return min(max(self.run_init >> c, min(self.run_init, 8)), nb(c), self.cap(c))

    def prefill(self):
        """R7 ("always populated"): slot q of class c holds blocks
        [q r, (q+1) r) of the class's segments, the classes' segments laid out
        one after another from segment 0; the class's partly used last segment
        keeps the rest, ascending, in its ring.  r = the largest power of two
        <= the first run, then -- while it all exceeds nseg / 8 segments --
        the class with the most segments (lowest on ties) whose r is above
        max(1, nb >> run_grow) halved; if none can be, nothing is filled."""
        r = [1 << (self.first_run(c).bit_length() - 1) for c in range(TREES)]

        def segs(c):
            return -(-self.nslot[c] * r[c] // nb(c))
        while sum(segs(c) for c in range(TREES)) > self.nseg // 8:
            cand = [c for c in range(TREES) if r[c] > max(1, nb(c) >> self.grow)]
            if not cand:
                return
            big = max(cand, key=lambda c: (segs(c), -c))
            r[big] //= 2
        base = 0
        for c in range(TREES):
            for s in range(base, base + segs(c)):
                self.tree[s] = c
            used = self.nslot[c] * r[c] - (segs(c) - 1) * nb(c)
            self.ring[base + segs(c) - 1] = deque(range(used, nb(c)))
            for q in range(self.nslot[c]):
                self.slot[self.off[c] + q] = [0, r[c], base * nb(c) + q * r[c]]
            base += segs(c)

    # ---- the trees, by scan --------------------------------------------
    def free_segs(self):
        return [s for s in range(self.nseg) if self.tree[s] == FREE]

    def tree_segs(self, t):
        return [s for s in range(self.nseg) if self.tree[s] == t and self.ring[s]]

    # ---- segments and blocks --------------------------------------------
    def claim_front(self):
        f = self.free_segs()
        if not f and self.runs:                                   # R6: idle formatted segments go back
            for s in range(self.nseg):
                if self.tree[s] < TREES and len(self.ring[s]) == nb(self.tree[s]):
                    self.tree[s] = FREE
                    self.ring[s] = deque()
            f = self.free_segs()
        if not f:
            return None
        s = f[0]                                                  # successor(0): front first
        self.tree[s] = "claimed"
        return s

    def format(self, s, t):
        self.tree[s] = t
        self.ring[s] = deque(range(nb(t)))                        # P:125-126, ring in order

    def return_block(self, s, j):
        t = self.tree[s]
        self.ring[s].append(j)                                    # FIFO enqueue
        if len(self.ring[s]) == nb(t):                            # every block home
            self.tree[s] = FREE
            self.ring[s] = deque()

    def freed(self, gid, n):
        self.cnt[gid] += n
        if self.cnt[gid] == SLICES:
            self.cnt[gid] = 0
            self.return_block(gid // NB_MAX, gid % NB_MAX)

    def gid(self, t, linear):
        return (linear // nb(t)) * NB_MAX + linear % nb(t)

    def get_run_once(self, t, want):
        """(blocks, first linear index); the paper's GetBlock at want = 1."""
        cand = self.tree_segs(t)
        if cand and self.runs and want >= nb(t) and len(self.ring[cand[0]]) < want and self.free_segs():
            cand = []                                             # R2: whole fresh segments first
        if cand:
            s = cand[0]
            av = len(self.ring[s])
            got = min(want, av)
            taken = [self.ring[s].popleft() for _ in range(got)]
            if self.fa and av >= nb(t) // 4 and av - got < nb(t) // 4 and not [x for x in self.tree_segs(t) if x > s]:
                f = self.claim_front()                            # R3 format-ahead
                if f is not None:
                    self.format(f, t)
            best = (0, 0)                                         # (length, -start): longest, lowest start
            for j in sorted(taken):
                L = 1
                while j + L in taken:
                    L += 1
                if j - 1 not in taken and (L, -j) > (best[0], -best[1]):
                    best = (L, j)
            bl, bs = best
            for j in sorted(taken):
                if not bs <= j < bs + bl:
                    self.return_block(s, j)
            return bl, s * nb(t) + bs
        if want >= nb(t):                                         # R2: whole segments, privately
            s0 = self.claim_front()
            if s0 is None:
                return 0, 0
            k = 1
            while k < want // nb(t) and s0 + k < self.nseg and self.tree[s0 + k] == FREE:
                self.tree[s0 + k] = "claimed"
                k += 1
            for q in range(k):
                self.tree[s0 + q] = t
                self.ring[s0 + q] = deque()
            return k * nb(t), s0 * nb(t)
        s1 = self.claim_front()
        if s1 is None:
            return 0, 0
        self.format(s1, t)
        for _ in range(want):
            self.ring[s1].popleft()
        return want, s1 * nb(t)

    def trim(self):
        back = 0
        for c in range(TREES):
            for q in range(self.nslot[c]):
                i = self.off[c] + q
                sl = self.slot[i]
                if sl and sl[0] < SLICES * sl[1]:
                    keep = -(-sl[0] // SLICES)
                    for k in range(keep, sl[1]):
                        self.freed(self.gid(c, sl[2] + k), SLICES)
                    back += sl[1] - keep
                    self.slot[i] = [sl[0], keep, sl[2]] if keep else None
                if self.pf and self.next[i]:
                    nx, self.next[i] = self.next[i], None
                    for k in range(nx[1]):
                        self.freed(self.gid(c, nx[2] + k), SLICES)
                    back += nx[1]
        return back

    def get_run(self, t, want):
        got, first = self.get_run_once(t, want)
        if not got and self.runs and self.trim():                 # R5
            got, first = self.get_run_once(t, 1)
        return got, first

    def cap(self, c):
        return max(1, min(self.run_max, self.run_bytes // (SEG // nb(c))))

    # ---- requests --------------------------------------------------------
    def malloc_slice(self, c, key):
        i = self.off[c] + key % self.nslot[c]
        while True:
            sl = self.slot[i]
            if sl and sl[0] < SLICES * sl[1]:                     # a valid index
                idx = sl[0]
                sl[0] += 1
                if self.pf and idx == SLICES * sl[1] // 2 and self.next[i] is None:
                    g, f = self.get_run_once(c, min(sl[1] << self.grow, self.cap(c)))   # R4
                    if g:
                        self.next[i] = [0, g, f]
                return sl[2] * (SEG // nb(c)) + idx * (16 << c)
            if self.next[i]:
                self.slot[i], self.next[i] = self.next[i], None
                continue
            if sl is None:                                        # first run (R1)
                want = self.first_run(c)
            else:
                want = min(sl[1] << self.grow, self.cap(c))
            got, first = self.get_run(c, want)
            if not got:
                self.slot[i] = None
                return None                                       # nullptr
            self.slot[i] = [0, got, first]

    def malloc(self, size, key=0):
        k = classify(size)
        if k is None:
            return None
        if k[0] == "slice":
            return self.malloc_slice(k[1], key)
        if k[0] == "block":
            got, first = self.get_run(k[1], 1)
            if not got:
                return None
            self.cnt[self.gid(k[1], first)] = SLICES - 1          # A-2
            return first * (SEG // nb(k[1]))
        kk = k[1]
        for attempt in range(2):
            for i in range(self.nseg - kk, -1, -1):               # the highest start (A-17)
                if all(self.tree[i + m] == FREE for m in range(kk)):
                    self.tree[i] = TREES + kk
                    for m in range(1, kk):
                        self.tree[i + m] = CONT
                    return i * SEG
            if not (self.runs and attempt == 0 and self.trim()):
                return None

    def free(self, off):
        if off is None:
            return
        if off >= self.nseg * SEG:
            self.err += 1
            return
        s = off // SEG
        t = self.tree[s]
        if t < TREES:
            self.freed(s * NB_MAX + (off % SEG) // (SEG // nb(t)), 1)
        elif t not in (FREE, CONT):
            for m in range(t - TREES):
                self.tree[s + m] = FREE
        else:
            self.err += 1

    def drain(self):
        for c in range(TREES):
            for q in range(self.nslot[c]):
                i = self.off[c] + q
                sl, nx = self.slot[i], self.next[i]
                self.slot[i] = self.next[i] = None
                if sl:
                    for k in range(sl[1]):
                        issued = min(max(sl[0] - SLICES * k, 0), SLICES)
                        if issued < SLICES:
                            self.freed(self.gid(c, sl[2] + k), SLICES - issued)
                if nx:
                    for k in range(nx[1]):
                        self.freed(self.gid(c, nx[2] + k), SLICES)
        if self.runs:
            for s in range(self.nseg):
                if self.tree[s] < TREES and len(self.ring[s]) == nb(self.tree[s]):
                    self.tree[s] = FREE
                    self.ring[s] = deque()

    def replay(self, kinds, args, keys):
        NONE = (1 << 64) - 1
        out = []
        for k, a, key in zip(kinds.tolist(), args.tolist(), keys.tolist()):
            if k == 0:
                r = self.malloc(a, key)
                out.append(NONE if r is None else r)
            elif k == 1:
                o = out[a]
                self.free(None if o == NONE else o)
                out.append(0)
            else:
                self.drain()
                out.append(0)
        return np.array(out, dtype=np.uint64)

    # ---- canonical image (include/gallatin.h "Snapshot image") ------------
    def image(self) -> np.ndarray:
        def bitmap_levels(members):
            wl = [(self.nseg + 63) // 64]
            while wl[-1] > 1:
                wl.append((wl[-1] + 63) // 64)
            bits = np.zeros(wl[0] * 64, dtype=np.uint8)
            bits[list(members)] = 1
            lv = [np.packbits(bits, bitorder="little").view(np.uint64)]
            for w in wl[1:]:
                nz = np.zeros(w * 64, dtype=np.uint8)
                nz[:len(lv[-1])] = lv[-1] != 0
                lv.append(np.packbits(nz, bitorder="little").view(np.uint64))
            return np.concatenate(lv), len(wl)

        seg, L = bitmap_levels(self.free_segs())
        W = len(seg)
        S = len(self.slot)
        hdr = np.array([0x47414C4C494D4731, self.nseg, L, W, S, self.err, 0, 0], dtype=np.uint64)
        bts = [bitmap_levels(self.tree_segs(t))[0] for t in range(TREES)]
        words = np.array([(self.tree[s] << 32) | (len(self.ring[s]) if self.tree[s] < TREES else 0)
                          for s in range(self.nseg)], dtype=np.uint64)
        q = np.zeros((self.nseg, 65), dtype=np.uint64)
        for s in range(self.nseg):
            e = np.full(256, 0xFFFF, dtype=np.uint16)
            e[:len(self.ring[s])] = list(self.ring[s])
            q[s, 0] = len(self.ring[s])
            q[s, 1:] = e.view(np.uint64)
        cnt = np.array(self.cnt, dtype=np.uint32).view(np.uint64)

        def word(sl):
            return EMPTY if sl is None else (sl[0] << 32) | (sl[1] << 22) | sl[2]

        slots = np.array([word(x) for x in self.slot], dtype=np.uint64)
        nxt = np.array([word(x) for x in self.next], dtype=np.uint64)
        return np.concatenate([hdr, seg] + bts + [words, q.reshape(-1), cnt, slots, nxt])
