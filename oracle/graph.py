"""O3 -- the streaming-graph oracle (TEST INFRASTRUCTURE ONLY; see oracle/__init__.py).

PAPER.md S6.12: per-vertex edge lists, each allocated as "the next
largest power of two region of memory".  The policy, evaluated once per batch
per vertex (reading A-29):
  insert batch : size += c_v; if size > cap: cap = nextpow2(max(size, 4))
  delete batch : one instance of each (src, dst) is removed if present; for a
                 vertex that had a deletion request and a non-empty list:
                 size == 0 -> cap = 0 (list freed); size <= cap/4 and cap > 4
                 -> cap = nextpow2(max(size, 4))
  expand round : every listed vertex appends max(size, 4) edges, edge j to
                 (v + size_before + j + 1) mod V; grow as for inserts.
  single edges : the same rules applied after every edge (insert_edges /
                 delete_edges; P:355's non-bulk "edge updates" and deletes).
The adjacency is kept as a multiset of keys src << 32 | dst (numpy).
"""
from __future__ import annotations

import numpy as np


def next_pow2(x: np.ndarray) -> np.ndarray:
    x = np.maximum(np.asarray(x, dtype=np.int64), 1)
    return (1 << np.ceil(np.log2(x)).astype(np.int64)).astype(np.int64)


def list_cap(size: np.ndarray) -> np.ndarray:
    return next_pow2(np.maximum(size, 4))


class GraphOracle:
    def __init__(self, num_vertices: int):
        self.V = num_vertices
        self.size = np.zeros(num_vertices, dtype=np.int64)
        self.cap = np.zeros(num_vertices, dtype=np.int64)
        self.keys = np.zeros(0, dtype=np.uint64)

    @staticmethod
    def _key(src, dst) -> np.ndarray:
        return (np.asarray(src, dtype=np.uint64) << np.uint64(32)) | np.asarray(dst, dtype=np.uint64)

    def insert(self, src: np.ndarray, dst: np.ndarray) -> None:
        c = np.bincount(np.asarray(src, dtype=np.int64), minlength=self.V)
        need = self.size + c
        grow = (c > 0) & (need > self.cap)
        self.cap[grow] = list_cap(need[grow])
        self.size = need
        self.keys = np.concatenate([self.keys, self._key(src, dst)])

    def delete(self, src: np.ndarray, dst: np.ndarray) -> None:
        req = np.bincount(np.asarray(src, dtype=np.int64), minlength=self.V)
        touched = (req > 0) & (self.size > 0)
        have_k, have_n = np.unique(self.keys, return_counts=True)
        del_k, del_n = np.unique(self._key(src, dst), return_counts=True)
        idx = np.searchsorted(have_k, del_k)
        idx_c = np.minimum(idx, len(have_k) - 1) if len(have_k) else idx
        present = (idx < len(have_k)) & (have_k[idx_c] == del_k) if len(have_k) else np.zeros(len(del_k), bool)
        removed = np.zeros_like(have_n)
        removed[idx[present]] = np.minimum(have_n[idx[present]], del_n[present])
        left = have_n - removed
        self.keys = np.repeat(have_k, left)
        rm_v = np.bincount((have_k >> np.uint64(32)).astype(np.int64), weights=removed, minlength=self.V)
        self.size = self.size - rm_v.astype(np.int64)
        zero = touched & (self.size == 0)
        self.cap[zero] = 0
        small = touched & (self.size > 0) & (self.size <= self.cap // 4) & (self.cap > 4)
        self.cap[small] = list_cap(self.size[small])

    def insert_edges(self, src: np.ndarray, dst: np.ndarray) -> None:
        """Single-edge inserts: a full list doubles at the edge that finds it
        full (0 -> 4 -> 8 ...); cap ends at the smallest power of two >= size
        reachable by doubling, which for caps that are 0 or powers of two >= 4
        is max(cap, nextpow2(max(size, 4)))."""
        c = np.bincount(np.asarray(src, dtype=np.int64), minlength=self.V)
        need = self.size + c
        grow = (c > 0) & (need > self.cap)
        cap = np.where(self.cap == 0, 4, self.cap)
        while True:                                      # doubling, step by step
            g = grow & (need > cap)
            if not g.any():
                break
            cap = np.where(g, cap * 2, cap)
        self.cap = np.where(grow, cap, self.cap)
        self.size = need
        self.keys = np.concatenate([self.keys, self._key(src, dst)])

    def delete_edges(self, src: np.ndarray, dst: np.ndarray) -> None:
        """Single-edge deletes: the per-vertex sizes go down one removal at a
        time; after each, size 0 frees the list (cap 0) and size <= cap/4 with
        cap > 4 reallocates to nextpow2(max(size, 4)).  Starting from
        size > cap/4 the shrinks happen when size reaches cap/4, so the final
        cap follows from the final size alone (iterated below)."""
        s0 = self.size.copy()
        cap0 = self.cap.copy()
        self.delete(src, dst)                            # multiset + sizes (caps recomputed below)
        s1 = self.size
        cap = cap0.copy()
        moved = s1 < s0
        while True:
            sh = moved & (cap > 4) & (s1 <= cap // 4)
            if not sh.any():
                break
            cap = np.where(sh, list_cap(cap // 4), cap)
        cap = np.where(moved & (s1 == 0), 0, cap)
        self.cap = np.where(moved, cap, cap0)

    def expand(self, vertices: np.ndarray) -> None:
        v = np.asarray(vertices, dtype=np.int64)
        s0 = self.size[v]
        add = np.maximum(s0, 4)
        need = s0 + add
        grow = need > self.cap[v]
        self.cap[v[grow]] = list_cap(need[grow])
        self.size[v] = need
        src = np.repeat(v, add)
        start = np.repeat(np.cumsum(add) - add, add)
        j = np.arange(len(src)) - start
        dst = (src + np.repeat(s0, add) + j + 1) % self.V
        self.keys = np.concatenate([self.keys, self._key(src, dst)])

    def sorted_keys(self) -> np.ndarray:
        return np.sort(self.keys)


class BruteGraph:
    """A one-edge-at-a-time Python simulation of the same policy (pins O3)."""

    def __init__(self, num_vertices: int):
        self.V = num_vertices
        self.lists = {v: [] for v in range(num_vertices)}
        self.cap = [0] * num_vertices

    @staticmethod
    def _cap(size: int) -> int:
        c = 4
        while c < size:
            c *= 2
        return c

    def insert(self, src, dst):
        for s, d in zip(src.tolist(), dst.tolist()):
            self.lists[s].append(d)
        for s in set(src.tolist()):
            if len(self.lists[s]) > self.cap[s]:
                self.cap[s] = self._cap(len(self.lists[s]))

    def delete(self, src, dst):
        had = {s for s in set(src.tolist()) if self.lists[s]}
        for s, d in zip(src.tolist(), dst.tolist()):
            if d in self.lists[s]:
                self.lists[s].remove(d)
        for s in had:
            n = len(self.lists[s])
            if n == 0:
                self.cap[s] = 0
            elif n <= self.cap[s] // 4 and self.cap[s] > 4:
                self.cap[s] = self._cap(n)

    def insert_edges(self, src, dst):
        for s, d in zip(src.tolist(), dst.tolist()):
            if len(self.lists[s]) == self.cap[s]:
                self.cap[s] = 4 if self.cap[s] == 0 else 2 * self.cap[s]
            self.lists[s].append(d)

    def delete_edges(self, src, dst):
        for s, d in zip(src.tolist(), dst.tolist()):
            if d not in self.lists[s]:
                continue
            self.lists[s].remove(d)
            n = len(self.lists[s])
            if n == 0:
                self.cap[s] = 0
            elif self.cap[s] > 4 and n <= self.cap[s] // 4:
                self.cap[s] = self._cap(n)

    def expand(self, vertices):
        for v in vertices.tolist():
            s0 = len(self.lists[v])
            add = max(s0, 4)
            self.lists[v] += [(v + s0 + j + 1) % self.V for j in range(add)]
            if len(self.lists[v]) > self.cap[v]:
                self.cap[v] = self._cap(len(self.lists[v]))

    def sorted_keys(self):
        return np.sort(np.array([(s << 32) | d for s, l in self.lists.items() for d in l], dtype=np.uint64))
