"""CPU oracle for the Gallatin hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ppopp_mccoyp24_b200``) never imports it, and it
never imports the product path: the two share no code, header or constant.

* O1 -- ``Veb``: the textbook (CLRS) van Emde Boas tree with min/max, summary
  and sqrt(U) clusters that PAPER.md S3.1 describes; ``succ`` is the
  paper's ">= x".  ``veb_oracle.c``.
* O2-P -- ``Allocator``: the sequential allocator following PAPER.md S4-S5
  (Alg. 1-4, policy POL) one request at a time.
  ``alloc_paper.c`` (+ ``alloc_state.c``: lifecycle, invariant checks, image).
* O2-R -- ``RunsAllocator``: the deviation model (DESIGN.md Deviations 5, 8:
  runs of blocks, format-ahead, prefetch, slot trims), built on O2-P's
  primitives.  ``alloc_runs.c``.
* O3 -- graph adjacency oracle (``graph.py``), per-vertex Python/numpy lists.

Parity status of every function is listed in DESIGN.md ("Oracle pins").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SOURCES = ["veb_oracle.c", "alloc_state.c", "alloc_paper.c", "alloc_runs.c"]
_HEADERS = ["alloc_state.h"]

NONE = (1 << 64) - 1
TREE_FREE = 0xFFFFFFFF
TREE_CONT = 0xFFFFFFFE
GID_NONE = 0xFFFFFFFF

OV_INSERT, OV_DELETE, OV_MEMBER, OV_SUCC, OV_PRED = range(5)

# violation bits of o2_check()
VIOLATIONS = {
    1: "front-first (P:138)", 2: "back-first large (P:138)", 4: "free of a non-live pointer",
    8: "overlap", 16: "alignment", 32: "outside heap", 64: "accounting", 128: "trees vs table",
    256: "ring queue",
}


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain C, -O2).  Building is not using it."""
    srcs = [os.path.join(_HERE, s) for s in _SOURCES]
    if not force and os.path.exists(_LIB_PATH):
        lib_m = os.path.getmtime(_LIB_PATH)
        if all(os.path.getmtime(s) <= lib_m for s in srcs + [os.path.join(_HERE, h) for h in _HEADERS]):
            return _LIB_PATH
    cmd = ["gcc", "-O2", "-std=c11", "-Wall", "-Wextra", "-fPIC", "-shared", "-o", _LIB_PATH] + srcs
    subprocess.check_call(cmd)
    return _LIB_PATH


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        u64, u32, vp, i32 = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_int
        sig = {
            "oracle_veb_create": ([ctypes.c_uint], vp),
            "oracle_veb_destroy": ([vp], None),
            "oracle_veb_size": ([vp], u64),
            "oracle_veb_member": ([vp, u64], i32),
            "oracle_veb_insert": ([vp, u64], i32),
            "oracle_veb_delete": ([vp, u64], i32),
            "oracle_veb_successor": ([vp, u64], u64),
            "oracle_veb_predecessor": ([vp, u64], u64),
            "oracle_veb_min": ([vp], u64),
            "oracle_veb_max": ([vp], u64),
            "oracle_veb_apply": ([vp, vp, vp, u64, vp], None),
            "oracle_veb_batch": ([vp, i32, vp, u64, vp], None),
            "oracle_veb_image": ([vp, vp, u64], u64),
            "oracle_veb_image_levels": ([ctypes.c_uint, vp], ctypes.c_uint),
            "o2_create_paper": ([u64, ctypes.c_uint, ctypes.c_uint], vp),
            "o2_create_runs": ([u64, ctypes.c_uint, ctypes.c_uint, ctypes.c_uint, u64, ctypes.c_uint, ctypes.c_uint,
                                ctypes.c_uint, ctypes.c_uint, ctypes.c_uint], vp),
            "o2_destroy": ([vp], None),
            "o2_nslot": ([vp, ctypes.c_uint], ctypes.c_uint),
            "o2_errors": ([vp], u64),
            "o2_violations": ([vp], u64),
            "o2_live_count": ([vp], u64),
            "o2_usable_live": ([vp], u64),
            "o2_usable_size": ([u64], u64),
            "o2_malloc": ([vp, u64, u64], u64),
            "o2_free": ([vp, u64], None),
            "o2_drain": ([vp], None),
            "o2_replay": ([vp, vp, vp, vp, u64, vp], None),
            "o2_malloc_batch": ([vp, vp, u64, u64, vp], None),
            "o2_free_batch": ([vp, vp, u64], None),
            "o2_check": ([vp], u64),
            "o2_image_words": ([vp], u64),
            "o2_image": ([vp, vp, u64], u64),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


class Veb:
    """O1: textbook vEB over U = {0 .. 2^k - 1}."""

    def __init__(self, k: int):
        self._h = None
        self.k = k
        self.u = 1 << k
        self._h = lib().oracle_veb_create(k)
        if not self._h:
            raise ValueError(f"bad universe 2^{k}")

    def close(self):
        if self._h:
            lib().oracle_veb_destroy(self._h)
            self._h = None

    __del__ = close

    def __len__(self):
        return lib().oracle_veb_size(self._h)

    def insert(self, x: int) -> int:
        return lib().oracle_veb_insert(self._h, x)

    def delete(self, x: int) -> int:
        return lib().oracle_veb_delete(self._h, x)

    def member(self, x: int) -> int:
        return lib().oracle_veb_member(self._h, x)

    def successor(self, x: int) -> int:
        return lib().oracle_veb_successor(self._h, x)

    def predecessor(self, x: int) -> int:
        return lib().oracle_veb_predecessor(self._h, x)

    def apply(self, ops: np.ndarray, keys: np.ndarray) -> np.ndarray:
        ops = np.ascontiguousarray(ops, dtype=np.uint8)
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        out = np.empty(len(keys), dtype=np.uint64)
        lib().oracle_veb_apply(self._h, _ptr(ops), _ptr(keys), len(keys), _ptr(out))
        return out

    def batch(self, op: int, keys: np.ndarray) -> np.ndarray:
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        out = np.empty(len(keys), dtype=np.uint64)
        lib().oracle_veb_batch(self._h, op, _ptr(keys), len(keys), _ptr(out))
        return out

    def image(self) -> np.ndarray:
        wpl = np.zeros(16, dtype=np.uint64)
        L = lib().oracle_veb_image_levels(self.k, _ptr(wpl))
        total = int(wpl[:L].sum())
        out = np.empty(total, dtype=np.uint64)
        got = lib().oracle_veb_image(self._h, _ptr(out), total)
        assert got == total
        return out


def veb_image_levels(k: int) -> list[int]:
    wpl = np.zeros(16, dtype=np.uint64)
    L = lib().oracle_veb_image_levels(k, _ptr(wpl))
    return [int(w) for w in wpl[:L]]


class Allocator:
    """O2-P: sequential Gallatin allocator, the paper's policy POL (PAPER.md
    S4-S5, Alg. 1-4; one-block buffer slots).

    Offsets are relative to the heap base; NONE (2^64-1) is NULL.
    """

    def __init__(self, nseg: int, slot_base: int = 148, slot_min: int = 4):
        self._h = None
        self.nseg = nseg
        self._h = lib().o2_create_paper(nseg, slot_base, slot_min)
        if not self._h:
            raise ValueError("bad allocator parameters")

    def close(self):
        if self._h:
            lib().o2_destroy(self._h)
            self._h = None

    __del__ = close

    def nslot(self, c: int) -> int:
        return lib().o2_nslot(self._h, c)

    def malloc(self, size: int, key: int = 0) -> int:
        return lib().o2_malloc(self._h, size, key)

    def free(self, off: int) -> None:
        lib().o2_free(self._h, off)

    def drain(self) -> None:
        lib().o2_drain(self._h)

    @property
    def errors(self) -> int:
        return lib().o2_errors(self._h)

    @property
    def live_count(self) -> int:
        return lib().o2_live_count(self._h)

    @property
    def usable_live(self) -> int:
        return lib().o2_usable_live(self._h)

    def check(self) -> int:
        return lib().o2_check(self._h)

    def replay(self, kinds: np.ndarray, args: np.ndarray, keys: np.ndarray) -> np.ndarray:
        kinds = np.ascontiguousarray(kinds, dtype=np.uint8)
        args = np.ascontiguousarray(args, dtype=np.uint64)
        keys = np.ascontiguousarray(keys, dtype=np.uint64)
        out = np.empty(len(kinds), dtype=np.uint64)
        lib().o2_replay(self._h, _ptr(kinds), _ptr(args), _ptr(keys), len(kinds), _ptr(out))
        return out

    def malloc_batch(self, sizes: np.ndarray, keydiv: int = 32) -> np.ndarray:
        sizes = np.ascontiguousarray(sizes, dtype=np.uint64)
        out = np.empty(len(sizes), dtype=np.uint64)
        lib().o2_malloc_batch(self._h, _ptr(sizes), len(sizes), keydiv, _ptr(out))
        return out

    def free_batch(self, offs: np.ndarray) -> None:
        offs = np.ascontiguousarray(offs, dtype=np.uint64)
        lib().o2_free_batch(self._h, _ptr(offs), len(offs))

    def image(self) -> np.ndarray:
        n = lib().o2_image_words(self._h)
        out = np.empty(n, dtype=np.uint64)
        got = lib().o2_image(self._h, _ptr(out), n)
        assert got == n
        return out


class RunsAllocator(Allocator):
    """O2-R: the deviation model (DESIGN.md Deviations 5, 8; alloc_runs.c):
    runs of consecutive blocks per slot, format-ahead, prefetch, slot trims
    before "no memory".  run_max=1, run_init=1, format_ahead=0, prefetch=0 is
    the paper's one-block buffer; run_grow = log2 of the growth per
    refill; prefill=1: every slot starts holding its first run (R7),
    when those runs fit in half the heap."""

    def __init__(self, nseg: int, slot_base: int = 148, slot_min: int = 4, run_max: int = 1,
                 run_bytes: int = 64 << 20, format_ahead: int = 0, run_init: int = 1, prefetch: int = 0,
                 run_grow: int = 1, prefill: int = 0):
        self._h = None
        self.nseg = nseg
        self._h = lib().o2_create_runs(nseg, slot_base, slot_min, run_max, run_bytes, format_ahead, run_init,
                                       prefetch, run_grow, prefill)
        if not self._h:
            raise ValueError("bad allocator parameters")


PAPER_KNOBS = {"run_max": 1, "run_init": 1, "format_ahead": 0, "prefetch": 0}


def is_paper_policy(params: dict) -> bool:
    """True if the knobs are the paper's one-block buffer, filled on demand."""
    return all(params.get(k, PAPER_KNOBS[k]) == v for k, v in PAPER_KNOBS.items()) and not params.get("prefill", 0)


def model(nseg: int, **params) -> Allocator:
    """The O2 model for a set of knobs: O2-P for the paper's policy, else O2-R
    (which at the paper's knobs adds only the prefilled buffer and the slot
    trims)."""
    if is_paper_policy(params):
        return Allocator(nseg, params.get("slot_base", 148), params.get("slot_min", 4))
    return RunsAllocator(nseg, **params)


def usable_size(size: int) -> int:
    return lib().o2_usable_size(size)


def violation_names(mask: int) -> list[str]:
    return [v for b, v in VIOLATIONS.items() if mask & b]
