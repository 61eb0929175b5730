"""ctypes binding of libgallatin.so (include/gallatin.h) -- argument marshalling only.

Every step of the hot path runs in the CUDA kernels of the library; this file
only converts torch tensors / numpy arrays to pointers and streams.  There is
no CPU fallback: if the library is missing the import fails.
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GALLATIN_LIB") or os.path.join(_PKG, "libgallatin.so")
HEADER = os.path.join(os.path.dirname(_PKG), "include", "gallatin.h")

OK, ERR_INVALID, ERR_CUDA, ERR_STATE, ERR_NOMEM = 0, -1, -2, -3, -4
NULL = 0
NONE = (1 << 64) - 1


class GallatinError(RuntimeError):
    pass


class Config(ctypes.Structure):
    _fields_ = [("heap_bytes", ctypes.c_uint64), ("run_bytes", ctypes.c_uint64), ("slot_base", ctypes.c_uint32),
                ("slot_min", ctypes.c_uint32), ("run_max", ctypes.c_uint32), ("format_ahead", ctypes.c_uint32),
                ("fence_free", ctypes.c_uint32), ("bulk_items", ctypes.c_uint32), ("run_init", ctypes.c_uint32),
                ("prefetch", ctypes.c_uint32), ("run_grow", ctypes.c_uint32), ("demand_hint", ctypes.c_uint32),
                ("oom_record", ctypes.c_uint32), ("prefill", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [("heap_base", ctypes.c_uint64), ("heap_bytes", ctypes.c_uint64), ("num_segments", ctypes.c_uint64),
                ("free_segments", ctypes.c_uint64), ("tree_segments", ctypes.c_uint64 * 9),
                ("large_segments", ctypes.c_uint64), ("errors", ctypes.c_uint64), ("run_bytes", ctypes.c_uint64),
                ("nslot", ctypes.c_uint32 * 9), ("run_cap", ctypes.c_uint32 * 9), ("slot_base", ctypes.c_uint32),
                ("slot_min", ctypes.c_uint32), ("run_max", ctypes.c_uint32), ("format_ahead", ctypes.c_uint32),
                ("fence_free", ctypes.c_uint32), ("run_init", ctypes.c_uint32), ("formatters", ctypes.c_uint32),
                ("prefetch", ctypes.c_uint32), ("run_grow", ctypes.c_uint32), ("demand_hint", ctypes.c_uint32),
                ("oom_record", ctypes.c_uint32), ("prefill_segments", ctypes.c_uint32)]


def declared_functions() -> list[str]:
    """Every function the include/*.h headers declare (for the export check)."""
    import glob
    names = set()
    for h in glob.glob(os.path.join(os.path.dirname(HEADER), "*.h")):
        text = re.sub(r"/\*.*?\*/", "", open(h).read(), flags=re.S)
        names |= set(re.findall(r"^\s*(?:const\s+)?[\w ]+?\**\s*\b((?:gallatin|veb)_\w+)\s*\(", text, flags=re.M))
    return sorted(names)


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                          "(there is no CPU fallback)")
    L = ctypes.CDLL(LIB_PATH)
    u64, u32, vp, i32, dp = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_int, ctypes.POINTER(ctypes.c_double)
    P64 = ctypes.POINTER(ctypes.c_uint64)
    sig = {
        "gallatin_init": ([u64], i32),
        "gallatin_init_ex": ([ctypes.POINTER(Config)], i32),
        "gallatin_destroy": ([], i32),
        "gallatin_is_initialized": ([], i32),
        "gallatin_malloc": ([vp, vp, u64, vp], i32),
        "gallatin_free": ([vp, u64, vp], i32),
        "gallatin_malloc_host": ([vp, vp, u64, vp], i32),
        "gallatin_free_host": ([vp, u64, vp], i32),
        "gallatin_reset": ([vp], i32),
        "gallatin_drain": ([vp], i32),
        "gallatin_replay": ([vp, vp, vp, u64, vp, vp], i32),
        "gallatin_stats": ([ctypes.POINTER(Stats)], i32),
        "gallatin_snapshot_words": ([P64], i32),
        "gallatin_snapshot": ([vp, u64, P64], i32),
        "gallatin_get_device_view": ([vp, u64], i32),
        "gallatin_device_view_bytes": ([], u64),
        "gallatin_stamp": ([vp, vp, u64, vp], i32),
        "gallatin_verify": ([vp, vp, u64, vp, vp], i32),
        "gallatin_usable": ([vp, vp, u64, vp, vp, vp, vp], i32),
        "veb_create": ([u32, ctypes.POINTER(vp)], i32),
        "veb_destroy": ([vp], i32),
        "veb_clear": ([vp, vp], i32),
        "veb_insert": ([vp, vp, vp, u64, vp], i32),
        "veb_delete": ([vp, vp, vp, u64, vp], i32),
        "veb_member": ([vp, vp, vp, u64, vp], i32),
        "veb_successor": ([vp, vp, vp, u64, vp], i32),
        "veb_predecessor": ([vp, vp, vp, u64, vp], i32),
        "veb_words": ([vp, P64], i32),
        "veb_set_concurrent": ([vp, i32], i32),
        "veb_snapshot": ([vp, vp, u64, P64], i32),
        "gallatin_probe": ([i32, u64, u64, dp, dp, vp], i32),
        "gallatin_version": ([], ctypes.c_char_p),
        "gallatin_error_string": ([i32], ctypes.c_char_p),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    _lib = L
    return L


def check(rc: int, what: str) -> None:
    if rc != OK:
        msg = lib().gallatin_error_string(rc).decode()
        raise GallatinError(f"{what} failed: {msg} ({rc})")


# ----------------------------------------------------------- marshalling ---
def _stream(stream) -> int | None:
    if stream is not None:
        return int(stream)
    import torch
    return torch.cuda.current_stream().cuda_stream


def _on_device(t) -> None:
    """Tensors must live on the current device (the allocator's, set at init)."""
    import torch
    if t.device.index != torch.cuda.current_device():
        raise ValueError(f"tensor on {t.device}, the library runs on cuda:{torch.cuda.current_device()}")


def _dptr(t) -> int:
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or not t.is_contiguous() or t.element_size() != 8:
        raise TypeError("expected a contiguous 8-byte-element CUDA tensor")
    _on_device(t)
    return t.data_ptr()


def _dptr1(t) -> int:
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or not t.is_contiguous() or t.element_size() != 1:
        raise TypeError("expected a contiguous 1-byte-element CUDA tensor")
    _on_device(t)
    return t.data_ptr()


def _hptr(a: np.ndarray) -> int:
    if a.dtype.itemsize != 8 or not a.flags.c_contiguous:
        raise TypeError("expected a contiguous 8-byte numpy array")
    return a.ctypes.data


def _need(t, n: int, what: str) -> None:
    """Raise unless tensor / array t holds at least n elements (the kernels
    index every output and every paired input by the request count)."""
    m = t.numel() if hasattr(t, "numel") else len(t)
    if m < n:
        raise ValueError(f"{what} holds {m} elements, {n} needed")


def _empty64(n: int):
    import torch
    return torch.empty(n, dtype=torch.int64, device="cuda")


# ------------------------------------------------------------- allocator ---
def gallatin_init(heap_bytes: int, slot_base: int = 0, slot_min: int = 0, run_max: int = 0, run_bytes: int = 0,
                  format_ahead: int = 0, fence_free: int = 0, bulk_items: int = 0, run_init: int = 0,
                  prefetch: int = 0, run_grow: int = 0, demand_hint: int = 0, oom_record: int = 0,
                  prefill: int = 0) -> None:
    """0 = library default for every knob (include/gallatin.h gallatin_config_t)."""
    cfg = Config(heap_bytes=heap_bytes, run_bytes=run_bytes, slot_base=slot_base, slot_min=slot_min,
                 run_max=run_max, format_ahead=format_ahead, fence_free=fence_free, bulk_items=bulk_items,
                 run_init=run_init, prefetch=prefetch, run_grow=run_grow, demand_hint=demand_hint,
                 oom_record=oom_record, prefill=prefill)
    check(lib().gallatin_init_ex(ctypes.byref(cfg)), "gallatin_init")


def gallatin_destroy() -> None:
    check(lib().gallatin_destroy(), "gallatin_destroy")


def gallatin_is_initialized() -> bool:
    return bool(lib().gallatin_is_initialized())


def gallatin_malloc(sizes, ptrs=None, stream=None):
    """ptrs[i] = device malloc(sizes[i]); int64 CUDA tensors holding u64 values."""
    if ptrs is None:
        ptrs = _empty64(sizes.numel())
    _need(ptrs, sizes.numel(), "ptrs")
    check(lib().gallatin_malloc(_dptr(sizes), _dptr(ptrs), sizes.numel(), _stream(stream)), "gallatin_malloc")
    return ptrs


def gallatin_free(ptrs, stream=None) -> None:
    check(lib().gallatin_free(_dptr(ptrs), ptrs.numel(), _stream(stream)), "gallatin_free")


def gallatin_malloc_host(sizes: np.ndarray, out: np.ndarray | None = None, stream=None) -> np.ndarray:
    if out is None:
        out = np.empty(len(sizes), dtype=np.uint64)
    _need(out, len(sizes), "out")
    check(lib().gallatin_malloc_host(_hptr(sizes), _hptr(out), len(sizes), _stream(stream)), "gallatin_malloc_host")
    return out


def gallatin_free_host(ptrs: np.ndarray, stream=None) -> None:
    check(lib().gallatin_free_host(_hptr(ptrs), len(ptrs), _stream(stream)), "gallatin_free_host")


def gallatin_reset(stream=None) -> None:
    check(lib().gallatin_reset(_stream(stream)), "gallatin_reset")


def gallatin_drain(stream=None) -> None:
    check(lib().gallatin_drain(_stream(stream)), "gallatin_drain")


def gallatin_replay(kinds, args, keys, out=None, stream=None):
    """Serialized replay of an op list (include/gallatin.h).  Device tensors."""
    n = kinds.numel()
    if out is None:
        out = _empty64(n)
    for t, what in ((args, "args"), (keys, "keys"), (out, "out")):
        _need(t, n, what)
    check(lib().gallatin_replay(_dptr1(kinds), _dptr(args), _dptr(keys), n, _dptr(out), _stream(stream)),
          "gallatin_replay")
    return out


def gallatin_stats() -> dict:
    s = Stats()
    check(lib().gallatin_stats(ctypes.byref(s)), "gallatin_stats")
    return {"heap_base": s.heap_base, "heap_bytes": s.heap_bytes, "num_segments": s.num_segments,
            "free_segments": s.free_segments, "tree_segments": list(s.tree_segments),
            "large_segments": s.large_segments, "errors": s.errors, "nslot": list(s.nslot),
            "run_cap": list(s.run_cap), "run_bytes": s.run_bytes, "slot_base": s.slot_base, "slot_min": s.slot_min,
            "run_max": s.run_max, "format_ahead": s.format_ahead, "fence_free": s.fence_free,
            "run_init": s.run_init, "formatters": s.formatters, "prefetch": s.prefetch, "run_grow": s.run_grow,
            "demand_hint": s.demand_hint, "oom_record": s.oom_record, "prefill_segments": s.prefill_segments}


def oracle_params() -> dict:
    """The effective policy knobs, as keyword arguments of oracle.model() (tests)."""
    st = gallatin_stats()
    return {"slot_base": st["slot_base"], "slot_min": st["slot_min"], "run_max": st["run_max"],
            "run_bytes": st["run_bytes"], "format_ahead": 1 if st["format_ahead"] == 1 else 0,
            "run_init": st["run_init"], "prefetch": st["prefetch"], "run_grow": st["run_grow"],
            "prefill": 1 if st["prefill_segments"] else 0}


def gallatin_snapshot() -> np.ndarray:
    n = ctypes.c_uint64()
    check(lib().gallatin_snapshot_words(ctypes.byref(n)), "gallatin_snapshot_words")
    out = np.empty(n.value, dtype=np.uint64)
    got = ctypes.c_uint64()
    check(lib().gallatin_snapshot(out.ctypes.data, n.value, ctypes.byref(got)), "gallatin_snapshot")
    return out


def gallatin_stamp(ptrs, sizes, stream=None) -> None:
    _need(sizes, ptrs.numel(), "sizes")
    check(lib().gallatin_stamp(_dptr(ptrs), _dptr(sizes), ptrs.numel(), _stream(stream)), "gallatin_stamp")


def gallatin_verify(ptrs, sizes, stream=None) -> int:
    import torch
    _need(sizes, ptrs.numel(), "sizes")
    bad = torch.zeros(1, dtype=torch.int64, device="cuda")
    check(lib().gallatin_verify(_dptr(ptrs), _dptr(sizes), ptrs.numel(), _dptr(bad), _stream(stream)),
          "gallatin_verify")
    return int(bad.item())


def gallatin_usable(ptrs, sizes, usable=None, stream=None) -> tuple[int, int]:
    """(sum of usable bytes read from the memory table, #pointers contradicting their request)."""
    import torch
    _need(sizes, ptrs.numel(), "sizes")
    if usable is not None:
        _need(usable, ptrs.numel(), "usable")
    acc = torch.zeros(2, dtype=torch.int64, device="cuda")
    up = _dptr(usable) if usable is not None else None
    check(lib().gallatin_usable(_dptr(ptrs), _dptr(sizes), ptrs.numel(), up, acc.data_ptr(), acc.data_ptr() + 8,
                                _stream(stream)), "gallatin_usable")
    s, b = acc.cpu().tolist()
    return s & ((1 << 64) - 1), b


def gallatin_probe(kind: int, n: int, param: int, stream=None) -> tuple[float, float]:
    ms, ops = ctypes.c_double(), ctypes.c_double()
    check(lib().gallatin_probe(kind, n, param, ctypes.byref(ms), ctypes.byref(ops), _stream(stream)), "gallatin_probe")
    return ms.value, ops.value


def gallatin_version() -> str:
    return lib().gallatin_version().decode()


# -------------------------------------------------------- standalone vEB ---
class Veb:
    """The concurrent GPU vEB tree over [0, 2^universe_log2)."""

    def __init__(self, universe_log2: int):
        h = ctypes.c_void_p()
        check(lib().veb_create(universe_log2, ctypes.byref(h)), "veb_create")
        self._h = h
        self.k = universe_log2

    def close(self):
        if self._h:
            lib().veb_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def clear(self, stream=None):
        check(lib().veb_clear(self._h, _stream(stream)), "veb_clear")

    def set_concurrent(self, on: bool = True):
        """Coherent query loads, so queries may overlap updates (include/gallatin.h)."""
        check(lib().veb_set_concurrent(self._h, 1 if on else 0), "veb_set_concurrent")

    def _flags(self, fn, keys, want_out, stream):
        import torch
        out = torch.empty(keys.numel(), dtype=torch.uint8, device="cuda") if want_out else None
        check(fn(self._h, _dptr(keys), _dptr1(out) if out is not None else None, keys.numel(), _stream(stream)),
              fn.__name__)
        return out

    def insert(self, keys, want_out=True, stream=None):
        return self._flags(lib().veb_insert, keys, want_out, stream)

    def delete(self, keys, want_out=True, stream=None):
        return self._flags(lib().veb_delete, keys, want_out, stream)

    def member(self, keys, stream=None):
        return self._flags(lib().veb_member, keys, True, stream)

    def successor(self, q, out=None, stream=None):
        out = _empty64(q.numel()) if out is None else out
        _need(out, q.numel(), "out")
        check(lib().veb_successor(self._h, _dptr(q), _dptr(out), q.numel(), _stream(stream)), "veb_successor")
        return out

    def predecessor(self, q, out=None, stream=None):
        out = _empty64(q.numel()) if out is None else out
        _need(out, q.numel(), "out")
        check(lib().veb_predecessor(self._h, _dptr(q), _dptr(out), q.numel(), _stream(stream)), "veb_predecessor")
        return out

    def snapshot(self) -> np.ndarray:
        n = ctypes.c_uint64()
        check(lib().veb_words(self._h, ctypes.byref(n)), "veb_words")
        out = np.empty(n.value, dtype=np.uint64)
        got = ctypes.c_uint64()
        check(lib().veb_snapshot(self._h, out.ctypes.data, n.value, ctypes.byref(got)), "veb_snapshot")
        return out


# ------------------------------------------------------ streaming graph ----
GRAPH_HEADER = os.path.join(os.path.dirname(_PKG), "include", "gallatin_graph.h")


def _graph_sigs(L):
    u64, u32, vp, i32 = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_int
    sig = {
        "gallatin_graph_create": ([u32, ctypes.POINTER(vp)], i32),
        "gallatin_graph_destroy": ([vp, vp], i32),
        "gallatin_graph_insert": ([vp, vp, vp, u64, vp], i32),
        "gallatin_graph_insert_edges": ([vp, vp, vp, u64, vp], i32),
        "gallatin_graph_delete_edges": ([vp, vp, vp, u64, vp], i32),
        "gallatin_graph_delete": ([vp, vp, vp, u64, vp], i32),
        "gallatin_graph_expand": ([vp, vp, u64, vp], i32),
        "gallatin_graph_export": ([vp, vp, vp, vp, vp], i32),
        "gallatin_graph_gather": ([vp, vp, vp, vp], i32),
        "gallatin_graph_counters": ([vp, ctypes.POINTER(ctypes.c_uint64)], i32),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res


def _dptr4(t) -> int:
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda or not t.is_contiguous() or t.element_size() != 4:
        raise TypeError("expected a contiguous 4-byte-element CUDA tensor")
    _on_device(t)
    return t.data_ptr()


class Graph:
    """Streaming graph of per-vertex edge lists kept by the DEVICE-side
    allocator (include/gallatin_graph.h; BASELINE configs[4])."""

    def __init__(self, num_vertices: int):
        L = lib()
        _graph_sigs(L)
        h = ctypes.c_void_p()
        check(L.gallatin_graph_create(num_vertices, ctypes.byref(h)), "gallatin_graph_create")
        self._h = h
        self.V = num_vertices

    def destroy(self, stream=None):
        if self._h:
            check(lib().gallatin_graph_destroy(self._h, _stream(stream)), "gallatin_graph_destroy")
            self._h = None

    def insert(self, src, dst, stream=None):
        _need(dst, src.numel(), "dst")
        check(lib().gallatin_graph_insert(self._h, _dptr4(src), _dptr4(dst), src.numel(), _stream(stream)),
              "gallatin_graph_insert")

    def delete(self, src, dst, stream=None):
        _need(dst, src.numel(), "dst")
        check(lib().gallatin_graph_delete(self._h, _dptr4(src), _dptr4(dst), src.numel(), _stream(stream)),
              "gallatin_graph_delete")

    def insert_edges(self, src, dst, stream=None):
        """Single-edge inserts (one thread per edge under a vertex lock)."""
        _need(dst, src.numel(), "dst")
        check(lib().gallatin_graph_insert_edges(self._h, _dptr4(src), _dptr4(dst), src.numel(), _stream(stream)),
              "gallatin_graph_insert_edges")

    def delete_edges(self, src, dst, stream=None):
        """Single-edge deletes (one thread per edge under a vertex lock)."""
        _need(dst, src.numel(), "dst")
        check(lib().gallatin_graph_delete_edges(self._h, _dptr4(src), _dptr4(dst), src.numel(), _stream(stream)),
              "gallatin_graph_delete_edges")

    def expand(self, vertices, stream=None):
        check(lib().gallatin_graph_expand(self._h, _dptr4(vertices), vertices.numel(), _stream(stream)),
              "gallatin_graph_expand")

    def export(self, stream=None):
        """(size uint32[V], cap uint32[V], list pointer int64[V]) CUDA tensors."""
        import torch
        size = torch.empty(self.V, dtype=torch.int32, device="cuda")
        cap = torch.empty(self.V, dtype=torch.int32, device="cuda")
        ptr = torch.empty(self.V, dtype=torch.int64, device="cuda")
        check(lib().gallatin_graph_export(self._h, size.data_ptr(), cap.data_ptr(), ptr.data_ptr(), _stream(stream)),
              "gallatin_graph_export")
        return size, cap, ptr

    def gather(self, offsets, total: int, stream=None):
        """CSR copy of every list given the exclusive prefix sum of the sizes."""
        import torch
        out = torch.empty(max(total, 1), dtype=torch.int32, device="cuda")
        check(lib().gallatin_graph_gather(self._h, _dptr(offsets), out.data_ptr(), _stream(stream)),
              "gallatin_graph_gather")
        return out[:total]

    def counters(self) -> dict:
        c = (ctypes.c_uint64 * 4)()
        check(lib().gallatin_graph_counters(self._h, c), "gallatin_graph_counters")
        return {"mallocs": c[0], "frees": c[1], "failed": c[2], "bad_vertex": c[3]}
