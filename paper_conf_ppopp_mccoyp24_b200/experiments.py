"""The paper's other evaluation modes (PAPER.md S6) on the bulk C-ABI calls.

Each function drives libgallatin.so through the same bulk calls bench.py
times; the allocator arithmetic all runs in the CUDA kernels.  Torch is used
for device buffers and events, and for harness-side reductions over the
returned pointer arrays (NULL counts, min/max) that are not part of the
method.

* utilization  -- E8: batches of 100,000 allocations of one
  size until the allocator returns NULL; successes x size / heap bytes.
* fragmentation -- E7: highest minus lowest address handed out
  by a static set of 2^20 allocations of one size.
* warm_vs_cold -- E6: the single-size test run with a reset before
  every round (cold, the paper's default) and without (warmed up).
* variance     -- E5: variance of the per-round time (ms^2) over
  the rounds of one cell.
* init_time    -- E1: one gallatin_init (heap + metadata + reset),
  excluded from every other measurement as in the paper.
"""
from __future__ import annotations

import statistics
import time

from . import _native as N

SEG = 1 << 24


def utilization(size: int, heap_bytes: int | None = None, batch: int = 100_000, max_batches: int = 1 << 20) -> dict:
    """E8 on the current allocator (call right after init or reset).

    Allocates `batch` requests of `size` per bulk call, keeping every pointer
    live, until a call returns at least one NULL.  Returns the
    successes (non-NULL pointers over all batches, the failing one included),
    the batches issued and utilization = successes * size / heap bytes (the
    fraction of the theoretical maximum number of allocations)."""
    import torch
    st = N.gallatin_stats()
    heap = heap_bytes or st["heap_bytes"]
    sizes = torch.full((batch,), size, dtype=torch.int64, device="cuda")
    keep = []
    succ = 0
    t0 = time.perf_counter()
    for b in range(max_batches):
        p = torch.empty(batch, dtype=torch.int64, device="cuda")
        N.gallatin_malloc(sizes, p)
        ok = int(torch.count_nonzero(p).item())
        succ += ok
        keep.append(p)
        if ok < batch:
            break
    dt = time.perf_counter() - t0
    return {"size": size, "successes": succ, "batches": len(keep), "heap_bytes": heap,
            "utilization": succ * size / heap, "seconds": dt, "ptrs": keep}


def fragmentation(size: int, n: int = 1 << 20) -> dict:
    """E7: one bulk call of n requests of `size`; the gap between the highest
    and lowest address handed out, and that gap over the bytes
    requested (1.0 = perfectly packed)."""
    import torch
    sizes = torch.full((n,), size, dtype=torch.int64, device="cuda")
    p = torch.empty_like(sizes)
    N.gallatin_malloc(sizes, p)
    live = p[p != 0]
    lo, hi = int(live.min().item()), int(live.max().item())
    rng = hi - lo
    return {"size": size, "n": n, "nulls": n - live.numel(), "range_bytes": rng,
            "range_over_requested": (rng + size) / (n * size), "ptrs": p, "sizes": sizes}


def _round_times(size: int, n: int, rounds: int, reset: bool) -> tuple[list[float], list[float]]:
    import torch
    sizes = torch.full((n,), size, dtype=torch.int64, device="cuda")
    p = torch.empty_like(sizes)
    s = torch.cuda.current_stream()                      # events and calls on one stream
    mm, fm = [], []
    for _ in range(rounds):
        if reset:
            N.gallatin_reset()
        a, b, c = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        a.record(s)
        N.gallatin_malloc(sizes, p)
        b.record(s)
        N.gallatin_free(p)
        c.record(s)
        torch.cuda.synchronize()
        mm.append(a.elapsed_time(b))
        fm.append(b.elapsed_time(c))
    return mm, fm


def warm_vs_cold(size: int, n: int, rounds: int = 20) -> dict:
    """E6: median malloc/free time per round with a reset before each round
    (cold) and after one untimed round without any reset (warm)."""
    N.gallatin_reset()
    cm, cf = _round_times(size, n, rounds, True)
    N.gallatin_reset()
    _round_times(size, n, 1, False)                 # the untimed first round
    wm, wf = _round_times(size, n, rounds, False)
    return {"size": size, "n": n, "rounds": rounds,
            "cold": {"malloc_ms": statistics.median(cm), "free_ms": statistics.median(cf),
                     "malloc_var_ms2": statistics.pvariance(cm), "free_var_ms2": statistics.pvariance(cf)},
            "warm": {"malloc_ms": statistics.median(wm), "free_ms": statistics.median(wf),
                     "malloc_var_ms2": statistics.pvariance(wm), "free_var_ms2": statistics.pvariance(wf)}}


def variance(size: int, n: int, rounds: int = 50) -> dict:
    """E5: per-round malloc and free times of `rounds` cold rounds (the paper's
    50 runs); median, variance and spread."""
    mm, fm = _round_times(size, n, rounds, True)
    return {"size": size, "n": n, "rounds": rounds,
            "malloc_ms_median": statistics.median(mm), "malloc_var_ms2": statistics.pvariance(mm),
            "malloc_ms_min": min(mm), "malloc_ms_max": max(mm),
            "free_ms_median": statistics.median(fm), "free_var_ms2": statistics.pvariance(fm),
            "free_ms_min": min(fm), "free_ms_max": max(fm)}


def init_time(heap_bytes: int, reps: int = 3, **knobs) -> dict:
    """E1: wall time of gallatin_init (heap + metadata cudaMalloc, pristine
    image written, synchronized) and of gallatin_destroy; the allocator is
    left destroyed."""
    import torch
    if N.gallatin_is_initialized():
        N.gallatin_destroy()
    ti, td = [], []
    for _ in range(reps):
        torch.cuda.synchronize()
        t = time.perf_counter()
        N.gallatin_init(heap_bytes, **knobs)
        torch.cuda.synchronize()
        ti.append((time.perf_counter() - t) * 1e3)
        t = time.perf_counter()
        N.gallatin_destroy()
        torch.cuda.synchronize()
        td.append((time.perf_counter() - t) * 1e3)
    return {"heap_bytes": heap_bytes, "init_ms_median": statistics.median(ti), "init_ms_min": min(ti),
            "destroy_ms_median": statistics.median(td), "reps": reps}
