"""Seeded synthetic inputs shared by the CUDA path's tests/bench and the oracle.

This module holds NO arithmetic of the method (no size classes, no trees, no
addresses): only random numbers and the shapes of the paper's workloads
(PAPER.md S6).  Both sides receive the arrays it
returns; neither side generates its own.

Seeds: base 0x6A11A7; the seed of (config, cell) is
``splitmix64(base ^ (config << 32) ^ cell)``.
"""
from __future__ import annotations

import numpy as np

BASE_SEED = 0x6A11A7
_M64 = (1 << 64) - 1


def splitmix64_scalar(x: int) -> int:
    x = (x + 0x9E3779B97F4A7C15) & _M64
    z = x
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def cell_seed(config: int, cell: int = 0) -> int:
    return splitmix64_scalar(BASE_SEED ^ (config << 32) ^ cell)


def splitmix64(seed: int, n: int) -> np.ndarray:
    """n uniform u64 words: the splitmix64 stream of `seed` (counter-based)."""
    with np.errstate(over="ignore"):
        i = np.arange(1, n + 1, dtype=np.uint64)
        z = np.uint64(seed & _M64) + i * np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def uniform_below(seed: int, n: int, bound: int) -> np.ndarray:
    """n integers uniform in [0, bound) (multiply-high; bias < 2^-40 for bound < 2^24)."""
    r = splitmix64(seed, n)
    if bound <= (1 << 32):
        return ((r >> np.uint64(32)) * np.uint64(bound)) >> np.uint64(32)
    return r % np.uint64(bound)


def distinct_below(seed: int, n: int, bound: int) -> np.ndarray:
    """n DISTINCT integers in [0, bound), in random order (a permutation sample)."""
    assert n <= bound
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.choice(bound, size=n, replace=False).astype(np.uint64)


def permutation(seed: int, n: int) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    return rng.permutation(n).astype(np.uint64)


# --------------------------------------------------------------- vEB (C1) ---
def veb_workload(k: int = 20, n: int = 1 << 16, seed: int | None = None) -> dict:
    """Config 1 vEB batches on a 2^k universe:
    I  = n distinct uniform keys (insert batch),
    S1 = n uniform queries + {0, u-1, max(I), max(I)+1} (successor batch),
    D  = n distinct keys, half drawn from I and half uniform (delete batch),
    S2 = n uniform queries (successor batch after the deletes)."""
    seed = cell_seed(1, 100 + k) if seed is None else seed
    u = 1 << k
    ins = distinct_below(seed ^ 1, n, u)
    q1 = uniform_below(seed ^ 2, n, u)
    edge = np.array([0, u - 1, int(ins.max()), min(int(ins.max()) + 1, u - 1)], dtype=np.uint64)
    q1 = np.concatenate([q1, edge])
    half = n // 2
    from_i = ins[distinct_below(seed ^ 3, half, n).astype(np.int64)]
    rest = uniform_below(seed ^ 4, 4 * n, u)
    rest = np.setdiff1d(np.unique(rest), from_i)
    rng = np.random.Generator(np.random.PCG64(seed ^ 5))
    rest = rng.permutation(rest)[: n - half]
    dele = np.concatenate([from_i, rest.astype(np.uint64)])
    dele = dele[rng.permutation(len(dele))]
    q2 = uniform_below(seed ^ 6, n, u)
    return {"k": k, "insert": ins, "succ1": q1, "delete": dele, "succ2": q2}


# ------------------------------------------------------ allocator sizes ---
SLICE_SIZES = [16 << i for i in range(9)]          # 16 B .. 4096 B
LARGE_SIZES = [(1 << 20) << i for i in range(7)]   # 1 MB .. 64 MB (BASELINE configs[2])


def single_sizes(size: int, n: int) -> np.ndarray:
    """Config 2 / 4: every thread asks for the same size."""
    return np.full(n, size, dtype=np.uint64)


def mixed_sizes(n: int, seed: int | None = None, upper: int = 4096, p_large: float = 2.0 ** -12,
                exact_pow2: bool = True) -> np.ndarray:
    """Config 3: per thread, with probability p_large a large size uniform over
    {1,2,4,8,16,32,64} MB, else a power of two uniform in [16, upper].
    exact_pow2=False draws sizes uniform in [1, 4096] B / [1, 64 MB] instead (C3b)."""
    seed = cell_seed(3) if seed is None else seed
    r_kind = splitmix64(seed ^ 11, n)
    large = r_kind < np.uint64(int(p_large * 2.0 ** 64))
    nsmall = int(np.log2(upper)) - 3
    if exact_pow2:
        small = np.uint64(16) << uniform_below(seed ^ 12, n, nsmall)
        big = np.uint64(1 << 20) << uniform_below(seed ^ 13, n, len(LARGE_SIZES))
    else:
        small = uniform_below(seed ^ 12, n, upper) + np.uint64(1)
        big = uniform_below(seed ^ 13, n, 64 << 20) + np.uint64(1)
    return np.where(large, big, small).astype(np.uint64)


def replay_ops(n_ops: int, seed: int, p_free: float = 0.4, p_drain: float = 0.0,
               sizes: list[int] | None = None, size_weights: list[float] | None = None,
               nkeys: int = 1 << 16) -> tuple[np.ndarray, np.ndarray, np.ndarray]:
    """A random sequential op list for serialized replay:
    kinds 0 = malloc(args[i]) with slot key keys[i]; 1 = free(result of op
    args[i]) -- each live allocation freed at most once; 2 = drain."""
    rng = np.random.Generator(np.random.PCG64(seed))
    if sizes is None:
        # every slice class, non-power-of-two slices (rounding, A-4), malloc(0)
        # (NULL), whole blocks, exactly one segment (A-3) and one byte more
        sizes = SLICE_SIZES + [0, 1, 17, 100, 4095, 5000, 70000, 1 << 20, 3 << 20, 16 << 20, (16 << 20) + 1,
                               40 << 20]
    sizes = np.asarray(sizes, dtype=np.uint64)
    w = None if size_weights is None else np.asarray(size_weights, dtype=float) / sum(size_weights)
    kinds = np.zeros(n_ops, dtype=np.uint8)
    args = np.zeros(n_ops, dtype=np.uint64)
    keys = rng.integers(0, nkeys, size=n_ops).astype(np.uint64)
    live: list[int] = []
    for i in range(n_ops):
        r = rng.random()
        if r < p_drain:
            kinds[i] = 2
        elif r < p_drain + p_free and live:
            j = int(rng.integers(len(live)))
            live[j], live[-1] = live[-1], live[j]
            kinds[i] = 1
            args[i] = live.pop()
        else:
            kinds[i] = 0
            args[i] = sizes[rng.choice(len(sizes), p=w)]
            live.append(i)
    return kinds, args, keys


# ------------------------------------------------------- streaming graph ---
def rmat_edges(scale: int, n: int, seed: int, device: str = "cpu", abcd=(0.57, 0.19, 0.19, 0.05),
               chunk: int = 1 << 24):
    """n R-MAT edges over 2^scale vertices (Chakrabarti et al.; SURVEY 8(d) C5:
    (a,b,c,d) = (0.57, 0.19, 0.19, 0.05), multi-edges kept) with a seeded
    vertex permutation.  Returns int32 torch tensors (src, dst) on `device`."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed & ((1 << 63) - 1))
    a, b, c, _ = abcd
    src = torch.empty(n, dtype=torch.int32, device=device)
    dst = torch.empty(n, dtype=torch.int32, device=device)
    for lo in range(0, n, chunk):
        m = min(chunk, n - lo)
        s = torch.zeros(m, dtype=torch.int64, device=device)
        d = torch.zeros(m, dtype=torch.int64, device=device)
        for _ in range(scale):
            r = torch.rand(m, generator=g, device=device)
            s = s * 2 + (r >= a + b).to(torch.int64)
            d = d * 2 + (((r >= a) & (r < a + b)) | (r >= a + b + c)).to(torch.int64)
        src[lo:lo + m] = s.to(torch.int32)
        dst[lo:lo + m] = d.to(torch.int32)
    perm = torch.randperm(1 << scale, generator=g, device=device).to(torch.int32)
    return perm[src.long()], perm[dst.long()]


def graph_workload(scale: int, n_edges: int, seed: int | None = None, device: str = "cpu", batches: int = 8,
                   n_expand: int = 1 << 16, rounds: int = 8) -> dict:
    """BASELINE configs[4] phases:
      init    : the first n/2 edges,
      insert  : the other n/2 in `batches` batches,
      delete  : `batches` batches of n/16 edges sampled without replacement
                from the inserted multiset,
      expand  : min(n_expand, V/4) distinct seeded vertices, `rounds` rounds."""
    import torch
    seed = cell_seed(5, scale) if seed is None else seed
    V = 1 << scale
    src, dst = rmat_edges(scale, n_edges, seed, device)
    half = n_edges // 2
    g = torch.Generator(device=device)
    g.manual_seed((seed ^ 0x5DEECE66D) & ((1 << 63) - 1))
    per = torch.randperm(n_edges, generator=g, device=device)
    db = n_edges // (2 * batches)
    ins_b = (n_edges - half) // batches
    nexp = min(n_expand, V // 4)
    exp_v = torch.randperm(V, generator=g, device=device)[:nexp].to(torch.int32)
    return {
        "V": V,
        "init": (src[:half], dst[:half]),
        "insert": [(src[half + k * ins_b: half + (k + 1) * ins_b], dst[half + k * ins_b: half + (k + 1) * ins_b])
                   for k in range(batches)],
        "delete": [(src[per[k * db:(k + 1) * db]], dst[per[k * db:(k + 1) * db]]) for k in range(batches)],
        "expand": exp_v,
        "rounds": rounds,
    }
