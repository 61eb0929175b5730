// graph.cu -- the streaming-graph workload (BASELINE configs[4]; PAPER.md
// S6.12) on the DEVICE-side allocator: every per-vertex edge list
// is malloc'd, grown, shrunk and freed by GPU threads through
// include/gallatin/device.cuh.  C-ABI: include/gallatin_graph.h.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "gallatin.h"
#include "gallatin/device.cuh"
#include "gallatin_graph.h"

using gallatin::gallatin_free;
using gallatin::gallatin_malloc;

struct gallatin_graph {
    uint32_t V;
    uint64_t *list;       // per-vertex uint32_t* (as u64)
    uint32_t *size, *cap, *cnt;
    uint64_t *old;        // list being replaced during a grow / shrink
    uint32_t *work;       // vertices to process (compacted)
    uint32_t *work2;      // big vertices (CTA-per-vertex deletes)
    uint32_t *nwork;      // [0] work, [1] work2
    unsigned long long *ctr;   // [0] mallocs [1] frees [2] failed mallocs [3] vertex ids >= V (ignored)
    uint32_t *hkeys;      // delete-batch hash, one region per source vertex: dst -> remaining count
    uint32_t *hcnt;
    uint64_t hcap;        // slots allocated (>= 4 x the batch)
    uint32_t *hoff;       // per vertex: first slot of its region (next_pow2(2 cnt) slots)
    uint32_t *hbump;      // region allocator
    uint32_t *lock;       // per-vertex lock word of the single-edge operations
};

namespace {
constexpr int kT = 256;
constexpr uint32_t kBig = 2048;        // lists at least this long delete with a whole CTA
#ifndef GALLATIN_GRAPH_MINB
#define GALLATIN_GRAPH_MINB 4
#endif
// kernels that call the device allocator: register cap for >= this many CTAs/SM
constexpr int kGraphMinBlocks = GALLATIN_GRAPH_MINB;

inline cudaStream_t S(void *s) { return reinterpret_cast<cudaStream_t>(s); }
inline unsigned blocks(uint64_t n) { return (unsigned)((n + kT - 1) / kT); }
int status() {
    const cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        fprintf(stderr, "gallatin_graph: %s\n", cudaGetErrorString(e));
        return GALLATIN_ERR_CUDA;
    }
    return GALLATIN_OK;
}

__device__ __forceinline__ uint32_t next_pow2(uint32_t x) { return x <= 1 ? 1u : 1u << (32 - __clz(x - 1)); }
__device__ __forceinline__ uint32_t list_cap(uint32_t size) { return next_pow2(size < 4 ? 4 : size); }
__device__ __forceinline__ uint32_t lane() { return threadIdx.x & 31; }

// one atomic per warp for the statistics counters (all lanes present)
__device__ __forceinline__ void count_warp(unsigned long long *ctr, bool m, bool f, bool fail) {
    const unsigned a = __ballot_sync(0xFFFFFFFFu, m), b = __ballot_sync(0xFFFFFFFFu, f),
                   c = __ballot_sync(0xFFFFFFFFu, fail);
    if (lane() == 0) {
        if (a) atomicAdd(ctr + 0, (unsigned long long)__popc(a));
        if (b) atomicAdd(ctr + 1, (unsigned long long)__popc(b));
        if (c) atomicAdd(ctr + 2, (unsigned long long)__popc(c));
    }
}

// cnt[src] += 1 per edge, one atomic per distinct source in a warp
// (a source id >= V is ignored by the whole batch and counted in ctr[3])
__global__ void k_count(gallatin_graph g, const uint32_t *src, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    uint32_t s = i < n ? src[i] : 0xFFFFFFFFu;
    if (s != 0xFFFFFFFFu && s >= g.V) {
        atomicAdd(g.ctr + 3, 1ull);
        s = 0xFFFFFFFFu;
    }
    const unsigned peers = __match_any_sync(0xFFFFFFFFu, s);
    if (s != 0xFFFFFFFFu && lane() == (uint32_t)__ffs((int)peers) - 1) atomicAdd(g.cnt + s, (uint32_t)__popc(peers));
}

// Per vertex with cnt new edges: a batch that overflows the list reallocates
// it to the next power of two (device malloc); non-empty old lists are queued
// for the copy + free.
__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_grow(gallatin_graph g) {
    const uint64_t v = blockIdx.x * (uint64_t)kT + threadIdx.x;
    bool m = false, fail = false;
    if (v < g.V) {
        const uint32_t c = g.cnt[v];
        if (c) {
            const uint32_t s = g.size[v], need = s + c;
            if (need > g.cap[v]) {
                const uint32_t nc = list_cap(need);
                void *p = gallatin_malloc((uint64_t)nc * 4);
                if (!p) {
                    fail = true;
                } else {
                    m = true;
                    if (s > 0) {
                        g.old[v] = g.list[v];
                        g.work[atomicAdd(g.nwork, 1u)] = (uint32_t)v;
                    }
                    g.list[v] = reinterpret_cast<uint64_t>(p);
                    g.cap[v] = nc;
                }
            }
        }
    }
    count_warp(g.ctr, m, false, fail);
}

// warp per queued vertex: copy size[v] entries old -> new, free the old list;
// lists of kHuge entries or more are left to the whole grid (k_copy_huge)
constexpr uint32_t kHuge = 1u << 16;
__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_copy(gallatin_graph g) {
    const uint32_t nw = *g.nwork;
    const uint64_t warps = (uint64_t)gridDim.x * (kT / 32);
    unsigned long long frees = 0;
    for (uint64_t w = (blockIdx.x * (uint64_t)kT + threadIdx.x) >> 5; w < nw; w += warps) {
        const uint32_t v = g.work[w], s = g.size[v];
        if (s >= kHuge) {
            if (lane() == 0) g.work2[atomicAdd(g.nwork + 1, 1u)] = v;
            continue;
        }
        const uint32_t *src = reinterpret_cast<const uint32_t *>(g.old[v]);
        uint32_t *dst = reinterpret_cast<uint32_t *>(g.list[v]);
        for (uint32_t k = lane(); k < s; k += 32) dst[k] = src[k];
        __syncwarp();
        if (lane() == 0) {
            gallatin_free((void *)src);
            frees++;
        }
    }
    if (lane() == 0 && frees) atomicAdd(g.ctr + 1, frees);
}

// Huge lists (a hub drawn by the expansion reaches hundreds of MB): every CTA
// takes 16 KB chunks of each in turn, 16-byte vector copies (lists come from
// the allocator 16-byte aligned); the old lists are freed afterwards.
constexpr uint32_t kChunk = 4096;                      // entries per CTA chunk
__global__ void k_copy_huge(gallatin_graph g) {
    const uint32_t nb = g.nwork[1];
    for (uint32_t b = 0; b < nb; b++) {
        const uint32_t v = g.work2[b], s = g.size[v];
        const uint4 *src = reinterpret_cast<const uint4 *>(g.old[v]);
        uint4 *dst = reinterpret_cast<uint4 *>(g.list[v]);
        const uint32_t q = s / 4, chunks = (s + kChunk - 1) / kChunk;
        for (uint32_t c = blockIdx.x; c < chunks; c += gridDim.x) {
            const uint32_t lo = c * (kChunk / 4), hi = min(q, lo + kChunk / 4);
            for (uint32_t k = lo + threadIdx.x; k < hi; k += kT) dst[k] = src[k];
            if (c == chunks - 1 && threadIdx.x < (s & 3))              // the last 1-3 entries
                reinterpret_cast<uint32_t *>(dst)[4 * q + threadIdx.x] =
                    reinterpret_cast<const uint32_t *>(src)[4 * q + threadIdx.x];
        }
    }
}
__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_free_huge(gallatin_graph g) {
    unsigned long long frees = 0;
    for (uint32_t b = blockIdx.x * kT + threadIdx.x; b < g.nwork[1]; b += gridDim.x * kT) {
        gallatin_free(reinterpret_cast<void *>(g.old[g.work2[b]]));
        frees++;
    }
    if (frees) atomicAdd(g.ctr + 1, frees);
}

// append: one atomic per distinct source in a warp reserves the positions
__global__ void k_scatter(gallatin_graph g, const uint32_t *src, const uint32_t *dst, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    uint32_t s = i < n ? src[i] : 0xFFFFFFFFu;
    if (s >= g.V) s = 0xFFFFFFFFu;                            // counted by k_count
    const unsigned peers = __match_any_sync(0xFFFFFFFFu, s);
    const uint32_t leader = (uint32_t)__ffs((int)peers) - 1;
    uint32_t base = 0;
    if (s != 0xFFFFFFFFu && lane() == leader) base = atomicAdd(g.size + s, (uint32_t)__popc(peers));
    base = __shfl_sync(peers, base, (int)leader);
    if (s == 0xFFFFFFFFu) return;
    const uint32_t pos = base + (uint32_t)__popc(peers & ((1u << lane()) - 1));
    reinterpret_cast<uint32_t *>(g.list[s])[pos] = dst[i];
}

// ---- delete batch ------------------------------------------------------------
__device__ __forceinline__ uint64_t hmix(uint64_t k) {
    k ^= k >> 33;
    k *= 0xff51afd7ed558ccdull;
    k ^= k >> 33;
    return k;
}

// The batch's deletions live in one small open-addressing region per source
// vertex (next_pow2(2 cnt) slots), so the probes of one vertex's list entries
// stay in a few cache lines instead of a batch-wide table in HBM (one random
// DRAM sector per list entry).
constexpr uint32_t kHEmpty = 0xFFFFFFFFu;
__device__ __forceinline__ uint32_t region_slots(uint32_t c) { return c ? next_pow2(2 * c) : 0u; }

// hoff[v] = a region of region_slots(cnt[v]) slots: one bump per CTA of the
// CTA's exclusive prefix (region order is irrelevant)
__global__ void k_hash_regions(gallatin_graph g) {
    __shared__ uint32_t wsum[kT / 32];
    __shared__ uint32_t base;
    const uint64_t v = blockIdx.x * (uint64_t)kT + threadIdx.x;
    const uint32_t r = v < g.V ? region_slots(g.cnt[v]) : 0u;
    uint32_t x = r;                                           // inclusive warp scan
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
        if (lane() >= (uint32_t)d) x += y;
    }
    if (lane() == 31) wsum[threadIdx.x >> 5] = x;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t t = 0;
        for (int w = 0; w < kT / 32; w++) { const uint32_t s = wsum[w]; wsum[w] = t; t += s; }
        base = t ? atomicAdd(g.hbump, t) : 0u;
    }
    __syncthreads();
    if (v < g.V && r) g.hoff[v] = base + wsum[threadIdx.x >> 5] + x - r;
}

__global__ void k_hash_insert(gallatin_graph g, const uint32_t *src, const uint32_t *dst, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    if (i >= n) return;
    const uint32_t s = src[i], key = dst[i];
    if (s >= g.V) return;                                     // counted by k_count
    uint32_t *keys = g.hkeys + g.hoff[s], *cnts = g.hcnt + g.hoff[s];
    const uint32_t mask = region_slots(g.cnt[s]) - 1;
    for (uint32_t h = (uint32_t)hmix(key) & mask;; h = (h + 1) & mask) {
        const uint32_t k = atomicCAS(keys + h, kHEmpty, key);
        if (k == kHEmpty || k == key) {
            atomicAdd(cnts + h, 1u);
            return;
        }
    }
}

// take one pending deletion of x from vertex v's region; true if this instance is deleted
__device__ __forceinline__ bool hash_take(const uint32_t *keys, uint32_t *cnts, uint32_t mask, uint32_t x) {
    for (uint32_t h = (uint32_t)hmix(x) & mask;; h = (h + 1) & mask) {
        const uint32_t k = keys[h];
        if (k == kHEmpty) return false;
        if (k != x) continue;
        uint32_t c = *(volatile uint32_t *)(cnts + h);
        while (c > 0) {
            const uint32_t o = atomicCAS(cnts + h, c, c - 1);
            if (o == c) return true;
            c = o;
        }
        return false;
    }
}

__global__ void k_list_work(gallatin_graph g) {
    const uint64_t v = blockIdx.x * (uint64_t)kT + threadIdx.x;
    if (v >= g.V || g.cnt[v] == 0 || g.size[v] == 0) return;
    if (g.size[v] >= kBig) g.work2[atomicAdd(g.nwork + 1, 1u)] = (uint32_t)v;
    else g.work[atomicAdd(g.nwork, 1u)] = (uint32_t)v;
}

// Shrink after a delete (once per batch per vertex): size 0 frees the list,
// size <= cap/4 reallocates to the next power of two; executed by one warp.
__device__ void shrink_warp(const gallatin_graph &g, uint32_t v, uint32_t out, bool &m, bool &f, bool &fail) {
    const uint32_t cap = g.cap[v];
    uint64_t np = 0;
    bool act = false;
    if (lane() == 0) {
        g.size[v] = out;
        if (out == 0) {
            gallatin_free(reinterpret_cast<void *>(g.list[v]));
            g.list[v] = 0;
            g.cap[v] = 0;
            f = true;
        } else if (out <= cap / 4 && cap > 4) {
            const uint32_t nc = list_cap(out);
            void *p = gallatin_malloc((uint64_t)nc * 4);
            if (p) {
                np = reinterpret_cast<uint64_t>(p);
                act = true;
                m = f = true;
            } else {
                fail = true;
            }
        }
    }
    act = __shfl_sync(0xFFFFFFFFu, act, 0);
    if (!act) return;
    np = __shfl_sync(0xFFFFFFFFu, np, 0);
    const uint32_t *src = reinterpret_cast<const uint32_t *>(g.list[v]);
    uint32_t *dst = reinterpret_cast<uint32_t *>(np);
    for (uint32_t k = lane(); k < out; k += 32) dst[k] = src[k];
    __syncwarp();
    if (lane() == 0) {
        gallatin_free((void *)src);
        g.list[v] = np;
        g.cap[v] = list_cap(out);
    }
}

// warp per vertex: scan, drop the deleted instances, compact in place
__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_delete_small(gallatin_graph g) {
    const uint32_t nw = g.nwork[0];
    const uint64_t warps = (uint64_t)gridDim.x * (kT / 32);
    bool m = false, f = false, fail = false;
    for (uint64_t w = (blockIdx.x * (uint64_t)kT + threadIdx.x) >> 5; w < nw; w += warps) {
        const uint32_t v = g.work[w], s = g.size[v];
        uint32_t *L = reinterpret_cast<uint32_t *>(g.list[v]);
        const uint32_t *hk = g.hkeys + g.hoff[v];
        uint32_t *hc = g.hcnt + g.hoff[v];
        const uint32_t hm = region_slots(g.cnt[v]) - 1;
        uint32_t out = 0;
        for (uint32_t b = 0; b < s; b += 32) {
            const uint32_t i = b + lane();
            uint32_t x = 0;
            bool keep = false;
            if (i < s) {
                x = L[i];
                keep = !hash_take(hk, hc, hm, x);
            }
            const unsigned km = __ballot_sync(0xFFFFFFFFu, keep);
            if (keep) L[out + __popc(km & ((1u << lane()) - 1))] = x;    // out <= b: never ahead of the reads
            out += (uint32_t)__popc(km);
        }
        __syncwarp();
        shrink_warp(g, v, out, m, f, fail);
    }
    count_warp(g.ctr, m, f, fail);
}

// CTA per big vertex: same, with a block-wide prefix per 256-entry chunk
__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_delete_big(gallatin_graph g) {
    __shared__ uint32_t wsum[kT / 32];
    __shared__ uint32_t out_s;
    const uint32_t nw = g.nwork[1], wid = threadIdx.x >> 5;
    bool m = false, f = false, fail = false;
    for (uint32_t w = blockIdx.x; w < nw; w += gridDim.x) {
        const uint32_t v = g.work2[w], s = g.size[v];
        uint32_t *L = reinterpret_cast<uint32_t *>(g.list[v]);
        const uint32_t *hk = g.hkeys + g.hoff[v];
        uint32_t *hc = g.hcnt + g.hoff[v];
        const uint32_t hm = region_slots(g.cnt[v]) - 1;
        if (threadIdx.x == 0) out_s = 0;
        __syncthreads();
        for (uint32_t b = 0; b < s; b += kT) {
            const uint32_t i = b + threadIdx.x;
            uint32_t x = 0;
            bool keep = false;
            if (i < s) {
                x = L[i];
                keep = !hash_take(hk, hc, hm, x);
            }
            const unsigned km = __ballot_sync(0xFFFFFFFFu, keep);
            if (lane() == 0) wsum[wid] = (uint32_t)__popc(km);
            __syncthreads();
            uint32_t before = out_s, tot = 0;
            for (uint32_t q = 0; q < kT / 32; q++) {
                if (q < wid) before += wsum[q];
                tot += wsum[q];
            }
            if (keep) L[before + __popc(km & ((1u << lane()) - 1))] = x;
            __syncthreads();
            if (threadIdx.x == 0) out_s += tot;
            __syncthreads();
        }
        if (wid == 0) shrink_warp(g, v, out_s, m, f, fail);
        __syncthreads();
    }
    count_warp(g.ctr, m, f, fail);
}

// ---- expansion ---------------------------------------------------------------
__global__ void k_expand_prep(gallatin_graph g, const uint32_t *vs, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    if (i >= n) return;
    if (vs[i] >= g.V) {                        // ignored, counted
        atomicAdd(g.ctr + 3, 1ull);
        return;
    }
    const uint32_t s = g.size[vs[i]];
    g.cnt[vs[i]] = s < 4 ? 4 : s;              // each round appends max(size, 4) edges
}

__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_expand_fill(gallatin_graph g, const uint32_t *vs, uint64_t n) {
    const uint64_t warps = (uint64_t)gridDim.x * (kT / 32);
    for (uint64_t w = (blockIdx.x * (uint64_t)kT + threadIdx.x) >> 5; w < n; w += warps) {
        const uint32_t v = vs[w];
        if (v >= g.V) continue;
        const uint32_t s0 = g.size[v], add = g.cnt[v];
        if (add >= kHuge) {                                   // the whole grid fills it (k_expand_huge)
            if (lane() == 0) g.work2[atomicAdd(g.nwork + 1, 1u)] = v;
            continue;
        }
        uint32_t *L = reinterpret_cast<uint32_t *>(g.list[v]);
        for (uint32_t j = lane(); j < add; j += 32) L[s0 + j] = (uint32_t)(((uint64_t)v + s0 + j + 1) % g.V);
        __syncwarp();
        if (lane() == 0) g.size[v] = s0 + add;
    }
}
__global__ void k_expand_huge(gallatin_graph g) {
    const uint32_t nb = g.nwork[1];
    for (uint32_t b = 0; b < nb; b++) {
        const uint32_t v = g.work2[b], s0 = g.size[v], add = g.cnt[v];
        uint32_t *L = reinterpret_cast<uint32_t *>(g.list[v]);
        for (uint64_t j = blockIdx.x * (uint64_t)kT + threadIdx.x; j < add; j += (uint64_t)gridDim.x * kT)
            L[s0 + j] = (uint32_t)(((uint64_t)v + s0 + j + 1) % g.V);
    }
}
__global__ void k_expand_huge_size(gallatin_graph g) {
    for (uint32_t b = blockIdx.x * kT + threadIdx.x; b < g.nwork[1]; b += gridDim.x * kT)
        g.size[g.work2[b]] += g.cnt[g.work2[b]];
}

__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_free_all(gallatin_graph g) {
    const uint64_t v = blockIdx.x * (uint64_t)kT + threadIdx.x;
    bool f = false;
    if (v < g.V && g.list[v]) {
        gallatin_free(reinterpret_cast<void *>(g.list[v]));
        g.list[v] = 0;
        g.size[v] = 0;
        g.cap[v] = 0;
        f = true;
    }
    count_warp(g.ctr, false, f, false);
}

__global__ void k_export(gallatin_graph g, uint32_t *size, uint32_t *cap, uint64_t *list) {
    const uint64_t v = blockIdx.x * (uint64_t)kT + threadIdx.x;
    if (v >= g.V) return;
    if (size) size[v] = g.size[v];
    if (cap) cap[v] = g.cap[v];
    if (list) list[v] = g.list[v];
}

__global__ void k_gather(gallatin_graph g, const uint64_t *off, uint32_t *out) {
    const uint64_t warps = (uint64_t)gridDim.x * (kT / 32);
    for (uint64_t v = (blockIdx.x * (uint64_t)kT + threadIdx.x) >> 5; v < g.V; v += warps) {
        const uint32_t s = g.size[v];
        const uint32_t *L = reinterpret_cast<const uint32_t *>(g.list[v]);
        for (uint32_t k = lane(); k < s; k += 32) out[off[v] + k] = L[k];
    }
}

// ---- single-edge operations ("edge updates" / "edge deletes") ---------
// One thread per edge, each under its source vertex's lock: the list grows by
// doubling when an append finds it full (malloc, copy, free: the allocator is
// called per overflowing edge, not per batch) and shrinks after every delete
// that leaves size <= cap/4 (reading A-29 applied per edge).
// [dev] The lanes of a warp that hold their vertex's lock are served one at a
// time by the WHOLE warp: the 32 lanes scan (delete) or copy (grow / shrink)
// the holder's list together; the holder alone updates size, cap and list,
// calls the allocator and releases the lock.  Same result as one thread per
// edge (the holder's operation is unchanged); a hub list is scanned 32 (x4
// in flight) entries per step instead of one.  Lanes whose lock is taken
// retry after the round.
__device__ __forceinline__ void warp_copy(uint32_t *dst, const uint32_t *src, uint32_t n) {
    // lists hold a multiple of 4 entries (caps are powers of two >= 4) and are 16 B aligned
    uint4 *d = reinterpret_cast<uint4 *>(dst);
    const uint4 *s = reinterpret_cast<const uint4 *>(src);
    for (uint32_t k = lane(); k < (n + 3) / 4; k += 32) d[k] = s[k];
}

// last index < s of x in L (all lanes get it), or -1
__device__ __forceinline__ int64_t warp_find_last(const uint32_t *L, uint32_t s, uint32_t x) {
    for (int64_t top = s; top > 0; top -= 128) {
        uint32_t e[4];
        bool in[4];
#pragma unroll
        for (int u = 0; u < 4; u++) {                         // 4 loads in flight per lane
            const int64_t idx = top - 128 + 32 * u + lane();
            in[u] = idx >= 0;
            e[u] = in[u] ? L[idx] : 0u;
        }
#pragma unroll
        for (int u = 3; u >= 0; u--) {
            const unsigned m = __ballot_sync(0xFFFFFFFFu, in[u] && e[u] == x);
            if (m) return top - 128 + 32 * u + (31 - __clz((int)m));
        }
    }
    return -1;
}

__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_edge_insert(gallatin_graph g, const uint32_t *src,
                                                                      const uint32_t *dst, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    bool m = false, f = false, fail = false;
    const bool in = i < n && src[i] < g.V;
    if (i < n && !in) atomicAdd(g.ctr + 3, 1ull);             // vertex id >= V: ignored, counted
    const bool active = in;
    const uint32_t v = active ? src[i] : 0u, x = active ? dst[i] : 0u;
    bool done = !active;
    uint32_t ns = 32;
    while (__any_sync(0xFFFFFFFFu, !done)) {
        const bool got = !done && atomicCAS(g.lock + v, 0u, 1u) == 0u;
        bool grow = false;
        if (got) {
            __threadfence();                                   // acquire the previous holder's writes
            const uint32_t s = g.size[v];
            if (s < g.cap[v]) {                                // room: the holder appends alone
                reinterpret_cast<uint32_t *>(g.list[v])[s] = x;
                g.size[v] = s + 1;
                __threadfence();
                atomicExch(g.lock + v, 0u);
                done = true;
            } else {
                grow = true;
            }
        }
        unsigned holders = __ballot_sync(0xFFFFFFFFu, grow);    // the warp doubles these lists together
        while (holders) {
            const int l = __ffs((int)holders) - 1;
            holders &= holders - 1;
            const uint32_t vv = __shfl_sync(0xFFFFFFFFu, v, l);
            const uint32_t s = g.size[vv], c = g.cap[vv];
            uint32_t *L = reinterpret_cast<uint32_t *>(g.list[vv]);
            if (s == c) {                                      // full (or no list): double
                uint64_t p = 0;
                if (lane() == (uint32_t)l) {
                    p = reinterpret_cast<uint64_t>(gallatin_malloc((uint64_t)(c ? 2 * c : 4) * 4));
                    if (!p) fail = true;
                    else m = true;
                }
                p = __shfl_sync(0xFFFFFFFFu, p, l);
                if (p && L) warp_copy(reinterpret_cast<uint32_t *>(p), L, s);
                __syncwarp();
                if (lane() == (uint32_t)l && p) {
                    if (L) {
                        gallatin_free(L);
                        f = true;
                    }
                    g.list[vv] = p;
                    g.cap[vv] = c ? 2 * c : 4;
                    L = reinterpret_cast<uint32_t *>(p);
                }
                if (!p) L = nullptr;
            }
            if (lane() == (uint32_t)l) {
                if (L) {
                    L[s] = x;
                    g.size[vv] = s + 1;
                }
                __threadfence();                               // release this holder's writes
                atomicExch(g.lock + vv, 0u);
                done = true;
            }
            __syncwarp();
        }
        if (!done && !got) {
            __nanosleep(ns);
            if (ns < 256) ns <<= 1;
        }
    }
    count_warp(g.ctr, m, f, fail);
}

__global__ void __launch_bounds__(kT, kGraphMinBlocks) k_edge_delete(gallatin_graph g, const uint32_t *src,
                                                                      const uint32_t *dst, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kT + threadIdx.x;
    bool m = false, f = false, fail = false;
    const bool in = i < n && src[i] < g.V;
    if (i < n && !in) atomicAdd(g.ctr + 3, 1ull);             // vertex id >= V: ignored, counted
    const bool active = in;
    const uint32_t v = active ? src[i] : 0u, x = active ? dst[i] : 0u;
    bool done = !active;
    uint32_t ns = 32;
    while (__any_sync(0xFFFFFFFFu, !done)) {
        const bool got = !done && atomicCAS(g.lock + v, 0u, 1u) == 0u;
        unsigned holders = __ballot_sync(0xFFFFFFFFu, got);
        if (holders) __threadfence();
        while (holders) {
            const int l = __ffs((int)holders) - 1;
            holders &= holders - 1;
            const uint32_t vv = __shfl_sync(0xFFFFFFFFu, v, l), xx = __shfl_sync(0xFFFFFFFFu, x, l);
            uint32_t s = g.size[vv];
            const uint32_t c = g.cap[vv];
            uint32_t *L = reinterpret_cast<uint32_t *>(g.list[vv]);
            // newest entries first (appends go to the end): remove one
            // instance, the last entry fills the hole (reading R-7)
            const int64_t j = s ? warp_find_last(L, s, xx) : -1;
            uint64_t p = 0;
            bool copy = false;
            if (lane() == (uint32_t)l && j >= 0) {
                L[j] = L[s - 1];
                s--;
                g.size[vv] = s;
                if (s == 0) {
                    gallatin_free(L);
                    g.list[vv] = 0;
                    g.cap[vv] = 0;
                    f = true;
                } else if (c > 4 && s <= c / 4) {
                    p = reinterpret_cast<uint64_t>(gallatin_malloc((uint64_t)list_cap(s) * 4));
                    if (p) copy = true;
                    else fail = true;
                }
            }
            copy = __shfl_sync(0xFFFFFFFFu, copy, l);
            if (copy) {
                p = __shfl_sync(0xFFFFFFFFu, p, l);
                s = __shfl_sync(0xFFFFFFFFu, s, l);
                __syncwarp();                                  // the hole fill precedes the copy
                warp_copy(reinterpret_cast<uint32_t *>(p), L, s);
                __syncwarp();
                if (lane() == (uint32_t)l) {
                    gallatin_free(L);
                    g.list[vv] = p;
                    g.cap[vv] = list_cap(s);
                    m = f = true;
                }
            }
            if (lane() == (uint32_t)l) {
                __threadfence();
                atomicExch(g.lock + vv, 0u);
                done = true;
            }
            __syncwarp();
        }
        if (!done && !got) {
            __nanosleep(ns);
            if (ns < 256) ns <<= 1;
        }
    }
    count_warp(g.ctr, m, f, fail);
}

int run_grow(gallatin_graph *g, cudaStream_t st) {
    k_grow<<<blocks(g->V), kT, 0, st>>>(*g);
    k_copy<<<148 * 8, kT, 0, st>>>(*g);
    k_copy_huge<<<148 * 8, kT, 0, st>>>(*g);
    k_free_huge<<<148, kT, 0, st>>>(*g);
    return status();
}
}  // namespace

extern "C" {

int gallatin_graph_create(uint32_t V, gallatin_graph_t **out) {
    if (!out || V == 0) return GALLATIN_ERR_INVALID;
    if (!gallatin_is_initialized()) return GALLATIN_ERR_STATE;
    const int rc = gallatin::bind_device();            // the device API's constant view
    if (rc != GALLATIN_OK) return rc;
    gallatin_graph *g = new gallatin_graph{};
    g->V = V;
    bool ok = cudaMalloc(&g->list, 8ull * V) == cudaSuccess && cudaMalloc(&g->size, 4ull * V) == cudaSuccess &&
              cudaMalloc(&g->cap, 4ull * V) == cudaSuccess && cudaMalloc(&g->cnt, 4ull * V) == cudaSuccess &&
              cudaMalloc(&g->old, 8ull * V) == cudaSuccess && cudaMalloc(&g->work, 4ull * V) == cudaSuccess &&
              cudaMalloc(&g->work2, 4ull * V) == cudaSuccess && cudaMalloc(&g->nwork, 8) == cudaSuccess &&
              cudaMalloc(&g->ctr, 32) == cudaSuccess && cudaMalloc(&g->lock, 4ull * V) == cudaSuccess &&
              cudaMalloc(&g->hoff, 4ull * V) == cudaSuccess && cudaMalloc(&g->hbump, 4) == cudaSuccess;
    if (!ok) {
        cudaGetLastError();
        gallatin_graph_destroy(g, nullptr);
        return GALLATIN_ERR_NOMEM;
    }
    cudaMemset(g->list, 0, 8ull * V);
    cudaMemset(g->size, 0, 4ull * V);
    cudaMemset(g->cap, 0, 4ull * V);
    cudaMemset(g->ctr, 0, 32);
    cudaMemset(g->lock, 0, 4ull * V);
    *out = g;
    return status();
}

int gallatin_graph_destroy(gallatin_graph_t *g, void *stream) {
    if (!g) return GALLATIN_ERR_INVALID;
    if (g->list && gallatin_is_initialized()) k_free_all<<<blocks(g->V), kT, 0, S(stream)>>>(*g);
    cudaStreamSynchronize(S(stream));
    void *ptrs[] = {g->list, g->size, g->cap, g->cnt, g->old, g->work, g->work2, g->nwork, g->ctr, g->hkeys, g->hcnt,
                    g->lock, g->hoff, g->hbump};
    for (void *p : ptrs)
        if (p) cudaFree(p);
    delete g;
    return status();
}

int gallatin_graph_insert(gallatin_graph_t *g, const uint32_t *src, const uint32_t *dst, uint64_t n, void *stream) {
    if (!g || (n && (!src || !dst))) return GALLATIN_ERR_INVALID;
    if (n == 0) return GALLATIN_OK;
    cudaStream_t st = S(stream);
    cudaMemsetAsync(g->cnt, 0, 4ull * g->V, st);
    cudaMemsetAsync(g->nwork, 0, 8, st);
    k_count<<<blocks(n), kT, 0, st>>>(*g, src, n);
    int rc = run_grow(g, st);
    if (rc) return rc;
    k_scatter<<<blocks(n), kT, 0, st>>>(*g, src, dst, n);
    return status();
}

int gallatin_graph_delete(gallatin_graph_t *g, const uint32_t *src, const uint32_t *dst, uint64_t n, void *stream) {
    if (!g || (n && (!src || !dst))) return GALLATIN_ERR_INVALID;
    if (n == 0) return GALLATIN_OK;
    cudaStream_t st = S(stream);
    if (n > (1ull << 29)) return GALLATIN_ERR_INVALID;          // region offsets are 32-bit
    const uint64_t cap = 4 * n;                                 // sum of next_pow2(2 cnt[v]) <= 4 n
    if (cap > g->hcap) {
        if (g->hkeys) cudaFree(g->hkeys);
        if (g->hcnt) cudaFree(g->hcnt);
        g->hkeys = nullptr;
        g->hcnt = nullptr;
        if (cudaMalloc(&g->hkeys, 4 * cap) != cudaSuccess || cudaMalloc(&g->hcnt, 4 * cap) != cudaSuccess) {
            cudaGetLastError();
            g->hcap = 0;
            return GALLATIN_ERR_NOMEM;
        }
        g->hcap = cap;
    }
    gallatin_graph gv = *g;
    cudaMemsetAsync(g->hkeys, 0xFF, 4 * cap, st);
    cudaMemsetAsync(g->hcnt, 0, 4 * cap, st);
    cudaMemsetAsync(g->hbump, 0, 4, st);
    cudaMemsetAsync(g->cnt, 0, 4ull * g->V, st);
    cudaMemsetAsync(g->nwork, 0, 8, st);
    k_count<<<blocks(n), kT, 0, st>>>(gv, src, n);
    k_hash_regions<<<blocks(g->V), kT, 0, st>>>(gv);
    k_hash_insert<<<blocks(n), kT, 0, st>>>(gv, src, dst, n);
    k_list_work<<<blocks(g->V), kT, 0, st>>>(gv);
    k_delete_small<<<148 * 8, kT, 0, st>>>(gv);
    k_delete_big<<<148 * 4, kT, 0, st>>>(gv);
    return status();
}

int gallatin_graph_expand(gallatin_graph_t *g, const uint32_t *vs, uint64_t n, void *stream) {
    if (!g || (n && !vs)) return GALLATIN_ERR_INVALID;
    if (n == 0) return GALLATIN_OK;
    cudaStream_t st = S(stream);
    cudaMemsetAsync(g->cnt, 0, 4ull * g->V, st);
    cudaMemsetAsync(g->nwork, 0, 8, st);
    k_expand_prep<<<blocks(n), kT, 0, st>>>(*g, vs, n);
    int rc = run_grow(g, st);
    if (rc) return rc;
    cudaMemsetAsync(g->nwork + 1, 0, 4, st);                    // huge lists of this round's fill
    k_expand_fill<<<148 * 8, kT, 0, st>>>(*g, vs, n);
    k_expand_huge<<<148 * 8, kT, 0, st>>>(*g);
    k_expand_huge_size<<<148, kT, 0, st>>>(*g);
    return status();
}

int gallatin_graph_insert_edges(gallatin_graph_t *g, const uint32_t *src, const uint32_t *dst, uint64_t n,
                                void *stream) {
    if (!g || (n && (!src || !dst))) return GALLATIN_ERR_INVALID;
    if (n == 0) return GALLATIN_OK;
    k_edge_insert<<<blocks(n), kT, 0, S(stream)>>>(*g, src, dst, n);
    return status();
}

int gallatin_graph_delete_edges(gallatin_graph_t *g, const uint32_t *src, const uint32_t *dst, uint64_t n,
                                void *stream) {
    if (!g || (n && (!src || !dst))) return GALLATIN_ERR_INVALID;
    if (n == 0) return GALLATIN_OK;
    k_edge_delete<<<blocks(n), kT, 0, S(stream)>>>(*g, src, dst, n);
    return status();
}

int gallatin_graph_export(const gallatin_graph_t *g, uint32_t *size, uint32_t *cap, uint64_t *list, void *stream) {
    if (!g) return GALLATIN_ERR_INVALID;
    k_export<<<blocks(g->V), kT, 0, S(stream)>>>(*g, size, cap, list);
    return status();
}

int gallatin_graph_gather(const gallatin_graph_t *g, const uint64_t *off, uint32_t *out, void *stream) {
    if (!g || !off || !out) return GALLATIN_ERR_INVALID;
    k_gather<<<148 * 16, kT, 0, S(stream)>>>(*g, off, out);
    return status();
}

int gallatin_graph_counters(const gallatin_graph_t *g, uint64_t out[4]) {
    if (!g || !out) return GALLATIN_ERR_INVALID;
    if (cudaDeviceSynchronize() != cudaSuccess) return GALLATIN_ERR_CUDA;
    unsigned long long c[4];
    if (cudaMemcpy(c, g->ctr, sizeof(c), cudaMemcpyDeviceToHost) != cudaSuccess) return GALLATIN_ERR_CUDA;
    for (int i = 0; i < 4; i++) out[i] = c[i];
    return GALLATIN_OK;
}

}  // extern "C"
