// gallatin_capi.cu -- libgallatin.so: the C-ABI of include/gallatin.h.
//
// Host plumbing (heap + metadata in HBM, reset, snapshot, stats) and the bulk
// kernels: one GPU thread per request, each running the same device code a
// user kernel gets from include/gallatin/device.cuh (one thread per
// allocation, 1M+ threads).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <vector>

#include "gallatin.h"
#include "gallatin/core.cuh"

using namespace gallatin;
using core::View;

namespace {

constexpr int kThreads = 256;
// ITEMS=4 per thread once the grid would still fill every SM several times
constexpr int kItemsMin = 148 * 1024 * 4;
// host-array calls are cut into at most kMaxChunks pieces of >= kChunkMin
// requests, so the copy in of piece i+1, the kernel of piece i and the copy
// out of piece i-1 overlap (PCIe is full duplex)
constexpr int kMaxChunks = 8;
constexpr uint64_t kChunkMin = 1ull << 20;

struct State {
    bool init = false;
    int device = 0;
    gallatin_config_t cfg{};
    void *heap_raw = nullptr;
    void *meta = nullptr;
    uint64_t meta_bytes = 0;
    View v{};
    void *scratch = nullptr;
    uint64_t scratch_bytes = 0;
    // host-array calls: copy-in / copy-out streams and per-chunk events
    cudaStream_t cin = nullptr, cout = nullptr;
    uint32_t launch_tag = 0;                          // bulk malloc launches (deferred-request queue owner)
    bool pdl = true;
    bool defer_big = true;
    cudaEvent_t ev_in[kMaxChunks] = {}, ev_k[kMaxChunks] = {};
};
State g;

// The allocator's device view lives in constant memory (set once by init):
// kernels and the slow paths they call read it through the constant cache
// instead of materializing a ~300 B kernel-parameter copy per thread.
__constant__ View c_view;

#define CUDA_TRY(x)                                                                 \
    do {                                                                            \
        cudaError_t e_ = (x);                                                       \
        if (e_ != cudaSuccess) {                                                    \
            fprintf(stderr, "gallatin: %s failed: %s\n", #x, cudaGetErrorString(e_)); \
            return GALLATIN_ERR_CUDA;                                               \
        }                                                                           \
    } while (0)

inline cudaStream_t S(void *s) { return reinterpret_cast<cudaStream_t>(s); }
inline unsigned grid_for(uint64_t n) { return (unsigned)((n + kThreads - 1) / kThreads); }
inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

int launch_status() {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        fprintf(stderr, "gallatin: launch failed: %s\n", cudaGetErrorString(e));
        return GALLATIN_ERR_CUDA;
    }
    return GALLATIN_OK;
}

// ------------------------------------------------------------ kernels ----
// The state a reset leaves, every word computed from its index: the
// pristine image (every segment free, trees and table consistent, rings and
// counters empty) or -- with a prefilled block buffer ("always
// populated", v.pf_segs > 0) -- the same with segments [0, pf_segs) carved
// into the slots' first runs, class by class (view.h).
__device__ __forceinline__ uint32_t pf_class_of(const View &v, uint64_t s) {
    uint32_t c = 0;
    while (c + 1 < core::kTrees && s >= v.pf_base[c + 1]) c++;
    return c;
}
__global__ void k_reset() {
    const View &v = c_view;
    const uint64_t W = v.tree_words, nseg = v.nseg, pf = v.pf_segs;
    const uint64_t S = v.nslot_total;
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    // one thread per 16 B of the largest arrays (block counters: 64 per
    // segment, ring entries: 32 per segment, slot lines: 8 per slot)
    uint64_t total = nseg * 64;
    if (S * 8 > total) total = S * 8;
    if (9 * W > total) total = 9 * W;
    if (9 * 32 > total) total = 9 * 32;
    const uint4 ones = make_uint4(~0u, ~0u, ~0u, ~0u), zeros = make_uint4(0u, 0u, 0u, 0u);
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < total; i += stride) {
        if (i < W) {
            // segment tree: leaf bit s set iff pf <= s < nseg; a summary bit
            // set iff its child covers such a segment: children ch of this
            // word with ch < nbits and (ch + 1) * span > pf, i.e. ch >= pf / span
            uint32_t lvl = 0;
            while (lvl + 1 < v.tree_levels && i >= v.level_off[lvl + 1]) lvl++;
            const uint64_t word = i - v.level_off[lvl];
            const uint64_t nbits = lvl == 0 ? nseg : (uint64_t)(v.level_off[lvl] - v.level_off[lvl - 1]);
            const uint64_t lo_ch = pf >> (6 * lvl);
            const uint64_t lo = lo_ch > word * 64 ? lo_ch : word * 64, hi = nbits < word * 64 + 64 ? nbits : word * 64 + 64;
            v.seg_tree[i] = lo < hi ? bit_range((uint32_t)(lo - word * 64), (uint32_t)(hi - word * 64)) : 0ull;
        }
        if (i < 9 * W) {
            // block tree t holds only its class's partly used prefill segment
            const uint32_t t = (uint32_t)(i / W), wi = (uint32_t)(i % W);
            uint64_t w = 0;
            if (pf && v.pf_last[t] != 0xFFFFFFFFu) {
                uint32_t lvl = 0;
                while (lvl + 1 < v.tree_levels && wi >= v.level_off[lvl + 1]) lvl++;
                const uint64_t idx = (uint64_t)v.pf_last[t] >> (6 * lvl);      // this level's bit index
                if (wi - v.level_off[lvl] == (idx >> 6)) w = 1ull << (idx & 63);
            }
            v.block_trees[i] = w;
        }
        if (i < nseg) {
            uint32_t t = core::kTreeFree;
            int32_t avail = 0;
            uint32_t tail = 0;
            if (i < pf) {
                t = pf_class_of(v, i);
                if (i == v.pf_last[t]) avail = (int32_t)(core::nb_of(t) - v.pf_used[t]);
                tail = (uint32_t)avail;
            }
            v.seg_word[i] = core::sw_make(t, t == core::kTreeFree ? 0 : avail);
            v.seg_tid[i] = t;
            v.q_head[i] = 0;
            v.q_tail[i] = tail;
        }
        if (i < nseg * 32) {                                             // ring entries, 8 per thread
            uint4 e = ones;
            const uint64_t s = i / 32;
            if (s < pf) {
                const uint32_t t = pf_class_of(v, s);
                if (s == v.pf_last[t]) {                                 // ring: blocks used..nb-1, ascending
                    const uint32_t u = v.pf_used[t], cnt = core::nb_of(t) - u, q0 = (uint32_t)(i % 32) * 8;
                    uint32_t h[4];
#pragma unroll
                    for (uint32_t k = 0; k < 4; k++) {
                        const uint32_t a0 = q0 + 2 * k, a1 = a0 + 1;
                        h[k] = (a0 < cnt ? (u + a0) : core::kRingEmpty) | ((a1 < cnt ? (u + a1) : core::kRingEmpty) << 16);
                    }
                    e = make_uint4(h[0], h[1], h[2], h[3]);
                }
            }
            reinterpret_cast<uint4 *>(v.q_entries)[i] = e;
        }
        if (i < nseg * 64) reinterpret_cast<uint4 *>(v.block_free)[i] = zeros;
        if (i < S * 8) {                                                 // slot lines: words 2j, 2j + 1
            const uint64_t j = i % 8, si = i / 8;
            uint64_t w0 = 0, w1 = 0;
            if (j == 0) {
                w0 = core::kSlotEmpty;
                w1 = core::kSlotEmpty;
                if (pf) {
                    uint32_t c = 0;
                    while (c + 1 < core::kTrees && si >= v.slot_off[c + 1]) c++;
                    const uint64_t first = (uint64_t)v.pf_base[c] * core::nb_of(c) + (si - v.slot_off[c]) * v.pf_run[c];
                    w0 = ((uint64_t)v.pf_run[c] << core::kRunShift) | first;
                }
            }
            reinterpret_cast<uint4 *>(v.slots)[i] =
                make_uint4((uint32_t)w0, (uint32_t)(w0 >> 32), (uint32_t)w1, (uint32_t)(w1 >> 32));
        }
        if (i < 9 * 32) v.fmt_token[i] = 0;
        if (i == 0) *v.err = 0;
        if (i < 16) v.oom[i] = 0;
        if (i < 2) v.bigq_ctl[i] = 0;
    }
}

// Slow items of one lane of the bulk malloc kernel.  Refill DUTIES (this lane
// drew exactly the end of a run) are discharged first, before this lane waits
// on anything: with pre-issued RMWs a later item's duty may be exactly the
// refill an earlier item would otherwise wait for.
// Then waits-and-retries, whole blocks and segment runs.
__device__ __noinline__ void bulk_malloc_slow(const uint64_t *sizes, void **ptrs, uint64_t n, uint64_t base,
                                              uint32_t key, uint32_t slow, const uint64_t *info, int items,
                                              unsigned callers, uint32_t stride = 32,
                                              const uint32_t *demand = nullptr, uint64_t ctas = 0) {
    const View &v = c_view;
    // pass 0: refill and prefetch duties only (never waits on another slot's refill)
    for (int k = 0; k < items; k++) {
        const uint32_t code = (uint32_t)(info[k >> 2] >> (16 * (k & 3))) & 0xFFFF;
        if (((slow >> k) & 1) && (code & 0x2000u)) {
            const uint32_t c = core::slice_class(sizes[base + (uint64_t)stride * k]);
            core::prefetch_slot(v, v.slot_off[c] + key % v.nslot[c], c, code & 0x3FF);
            slow &= ~(1u << k);                                     // its slice was stored already
            continue;
        }
        if (!((slow >> k) & 1) || !(code & 0x400u)) continue;
        const uint64_t i = base + (uint64_t)stride * k;
        const uint32_t c = core::slice_class(sizes[i]);
        // demand hint: this CTA's requests of class c x CTAs / slots of c, in blocks
        const uint32_t hint =
            demand ? (uint32_t)(((uint64_t)demand[c] * ctas / v.nslot[c] + core::kSlices - 1) >> core::kSliceLog2) : 0;
        if (!core::refill_slot(v, v.slot_off[c] + key % v.nslot[c], c, code & 0x3FF, hint)) {
            __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i, 0ull);   // heap exhausted: NULL
            slow &= ~(1u << k);
        }
    }
    // every duty of this warp is discharged before any of its lanes spins
    // (a sleeping lane stalls its warp-mates' diverged refill path)
    __syncwarp(callers);
    // pass 1: retries after a refill, waits, whole blocks and segment runs
    for (int k = 0; k < items; k++) {
        if (!((slow >> k) & 1)) continue;
        const uint32_t code = (uint32_t)(info[k >> 2] >> (16 * (k & 3))) & 0xFFFF;
        const uint64_t i = base + (uint64_t)stride * k;
        const uint64_t sz = sizes[i];
        void *p;
        if (code & 0x800u) {
            p = core::malloc_impl(v, sz, key);
        } else {
            const uint32_t c = core::slice_class(sz);
            if (code & 0x1000u) core::slot_exhausted(v, v.slot_off[c] + key % v.nslot[c], c, 0, ~0u);  // wait
            p = core::malloc_slice(v, c, key);
        }
        __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i, reinterpret_cast<unsigned long long>(p));
    }
}

// Bulk malloc, ITEMS requests per thread: all slice requests first issue their
// team RMW (one per team per item, back to back: memory-level parallelism),
// then take their slice; refills, waits, blocks and large requests follow on
// the per-request device path.  Lane l of warp w handles w*32*ITEMS + k*32 + l.
template <int ITEMS>
__global__ void __launch_bounds__(kThreads, 5) k_bulk_malloc(const uint64_t *__restrict__ sizes, void **__restrict__ ptrs,
                                                          uint64_t n) {
    const View &v = c_view;
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t base = ((blockIdx.x * (uint64_t)kThreads + threadIdx.x) >> 5) * (32 * ITEMS) + lane;
    const uint32_t key = ptx::smid();
    uint64_t sz[ITEMS], old[ITEMS];
    uint32_t si[ITEMS];
    unsigned peers[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + 32ull * k;
        // unconditional load of a clamped index: the ITEMS loads issue back to back
        const uint64_t x = __ldcs(reinterpret_cast<const unsigned long long *>(sizes) + (i < n ? i : n - 1));
        sz[k] = i < n ? x : 0;
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const bool slice = sz[k] - 1 < core::kMaxSlice;               // 1 .. 4096
        const uint32_t c = core::slice_class(sz[k]);
        si[k] = slice ? v.slot_off[c] + key % v.nslot[c] : 0xFFFFFFFFu;
        peers[k] = __match_any_sync(0xFFFFFFFFu, si[k]);
        old[k] = 0;
        if (slice && lane == (uint32_t)__ffs((int)peers[k]) - 1)
            old[k] = ptx::atom_add(core::slot_word(v, si[k]), (uint64_t)__popc(peers[k]) << 32);
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) old[k] = __shfl_sync(0xFFFFFFFFu, old[k], __ffs((int)peers[k]) - 1);
    // Fast path: every valid slice is computed and stored here; what a slow
    // item needs later is packed into 16 bits per item (bits 9..0: run length
    // of a refill duty, 0x400 duty flag, 0x800 not-a-slice, 0x1000 wait), so
    // no fast-path state is live across the slow path's calls.
    const uint32_t lt = ptx::lanemask_lt();
    uint32_t slow = 0;
    uint64_t info = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + 32ull * k;
        void *p = nullptr;
        uint32_t code = 0;
        if (si[k] != 0xFFFFFFFFu) {
            const uint32_t c = core::slice_class(sz[k]);
            const uint32_t m = core::run_len(old[k]);
            const uint32_t idx = (uint32_t)(old[k] >> 32) + (uint32_t)__popc(peers[k] & lt);
            if (idx < (m << core::kSliceLog2)) {
                p = core::slice_ptr(v, c, old[k] & core::kRunNone, idx);
                if (v.prefetch && idx == (m << (core::kSliceLog2 - 1))) code = 0x2000u | m;   // prefetch duty
            } else {
                code = idx == (m << core::kSliceLog2) ? (0x400u | m) : 0x1000u;
            }
        } else if (sz[k] != 0) {
            code = 0x800u;
        }
        if (code) {
            slow |= 1u << k;
            info |= (uint64_t)code << (16 * k);
        }
        if (!(code & 0x1C00u) && i < n)                           // valid (maybe with a prefetch duty)
            __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i, reinterpret_cast<unsigned long long>(p));
    }
    const unsigned callers = __ballot_sync(0xFFFFFFFFu, slow != 0);
    if (slow) bulk_malloc_slow(sizes, ptrs, n, base, key, slow, &info, ITEMS, callers);
}

// [dev] Deferred big requests (DESIGN.md Deviations 20): a bulk launch's
// whole-block and segment requests go into one device queue -- claimed by the
// launch's tag (concurrent launches on other streams find it taken and serve
// theirs inline) -- and the batch kernel k_big that follows the launch serves
// them together.  Returns false (serve inline) if the queue is another
// launch's or full.
__device__ __noinline__ bool defer_big(const View &v, uint32_t tag, uint64_t addr, uint64_t size) {
    const uint32_t own = atomicCAS(v.bigq_ctl, 0u, tag);
    if (own != 0u && own != tag) return false;
    const uint32_t q = atomicAdd(v.bigq_ctl + 1, 1u);
    if (q >= v.bigq_cap) return false;
    v.bigq[2 * (uint64_t)q] = addr;
    v.bigq[2 * (uint64_t)q + 1] = size;
    return true;
}

// The slow remainder of one k_bulk_malloc_cta tile (called by every thread
// of the tile, or by none).  Thread c_me < 9 serves class c_me: its slot si,
// the tile's my_cnt requests of the class, the RMW's lo/run (my_lo, my_m),
// duty = this tile drew the run's end.
template <int ITEMS, int NT>
__device__ __noinline__ void tile_slow(const uint64_t *sizes, void **ptrs, uint64_t base, uint32_t key,
                                       const uint32_t *cr, uint32_t pend, uint32_t big, uint32_t pfd,
                                       const uint32_t *cnt, uint64_t *lim_lo, uint64_t *run_base, uint32_t *roff,
                                       uint32_t *failed, bool rounds, uint32_t tag) {
    const View &v = c_view;
    // [dev] prefetch duties (knob prefetch=1): the item that drew the middle of a run
    for (int k = 0; k < ITEMS; k++) {
        if (!((pfd >> k) & 1)) continue;
        const uint32_t c = cr[k] & 0xFFu;
        core::prefetch_slot(v, v.slot_off[c] + key % v.nslot[c], c, (uint32_t)(lim_lo[c] >> 32) >> core::kSliceLog2);
    }
    const uint32_t c_me = (threadIdx.x & 31) * (NT / 32) + (threadIdx.x >> 5);
    const bool cls_thread = c_me < core::kTrees;
    uint32_t my_cnt = cls_thread ? cnt[c_me] : 0u;
    const uint64_t ll0 = my_cnt ? lim_lo[c_me] : 0ull;
    uint32_t my_lo = (uint32_t)ll0, my_limit = (uint32_t)(ll0 >> 32), my_m = my_limit >> core::kSliceLog2;
    const uint32_t si = cls_thread ? v.slot_off[c_me] + key % v.nslot[c_me] : 0u;
    bool duty = my_cnt && my_lo <= my_limit && my_limit < my_lo + my_cnt;
    // Refill duty (Alg.3: the request that draws the end replaces
    // the run) -- discharged by the class thread before it ever waits, so no
    // tile waits on a refill while holding one.  [dev] The refill is sized to
    // this slot's share of the launch (demand hint, DESIGN.md Deviations 10).
    bool dutyfail = false;
    const uint32_t hint_of = cls_thread && v.demand_hint
                                 ? (uint32_t)(((uint64_t)my_cnt * gridDim.x / v.nslot[c_me] + core::kSlices - 1) >>
                                              core::kSliceLog2)
                                 : 0u;
    if (duty) dutyfail = !core::refill_slot(v, si, c_me, my_m, hint_of);
    // [dev] demand prefetch (DESIGN.md Deviations 19): what the rest of the
    // launch will ask of this slot (this tile's count x the tiles not yet
    // started / slots -- CTAs start in index order) exceeds what is left of
    // the run by a block or more, the run still covers 16+ tiles (a run about
    // to end is refilled as usual) and the launch is not in its last quarter
    // (the fetch would only lengthen the tail): fetch the missing blocks
    // into the slot's second word now -- before this thread waits on anything
    if (cls_thread && v.demand_hint && my_cnt && my_lo + my_cnt < my_limit &&
        my_limit - (my_lo + my_cnt) >= 16u * my_cnt && blockIdx.x < gridDim.x - gridDim.x / 4) {
        const uint32_t pf_rem = my_limit - (my_lo + my_cnt);
        const float rest = (float)my_cnt * (float)(gridDim.x - blockIdx.x) * v.nslot_rcp[c_me];
        if (rest >= (float)(pf_rem + core::kSlices) && ptx::ld_relaxed(core::slot_word(v, si) + 1) == core::kSlotEmpty)
            core::demand_prefetch(v, si, c_me, my_m, (uint32_t)((rest - (float)pf_rem) * (1.0f / core::kSlices)) + 1u);
    }
    // Rounds: the class thread retires what the last round served, waits for
    // the slot's refill (another tile's duty), takes the tile's remaining
    // requests of its class with ONE more RMW, and the items retry -- one RMW
    // and one barrier per round for the whole tile, not one per warp and item.
    // (rounds is CTA-uniform: no class past its run's end -> no duty, no round, no barrier)
    bool still = my_cnt && (dutyfail || my_lo + my_cnt > my_limit);
    while (rounds && __syncthreads_or(still)) {
        if (still) {
            const uint32_t served = my_lo < my_limit ? min(my_limit - my_lo, my_cnt) : 0u;
            if (dutyfail) {
                failed[c_me] = 1;                             // the team's refill found no memory
                my_cnt = 0;
            } else {
                roff[c_me] += served;
                my_cnt -= served;
                // wait for the refill; false: tree c is recorded exhausted [dev]
                if (!core::slot_exhausted(v, si, c_me, 0, ~0u)) {
                    failed[c_me] = 1;
                    my_cnt = 0;
                } else {
                    const uint64_t old = ptx::atom_add(core::slot_word(v, si), (uint64_t)my_cnt << 32);
                    my_m = core::run_len(old);
                    my_limit = my_m << core::kSliceLog2;
                    my_lo = (uint32_t)(old >> 32);
                    lim_lo[c_me] = ((uint64_t)my_limit << 32) | my_lo;
                    run_base[c_me] = reinterpret_cast<uint64_t>(core::slice_ptr(v, c_me, old & core::kRunNone, 0));
                    // a duty is discharged at once, before the barrier: a
                    // sibling class thread may be waiting in this phase for a
                    // refill whose holder waits for this one (no cycle)
                    duty = my_lo <= my_limit && my_limit < my_lo + my_cnt;
                    dutyfail = duty && !core::refill_slot(v, si, c_me, my_m, hint_of);
                }
            }
        }
        __syncthreads();
        for (int k = 0; k < ITEMS; k++) {
            if (!((pend >> k) & 1)) continue;
            const uint64_t i = base + (uint64_t)NT * k;
            const uint32_t c = cr[k] & 0xFFu;
            if (failed[c]) {
                __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i, 0ull);   // heap exhausted: NULL
                pend &= ~(1u << k);
                continue;
            }
            const uint64_t ll = lim_lo[c];
            const uint32_t limit = (uint32_t)(ll >> 32);
            const uint32_t idx = (uint32_t)ll + (cr[k] >> 8) - roff[c];
            if (idx < limit) {
                __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i,
                       run_base[c] + ((uint64_t)idx << (core::kMinSliceLog2 + c)));
                pend &= ~(1u << k);
            }
        }
        still = my_cnt && (dutyfail || my_lo + my_cnt > my_limit);
    }
    // whole blocks and segment runs: the device path, per lane
    if (big) {
        for (int k = 0; k < ITEMS; k++) {
            if (!((big >> k) & 1)) continue;
            const uint64_t i = base + (uint64_t)NT * k;
            // [dev] deferred to the launch's batch kernel (k_big) while the
            // queue is this launch's and has room (DESIGN.md Deviations 20)
            if (tag && defer_big(v, tag, reinterpret_cast<uint64_t>(ptrs + i), sizes[i])) continue;
#ifdef GALLATIN_TRACE
            const uint64_t tb0 = ptx::globaltimer();
#endif
            __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i,
                   reinterpret_cast<unsigned long long>(core::malloc_impl(v, sizes[i], key)));
#ifdef GALLATIN_TRACE
            ptx::trace(tb0, ptx::globaltimer(), (12ull << 60) | (sizes[i] >> 20));
#endif
        }
    }
}

// Bulk malloc with CTA-level aggregation: every warp of a CTA runs on one SM,
// hence uses one block-buffer slot per class; the CTA's requests of a class
// are counted in shared memory (one shared atomic per warp team) and ONE
// global RMW per class per CTA takes their slices (1024 requests at
// ITEMS=4), so the hot slot words see 32x fewer RMWs than with warp teams.
// Item k of thread t is request blockIdx*256*ITEMS + k*256 + t.
template <int ITEMS, int MINB = 5, int NT = kThreads>
__global__ void __launch_bounds__(NT, MINB) k_bulk_malloc_cta(const uint64_t *__restrict__ sizes,
                                                                  void **__restrict__ ptrs, uint64_t n,
                                                                  uint32_t tag) {
    const View &v = c_view;
    __shared__ uint32_t cnt[core::kTrees];
    __shared__ uint32_t tile_flags;
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t base = blockIdx.x * (uint64_t)(NT * ITEMS) + threadIdx.x;
#ifdef GALLATIN_TRACE
    const uint64_t tk0 = ptx::globaltimer();
#endif
    const uint32_t key = ptx::smid();
    // the launch's batch kernel (k_big) may become resident once every tile has started
    asm volatile("griddepcontrol.launch_dependents;");
    if (threadIdx.x < core::kTrees) cnt[threadIdx.x] = 0;
    if (threadIdx.x == 32) tile_flags = 0;
    // a tile entirely inside the array needs no per-item range checks (CTA-uniform)
    const bool full = (blockIdx.x + 1ull) * (NT * ITEMS) <= n;
    // per item: class (0..8 slice class, 0xFE nothing to do, 0xFF block or
    // segment request) | rank << 8; the sizes themselves are not kept
    uint32_t cr[ITEMS];
    uint64_t x[ITEMS];
    // all loads issued before any is used (clamped indices in a ragged tile)
    if (full) {
#pragma unroll
        for (int k = 0; k < ITEMS; k++) x[k] = __ldcs(reinterpret_cast<const unsigned long long *>(sizes) + base + NT * k);
    } else {
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            const uint64_t i = base + (uint64_t)NT * k;
            x[k] = __ldcs(reinterpret_cast<const unsigned long long *>(sizes) + (i < n ? i : n - 1));
            if (i >= n) x[k] = 0;
        }
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t s = x[k];
        const uint32_t lg = 64u - (uint32_t)__clzll((long long)(s - 1));      // ceil(log2 s) for s >= 2
        const uint32_t sc = (lg > core::kMinSliceLog2 ? lg : core::kMinSliceLog2) - core::kMinSliceLog2;
        cr[k] = s - 1 < core::kMaxSlice ? sc : (s == 0 ? 0xFEu : 0xFFu);   // branch-free slice_class
    }
    __syncthreads();
    // A warp whose 32 x ITEMS requests are all of one slice class (single-size
    // launches: every warp) takes 32 x ITEMS consecutive ranks of its class
    // with one shared atomic -- any bijection onto [0, count) serves (the tile
    // ranks are only offsets into the run) -- instead of one match, shared
    // atomic and shuffle per item; the item pass then reads its class's run
    // once.  Other warps rank per item by warp teams.
    const uint32_t cw = __shfl_sync(0xFFFFFFFFu, cr[0], 0);
    bool mine = cw < core::kTrees;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) mine &= cr[k] == cw;
    const bool uni = __all_sync(0xFFFFFFFFu, mine);
    if (uni) {
        uint32_t b = 0;
        if (lane == 0) b = atomicAdd(&cnt[cw], 32u * ITEMS);
        b = __shfl_sync(0xFFFFFFFFu, b, 0) + lane;
#pragma unroll
        for (int k = 0; k < ITEMS; k++) cr[k] = cw | ((b + 32u * k) << 8);
    } else {
        const uint32_t lt = ptx::lanemask_lt();
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            const uint32_t c = cr[k];
            const unsigned peers = __match_any_sync(0xFFFFFFFFu, c);
            const uint32_t leader = (uint32_t)__ffs((int)peers) - 1;
            uint32_t b = 0;
            if (c < core::kTrees && lane == leader) b = atomicAdd(&cnt[c], (uint32_t)__popc(peers));
            cr[k] = c | ((__shfl_sync(0xFFFFFFFFu, b, (int)leader) + (uint32_t)__popc(peers & lt)) << 8);
        }
    }
    __syncthreads();
    // Class c is served by thread (c % warps) * 32 + c / warps (one per warp
    // in turn: refills of different classes run in different warps).  Per
    // class, shared: the slot RMW's {limit : 32 | first index : 32}, the
    // address of the run's slice 0 (an item's pointer is one shift-add), the
    // rank of the lowest request still unserved, and a failed flag.
    __shared__ uint64_t lim_lo[core::kTrees];
    __shared__ uint64_t run_base[core::kTrees];
    __shared__ uint32_t roff[core::kTrees];
    __shared__ uint32_t failed[core::kTrees];
    constexpr uint32_t NW = NT / 32;
    const uint32_t c_me = lane * NW + (threadIdx.x >> 5);
    const bool cls_thread = c_me < core::kTrees;
    bool cls_over = false;      // requests of this class past the run's end: the tile needs rounds
    bool cls_slow = false;      // this class thread has a prefetch or a demand prefetch to do
    if (cls_thread) {
        roff[c_me] = 0;
        failed[c_me] = 0;
        const uint32_t my_cnt = cnt[c_me];
        if (my_cnt) {
            const uint64_t old = ptx::atom_add(core::slot_word(v, v.slot_off[c_me] + key % v.nslot[c_me]),
                                               (uint64_t)my_cnt << 32);
            const uint32_t my_limit = core::run_len(old) << core::kSliceLog2, my_lo = (uint32_t)(old >> 32);
            lim_lo[c_me] = ((uint64_t)my_limit << 32) | my_lo;
            run_base[c_me] = reinterpret_cast<uint64_t>(core::slice_ptr(v, c_me, old & core::kRunNone, 0));
            cls_over = my_lo + my_cnt > my_limit;
            cls_slow = (v.prefetch && my_lo <= (my_limit >> 1) && (my_limit >> 1) < my_lo + my_cnt) ||
                       // (checked by the tile whose draw crosses a 4-block mark only: every
                       // check reads the slot's second word, a round trip the tile waits for)
                       (v.demand_hint && (my_lo >> 14) != ((my_lo + my_cnt) >> 14) &&
                        my_limit - (my_lo + my_cnt) >= 16u * my_cnt &&
                        blockIdx.x < gridDim.x - gridDim.x / 4 &&
                        (float)my_cnt * (float)(gridDim.x - blockIdx.x) * v.nslot_rcp[c_me] >=
                            (float)(my_limit - (my_lo + my_cnt) + core::kSlices));   // demand prefetch (tile_slow)
        }
    }
    bool big_any = false;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) big_any |= (cr[k] & 0xFFu) == 0xFFu;
    // the tile's slow remainder is known here, before any store: the fast
    // path ends with its stores (no barrier behind them)
    if (cls_over) atomicOr(&tile_flags, 1u);
    if (cls_slow || big_any) atomicOr(&tile_flags, 2u);
    __syncthreads();
    const uint32_t slow_tile = tile_flags;                    // bit 0: rounds, bit 1: barrier-free slow work
    // items whose slice lies inside the run are stored now; the rest wait in
    // `pend` for the tile's next round (bit k: item k)
    uint32_t pend = 0, big = 0, pfd = 0;
    if (uni) {                                            // one class: its run read once
        const uint64_t ll = lim_lo[cw], rb = run_base[cw];
        const uint32_t limit = (uint32_t)(ll >> 32);
#pragma unroll
        for (int k = 0; k < ITEMS; k++) {
            const uint32_t idx = (uint32_t)ll + (cr[k] >> 8);
            if (idx < limit) {
                __stcs(reinterpret_cast<unsigned long long *>(ptrs) + base + (uint64_t)NT * k,
                       rb + ((uint64_t)idx << (core::kMinSliceLog2 + cw)));
                if (v.prefetch && idx == (limit >> 1)) pfd |= 1u << k;
            } else {
                pend |= 1u << k;
            }
        }
    } else
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + (uint64_t)NT * k;
        const uint32_t c = cr[k] & 0xFFu;
        if (c < core::kTrees) {
            const uint64_t ll = lim_lo[c];
            const uint32_t limit = (uint32_t)(ll >> 32);
            const uint32_t idx = (uint32_t)ll + (cr[k] >> 8);
            if (idx < limit) {
                __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i,
                       run_base[c] + ((uint64_t)idx << (core::kMinSliceLog2 + c)));
                if (v.prefetch && idx == (limit >> 1)) pfd |= 1u << k;
            } else {
                pend |= 1u << k;
            }
        } else if (c == 0xFFu) {
            big |= 1u << k;                                   // a whole block or segments
        } else if (full || i < n) {
            __stcs(reinterpret_cast<unsigned long long *>(ptrs) + i, 0ull);   // malloc(0): NULL
        }
    }
    // the rest -- refill duties, demand prefetch, further rounds, blocks and
    // segments -- only if some thread of the tile has any of it (its frame
    // is not the fast path's)
    if (slow_tile) {
        uint32_t crs[ITEMS];
#pragma unroll
        for (int k = 0; k < ITEMS; k++) crs[k] = cr[k];
        tile_slow<ITEMS, NT>(sizes, ptrs, base, key, crs, pend, big, pfd, cnt, lim_lo, run_base, roff, failed,
                             slow_tile & 1, tag);
    }
#ifdef GALLATIN_TRACE
    __syncthreads();
    if (threadIdx.x == 0) ptx::trace(tk0, ptx::globaltimer(), (7ull << 60) | blockIdx.x);   // CTA start, end
#endif
}

// ---- the batch kernel of a bulk malloc launch's deferred big requests ------
// [dev] (DESIGN.md Deviations 20).  One CTA, after the launch (stream order):
//   1. rank every request within its block tree (4 KB < size < 16 MB: one
//      whole block of tree t, reading A-2) and sum the segment requests' k;
//   2. ONE claim of consecutive free segments from the front for all the
//      trees' blocks (tree after tree, ceil(requests / nb) segments each,
//      taken privately like a whole-segment run, O2-R R2; a tree's partly
//      used last segment keeps the rest of its blocks in its ring and block
//      tree, initSegment P:125) and ONE claimMultiple from the back (P:110-113,
//      P:138) of the sum of the segment requests' k -- both as one atomicAnd
//      per leaf word, the words spread over a warp's lanes;
//   3. every request's pointer in rank order (a block's free counter preset
//      to 4095, reading A-2; a segment run's table entries, P:143 / P:235).
// A claim that finds no such range (fragmented or nearly full heap) leaves
// its requests to the per-request device path (malloc_impl: GetBlock /
// claimMultiple, NULL on exhaustion).
constexpr int kBigThreads = 1024;
constexpr uint32_t kBigCap = 8192;
constexpr uint32_t kMaxLeafWords = 256;                      // nseg <= 2^14 (gallatin_init_ex)

__device__ __noinline__ void *big_inline(const View &v, uint64_t size) { return core::malloc_impl(v, size, 0u); }

// lowest start of k consecutive set bits among the nw words of lw (shared
// copy of the segment tree's leaves); kNone if none
__device__ uint64_t lowest_run_of(const uint64_t *lw, uint64_t nw, uint64_t k) {
    uint64_t run = 0, start = 0;
    if (k > 64) {
        // a run longer than a word is the leading ones of one word, whole
        // words, and the trailing ones of another: O(1) per word
        for (uint64_t wi = 0; wi < nw; wi++) {
            const uint64_t x = lw[wi], base = wi << 6;
            if (x == ~0ull) {
                if (!run) start = base;
                run += 64;
                if (run >= k) return start;
                continue;
            }
            const uint32_t tr = (uint32_t)__ffsll((long long)~x) - 1;
            if (run + tr >= k) return start;
            const uint32_t lead = (uint32_t)__clzll((long long)~x);          // ones from bit 63 down
            run = lead;
            start = base + 64 - lead;
        }
        return kNone;
    }
    for (uint64_t wi = 0; wi < nw; wi++) {
        const uint64_t x = lw[wi], base = wi << 6;
        if (x == ~0ull) {
            if (!run) start = base;
            run += 64;
            if (run >= k) return start;
            continue;
        }
        const uint32_t tr = (uint32_t)__ffsll((long long)~x) - 1;   // ones at the bottom continue the run
        if (tr) {
            if (!run) start = base;
            run += tr;
            if (run >= k) return start;
        }
        run = 0;
        uint64_t rest = x & (~0ull << tr);                          // bit tr is 0
        while (rest) {
            const uint32_t lo = (uint32_t)__ffsll((long long)rest) - 1;
            const uint64_t sh = rest >> lo;
            const uint32_t len = (uint32_t)__ffsll((long long)~sh) - 1;
            if (len >= k) return base + lo;
            if (lo + len == 64) {                                      // continues into the next word
                run = len;
                start = base + lo;
                break;
            }
            rest &= ~bit_range(lo, lo + len);
        }
    }
    return kNone;
}

// Warp-parallel fast path of lowest_run_of / bt_find_highest_run: if the k
// bits from the lowest set bit (back = false) or ending at the highest set
// bit (back = true) are all set, their start; else kNone (the caller scans).
__device__ uint64_t edge_run_warp(const uint64_t *lw, uint64_t nw, uint64_t k, bool back, uint32_t lane) {
    uint64_t edge = kNone;
    for (uint64_t b = 0; b < nw && edge == kNone; b += 32) {
        const uint64_t wi = back ? nw - 1 - (b + lane) : b + lane;
        const uint64_t x = (b + lane < nw) ? lw[wi] : 0ull;
        const unsigned any = __ballot_sync(0xFFFFFFFFu, x != 0);
        if (any) {
            const uint32_t src = (uint32_t)__ffs((int)any) - 1;
            const uint64_t xs = __shfl_sync(0xFFFFFFFFu, x, (int)src);
            const uint64_t ws = back ? nw - 1 - (b + src) : b + src;
            edge = (ws << 6) + (back ? 63 - (uint64_t)__clzll((long long)xs) : (uint64_t)(__ffsll((long long)xs) - 1));
        }
    }
    if (edge == kNone) return kNone;
    if (back && edge + 1 < k) return kNone;
    const uint64_t i0 = back ? edge + 1 - k : edge;
    if (i0 + k > nw * 64) return kNone;
    const uint64_t w0 = i0 >> 6, w1 = (i0 + k - 1) >> 6;
    bool ok = true;
    for (uint64_t wi = w0 + lane; wi <= w1; wi += 32) {
        const uint32_t lo = wi == w0 ? (uint32_t)(i0 & 63) : 0u;
        const uint32_t hi = wi == w1 ? (uint32_t)((i0 + k - 1) & 63) + 1 : 64u;
        const uint64_t m = bit_range(lo, hi);
        ok &= (lw[wi] & m) == m;
    }
    return __all_sync(0xFFFFFFFFu, ok) ? i0 : kNone;
}

// Claim [i0, i0+k) of the segment tree, one atomicAnd per leaf word spread
// over the lanes of the calling warp; on a conflict every bit taken is given
// back (claimMultiple, for the whole range at once).  On success the
// words this lane's RMWs emptied are left in *emptied (bit r: word w0 + lane
// + 32 r): their summary repair (bt_reconcile_up) is the caller's, later --
// a stale summary over an empty word only makes a search restart.
__device__ bool claim_range_warp(const BitTree &st, uint64_t i0, uint64_t k, uint32_t lane, uint32_t *emptied) {
    const uint64_t w0 = i0 >> 6, w1 = (i0 + k - 1) >> 6;
    constexpr int R = (int)(kMaxLeafWords / 32);
    uint64_t old[R], msk[R];
    bool ok = true;
#pragma unroll
    for (int r = 0; r < R; r++) {
        const uint64_t wi = w0 + lane + 32u * r;
        msk[r] = 0;
        old[r] = 0;
        if (wi <= w1) {
            const uint32_t lo = wi == w0 ? (uint32_t)(i0 & 63) : 0u;
            const uint32_t hi = wi == w1 ? (uint32_t)((i0 + k - 1) & 63) + 1 : 64u;
            msk[r] = bit_range(lo, hi);
            old[r] = ptx::atom_and(st.w + st.off[0] + wi, ~msk[r]);
            ok &= (old[r] & msk[r]) == msk[r];
        }
    }
    ok = __all_sync(0xFFFFFFFFu, ok);
    *emptied = 0;
#pragma unroll
    for (int r = 0; r < R; r++) {
        if (!msk[r]) continue;
        const uint64_t wi = w0 + lane + 32u * r;
        bool flip = (old[r] & ~msk[r]) == 0 && (old[r] & msk[r]) != 0;   // our RMW emptied the word
        if (ok) {
            if (flip) *emptied |= 1u << r;
            continue;
        }
        if (old[r] & msk[r]) flip |= ptx::atom_or(st.w + st.off[0] + wi, old[r] & msk[r]) == 0;
        if (flip) bt_reconcile_up(st, 0, wi);
    }
    return ok;
}

// the summary repair claim_range_warp left to its caller
__device__ __forceinline__ void claim_range_repair(const BitTree &st, uint64_t i0, uint32_t lane, uint32_t emptied) {
    for (; emptied; emptied &= emptied - 1)
        bt_reconcile_up(st, 0, (i0 >> 6) + lane + 32u * (uint32_t)(__ffs((int)emptied) - 1));
}

__global__ void __launch_bounds__(kBigThreads, 1) k_big(uint32_t tag) {
    const View &v = c_view;
    __shared__ uint32_t own, nq;
    __shared__ uint32_t tcnt[core::kTrees], tsegs[core::kTrees], tbase[core::kTrees];
    __shared__ uint32_t ksum;
    __shared__ uint64_t front, back;                  // claimed ranges (kNone: serve inline)
    __shared__ uint64_t leaf[kMaxLeafWords];
    __shared__ uint32_t erank[kBigCap];               // tree << 28 | rank, or 0xF << 28 | segment offset
    const uint32_t tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // launched as the bulk malloc kernel's programmatic dependent: resident
    // before that kernel ends, it waits here for its completion (and memory)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    if (tid == 0) {
        own = ptx::ld_relaxed(v.bigq_ctl);
        const uint32_t c = ptx::ld_relaxed(v.bigq_ctl + 1);
        nq = c < v.bigq_cap ? c : v.bigq_cap;
        ksum = 0;
        front = kNone;
        back = kNone;
    }
    if (tid < core::kTrees) tcnt[tid] = 0;
    __syncthreads();
    if (own != tag) return;                                   // nothing of this launch's was deferred
    const uint32_t n = nq;
#ifdef GALLATIN_TRACE
    const uint64_t tb0 = ptx::globaltimer();
#endif
    const BitTree st = core::seg_tree(v);
    const uint64_t nw = (v.nseg + 63) / 64;
    if (tid < nw) leaf[tid] = ptx::ld_relaxed(st.w + st.off[0] + tid);
    // 1. ranks
    for (uint32_t e = tid; e < n; e += kBigThreads) {
        const uint64_t size = v.bigq[2 * (uint64_t)e + 1];
        if (size < core::kSegBytes) {
            const uint32_t t = core::block_class(size);
            erank[e] = (t << 28) | atomicAdd(&tcnt[t], 1u);
        } else {
            const uint64_t k = (size >> core::kSegLog2) + ((size & (core::kSegBytes - 1)) != 0);
            erank[e] = k <= v.nseg ? ((0xFu << 28) | atomicAdd(&ksum, (uint32_t)k)) : 0xFFFFFFFFu;
        }
    }
    __syncthreads();
#ifdef GALLATIN_TRACE
    if (tid == 0) ptx::trace(tb0, ptx::globaltimer(), (13ull << 60) | 1);
#endif
    uint64_t T = 0;                                           // segments for the trees' blocks
#pragma unroll
    for (uint32_t t = 0; t < core::kTrees; t++) {
        const uint32_t sg = (tcnt[t] + core::nb_of(t) - 1) / core::nb_of(t);
        if (tid == 0) {
            tsegs[t] = sg;
            tbase[t] = (uint32_t)T;                           // offset from `front` for now
        }
        T += sg;
    }
    // 2. the two claims (warp 0: front, warp 1: back), each retried once on a lost race
    uint32_t emptied = 0;
    uint64_t claimed = kNone;
    if (warp == 0 && T) {
        for (int attempt = 0; attempt < 2; attempt++) {
            uint64_t s0 = edge_run_warp(leaf, nw, T, false, lane);   // the free segments from the lowest on
            if (s0 == kNone) {
                s0 = lane == 0 ? lowest_run_of(leaf, nw, T) : 0;
                s0 = __shfl_sync(0xFFFFFFFFu, s0, 0);
            }
            if (s0 == kNone) break;
            if (claim_range_warp(st, s0, T, lane, &emptied)) {
                claimed = s0;
                if (lane == 0) front = s0;
                break;
            }
            for (uint64_t w = lane; w < nw; w += 32) leaf[w] = ptx::ld_relaxed(st.w + st.off[0] + w);
            __syncwarp();
        }
    }
    if (warp == 1 && ksum) {
        for (int attempt = 0; attempt < 2; attempt++) {
            uint64_t s0 = edge_run_warp(leaf, nw, ksum, true, lane);   // the free segments up to the highest
            if (s0 == kNone) {
                s0 = lane == 0 ? bt_find_highest_run(st, ksum) : 0;
                s0 = __shfl_sync(0xFFFFFFFFu, s0, 0);
            }
            if (s0 == kNone) break;
            if (claim_range_warp(st, s0, ksum, lane, &emptied)) {
                claimed = s0;
                if (lane == 0) back = s0;
                break;
            }
        }
    }
    __syncthreads();
#ifdef GALLATIN_TRACE
    if (tid == 0) ptx::trace(tb0, ptx::globaltimer(), (13ull << 60) | 2);
#endif
    // the trees' segments, taken privately ({t, 0 available}, tree-id copy);
    // (a tree's partly used last segment too: its other blocks are placed below)
    const uint64_t fr = front;
    if (fr != kNone) {
        for (uint64_t x = tid; x < T; x += kBigThreads) {
            uint32_t t = 0;
            while (x >= (uint64_t)tbase[t] + tsegs[t]) t++;
            const uint64_t s = fr + x;
            ptx::st_relaxed(v.seg_tid + s, t);
            ptx::atom_add(v.seg_word + s, core::sw_retree(core::kTreeFree, t));
        }
        ptx::fence_acq_rel();
    }
    __syncthreads();
    // summaries over the words the claims emptied (warps 0-1), the rest of
    // each tree's partly used segment made available -- it joins the tree's
    // block tree (warp 2) -- and the pointers, all at once
    if (claimed != kNone) claim_range_repair(st, claimed, lane, emptied);
    if (warp == 2 && fr != kNone && lane < core::kTrees && tsegs[lane]) {
        const uint32_t t = lane, nb = core::nb_of(t), used = tcnt[t] - (tsegs[t] - 1) * nb;
        if (used < nb) {
            const uint64_t s = fr + tbase[t] + tsegs[t] - 1;
            // the rest of the segment's blocks, consecutive: a run for the
            // next-run word of class t's first slot when that word is free
            // (one CAS; it is swapped in at the slot's next refill, trims and
            // the drain give it back like any fetched run), else into the
            // segment's ring and block tree (initSegment)
            const uint64_t run = ((uint64_t)(nb - used) << core::kRunShift) | (s * nb + used);
            if (ptx::atom_cas(core::slot_word(v, v.slot_off[t]) + 1, core::kSlotEmpty, run) != core::kSlotEmpty) {
                uint16_t *e = v.q_entries + s * core::kMaxBlocks;
                for (uint32_t q = 0; q < nb - used; q++) e[q] = (uint16_t)(used + q);
                ptx::st_relaxed(v.q_head + s, 0u);
                ptx::st_relaxed(v.q_tail + s, nb - used);
                ptx::fence_acq_rel();                         // ring entries before the count
                const uint64_t old = ptx::atom_add(v.seg_word + s, (uint64_t)(nb - used));
                core::seg_after_rmw(v, s, old, old + (nb - used));
                core::oom_notify(v);
            }
        }
    }
    // 3. pointers (read by the caller after this kernel: its end orders the
    // table writes before them)
    for (uint32_t e = tid; e < n; e += kBigThreads) {
        const uint32_t er = erank[e];
        const uint64_t addr = v.bigq[2 * (uint64_t)e];
        void *p = nullptr;
        if (er == 0xFFFFFFFFu) {
            p = nullptr;                                      // more segments than the heap
        } else if ((er >> 28) < core::kTrees) {
            const uint32_t t = er >> 28, r = er & 0x0FFFFFFFu;
            if (fr != kNone) {
                const uint64_t lin = (fr + tbase[t]) * core::nb_of(t) + r;
                ptx::st_relaxed(v.block_free + core::gid_of(t, lin), core::kSlices - 1);   // reading A-2 (block is ours)
                p = reinterpret_cast<void *>(v.heap + (lin << (16 + t)));
            } else {
                p = big_inline(v, v.bigq[2 * (uint64_t)e + 1]);
            }
        } else {
            const uint64_t size = v.bigq[2 * (uint64_t)e + 1];
            const uint64_t k = (size >> core::kSegLog2) + ((size & (core::kSegBytes - 1)) != 0);
            if (back != kNone) {
                const uint64_t i = back + (er & 0x0FFFFFFFu);
                ptx::st_relaxed(v.seg_tid + i, core::kTrees + (uint32_t)k);
                for (uint64_t m = 1; m < k; m++) ptx::st_relaxed(v.seg_tid + i + m, core::kTreeCont);
                ptx::atom_add(v.seg_word + i, core::sw_retree(core::kTreeFree, core::kTrees + (uint32_t)k));
                for (uint64_t m = 1; m < k; m++)
                    ptx::atom_add(v.seg_word + i + m, core::sw_retree(core::kTreeFree, core::kTreeCont));
                p = reinterpret_cast<void *>(v.heap + (i << core::kSegLog2));
            } else {
                p = big_inline(v, size);
            }
        }
        *reinterpret_cast<uint64_t *>(addr) = reinterpret_cast<uint64_t>(p);
    }
    __syncthreads();
#ifdef GALLATIN_TRACE
    if (tid == 0) ptx::trace(tb0, ptx::globaltimer(), (15ull << 60) | n);
#endif
    if (tid == 0) {                                           // the queue is free for the next launch
        ptx::st_relaxed(v.bigq_ctl + 1, 0u);
        ptx::fence_acq_rel();
        ptx::st_relaxed(v.bigq_ctl, 0u);
    }
}

__device__ __noinline__ void free_slow(const View &v, uint64_t p) {
    const uint64_t off = p - v.heap;
    if (off >= (v.nseg << core::kSegLog2)) { atomicAdd(v.err, 1ull); return; }
    const uint64_t s = off >> core::kSegLog2;
    const uint32_t t = core::sw_tree(ptx::ld_relaxed(v.seg_word + s));
    if (t == core::kTreeFree || t == core::kTreeCont || t < core::kTrees) { atomicAdd(v.err, 1ull); return; }
    core::free_large(v, s, t);
}

// Rare items of one lane of the bulk free kernel: block returns (this team's
// free completed 4096) and frees that are not slices/blocks.  The block id is
// re-derived from the pointer: a segment's tree id cannot change while one of
// its blocks is out.
__device__ __noinline__ void bulk_free_slow(void *const *ptrs, uint64_t base, uint32_t done, uint32_t slow, int items) {
    const View &v = c_view;
    for (int k = 0; k < items; k++) {
        const uint64_t p = reinterpret_cast<uint64_t>(ptrs[base + 32ull * k]);
        if ((done >> k) & 1) {
            const uint64_t off = p - v.heap;
            const uint32_t t = core::sw_tree(ptx::ld_relaxed(v.seg_word + (off >> core::kSegLog2)));
            const uint32_t gid =
                (uint32_t)((off >> core::kSegLog2) * core::kMaxBlocks + ((off & (core::kSegBytes - 1)) >> (16 + t)));
            atomicExch(v.block_free + gid, 0u);
            ptx::fence_acq_rel();
            core::return_block(v, gid);
        }
        if ((slow >> k) & 1) free_slow(v, p);
    }
}

// Bulk free, ITEMS pointers per thread: load pointers, then their segments'
// table words, team the lanes freeing one block, one release fence
// per leading lane, then the team counter RMWs back to back.
template <int ITEMS, int NT = kThreads>
__global__ void __launch_bounds__(NT, (ITEMS <= 4 ? 6 : 4) * kThreads / NT) k_bulk_free(void *const *__restrict__ ptrs, uint64_t n) {
    const View &v = c_view;
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t base = ((blockIdx.x * (uint64_t)NT + threadIdx.x) >> 5) * (32 * ITEMS) + lane;
    const uint64_t heap_bytes = v.nseg << core::kSegLog2;
    uint64_t p[ITEMS], w[ITEMS];
    uint32_t gid[ITEMS], oldc[ITEMS];
    unsigned peers[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + 32ull * k;
        const uint64_t x = __ldcs(reinterpret_cast<const unsigned long long *>(ptrs) + (i < n ? i : n - 1));
        p[k] = i < n ? x : 0;
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t off = p[k] - v.heap;
        // tree id of a segment holding a live block cannot change while the
        // block is out, and L1 is invalidated at launch: a cached read is exact
        w[k] = (p[k] && off < heap_bytes) ? ((uint64_t)__ldca(v.seg_tid + (off >> core::kSegLog2)) << 32) : ~0ull;
    }
    bool lead_any = false;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t off = p[k] - v.heap;
        const uint32_t t = core::sw_tree(w[k]);
        const bool blk = p[k] && t < core::kTrees;                  // slice or whole block
        gid[k] = blk ? (uint32_t)((off >> core::kSegLog2) * core::kMaxBlocks + ((off & (core::kSegBytes - 1)) >> (16 + t)))
                     : (0x80000000u | (uint32_t)(k << 5) | lane);
        peers[k] = __match_any_sync(0xFFFFFFFFu, gid[k]);
        if (!blk) peers[k] = 0;
        lead_any |= blk && lane == (uint32_t)__ffs((int)peers[k]) - 1;
    }
    // No release fence here: every write to the memory being freed was made by
    // an earlier kernel, and the kernel boundary orders it (the device-API free,
    // core::free_impl, fences per team instead).
    (void)lead_any;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        oldc[k] = 0;
        if (peers[k] && lane == (uint32_t)__ffs((int)peers[k]) - 1)
            oldc[k] = atomicAdd(v.block_free + gid[k], (uint32_t)__popc(peers[k]));
    }
    uint32_t done = 0, slow = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        if (peers[k] && lane == (uint32_t)__ffs((int)peers[k]) - 1 && oldc[k] + __popc(peers[k]) == core::kSlices)
            done |= 1u << k;                                         // the 4096th free
        if (p[k] && !peers[k]) slow |= 1u << k;
    }
    if (done | slow) bulk_free_slow(ptrs, base, done, slow, ITEMS);
}

// One warp tile of the bulk free (lane l frees p[k] = ptrs[base + 32k], base
// = tile * 32 * ITEMS + l): k_bulk_free's protocol on pointers already loaded.
// The block id is computed in 32 bits from off >> 16 (segments < 2^22).
template <int ITEMS>
__device__ __forceinline__ void free_warp_tile(const View &v, void *const *ptrs, const uint64_t (&p)[ITEMS],
                                               uint64_t base, uint32_t lane, uint64_t heap_bytes) {
    uint32_t o16[ITEMS], t[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t off = p[k] - v.heap;                        // NULL: 2^64 - heap, out of range
        const bool in = off < heap_bytes;
        o16[k] = (uint32_t)(off >> 16);                            // segment << 8 | 64 KB unit
        t[k] = in ? __ldca(v.seg_tid + (o16[k] >> 8)) : core::kTreeFree;
    }
    uint32_t gid[ITEMS], oldc[ITEMS];
    unsigned peers[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const bool blk = t[k] < core::kTrees;                       // slice or whole block
        gid[k] = blk ? ((o16[k] & ~0xFFu) | ((o16[k] & 0xFFu) >> t[k])) : (0x80000000u | (uint32_t)(k << 5) | lane);
        peers[k] = __match_any_sync(0xFFFFFFFFu, gid[k]);
        if (!blk) peers[k] = 0;
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        oldc[k] = 0;
        if (peers[k] && lane == (uint32_t)__ffs((int)peers[k]) - 1)
            oldc[k] = atomicAdd(v.block_free + gid[k], (uint32_t)__popc(peers[k]));
    }
    uint32_t done = 0, slow = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        if (peers[k] && lane == (uint32_t)__ffs((int)peers[k]) - 1 && oldc[k] + __popc(peers[k]) == core::kSlices)
            done |= 1u << k;                                         // the 4096th free
        if (p[k] && !peers[k]) slow |= 1u << k;
    }
    if (done | slow) bulk_free_slow(ptrs, base, done, slow, ITEMS);
}

// k_bulk_free's protocol through free_warp_tile (32-bit block-id math, one
// range check per item) with the warp's loads unclamped when its whole tile
// is in range.
constexpr uint64_t kFreeWideMin = 1ull << 23;     // bulk frees from here on take the 64-warp/SM kernel
template <int ITEMS, int NT = kThreads, int MINB = 6 * kThreads / NT>
__global__ void __launch_bounds__(NT, MINB) k_bulk_free_w(void *const *__restrict__ ptrs, uint64_t n) {
    const View &v = c_view;
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t wbase = ((blockIdx.x * (uint64_t)NT + threadIdx.x) >> 5) * (32 * ITEMS);
    const uint64_t base = wbase + lane;
    const unsigned long long *src = reinterpret_cast<const unsigned long long *>(ptrs);
    uint64_t p[ITEMS];
    if (wbase + 32 * ITEMS <= n) {
#pragma unroll
        for (int k = 0; k < ITEMS; k++) p[k] = __ldcs(src + base + 32ull * k);
    } else {
#pragma unroll
        for (int k = 0; k < ITEMS; k++) p[k] = base + 32ull * k < n ? __ldcs(src + base + 32ull * k) : 0;
    }
    free_warp_tile<ITEMS>(v, ptrs, p, base, lane, v.nseg << core::kSegLog2);
}


__global__ void k_replay(const uint8_t *kinds, const uint64_t *args, const uint64_t *keys, uint64_t n,
                         uint64_t *out) {
    const View &v = c_view;
    for (uint64_t i = 0; i < n; i++) {
        const uint8_t k = kinds[i];
        if (k == 0) {
            void *p = core::malloc_impl(v, args[i], (uint32_t)keys[i]);
            out[i] = p ? reinterpret_cast<uint64_t>(p) - v.heap : ~0ull;
        } else if (k == 1) {
            const uint64_t o = out[args[i]];
            core::free_impl(v, o == ~0ull ? nullptr : reinterpret_cast<void *>(v.heap + o));
            out[i] = 0;
        } else {
            core::drain_slots(v);
            for (uint64_t s = 0; s < v.nseg; s++) core::retire_idle(v, s);
            out[i] = 0;
        }
    }
}

__global__ void k_drain_slots() { core::drain_slots(c_view); }

__global__ void k_retire_idle() {
    const View &v = c_view;
    const uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (s < v.nseg) core::retire_idle(v, s);
}

// -- correctness harness ("checks the correctness of allocated memory")
__global__ void k_stamp(void *const *ptrs, const uint64_t *sizes, uint64_t n) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    for (uint32_t a = 0; a < 32; a++) {
        const uint64_t i = warp * 32 + a;
        if (i >= n) break;
        uint32_t *p = reinterpret_cast<uint32_t *>(ptrs[i]);
        if (!p) continue;
        const uint64_t words = (sizes[i] + 3) / 4, n16 = words / 4;
        const uint32_t val = (uint32_t)i;
        uint4 *q = reinterpret_cast<uint4 *>(p);
        for (uint64_t w = lane; w < n16; w += 32) q[w] = make_uint4(val, val, val, val);
        for (uint64_t w = n16 * 4 + lane; w < words; w += 32) p[w] = val;
    }
}

__global__ void k_verify(void *const *ptrs, const uint64_t *sizes, uint64_t n, unsigned long long *bad) {
    const uint64_t warp = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    unsigned long long mine = 0;
    for (uint32_t a = 0; a < 32; a++) {
        const uint64_t i = warp * 32 + a;
        if (i >= n) break;
        const uint32_t *p = reinterpret_cast<const uint32_t *>(ptrs[i]);
        if (!p) continue;
        const uint64_t words = (sizes[i] + 3) / 4, n16 = words / 4;
        const uint32_t val = (uint32_t)i;
        const uint4 *q = reinterpret_cast<const uint4 *>(p);
        for (uint64_t w = lane; w < n16; w += 32) {
            const uint4 x = __ldcg(q + w);
            mine += (x.x != val) + (x.y != val) + (x.z != val) + (x.w != val);
        }
        for (uint64_t w = n16 * 4 + lane; w < words; w += 32) mine += __ldcg(p + w) != val;
    }
    for (int o = 16; o; o >>= 1) mine += __shfl_down_sync(0xFFFFFFFFu, mine, o);
    if (lane == 0 && mine) atomicAdd(bad, mine);
}

__global__ void k_usable(void *const *ptrs, const uint64_t *sizes, uint64_t n, uint64_t *usable,
                         unsigned long long *sum, unsigned long long *bad) {
    const View &v = c_view;
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t p = reinterpret_cast<uint64_t>(ptrs[i]);
    uint64_t u = 0;
    bool wrong = false;
    if (p) {
        const uint64_t off = p - v.heap, req = sizes[i];
        if (off >= (v.nseg << core::kSegLog2)) {
            wrong = true;
        } else {
            const uint32_t t = core::sw_tree(ptx::ld_relaxed(v.seg_word + (off >> core::kSegLog2)));
            if (req <= core::kMaxSlice) {
                const uint32_t c = req <= 16 ? 0u : (uint32_t)(64 - __clzll((long long)(req - 1))) - 4;
                u = t < core::kTrees ? (16ull << t) : 0;
                wrong = t != c;
            } else if (req < core::kSegBytes) {
                const uint32_t tb = req <= 65536 ? 0u : (uint32_t)(64 - __clzll((long long)(req - 1))) - 16;
                u = t < core::kTrees ? (65536ull << t) : 0;
                wrong = t != tb;
            } else {
                const uint64_t k = (req >> core::kSegLog2) + ((req & (core::kSegBytes - 1)) != 0);
                u = (t >= core::kTrees && t < core::kTreeCont) ? ((uint64_t)(t - core::kTrees) << core::kSegLog2) : 0;
                wrong = t != core::kTrees + k;
            }
            if (u == 0 || (off & ((u < core::kSegBytes ? u : core::kSegBytes) - 1)) || u < req) wrong = true;
            if (off + u > (v.nseg << core::kSegLog2)) wrong = true;
        }
    }
    if (usable) usable[i] = u;
    if (u) atomicAdd(sum, (unsigned long long)u);
    if (wrong) atomicAdd(bad, 1ull);
}

// ------------------------------------------------------- host helpers ----
uint64_t image_words(const View &v) {
    return 8 + 10ull * v.tree_words + v.nseg * (1 + 65 + 128) + 2ull * v.nslot_total;
}

struct HostCopy {
    std::vector<uint64_t> seg_tree, block_trees, seg_word, slots;
    std::vector<uint32_t> q_head, q_tail, block_free, seg_tid;
    std::vector<uint16_t> q_entries;
    unsigned long long err = 0;
};

int copy_state(HostCopy &h) {
    const View &v = g.v;
    const uint64_t W = v.tree_words, nseg = v.nseg;
    h.seg_tree.resize(W);
    h.block_trees.resize(9 * W);
    h.seg_word.resize(nseg);
    h.q_head.resize(nseg);
    h.q_tail.resize(nseg);
    h.q_entries.resize(nseg * 256);
    h.block_free.resize(nseg * 256);
    h.slots.resize((uint64_t)v.nslot_total * 16);
    CUDA_TRY(cudaDeviceSynchronize());
    CUDA_TRY(cudaMemcpy(h.seg_tree.data(), v.seg_tree, W * 8, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.block_trees.data(), v.block_trees, 9 * W * 8, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.seg_word.data(), v.seg_word, nseg * 8, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.q_head.data(), v.q_head, nseg * 4, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.q_tail.data(), v.q_tail, nseg * 4, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.q_entries.data(), v.q_entries, nseg * 512, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.block_free.data(), v.block_free, nseg * 1024, cudaMemcpyDeviceToHost));
    h.seg_tid.resize(nseg);
    CUDA_TRY(cudaMemcpy(h.seg_tid.data(), v.seg_tid, nseg * 4, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(h.slots.data(), v.slots, h.slots.size() * 8, cudaMemcpyDeviceToHost));
    CUDA_TRY(cudaMemcpy(&h.err, v.err, 8, cudaMemcpyDeviceToHost));
    return GALLATIN_OK;
}

int free_all() {
    if (g.cin) cudaStreamDestroy(g.cin);
    if (g.cout) cudaStreamDestroy(g.cout);
    for (int i = 0; i < kMaxChunks; i++) {
        if (g.ev_in[i]) cudaEventDestroy(g.ev_in[i]);
        if (g.ev_k[i]) cudaEventDestroy(g.ev_k[i]);
    }
    if (g.heap_raw) cudaFree(g.heap_raw);
    if (g.meta) cudaFree(g.meta);
    if (g.scratch) cudaFree(g.scratch);
    g = State{};
    return GALLATIN_OK;
}

}  // namespace

// ================================================================ C-ABI ====
extern "C" {

const char *gallatin_version(void) { return "gallatin-b200 0.1 (sm_100a)"; }

const char *gallatin_error_string(int code) {
    switch (code) {
    case GALLATIN_OK: return "ok";
    case GALLATIN_ERR_INVALID: return "invalid argument";
    case GALLATIN_ERR_CUDA: return "CUDA error";
    case GALLATIN_ERR_STATE: return "bad allocator state";
    case GALLATIN_ERR_NOMEM: return "out of device memory";
    default: return "unknown";
    }
}

int gallatin_is_initialized(void) { return g.init ? 1 : 0; }

int gallatin_init_ex(const gallatin_config_t *cfg_in) {
    if (g.init) return GALLATIN_ERR_STATE;
    if (!cfg_in) return GALLATIN_ERR_INVALID;
    gallatin_config_t cfg = *cfg_in;
    const uint64_t nseg = cfg.heap_bytes >> core::kSegLog2;
    if (nseg < 1 || nseg > (1ull << 22)) return GALLATIN_ERR_INVALID;
    int dev = 0, sms = 148;
    CUDA_TRY(cudaGetDevice(&dev));
    CUDA_TRY(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
    if (!cfg.slot_base) cfg.slot_base = (uint32_t)sms;      // one slot per SM
    if (!cfg.slot_min) cfg.slot_min = (uint32_t)(nseg / 32 < 4 ? 4 : (nseg / 32 > 32 ? 32 : nseg / 32));
    if (!cfg.fence_free) cfg.fence_free = 1;
    if (!cfg.format_ahead) cfg.format_ahead = 1;
    if (!cfg.run_max) cfg.run_max = 256;
    if (!cfg.run_bytes) {
        cfg.run_bytes = (nseg << core::kSegLog2) / 64;
        if (cfg.run_bytes > (256ull << 20)) cfg.run_bytes = 256ull << 20;
    }
    if (cfg.run_max > core::kMaxRun || cfg.fence_free > 2 || cfg.format_ahead > 2) return GALLATIN_ERR_INVALID;
    if (cfg.bulk_items != 0 && cfg.bulk_items != 1 && cfg.bulk_items != 4) return GALLATIN_ERR_INVALID;
    if (cfg.prefetch > 2 || cfg.demand_hint > 2 || cfg.oom_record > 2 || cfg.prefill > 2) return GALLATIN_ERR_INVALID;
    if (!cfg.run_grow) cfg.run_grow = 3;
    if (cfg.run_grow > 8) return GALLATIN_ERR_INVALID;
    if (nseg > (1ull << 14)) return GALLATIN_ERR_INVALID;        // 22-bit run index at 64 KB blocks (256 GiB)

    View v{};
    v.nseg = nseg;
    uint32_t levels = 0;
    const uint64_t W = bittree_geometry(nseg, &levels, v.level_off);
    v.tree_levels = levels;
    v.tree_words = (uint32_t)W;
    uint32_t off = 0;
    for (uint32_t c = 0; c < core::kTrees; c++) {
        uint32_t n = cfg.slot_base >> c;
        if (n < cfg.slot_min) n = cfg.slot_min;
        if (n < 1) n = 1;
        v.nslot[c] = n;
        v.slot_off[c] = off;
        v.nslot_rcp[c] = 1.0f / (float)n;
        off += n;
    }
    v.nslot_total = off;
    for (uint32_t c = 0; c < core::kTrees; c++) {
        uint64_t m = cfg.run_bytes >> (16 + c);
        if (m > cfg.run_max) m = cfg.run_max;
        v.run_cap[c] = m < 1 ? 1u : (uint32_t)m;
    }
    if (!cfg.run_init) {
        // [dev] the largest first run (power of two <= 256 blocks) whose
        // worst case -- every slot of every class holding a fresh first run --
        // stays within half the heap: whole-segment first runs on big heaps,
        // the paper's one block on small ones (DESIGN.md Deviations 5)
        uint32_t r = 256;
        for (; r > 1; r >>= 1) {
            uint64_t hoard = 0;
            for (uint32_t c = 0; c < core::kTrees; c++) {
                const uint32_t fl = r < 8 ? r : 8u, fs = (r >> c) > fl ? (r >> c) : fl;
                const uint32_t fr = fs < (256u >> c) ? fs : (256u >> c);
                const uint32_t first = fr < v.run_cap[c] ? fr : v.run_cap[c];
                hoard += (uint64_t)v.nslot[c] * first * (65536ull << c);
            }
            if (hoard <= (nseg << core::kSegLog2) / 2) break;
        }
        cfg.run_init = r;
    }
    v.format_ahead = cfg.format_ahead == 1 ? 1u : 0u;
    v.formatters = (uint32_t)(nseg / 32 < 1 ? 1 : (nseg / 32 > 32 ? 32 : nseg / 32));
    v.run_init = cfg.run_init;
    v.run_grow = cfg.run_grow;
    v.prefetch = cfg.prefetch == 1 ? 1u : 0u;              // default off (measured: DESIGN.md)
    v.fence_free = cfg.fence_free;
    v.demand_hint = cfg.demand_hint == 2 ? 0u : 1u;
    v.oom_record = cfg.oom_record == 2 ? 0u : 1u;
    v.nsm = (uint32_t)sms;
    // prefilled block buffer (include/gallatin.h "prefill"): every
    // slot's first run (rounded down to a power of two), shrunk to fit nseg/8
    // segments, laid out class by class
    {
        uint32_t r[core::kTrees];
        for (uint32_t c = 0; c < core::kTrees; c++) {
            const uint32_t nb = 256u >> c;
            const uint32_t fl = cfg.run_init < 8 ? cfg.run_init : 8u;
            const uint32_t fs = (cfg.run_init >> c) > fl ? (cfg.run_init >> c) : fl;
            uint32_t fr = fs < nb ? fs : nb;
            if (fr > v.run_cap[c]) fr = v.run_cap[c];
            r[c] = 1u << (31 - __builtin_clz(fr));                  // largest power of two <= fr
        }
        auto segs_of = [&](uint32_t c) { return ((uint64_t)v.nslot[c] * r[c] + (256u >> c) - 1) / (256u >> c); };
        // over budget: halve the class holding the most segments (lowest class
        // on ties) whose run is above max(1, nb >> run_grow) -- the refill
        // after such a run grows to whole segments
        bool fits = true;
        for (;;) {
            uint64_t total = 0;
            for (uint32_t c = 0; c < core::kTrees; c++) total += segs_of(c);
            if (total <= nseg / 8) break;
            int big = -1;
            for (uint32_t c = 0; c < core::kTrees; c++) {
                const uint32_t floor_ = ((256u >> c) >> cfg.run_grow) > 1 ? ((256u >> c) >> cfg.run_grow) : 1u;
                if (r[c] > floor_ && (big < 0 || segs_of(c) > segs_of((uint32_t)big))) big = (int)c;
            }
            if (big < 0) { fits = false; break; }
            r[big] >>= 1;
        }
        uint64_t seg = 0;
        for (uint32_t c = 0; c < core::kTrees; c++) {
            const uint32_t nb = 256u >> c;
            const uint64_t blocks = (uint64_t)v.nslot[c] * r[c], segs = segs_of(c);
            v.pf_base[c] = (uint32_t)seg;
            v.pf_run[c] = r[c];
            v.pf_used[c] = (uint32_t)(blocks - (segs - 1) * nb);
            v.pf_last[c] = v.pf_used[c] < nb ? (uint32_t)(seg + segs - 1) : 0xFFFFFFFFu;
            seg += segs;
        }
        v.pf_segs = (cfg.prefill != 2 && fits) ? (uint32_t)seg : 0u;
    }

    // metadata: one allocation, 256 B aligned sections
    uint64_t sz[14] = {W * 8, 9 * W * 8, nseg * 8, nseg * 4, nseg * 4, nseg * 512, nseg * 1024,
                       (uint64_t)off * 128, 9 * 128, 128, nseg * 4, 128, (uint64_t)kBigCap * 16, 128};
    uint64_t total = 0, offs[14];
    for (int i = 0; i < 14; i++) { offs[i] = total; total += align_up(sz[i], 256); }
    void *meta = nullptr;
    if (cudaMalloc(&meta, total) != cudaSuccess) { cudaGetLastError(); return GALLATIN_ERR_NOMEM; }
    void *heap = nullptr;
    if (cudaMalloc(&heap, (nseg << core::kSegLog2) + core::kSegBytes) != cudaSuccess) {
        cudaGetLastError();
        cudaFree(meta);
        return GALLATIN_ERR_NOMEM;
    }
    char *m = static_cast<char *>(meta);
    v.seg_tree = reinterpret_cast<uint64_t *>(m + offs[0]);
    v.block_trees = reinterpret_cast<uint64_t *>(m + offs[1]);
    v.seg_word = reinterpret_cast<uint64_t *>(m + offs[2]);
    v.q_head = reinterpret_cast<uint32_t *>(m + offs[3]);
    v.q_tail = reinterpret_cast<uint32_t *>(m + offs[4]);
    v.q_entries = reinterpret_cast<uint16_t *>(m + offs[5]);
    v.block_free = reinterpret_cast<uint32_t *>(m + offs[6]);
    v.slots = reinterpret_cast<uint64_t *>(m + offs[7]);
    v.fmt_token = reinterpret_cast<uint32_t *>(m + offs[8]);
    v.err = reinterpret_cast<unsigned long long *>(m + offs[9]);
    v.seg_tid = reinterpret_cast<uint32_t *>(m + offs[10]);
    v.oom = reinterpret_cast<uint64_t *>(m + offs[11]);
    v.bigq = reinterpret_cast<uint64_t *>(m + offs[12]);
    v.bigq_ctl = reinterpret_cast<uint32_t *>(m + offs[13]);
    v.bigq_cap = kBigCap;
    v.heap = align_up(reinterpret_cast<uint64_t>(heap), core::kSegBytes);   // 16 MiB aligned base

    g.init = true;
    g.device = dev;
    {
        const char *e = getenv("GALLATIN_PDL");
        g.pdl = !(e && e[0] == '0');
        const char *b = getenv("GALLATIN_DEFER_BIG");             // measurement: 0 = serve big requests inline
        g.defer_big = !(b && b[0] == '0');
    }
    g.cfg = cfg;
    g.heap_raw = heap;
    g.meta = meta;
    g.meta_bytes = total;
    g.v = v;
    if (cudaMemcpyToSymbol(c_view, &v, sizeof(View)) != cudaSuccess) { free_all(); return GALLATIN_ERR_CUDA; }
    const int rc = gallatin_reset(nullptr);
    if (rc != GALLATIN_OK) { free_all(); return rc; }
    CUDA_TRY(cudaDeviceSynchronize());
    return GALLATIN_OK;
}

int gallatin_init(uint64_t heap_bytes) {
    gallatin_config_t cfg{};
    cfg.heap_bytes = heap_bytes;
    return gallatin_init_ex(&cfg);
}

int gallatin_destroy(void) {
    if (!g.init) return GALLATIN_ERR_STATE;
    cudaDeviceSynchronize();
    return free_all();
}

int gallatin_reset(void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    uint64_t n = g.v.nseg * 64;
    if ((uint64_t)g.v.nslot_total * 8 > n) n = (uint64_t)g.v.nslot_total * 8;
    unsigned grid = grid_for(n);
    if (grid > 148 * 16) grid = 148 * 16;
    k_reset<<<grid, kThreads, 0, S(stream)>>>();
    return launch_status();
}

int gallatin_malloc(const uint64_t *d_sizes, void **d_ptrs, uint64_t n, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!d_sizes || !d_ptrs || n > (1ull << 40)) return GALLATIN_ERR_INVALID;
    const uint32_t items = g.cfg.bulk_items ? g.cfg.bulk_items : (n >= (uint64_t)kItemsMin ? 4u : 1u);
    if (items == 4) {  // 128-thread CTAs, 8 requests per thread, one slot RMW per class per CTA
        // the launch's tag claims the deferred-request queue; its batch kernel follows
        if (++g.launch_tag == 0) g.launch_tag = 1;
        k_bulk_malloc_cta<8, 10, 128><<<(unsigned)((n + 1023) / 1024), 128, 0, S(stream)>>>(
            d_sizes, d_ptrs, n, g.defer_big ? g.launch_tag : 0u);
        const int rc = launch_status();
        if (rc || !g.defer_big) return rc;
        // programmatic dependent launch: k_big's launch overlaps the tail of
        // the malloc kernel; it waits for that kernel with griddepcontrol.wait
        cudaLaunchConfig_t lc = {};
        lc.gridDim = dim3(1);
        lc.blockDim = dim3(kBigThreads);
        lc.stream = S(stream);
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        at[0].val.programmaticStreamSerializationAllowed = 1;
        lc.attrs = at;
        lc.numAttrs = g.pdl ? 1 : 0;
        CUDA_TRY(cudaLaunchKernelEx(&lc, k_big, g.launch_tag));
    } else
        k_bulk_malloc<1><<<grid_for(n), kThreads, 0, S(stream)>>>(d_sizes, d_ptrs, n);
    return launch_status();
}

int gallatin_free(void *const *d_ptrs, uint64_t n, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!d_ptrs || n > (1ull << 40)) return GALLATIN_ERR_INVALID;
    const uint32_t items = g.cfg.bulk_items ? g.cfg.bulk_items : (n >= (uint64_t)kItemsMin ? 4u : 1u);
    if (items == 4 && n >= kFreeWideMin)
        // 64-thread CTAs at 32 registers (64 warps per SM): more frees in
        // flight shorten a throughput-bound launch
        k_bulk_free_w<4, 64, 32><<<(unsigned)((n + 255) / 256), 64, 0, S(stream)>>>(d_ptrs, n);
    else if (items == 4)
        // 128-thread CTAs at 40 registers (48 warps): smaller launches end on
        // the block-return tail, which the 32-register kernel lengthens
        k_bulk_free_w<4, 128><<<(unsigned)((n + 511) / 512), 128, 0, S(stream)>>>(d_ptrs, n);
    else
        k_bulk_free<1><<<grid_for(n), kThreads, 0, S(stream)>>>(d_ptrs, n);
    return launch_status();
}

static int ensure_scratch(uint64_t bytes) {
    if (!g.cin) {
        CUDA_TRY(cudaStreamCreateWithFlags(&g.cin, cudaStreamNonBlocking));
        CUDA_TRY(cudaStreamCreateWithFlags(&g.cout, cudaStreamNonBlocking));
        for (int i = 0; i < kMaxChunks; i++) {
            CUDA_TRY(cudaEventCreateWithFlags(&g.ev_in[i], cudaEventDisableTiming));
            CUDA_TRY(cudaEventCreateWithFlags(&g.ev_k[i], cudaEventDisableTiming));
        }
    }
    if (g.scratch_bytes >= bytes) return GALLATIN_OK;
    if (g.scratch) cudaFree(g.scratch);
    g.scratch = nullptr;
    g.scratch_bytes = 0;
    if (cudaMalloc(&g.scratch, bytes) != cudaSuccess) { cudaGetLastError(); return GALLATIN_ERR_NOMEM; }
    g.scratch_bytes = bytes;
    return GALLATIN_OK;
}

static uint64_t chunk_of(uint64_t n) {
    uint64_t c = (n + kMaxChunks - 1) / kMaxChunks;
    return c < kChunkMin ? kChunkMin : c;
}

// Pipelined over chunks: copy-in stream -> the caller's stream (kernels, in
// request order) -> copy-out stream; the call returns after everything landed.
int gallatin_malloc_host(const uint64_t *h_sizes, uint64_t *h_ptrs, uint64_t n, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!h_sizes || !h_ptrs) return GALLATIN_ERR_INVALID;
    int rc = ensure_scratch(16 * n);
    if (rc) return rc;
    uint64_t *d_sizes = static_cast<uint64_t *>(g.scratch);
    uint64_t *d_ptrs = d_sizes + n;
    const uint64_t ch = chunk_of(n);
    int q = 0;
    for (uint64_t lo = 0; lo < n; lo += ch, q++) {
        const uint64_t m = n - lo < ch ? n - lo : ch;
        CUDA_TRY(cudaMemcpyAsync(d_sizes + lo, h_sizes + lo, 8 * m, cudaMemcpyHostToDevice, g.cin));
        CUDA_TRY(cudaEventRecord(g.ev_in[q], g.cin));
        CUDA_TRY(cudaStreamWaitEvent(S(stream), g.ev_in[q], 0));
        rc = gallatin_malloc(d_sizes + lo, reinterpret_cast<void **>(d_ptrs + lo), m, stream);
        if (rc) return rc;
        CUDA_TRY(cudaEventRecord(g.ev_k[q], S(stream)));
        CUDA_TRY(cudaStreamWaitEvent(g.cout, g.ev_k[q], 0));
        CUDA_TRY(cudaMemcpyAsync(h_ptrs + lo, d_ptrs + lo, 8 * m, cudaMemcpyDeviceToHost, g.cout));
    }
    CUDA_TRY(cudaStreamSynchronize(g.cout));
    CUDA_TRY(cudaStreamSynchronize(S(stream)));
    return GALLATIN_OK;
}

int gallatin_free_host(const uint64_t *h_ptrs, uint64_t n, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!h_ptrs) return GALLATIN_ERR_INVALID;
    int rc = ensure_scratch(16 * n);
    if (rc) return rc;
    uint64_t *d_ptrs = static_cast<uint64_t *>(g.scratch);
    const uint64_t ch = chunk_of(n);
    int q = 0;
    for (uint64_t lo = 0; lo < n; lo += ch, q++) {
        const uint64_t m = n - lo < ch ? n - lo : ch;
        CUDA_TRY(cudaMemcpyAsync(d_ptrs + lo, h_ptrs + lo, 8 * m, cudaMemcpyHostToDevice, g.cin));
        CUDA_TRY(cudaEventRecord(g.ev_in[q], g.cin));
        CUDA_TRY(cudaStreamWaitEvent(S(stream), g.ev_in[q], 0));
        rc = gallatin_free(reinterpret_cast<void *const *>(d_ptrs + lo), m, stream);
        if (rc) return rc;
    }
    CUDA_TRY(cudaStreamSynchronize(S(stream)));
    return GALLATIN_OK;
}

int gallatin_drain(void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    k_drain_slots<<<1, 1, 0, S(stream)>>>();
    int rc = launch_status();
    if (rc) return rc;
    k_retire_idle<<<grid_for(g.v.nseg), kThreads, 0, S(stream)>>>();
    return launch_status();
}

int gallatin_replay(const uint8_t *d_kinds, const uint64_t *d_args, const uint64_t *d_keys, uint64_t n,
                    uint64_t *d_out, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!d_kinds || !d_args || !d_keys || !d_out) return GALLATIN_ERR_INVALID;
    k_replay<<<1, 1, 0, S(stream)>>>(d_kinds, d_args, d_keys, n, d_out);
    return launch_status();
}

int gallatin_snapshot_words(uint64_t *words) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (!words) return GALLATIN_ERR_INVALID;
    *words = image_words(g.v);
    return GALLATIN_OK;
}

int gallatin_snapshot(uint64_t *out, uint64_t cap, uint64_t *len) {
    if (!g.init) return GALLATIN_ERR_STATE;
    const View &v = g.v;
    const uint64_t need = image_words(v);
    if (len) *len = need;
    if (!out || cap < need) return GALLATIN_ERR_INVALID;
    HostCopy h;
    int rc = copy_state(h);
    if (rc) return rc;
    uint64_t *p = out;
    p[0] = 0x47414C4C494D4731ull;
    p[1] = v.nseg;
    p[2] = v.tree_levels;
    p[3] = v.tree_words;
    p[4] = v.nslot_total;
    p[5] = h.err;
    // [6]: segments whose read-mostly tree-id copy disagrees with the table (must be 0)
    uint64_t mism = 0;
    for (uint64_t s = 0; s < v.nseg; s++) mism += h.seg_tid[s] != (uint32_t)(h.seg_word[s] >> 32);
    p[6] = mism;
    p[7] = 0;
    p += 8;
    memcpy(p, h.seg_tree.data(), v.tree_words * 8ull);
    p += v.tree_words;
    memcpy(p, h.block_trees.data(), 9ull * v.tree_words * 8);
    p += 9ull * v.tree_words;
    for (uint64_t s = 0; s < v.nseg; s++) {
        const uint64_t w = h.seg_word[s];
        *p++ = (w & 0xFFFFFFFF00000000ull) | (uint32_t)((uint32_t)w - core::kAvailBias);
    }
    for (uint64_t s = 0; s < v.nseg; s++) {
        const uint32_t cnt = h.q_tail[s] - h.q_head[s];
        *p++ = cnt;
        uint16_t e[256];
        for (uint32_t q = 0; q < 256; q++) e[q] = q < cnt ? h.q_entries[s * 256 + ((h.q_head[s] + q) & 255)] : 0xFFFF;
        for (uint32_t q = 0; q < 64; q++)
            *p++ = (uint64_t)e[4 * q] | ((uint64_t)e[4 * q + 1] << 16) | ((uint64_t)e[4 * q + 2] << 32) |
                   ((uint64_t)e[4 * q + 3] << 48);
    }
    memcpy(p, h.block_free.data(), v.nseg * 1024);
    p += v.nseg * 128;
    for (uint32_t i = 0; i < v.nslot_total; i++) *p++ = h.slots[(uint64_t)i * 16];
    for (uint32_t i = 0; i < v.nslot_total; i++) *p++ = h.slots[(uint64_t)i * 16 + 1];
    return GALLATIN_OK;
}

int gallatin_stats(gallatin_stats_t *out) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (!out) return GALLATIN_ERR_INVALID;
    HostCopy h;
    int rc = copy_state(h);
    if (rc) return rc;
    memset(out, 0, sizeof(*out));
    const View &v = g.v;
    out->heap_base = v.heap;
    out->heap_bytes = v.nseg << core::kSegLog2;
    out->num_segments = v.nseg;
    for (uint64_t s = 0; s < v.nseg; s++) {
        if ((h.seg_tree[s >> 6] >> (s & 63)) & 1) out->free_segments++;
        const uint32_t t = (uint32_t)(h.seg_word[s] >> 32);
        if (t < core::kTrees) out->tree_segments[t]++;
        else if (t != core::kTreeFree) out->large_segments++;
    }
    out->errors = h.err;
    for (int c = 0; c < 9; c++) out->nslot[c] = v.nslot[c];
    for (int c = 0; c < 9; c++) out->run_cap[c] = v.run_cap[c];
    out->run_bytes = g.cfg.run_bytes;
    out->slot_base = g.cfg.slot_base;
    out->slot_min = g.cfg.slot_min;
    out->run_max = g.cfg.run_max;
    out->format_ahead = g.cfg.format_ahead;
    out->fence_free = v.fence_free;
    out->run_init = v.run_init;
    out->run_grow = v.run_grow;
    out->formatters = v.formatters;
    out->prefetch = v.prefetch;
    out->demand_hint = v.demand_hint;
    out->oom_record = v.oom_record;
    out->prefill_segments = v.pf_segs;
    return GALLATIN_OK;
}

uint64_t gallatin_device_view_bytes(void) { return sizeof(gallatin_device_view); }

int gallatin_get_device_view(struct gallatin_device_view *out, uint64_t out_bytes) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (!out || out_bytes != sizeof(gallatin_device_view)) return GALLATIN_ERR_INVALID;
    *out = g.v;
    return GALLATIN_OK;
}

int gallatin_stamp(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n, void *stream) {
    if (n == 0) return GALLATIN_OK;
    if (!d_ptrs || !d_sizes) return GALLATIN_ERR_INVALID;
    const uint64_t threads = (n + 31) / 32 * 32;
    k_stamp<<<grid_for(threads), kThreads, 0, S(stream)>>>(d_ptrs, d_sizes, n);
    return launch_status();
}

int gallatin_verify(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n, uint64_t *d_bad, void *stream) {
    if (n == 0) return GALLATIN_OK;
    if (!d_ptrs || !d_sizes || !d_bad) return GALLATIN_ERR_INVALID;
    const uint64_t threads = (n + 31) / 32 * 32;
    k_verify<<<grid_for(threads), kThreads, 0, S(stream)>>>(d_ptrs, d_sizes, n,
                                                           reinterpret_cast<unsigned long long *>(d_bad));
    return launch_status();
}

int gallatin_usable(void *const *d_ptrs, const uint64_t *d_sizes, uint64_t n, uint64_t *d_usable, uint64_t *d_sum,
                    uint64_t *d_bad, void *stream) {
    if (!g.init) return GALLATIN_ERR_STATE;
    if (n == 0) return GALLATIN_OK;
    if (!d_ptrs || !d_sizes || !d_sum || !d_bad) return GALLATIN_ERR_INVALID;
    k_usable<<<grid_for(n), kThreads, 0, S(stream)>>>(d_ptrs, d_sizes, n, d_usable,
                                                     reinterpret_cast<unsigned long long *>(d_sum),
                                                     reinterpret_cast<unsigned long long *>(d_bad));
    return launch_status();
}

}  // extern "C"

#ifdef GALLATIN_DEBUG_SPIN
// Debug builds only (not part of include/gallatin.h): point the spin-loop
// watchdog records at host-mapped (pinned) memory of 148*32*2 words.
extern "C" int gallatin_debug_spin_log(void *host_mapped) {
    if (cudaMemcpyToSymbol(gallatin::ptx::g_spin_log, &host_mapped, sizeof(void *)) != cudaSuccess)
        return GALLATIN_ERR_CUDA;
    return GALLATIN_OK;
}
#endif

#ifdef GALLATIN_TRACE
// Debug builds only: device buffer of cap records (3 words each) for refill
// traces; returns the number of records written so far through *n.
extern "C" int gallatin_debug_trace(void *dev_buf, uint64_t cap, uint64_t *n) {
    if (dev_buf) {
        unsigned long long z = 0;
        cudaMemcpyToSymbol(gallatin::ptx::g_trace, &dev_buf, sizeof(void *));
        cudaMemcpyToSymbol(gallatin::ptx::g_trace_cap, &cap, sizeof(cap));
        cudaMemcpyToSymbol(gallatin::ptx::g_trace_n, &z, sizeof(z));
    }
    if (n) {
        cudaDeviceSynchronize();
        unsigned long long v = 0;
        cudaMemcpyFromSymbol(&v, gallatin::ptx::g_trace_n, sizeof(v));
        *n = v;
    }
    return GALLATIN_OK;
}
#endif
