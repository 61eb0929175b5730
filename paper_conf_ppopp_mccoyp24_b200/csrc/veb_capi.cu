// veb_capi.cu -- the standalone concurrent GPU vEB tree of PAPER.md S3.2
// behind the C-ABI of include/gallatin.h: bulk insert / delete /
// member / successor / predecessor, one GPU thread per key.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "gallatin.h"
#include "gallatin/bittree.cuh"

using namespace gallatin;

struct veb {
    uint32_t k;
    BitTree t;
    uint64_t words;
    int concurrent;       // 1: queries read coherently (ld.relaxed.gpu), may overlap updates
};

namespace {
constexpr int kThreads = 256;
inline cudaStream_t S(void *s) { return reinterpret_cast<cudaStream_t>(s); }
inline unsigned grid_for(uint64_t n) { return (unsigned)((n + kThreads - 1) / kThreads); }
int launch_status() {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        fprintf(stderr, "veb: launch failed: %s\n", cudaGetErrorString(e));
        return GALLATIN_ERR_CUDA;
    }
    return GALLATIN_OK;
}

// Bulk insert / delete, ITEMS keys per thread (keys loaded first, then the
// ITEMS leaf RMWs issued back to back: several L2 round trips in flight per
// warp).  When neighbouring lanes' keys share a leaf word (sorted or
// clustered batches; one shfl + ballot decides per warp and item) the lanes
// of a warp on one word combine: one atomicOr / atomicAnd of the OR of their
// bits by the lowest such lane, the old word broadcast back, and of several
// lanes with the SAME key only the lowest reports.  Otherwise every lane
// issues its own RMW (random batches: the match would only cost issue
// slots); equal keys then still report once -- the second RMW sees the bit
// (exactly one op per distinct key returns 1, reading A-23).  The
// lane whose RMW flipped the word's emptiness repairs the summaries: set side
// bt_set_up (release fence, no re-read), clear side bt_reconcile_up.
template <bool INSERT, int ITEMS>
__global__ void __launch_bounds__(kThreads) k_update(BitTree t, const uint64_t *__restrict__ keys, uint8_t *__restrict__ out,
                                                     uint64_t n) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t base = blockIdx.x * (uint64_t)(kThreads * ITEMS) + threadIdx.x;
    uint64_t x[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + (uint64_t)kThreads * k;
        x[k] = i < n ? __ldcs(reinterpret_cast<const unsigned long long *>(keys) + i) : kNone;
    }
    uint64_t old[ITEMS], bit[ITEMS], msk[ITEMS];
    unsigned wp[ITEMS];
    bool comb[ITEMS];                                              // warp-uniform per item
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const bool valid = x[k] < t.nbits;
        const uint64_t wi = valid ? x[k] >> 6 : ~0ull - lane;       // invalid keys: a word of their own
        bit[k] = valid ? 1ull << (x[k] & 63) : 0;
        const bool adj = __shfl_up_sync(0xFFFFFFFFu, wi, 1) == wi && lane > 0;
        comb[k] = __ballot_sync(0xFFFFFFFFu, adj) != 0;
        if (comb[k]) {
            wp[k] = __match_any_sync(0xFFFFFFFFu, wi);
            msk[k] = ((uint64_t)__reduce_or_sync(wp[k], (uint32_t)(bit[k] >> 32)) << 32) |
                     __reduce_or_sync(wp[k], (uint32_t)bit[k]);
        } else {
            wp[k] = 1u << lane;
            msk[k] = bit[k];
        }
        old[k] = 0;
        if (valid && lane == (uint32_t)__ffs((int)wp[k]) - 1)
            old[k] = INSERT ? ptx::atom_or(t.w + t.off[0] + wi, msk[k]) : ptx::atom_and(t.w + t.off[0] + wi, ~msk[k]);
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint32_t leader = (uint32_t)__ffs((int)wp[k]) - 1;
        uint64_t o = old[k];
        bool first = true;                                          // the lowest lane with this key
        if (comb[k]) {
            o = __shfl_sync(0xFFFFFFFFu, old[k], (int)leader);
            const unsigned kp = __match_any_sync(0xFFFFFFFFu, x[k]);
            first = lane == (uint32_t)__ffs((int)kp) - 1;
        }
        const uint64_t i = base + (uint64_t)kThreads * k;
        const bool valid = bit[k] != 0;
        if (out && i < n) out[i] = valid && first && (INSERT ? !(o & bit[k]) : (o & bit[k]) != 0);
        if (valid && lane == leader) {
            if (INSERT && o == 0) bt_set_up(t, 0, x[k] >> 6);                          // empty -> non-empty
            if (!INSERT && (o & msk[k]) != 0 && (o & ~msk[k]) == 0) bt_reconcile_up(t, 0, x[k] >> 6);   // -> empty
        }
    }
}
// Queries, ITEMS per thread: the ITEMS query keys are loaded before any is
// walked (their HBM latency paid once, not ITEMS times).  NC: the tree words
// come through the read-only path (L1-resident at u <= 2^24) -- only while no
// update runs on the tree; otherwise coherent ld.relaxed.gpu loads
// (veb_set_concurrent), with which a set summary bit over a just-emptied
// child restarts the search past it (bt_successor / bt_predecessor).
enum QueryOp { kMember, kSucc, kPred };
template <QueryOp OP, int ITEMS, bool NC, typename OUT>
__global__ void __launch_bounds__(kThreads) k_query(BitTree t, const uint64_t *__restrict__ q, OUT *__restrict__ out,
                                                    uint64_t n) {
    const uint64_t base = blockIdx.x * (uint64_t)(kThreads * ITEMS) + threadIdx.x;
    uint64_t x[ITEMS];
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + (uint64_t)kThreads * k;
        x[k] = __ldcs(reinterpret_cast<const unsigned long long *>(q) + (i < n ? i : n - 1));
    }
#pragma unroll
    for (int k = 0; k < ITEMS; k++) {
        const uint64_t i = base + (uint64_t)kThreads * k;
        if (i >= n) break;
        if (OP == kMember) out[i] = (OUT)bt_member<NC>(t, x[k]);
        else if (OP == kSucc) out[i] = (OUT)bt_successor<NC>(t, x[k]);
        else out[i] = (OUT)bt_predecessor<NC>(t, x[k]);
    }
}
template <QueryOp OP, bool NC, typename OUT>
void launch_query_nc(const BitTree &t, const uint64_t *q, OUT *out, uint64_t n, cudaStream_t st) {
    if (n >= (1ull << 20))                                    // enough queries to fill every SM 4-deep
        k_query<OP, 4, NC, OUT><<<(unsigned)((n + 4 * kThreads - 1) / (4 * kThreads)), kThreads, 0, st>>>(t, q, out, n);
    else
        k_query<OP, 1, NC, OUT><<<grid_for(n), kThreads, 0, st>>>(t, q, out, n);
}
template <QueryOp OP, typename OUT>
int launch_query(const veb *h, const uint64_t *q, OUT *out, uint64_t n, cudaStream_t st) {
    if (h->concurrent) launch_query_nc<OP, false, OUT>(h->t, q, out, n, st);
    else launch_query_nc<OP, true, OUT>(h->t, q, out, n, st);
    return launch_status();
}
template <bool INSERT>
void launch_update(const BitTree &t, const uint64_t *keys, uint8_t *out, uint64_t n, cudaStream_t st) {
    if (n >= (1ull << 20))                                    // enough keys to fill every SM 4-deep
        k_update<INSERT, 4><<<(unsigned)((n + 4 * kThreads - 1) / (4 * kThreads)), kThreads, 0, st>>>(t, keys, out, n);
    else
        k_update<INSERT, 1><<<grid_for(n), kThreads, 0, st>>>(t, keys, out, n);
}

}  // namespace

extern "C" {

int veb_create(uint32_t universe_log2, veb_t **out) {
    if (!out || universe_log2 < 1 || universe_log2 > 32) return GALLATIN_ERR_INVALID;
    veb *h = new veb();
    h->k = universe_log2;
    h->t.nbits = 1ull << universe_log2;
    h->words = bittree_geometry(h->t.nbits, &h->t.levels, h->t.off);
    if (cudaMalloc(&h->t.w, h->words * 8) != cudaSuccess) {
        cudaGetLastError();
        delete h;
        return GALLATIN_ERR_NOMEM;
    }
    if (cudaMemset(h->t.w, 0, h->words * 8) != cudaSuccess) {
        cudaFree(h->t.w);
        delete h;
        return GALLATIN_ERR_CUDA;
    }
    *out = h;
    return GALLATIN_OK;
}

int veb_destroy(veb_t *h) {
    if (!h) return GALLATIN_ERR_INVALID;
    cudaDeviceSynchronize();
    cudaFree(h->t.w);
    delete h;
    return GALLATIN_OK;
}

int veb_clear(veb_t *h, void *stream) {
    if (!h) return GALLATIN_ERR_INVALID;
    if (cudaMemsetAsync(h->t.w, 0, h->words * 8, S(stream)) != cudaSuccess) return GALLATIN_ERR_CUDA;
    return GALLATIN_OK;
}

#define VEB_UPDATE(name, insert)                                                           \
    int name(veb_t *h, const uint64_t *d_keys, uint8_t *d_out, uint64_t n, void *stream) { \
        if (!h) return GALLATIN_ERR_INVALID;                                                \
        if (n == 0) return GALLATIN_OK;                                                     \
        if (!d_keys) return GALLATIN_ERR_INVALID;                                           \
        launch_update<insert>(h->t, d_keys, d_out, n, S(stream));                          \
        return launch_status();                                                             \
    }

VEB_UPDATE(veb_insert, true)
VEB_UPDATE(veb_delete, false)

#define VEB_QUERY(name, op, out_t)                                                         \
    int name(veb_t *h, const uint64_t *d_keys, out_t *d_out, uint64_t n, void *stream) {   \
        if (!h) return GALLATIN_ERR_INVALID;                                                \
        if (n == 0) return GALLATIN_OK;                                                     \
        if (!d_keys || !d_out) return GALLATIN_ERR_INVALID;                                 \
        return launch_query<op, out_t>(h, d_keys, d_out, n, S(stream));                    \
    }

VEB_QUERY(veb_member, kMember, uint8_t)
VEB_QUERY(veb_successor, kSucc, uint64_t)
VEB_QUERY(veb_predecessor, kPred, uint64_t)

int veb_set_concurrent(veb_t *h, int on) {
    if (!h || (on != 0 && on != 1)) return GALLATIN_ERR_INVALID;
    h->concurrent = on;
    return GALLATIN_OK;
}

int veb_words(const veb_t *h, uint64_t *words) {
    if (!h || !words) return GALLATIN_ERR_INVALID;
    *words = h->words;
    return GALLATIN_OK;
}

int veb_snapshot(const veb_t *h, uint64_t *out, uint64_t cap, uint64_t *len) {
    if (!h) return GALLATIN_ERR_INVALID;
    if (len) *len = h->words;
    if (!out || cap < h->words) return GALLATIN_ERR_INVALID;
    if (cudaDeviceSynchronize() != cudaSuccess) return GALLATIN_ERR_CUDA;
    if (cudaMemcpy(out, h->t.w, h->words * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return GALLATIN_ERR_CUDA;
    return GALLATIN_OK;
}

}  // extern "C"
