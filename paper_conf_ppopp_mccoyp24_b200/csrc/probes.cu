// probes.cu -- peak probes for the roofline of the allocator path
// (DESIGN.md 5 "Roofline").
//
// Every probe is a persistent microkernel: a grid of 148 x 8 CTAs of 256
// threads (all SMs, 64 warps each) in which every thread loops over many
// operations, so the number is the unit's throughput, not the CTA launch rate.
// Independent operations are issued 4 at a time (unrolled, results consumed
// after all four) so a warp keeps several in flight.  gallatin_probe() times
// one launch with CUDA events on `stream` after one untimed warm-up launch.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "gallatin.h"
#include "gallatin/ptx.cuh"

using namespace gallatin;

namespace {
constexpr int kThreads = 256;
constexpr int kCtasPerSm = 8;
constexpr int kUnroll = 4;

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    return x;
}
__device__ __forceinline__ uint64_t gtid() { return blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; }
__device__ __forceinline__ uint64_t gthreads() { return (uint64_t)gridDim.x * blockDim.x; }

// PK1: distinct-address atom.add with return; `words` words (L2-resident at
// 16 MB); RANDOM: hashed addresses, else coalesced (thread-consecutive).
template <typename T, bool RANDOM>
__global__ void __launch_bounds__(kThreads) pk_atom_distinct(T *arr, uint64_t words, uint32_t iters, T *sink) {
    const uint64_t t = gtid(), T_ = gthreads();
    T acc = 0;
    for (uint32_t it = 0; it < iters; it += kUnroll) {
        T r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            const uint64_t j = (uint64_t)(it + u) * T_ + t;
            const uint64_t a = RANDOM ? mix64(j) % words : j % words;
            r[u] = atomicAdd(arr + a, (T)1);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; u++) acc += r[u];
    }
    if (acc == (T)0x7FFFFFFF) *sink = acc;
}

// PK2/PK3/PK4: the leader lane of every warp RMWs one of `nlines` hot 128 B
// lines chosen by smid (as the block buffer does); the 4 unrolled RMWs of an
// iteration go to lines smid, smid+1, ... (mod nlines).  MODE 0 = atom.add
// with return, 1 = red.add (no return), 2 = atom.cas (old-value guess).
template <int MODE>
__global__ void __launch_bounds__(kThreads) pk_atom_hot(uint64_t *lines, uint32_t nlines, uint32_t iters, uint64_t *sink) {
    if ((threadIdx.x & 31) != 0) return;
    const uint32_t sm = ptx::smid();
    uint64_t acc = 0, guess[kUnroll] = {0, 0, 0, 0};
    for (uint32_t it = 0; it < iters; it += kUnroll) {
        uint64_t r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            uint64_t *p = lines + (uint64_t)((sm + u) % nlines) * 16;
            if (MODE == 0) r[u] = ptx::atom_add(p, 32);
            else if (MODE == 1) { atomicAdd(reinterpret_cast<unsigned long long *>(p), 32ull); r[u] = 0; }
            else r[u] = ptx::atom_cas(p, guess[u], guess[u] + 32);
        }
#pragma unroll
        for (int u = 0; u < kUnroll; u++) {
            acc += r[u];
            if (MODE == 2) guess[u] = r[u];
        }
    }
    if (acc == 0x7FFFFFFFFFFFull) *sink = acc;
}

// PK5a: the paper's "one atomic per warp" bump allocator (RegEff-AW analogue,
// P:292): per request 8 B size in, one team RMW per warp on the SM's line,
// __shfl_sync, 8 B pointer out.
__global__ void __launch_bounds__(kThreads) pk_bump_warp(uint64_t *lines, uint32_t nlines, const uint64_t *__restrict__ sizes,
                                                         uint64_t *__restrict__ out, uint64_t n) {
    const uint32_t lane = ptx::lane_id();
    uint64_t *line = lines + (uint64_t)(ptx::smid() % nlines) * 16;
    for (uint64_t i = gtid(); i - lane < n; i += gthreads()) {
        const bool in = i < n;
        const uint64_t sz = in ? __ldcs(reinterpret_cast<const unsigned long long *>(sizes) + i) : 0;
        uint64_t old = 0;
        if (lane == 0) old = ptx::atom_add(line, (uint64_t)32 * 16);
        old = __shfl_sync(0xFFFFFFFFu, old, 0);
        if (in) __stcs(reinterpret_cast<unsigned long long *>(out) + i, old + lane * sz);
    }
}

// PK5b: this design's ceiling -- k_bulk_malloc_cta's structure without the
// allocator: 128-thread CTAs, 4 requests per thread (512-request tiles), the
// class ranked in shared memory, ONE global RMW per class per tile on the
// SM's slot line, the pointer computed by one shift-add and stored.  What a
// malloc costs at 1 RMW per 512 requests and 16 B of I/O.
__global__ void __launch_bounds__(128) pk_bump_cta(uint64_t *lines, uint32_t nlines, const uint64_t *__restrict__ sizes,
                                                   uint64_t *__restrict__ out, uint64_t n) {
    __shared__ uint32_t cnt[9];
    __shared__ uint64_t base[9];
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t b0 = blockIdx.x * 512ull + threadIdx.x;
    if (threadIdx.x < 9) cnt[threadIdx.x] = 0;
    uint64_t x[4];
    uint32_t cr[4];
#pragma unroll
    for (int k = 0; k < 4; k++) {
        const uint64_t i = b0 + 128ull * k;
        x[k] = i < n ? __ldcs(reinterpret_cast<const unsigned long long *>(sizes) + i) : 0;
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 4; k++) {
        const uint32_t lg = 64u - (uint32_t)__clzll((long long)(x[k] - 1));
        const uint32_t c = x[k] - 1 < 4096 ? (lg > 4 ? lg : 4u) - 4 : 0xFFu;
        const unsigned peers = __match_any_sync(0xFFFFFFFFu, c);
        const uint32_t leader = (uint32_t)__ffs((int)peers) - 1;
        uint32_t b = 0;
        if (c < 9 && lane == leader) b = atomicAdd(&cnt[c], (uint32_t)__popc(peers));
        cr[k] = c | ((__shfl_sync(0xFFFFFFFFu, b, (int)leader) + (uint32_t)__popc(peers & ptx::lanemask_lt())) << 8);
    }
    __syncthreads();
    if (threadIdx.x < 9 && cnt[threadIdx.x])
        base[threadIdx.x] = ptx::atom_add(lines + (uint64_t)((ptx::smid() + 37 * threadIdx.x) % nlines) * 16,
                                          (uint64_t)cnt[threadIdx.x] << (4 + threadIdx.x));
    __syncthreads();
#pragma unroll
    for (int k = 0; k < 4; k++) {
        const uint64_t i = b0 + 128ull * k;
        const uint32_t c = cr[k] & 0xFF;
        if (i < n) __stcs(reinterpret_cast<unsigned long long *>(out) + i,
                          c < 9 ? base[c] + ((uint64_t)(cr[k] >> 8) << (4 + c)) : 0ull);
    }
}

// PK7: one fence per warp per iteration (plus a store so the fence has work).
template <bool SC>
__global__ void __launch_bounds__(kThreads) pk_fence(uint64_t *buf, uint32_t iters) {
    const uint64_t t = gtid();
    for (uint32_t it = 0; it < iters; it++) {
        buf[t] = it;
        if ((threadIdx.x & 31) == 0) {
            if (SC) ptx::fence_sc();
            else ptx::fence_acq_rel();
        }
    }
}

// PK6a: random 8 B loads over `words` words (L2-resident at 16 MB; HBM
// random-sector bound at GBs), 4 independent loads in flight per thread.
__global__ void __launch_bounds__(kThreads) pk_load_random(const uint64_t *arr, uint64_t words, uint32_t iters,
                                                           uint64_t *sink) {
    const uint64_t t = gtid(), T_ = gthreads();
    uint64_t acc = 0;
    for (uint32_t it = 0; it < iters; it += kUnroll) {
        uint64_t r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; u++) r[u] = ptx::ld_relaxed(arr + mix64((uint64_t)(it + u) * T_ + t) % words);
#pragma unroll
        for (int u = 0; u < kUnroll; u++) acc += r[u];
    }
    if (acc == 0x7FFFFFFFFFFFull) *sink = acc;
}

__global__ void pk_fill(uint64_t *p, uint64_t n, uint64_t v) {
    for (uint64_t i = gtid(); i < n; i += gthreads()) p[i] = v;
}

// PK6b: HBM copy, 4 x 16 B per thread per iteration in flight.
__global__ void __launch_bounds__(kThreads) pk_copy(const uint4 *__restrict__ a, uint4 *__restrict__ b, uint64_t n16) {
    const uint64_t T_ = gthreads();
    uint64_t i = gtid();
    for (; i + 3 * T_ < n16; i += 4 * T_) {
        uint4 v[4];
#pragma unroll
        for (int u = 0; u < 4; u++) v[u] = __ldcs(a + i + u * T_);
#pragma unroll
        for (int u = 0; u < 4; u++) __stcs(b + i + u * T_, v[u]);
    }
    for (; i < n16; i += T_) b[i] = a[i];
}
}  // namespace

extern "C" int gallatin_probe(int kind, uint64_t n, uint64_t param, double *ms, double *ops, void *stream) {
    if (!ms || !ops || n == 0 || param == 0) return GALLATIN_ERR_INVALID;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const unsigned grid = (unsigned)(sms * kCtasPerSm);
    const uint64_t threads = (uint64_t)grid * kThreads, warps = threads / 32;
    // iterations per thread (per warp for the leader-only probes), multiple of kUnroll
    auto iters_for = [&](uint64_t per) {
        uint64_t it = (n + per - 1) / per;
        it = (it + kUnroll - 1) / kUnroll * kUnroll;
        return (uint32_t)(it < kUnroll ? kUnroll : (it > (1u << 30) ? (1u << 30) : it));
    };
    void *a = nullptr, *b = nullptr, *sink = nullptr;
    uint64_t abytes = 0, bbytes = 0;
    switch (kind) {
    case GALLATIN_PROBE_ATOM_U64_RANDOM: case GALLATIN_PROBE_ATOM_U64_COALESCED:
    case GALLATIN_PROBE_LOAD_RANDOM: abytes = param * 8; break;
    case GALLATIN_PROBE_ATOM_U32_RANDOM: case GALLATIN_PROBE_ATOM_U32_COALESCED: abytes = param * 4; break;
    case GALLATIN_PROBE_ATOM_HOT: case GALLATIN_PROBE_RED_HOT: case GALLATIN_PROBE_CAS_HOT: abytes = param * 128; break;
    case GALLATIN_PROBE_BUMP_WARP: case GALLATIN_PROBE_BUMP_CTA: abytes = param * 128; bbytes = n * 16; break;
    case GALLATIN_PROBE_FENCE_ACQ_REL: case GALLATIN_PROBE_FENCE_SC: abytes = threads * 8; break;
    case GALLATIN_PROBE_HBM_COPY: abytes = param; bbytes = param; break;
    default: return GALLATIN_ERR_INVALID;
    }
    if (cudaMalloc(&a, abytes) != cudaSuccess) { cudaGetLastError(); return GALLATIN_ERR_NOMEM; }
    if (bbytes && cudaMalloc(&b, bbytes) != cudaSuccess) { cudaGetLastError(); cudaFree(a); return GALLATIN_ERR_NOMEM; }
    cudaMalloc(&sink, 64);
    cudaMemsetAsync(a, 0, abytes, s);
    if (kind == GALLATIN_PROBE_BUMP_WARP || kind == GALLATIN_PROBE_BUMP_CTA) {
        pk_fill<<<grid, kThreads, 0, s>>>(static_cast<uint64_t *>(b), n, 16);   // sizes: 16 B each
    }
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double count = 0;
    for (int rep = 0; rep < 2; rep++) {
        if (rep == 1) cudaEventRecord(e0, s);
        switch (kind) {
        case GALLATIN_PROBE_ATOM_U64_RANDOM: {
            const uint32_t it = iters_for(threads);
            pk_atom_distinct<unsigned long long, true><<<grid, kThreads, 0, s>>>((unsigned long long *)a, param, it,
                                                                                (unsigned long long *)sink);
            count = (double)threads * it;
            break;
        }
        case GALLATIN_PROBE_ATOM_U64_COALESCED: {
            const uint32_t it = iters_for(threads);
            pk_atom_distinct<unsigned long long, false><<<grid, kThreads, 0, s>>>((unsigned long long *)a, param, it,
                                                                                 (unsigned long long *)sink);
            count = (double)threads * it;
            break;
        }
        case GALLATIN_PROBE_ATOM_U32_RANDOM: {
            const uint32_t it = iters_for(threads);
            pk_atom_distinct<unsigned int, true><<<grid, kThreads, 0, s>>>((unsigned int *)a, param, it, (unsigned int *)sink);
            count = (double)threads * it;
            break;
        }
        case GALLATIN_PROBE_ATOM_U32_COALESCED: {
            const uint32_t it = iters_for(threads);
            pk_atom_distinct<unsigned int, false><<<grid, kThreads, 0, s>>>((unsigned int *)a, param, it, (unsigned int *)sink);
            count = (double)threads * it;
            break;
        }
        case GALLATIN_PROBE_ATOM_HOT: case GALLATIN_PROBE_RED_HOT: case GALLATIN_PROBE_CAS_HOT: {
            const uint32_t it = iters_for(warps);
            if (kind == GALLATIN_PROBE_ATOM_HOT) pk_atom_hot<0><<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, it, (uint64_t *)sink);
            else if (kind == GALLATIN_PROBE_RED_HOT) pk_atom_hot<1><<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, it, (uint64_t *)sink);
            else pk_atom_hot<2><<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, it, (uint64_t *)sink);
            count = (double)warps * it;
            break;
        }
        case GALLATIN_PROBE_BUMP_WARP:
            pk_bump_warp<<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, (const uint64_t *)b, (uint64_t *)b + n, n);
            count = (double)n;
            break;
        case GALLATIN_PROBE_BUMP_CTA:
            pk_bump_cta<<<(unsigned)((n + 511) / 512), 128, 0, s>>>((uint64_t *)a, (uint32_t)param, (const uint64_t *)b,
                                                                   (uint64_t *)b + n, n);
            count = (double)n;
            break;
        case GALLATIN_PROBE_FENCE_ACQ_REL: case GALLATIN_PROBE_FENCE_SC: {
            const uint32_t it = (uint32_t)((n + warps - 1) / warps);
            if (kind == GALLATIN_PROBE_FENCE_SC) pk_fence<true><<<grid, kThreads, 0, s>>>((uint64_t *)a, it);
            else pk_fence<false><<<grid, kThreads, 0, s>>>((uint64_t *)a, it);
            count = (double)warps * it;
            break;
        }
        case GALLATIN_PROBE_LOAD_RANDOM: {
            const uint32_t it = iters_for(threads);
            pk_load_random<<<grid, kThreads, 0, s>>>((const uint64_t *)a, param, it, (uint64_t *)sink);
            count = (double)threads * it;
            break;
        }
        case GALLATIN_PROBE_HBM_COPY: {
            const uint64_t n16 = param / 16;
            pk_copy<<<grid, kThreads, 0, s>>>((const uint4 *)a, (uint4 *)b, n16);
            count = 2.0 * (double)(n16 * 16);
            break;
        }
        }
        if (rep == 1) cudaEventRecord(e1, s);
    }
    cudaError_t err = cudaEventSynchronize(e1);
    float t = 0;
    cudaEventElapsedTime(&t, e0, e1);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaFree(a);
    if (b) cudaFree(b);
    cudaFree(sink);
    if (err != cudaSuccess || cudaGetLastError() != cudaSuccess) return GALLATIN_ERR_CUDA;
    *ms = t;
    *ops = count;
    return GALLATIN_OK;
}
