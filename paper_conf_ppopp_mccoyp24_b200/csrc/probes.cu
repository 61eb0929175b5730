// probes.cu -- peak probes for the roofline of the allocator path
// (SURVEY 8(d) PK1-PK7).  Each probe is a microkernel
// filling all 148 SMs; gallatin_probe() times one launch with CUDA events
// after one untimed warm-up launch.
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "gallatin.h"
#include "gallatin/ptx.cuh"

using namespace gallatin;

namespace {
constexpr int kThreads = 256;

__device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x ^= x >> 33;
    x *= 0xff51afd7ed558ccdull;
    x ^= x >> 33;
    return x;
}

// PK1: distinct-address atom.add with return, random addresses over `words`.
__global__ void pk_atom_distinct(uint64_t *arr, uint64_t words, uint64_t n, uint64_t *sink) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t r = ptx::atom_add(arr + mix64(i) % words, 1);
    if (r == 0xFFFFFFFFFFFFull) *sink = r;
}

// PK2/PK3: one lane per warp RMWs one of `lines` hot 128 B lines (by smid, as
// the block buffer does); with_return selects ATOM vs RED.
template <bool with_return>
__global__ void pk_atom_hot(uint64_t *lines, uint32_t nlines, uint64_t n, uint64_t *sink) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    if ((threadIdx.x & 31) == 0) {
        uint64_t *p = lines + (uint64_t)(ptx::smid() % nlines) * 16;
        if (with_return) {
            const uint64_t r = ptx::atom_add(p, 32);
            if (r == 0xFFFFFFFFFFFFull) *sink = r;
        } else {
            atomicAdd(reinterpret_cast<unsigned long long *>(p), 32ull);
        }
    }
}

// PK5 (the survey's bump ceiling, RegEff-AW analogue P:292): what an allocator
// that is "one atomic per warp" costs with the same 8 B in / 8 B out per request.
__global__ void pk_bump(uint64_t *lines, uint32_t nlines, const uint64_t *__restrict__ sizes,
                        uint64_t *__restrict__ out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const uint64_t sz = sizes[i];
    const unsigned act = __activemask();
    const uint32_t lane = ptx::lane_id();
    const uint32_t leader = (uint32_t)__ffs((int)act) - 1;
    uint64_t old = 0;
    if (lane == leader) old = ptx::atom_add(lines + (uint64_t)(ptx::smid() % nlines) * 16, (uint64_t)__popc(act) * sz);
    old = __shfl_sync(act, old, (int)leader);
    out[i] = old + (uint64_t)__popc(act & ptx::lanemask_lt()) * sz;
}

// PK7: one fence.acq_rel.gpu per warp (plus a store, so the fence has work).
__global__ void pk_fence(uint64_t *buf, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i >= n) return;
    buf[i] = i;
    if ((threadIdx.x & 31) == 0) ptx::fence_acq_rel();
}

// PK6: HBM copy (cross-check of MEASURED_PEAKS.json hbm_gbs).
__global__ void pk_copy(const uint4 *__restrict__ a, uint4 *__restrict__ b, uint64_t n16) {
    const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n16; i += stride) b[i] = a[i];
}
}  // namespace

extern "C" int gallatin_probe(int kind, uint64_t n, uint64_t param, double *ms, double *ops, void *stream) {
    if (!ms || !ops || n == 0) return GALLATIN_ERR_INVALID;
    cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
    const unsigned grid = (unsigned)((n + kThreads - 1) / kThreads);
    void *a = nullptr, *b = nullptr, *sink = nullptr;
    uint64_t abytes = 0, bbytes = 0;
    switch (kind) {
    case 1: abytes = param * 8; break;
    case 2: case 3: abytes = param * 128; break;
    case 4: abytes = param * 128; bbytes = n * 16; break;
    case 5: abytes = n * 8; break;
    case 6: abytes = param; bbytes = param; break;
    default: return GALLATIN_ERR_INVALID;
    }
    if (param == 0) return GALLATIN_ERR_INVALID;
    if (cudaMalloc(&a, abytes) != cudaSuccess) return GALLATIN_ERR_NOMEM;
    if (bbytes && cudaMalloc(&b, bbytes) != cudaSuccess) { cudaFree(a); return GALLATIN_ERR_NOMEM; }
    cudaMalloc(&sink, 64);
    cudaMemsetAsync(a, 0, abytes, s);
    if (kind == 4) {
        // sizes = 16 B each (the first half of b), outputs in the second half
        uint64_t *sz = static_cast<uint64_t *>(b);
        cudaMemsetAsync(sz, 0, n * 8, s);
    }
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    double count = 0;
    for (int rep = 0; rep < 2; rep++) {
        if (rep == 1) cudaEventRecord(e0, s);
        switch (kind) {
        case 1:
            pk_atom_distinct<<<grid, kThreads, 0, s>>>((uint64_t *)a, param, n, (uint64_t *)sink);
            count = (double)n;
            break;
        case 2:
            pk_atom_hot<true><<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, n, (uint64_t *)sink);
            count = (double)((n + 31) / 32);
            break;
        case 3:
            pk_atom_hot<false><<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, n, (uint64_t *)sink);
            count = (double)((n + 31) / 32);
            break;
        case 4:
            pk_bump<<<grid, kThreads, 0, s>>>((uint64_t *)a, (uint32_t)param, (const uint64_t *)b,
                                              (uint64_t *)b + n, n);
            count = (double)n;
            break;
        case 5:
            pk_fence<<<grid, kThreads, 0, s>>>((uint64_t *)a, n);
            count = (double)((n + 31) / 32);
            break;
        case 6: {
            const uint64_t n16 = param / 16;
            pk_copy<<<148 * 8, kThreads, 0, s>>>((const uint4 *)a, (uint4 *)b, n16);
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
