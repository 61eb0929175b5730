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

__global__ void __launch_bounds__(kThreads) k_insert(BitTree t, const uint64_t *keys, uint8_t *out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x;
    if (i >= n) return;
    const bool r = bt_insert(t, keys[i]);
    if (out) out[i] = r;
}
__global__ void __launch_bounds__(kThreads) k_delete(BitTree t, const uint64_t *keys, uint8_t *out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x;
    if (i >= n) return;
    const bool r = bt_delete(t, keys[i]);
    if (out) out[i] = r;
}
__global__ void __launch_bounds__(kThreads) k_member(BitTree t, const uint64_t *keys, uint8_t *out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x;
    if (i >= n) return;
    out[i] = bt_member<true>(t, keys[i]);
}
__global__ void __launch_bounds__(kThreads) k_successor(BitTree t, const uint64_t *__restrict__ q,
                                                        uint64_t *__restrict__ out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x;
    if (i >= n) return;
    out[i] = bt_successor<true>(t, q[i]);
}
__global__ void __launch_bounds__(kThreads) k_predecessor(BitTree t, const uint64_t *__restrict__ q,
                                                          uint64_t *__restrict__ out, uint64_t n) {
    const uint64_t i = blockIdx.x * (uint64_t)kThreads + threadIdx.x;
    if (i >= n) return;
    out[i] = bt_predecessor<true>(t, q[i]);
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

#define VEB_BULK(name, kern, out_t, need_out)                                               \
    int name(veb_t *h, const uint64_t *d_keys, out_t *d_out, uint64_t n, void *stream) {   \
        if (!h) return GALLATIN_ERR_INVALID;                                                \
        if (n == 0) return GALLATIN_OK;                                                     \
        if (!d_keys || (need_out && !d_out)) return GALLATIN_ERR_INVALID;                   \
        kern<<<grid_for(n), kThreads, 0, S(stream)>>>(h->t, d_keys, d_out, n);              \
        return launch_status();                                                             \
    }

VEB_BULK(veb_insert, k_insert, uint8_t, false)
VEB_BULK(veb_delete, k_delete, uint8_t, false)
VEB_BULK(veb_member, k_member, uint8_t, true)
VEB_BULK(veb_successor, k_successor, uint64_t, true)
VEB_BULK(veb_predecessor, k_predecessor, uint64_t, true)

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
