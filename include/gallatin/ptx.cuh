// gallatin/ptx.cuh -- memory-model primitives for the allocator metadata.
//
// Every metadata RMW is a relaxed gpu-scope atomic performed at L2, the
// coherence point (the paper's "one atomic per node").  Plain
// metadata reads are ld.relaxed.gpu -- the role of the paper's `ldcv` (P:158,
// P:180): they never hit a possibly stale L1 line.  Publication uses
// fence.acq_rel.gpu; the reconcile re-read
// uses fence.sc.gpu.
#pragma once
#include <stdint.h>

namespace gallatin {
namespace ptx {

__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed(const uint32_t *p) {
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint16_t ld_relaxed(const uint16_t *p) {
    uint16_t v;
    asm volatile("ld.relaxed.gpu.global.u16 %0, [%1];" : "=h"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(uint16_t *p, uint16_t v) {
    asm volatile("st.relaxed.gpu.global.u16 [%0], %1;" ::"l"(p), "h"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint32_t *p, uint32_t v) {
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// read-only path for query batches on a tree nobody mutates meanwhile
__device__ __forceinline__ uint64_t ld_nc(const uint64_t *p) { return __ldg(reinterpret_cast<const unsigned long long *>(p)); }

__device__ __forceinline__ void fence_acq_rel() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ void fence_sc() { asm volatile("fence.sc.gpu;" ::: "memory"); }

__device__ __forceinline__ uint64_t atom_add(uint64_t *p, uint64_t v) {
    return atomicAdd(reinterpret_cast<unsigned long long *>(p), (unsigned long long)v);
}
__device__ __forceinline__ uint64_t atom_or(uint64_t *p, uint64_t v) {
    return atomicOr(reinterpret_cast<unsigned long long *>(p), (unsigned long long)v);
}
__device__ __forceinline__ uint64_t atom_and(uint64_t *p, uint64_t v) {
    return atomicAnd(reinterpret_cast<unsigned long long *>(p), (unsigned long long)v);
}
__device__ __forceinline__ uint64_t atom_exch(uint64_t *p, uint64_t v) {
    return atomicExch(reinterpret_cast<unsigned long long *>(p), (unsigned long long)v);
}
__device__ __forceinline__ uint64_t atom_cas(uint64_t *p, uint64_t cmp, uint64_t v) {
    return atomicCAS(reinterpret_cast<unsigned long long *>(p), (unsigned long long)cmp, (unsigned long long)v);
}

__device__ __forceinline__ uint32_t smid() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t lane_id() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%laneid;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t lanemask_lt() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(r));
    return r;
}

__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

#ifdef GALLATIN_TRACE
// Debug builds only: refill trace records {t0, t1, slot|class|want|got} in a
// device buffer (gallatin_debug_trace).
static __device__ uint64_t *g_trace = nullptr;
static __device__ unsigned long long g_trace_n = 0;
static __device__ uint64_t g_trace_cap = 0;
__device__ __forceinline__ void trace(uint64_t t0, uint64_t t1, uint64_t info) {
    if (!g_trace) return;
    const unsigned long long i = atomicAdd(&g_trace_n, 1ull);
    if (i < g_trace_cap) {
        g_trace[3 * i] = t0;
        g_trace[3 * i + 1] = t1;
        g_trace[3 * i + 2] = info;
    }
}
#endif

#ifdef GALLATIN_DEBUG_SPIN
// Debug builds only: a spin loop that exceeds GALLATIN_DEBUG_SPIN pauses writes
// one record {site, smid, lane, value} per (SM, lane) into host-mapped memory
// the host can read while the kernel is still spinning.
static __device__ uint64_t *g_spin_log = nullptr;
#endif

// Bounded exponential backoff for spin loops (waiting on another thread's
// in-flight refill / ring slot): keeps the spinners off the L2 atomic unit.
struct Backoff {
    uint32_t ns = 32;
#ifdef GALLATIN_DEBUG_SPIN
    uint32_t n = 0, site = 0;
    uint64_t val = 0;
    __device__ __forceinline__ Backoff() {}
    __device__ __forceinline__ Backoff(uint32_t s, uint64_t v) : site(s), val(v) {}
    __device__ __forceinline__ void note(uint64_t v) { val = v; }
#else
    __device__ __forceinline__ Backoff() {}
    __device__ __forceinline__ Backoff(uint32_t, uint64_t) {}
    __device__ __forceinline__ void note(uint64_t) {}
#endif
    __device__ __forceinline__ void pause() {
        __nanosleep(ns);
        if (ns < 256) ns <<= 1;
#ifdef GALLATIN_DEBUG_SPIN
        if (++n == GALLATIN_DEBUG_SPIN && g_spin_log) {
            uint32_t sm, ln;
            asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
            asm volatile("mov.u32 %0, %%laneid;" : "=r"(ln));
            volatile uint64_t *r = g_spin_log + 2 * ((uint64_t)sm * 32 + ln);
            r[1] = val;
            r[0] = ((uint64_t)site << 48) | ((uint64_t)sm << 8) | ln | (1ull << 63);
        }
#endif
    }
};

}  // namespace ptx
}  // namespace gallatin
