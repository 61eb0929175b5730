// gallatin/device.cuh -- header-only device API: malloc/free from any kernel.
//
// Gallatin is a header-only library with a global variant
// whose malloc/free "can be used in any device function".  Usage:
//
//   #include "gallatin/device.cuh"
//   __global__ void k(...) {
//       void *p = gallatin::gallatin_malloc(bytes);   // nullptr on exhaustion
//       ...
//       gallatin::gallatin_free(p);
//   }
//   host:  gallatin_init(heap_bytes);  gallatin::bind_device();  k<<<...>>>(...);
//
// bind_device() copies the library's device view (gallatin_get_device_view)
// into this translation unit's __constant__ copy; call it again after
// gallatin_init in every TU that launches kernels using the API.  Overloads
// taking an explicit view exist for code that passes the view as a kernel
// argument.  Calls may come from divergent code; same-class requests of the
// lanes active together share one atomic, frees of one block share one
// atomic.  Calls are legal concurrently with the bulk C-ABI calls.
#pragma once
#include <cuda_runtime.h>

#include "gallatin.h"
#include "gallatin/core.cuh"

namespace gallatin {

static __constant__ gallatin_device_view g_device_view;

__device__ __forceinline__ void *gallatin_malloc(const gallatin_device_view &v, uint64_t bytes) {
    return core::malloc_impl(v, bytes, ptx::smid());
}
__device__ __forceinline__ void gallatin_free(const gallatin_device_view &v, void *p) { core::free_impl(v, p); }

__device__ __forceinline__ void *gallatin_malloc(uint64_t bytes) { return gallatin_malloc(g_device_view, bytes); }
__device__ __forceinline__ void gallatin_free(void *p) { gallatin_free(g_device_view, p); }

// Host: fetch the device view of the initialized allocator.
inline int get_view(gallatin_device_view *v) { return gallatin_get_device_view(v, sizeof(*v)); }

// Host: bind this TU's __constant__ view (after gallatin_init).
inline int bind_device() {
    gallatin_device_view v;
    const int rc = get_view(&v);
    if (rc != GALLATIN_OK) return rc;
    return cudaMemcpyToSymbol(g_device_view, &v, sizeof(v)) == cudaSuccess ? GALLATIN_OK : GALLATIN_ERR_CUDA;
}

}  // namespace gallatin
