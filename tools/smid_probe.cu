// Which %smid values exist, and how many CTAs of a 4096 x 128 launch each SM runs.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void k(unsigned *cnt, unsigned long long *sink) {
    unsigned s; asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
    if (threadIdx.x == 0) atomicAdd(cnt + s, 1u);
    unsigned long long x = clock64();
    for (int i = 0; i < 2000; i++) x = x * 6364136223846793005ull + 1;
    if (x == 42) sink[0] = x;
}
int main() {
    unsigned *d; unsigned long long *sink; cudaMalloc(&d, 1024 * 4); cudaMalloc(&sink, 8);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    for (int rep = 0; rep < 2; rep++) {
        cudaMemset(d, 0, 4096);
        k<<<4096, 128>>>(d, sink); cudaDeviceSynchronize();
        unsigned h[1024]; cudaMemcpy(h, d, 4096, cudaMemcpyDeviceToHost);
        int n = 0, mx = -1, mn = 1 << 30, mxc = 0;
        printf("sms=%d ids:", sms);
        for (int i = 0; i < 1024; i++) if (h[i]) { n++; mx = i; if ((int)h[i] < mn) mn = h[i]; if ((int)h[i] > mxc) mxc = h[i]; printf(" %d:%u", i, h[i]); }
        printf("\ncount=%d max_id=%d min_ctas=%d max_ctas=%d\n", n, mx, mn, mxc);
    }
}
