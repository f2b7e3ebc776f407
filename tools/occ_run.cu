// Does the hardware co-schedule two tcgen05 (TMEM-allocating) CTAs per SM?
// 296 CTAs x 192 threads each spin ~20 us; with two resident per SM the grid
// takes ~20 us, with one ~40 us.  k_tmem allocates 32 TMEM columns, k_plain not.
#include <cstdio>
#include <cuda_runtime.h>
__device__ void spin(long long cycles) { long long t0 = clock64(); while (clock64() - t0 < cycles) {} }
__global__ void __launch_bounds__(192, 1) k_tmem(int* p, long long cyc) {
    __shared__ unsigned base;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" :: "r"((unsigned)__cvta_generic_to_shared(&base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    __syncthreads();
    spin(cyc);
    if (p && threadIdx.x == 0) p[blockIdx.x] = base;
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" :: "r"(base));
}
__global__ void __launch_bounds__(192, 1) k_plain(int* p, long long cyc) {
    spin(cyc);
    if (p && threadIdx.x == 0) p[blockIdx.x] = 1;
}
int main() {
    int* d; cudaMalloc(&d, 4096 * 4);
    long long cyc = 40000;   // ~20 us at 1.9 GHz
    int smem = 100000;
    for (auto f : {(void*)k_tmem, (void*)k_plain}) {
        cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
        cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    }
    cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
    for (int grid : {148, 296}) {
        for (int which = 0; which < 2; ++which) {
            float best = 1e9;
            for (int r = 0; r < 5; ++r) {
                cudaEventRecord(a);
                if (which == 0) k_tmem<<<grid, 192, smem>>>(d, cyc); else k_plain<<<grid, 192, smem>>>(d, cyc);
                cudaEventRecord(b); cudaEventSynchronize(b);
                float ms; cudaEventElapsedTime(&ms, a, b); if (ms < best) best = ms;
            }
            printf("grid %d %s: %.1f us (%s)\n", grid, which ? "plain" : "tmem", best * 1000, cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
