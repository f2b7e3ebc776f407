// Occupancy probe: how many 192-thread CTAs with D bytes of dynamic shared
// memory fit on one sm_100a SM (max carveout), for a trivial kernel.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void __launch_bounds__(192, 1) k1(int* p) { extern __shared__ int s[]; if (p) p[threadIdx.x] = s[threadIdx.x]; }
__global__ void __launch_bounds__(192) k2(int* p) { extern __shared__ int s[]; if (p) p[threadIdx.x] = s[threadIdx.x]; }
// the same with a TMEM allocation (tcgen05.alloc / relinquish / dealloc)
__global__ void __launch_bounds__(192, 1) k3(int* p) {
    extern __shared__ int s[];
    __shared__ unsigned base;
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" :: "r"((unsigned)__cvta_generic_to_shared(&base)));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    __syncthreads();
    if (p) p[threadIdx.x] = s[threadIdx.x] + base;
    __syncthreads();
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" :: "r"(base));
}
int main() {
    int dev = 0, smem_sm = 0, smem_blk_optin = 0, reserved = 0;
    cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
    cudaDeviceGetAttribute(&smem_blk_optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev);
    printf("smem/SM %d, optin/block %d, reserved/block %d\n", smem_sm, smem_blk_optin, reserved);
    for (int d : {0, 16384, 50000, 80000, 100000, 107904, 110000, 113000, 115000}) {
        for (int which = 0; which < 3; ++which) {
            void* f = which == 2 ? (void*)k3 : which ? (void*)k2 : (void*)k1;
            cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, d);
            cudaFuncSetAttribute(f, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
            int n = 0;
            cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, 192, d);
            printf("dyn %d kernel %s: %d blocks/SM (%s)\n", d, which == 2 ? "k3(tmem)" : which ? "k2" : "k1(lb 192,1)", n, cudaGetErrorString(e));
        }
    }
    return 0;
}
