// mma_probe.cu -- how long a chain of small tcgen05.mma.cta_group::1.kind::f16
// takes on one SM, as a function of the UMMA shape (M x N, K = 16) and of the
// number of independent TMEM accumulators the chain rotates over.
// Question it answers: is the decode GEMM's ~57 cycles per M=64,N=32 MMA an
// accumulator dependency (more accumulators -> faster) or issue/throughput?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I ../paper_conf_hpdc_sunzmg00y25_b200/csrc mma_probe.cu -o mma_probe
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "sm100_ptx.cuh"
using namespace ft2dev;

template <int M, int N, int NACC>
__global__ void __launch_bounds__(128, 1) probe(int nmma, unsigned long long* out) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    __shared__ uint64_t bar;
    __shared__ uint32_t tbase;
    const int tid = threadIdx.x;
    for (int i = tid; i < (M + N) * 128 / 4; i += 128) reinterpret_cast<uint32_t*>(smem)[i] = 0u;
    if (tid == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
    if (tid < 32) tmem_alloc(&tbase, 256);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tbase;
    if (tid == 0) {
        constexpr uint32_t idesc = make_idesc(M, N);
        const uint32_t sa = smem_u32(smem);
        const uint64_t da = make_sdesc(sa), db = make_sdesc(sa + M * 128);
        unsigned long long t0, t1, t2;
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t0));
        for (int i = 0; i < nmma; ++i) {
            const int a = i % NACC;
            tc_mma(tmem + (uint32_t)(a * N), da + (uint64_t)((i & 3) * 2), db + (uint64_t)((i & 3) * 2), idesc,
                   i >= NACC ? 1u : 0u);
        }
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t1));
        tc_commit(&bar);
        mbar_wait(&bar, 0);
        asm volatile("mov.u64 %0, %%clock64;" : "=l"(t2));
        out[blockIdx.x * 2 + 0] = t1 - t0;
        out[blockIdx.x * 2 + 1] = t2 - t0;
    }
    tc_fence_before();
    __syncthreads();
    if (tid < 32) { tc_fence_after(); tmem_dealloc(tmem, 256); }
}

// NW warps issue nmma / NW MMAs each into their own accumulator: does the
// ~50-cycle cost belong to the issuing thread (overlaps across warps) or to
// the SM's tensor pipe (does not)?
template <int M, int N, int NW>
__global__ void __launch_bounds__(128, 1) probe_mw(int nmma, unsigned long long* out) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    __shared__ uint64_t bar[4];
    __shared__ uint32_t tbase;
    __shared__ unsigned long long t0s;
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int i = tid; i < (M + N) * 128 / 4; i += 128) reinterpret_cast<uint32_t*>(smem)[i] = 0u;
    if (tid == 0) { for (int w = 0; w < 4; ++w) mbar_init(&bar[w], 1); fence_mbar_init(); }
    if (tid < 32) tmem_alloc(&tbase, 256);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = tbase;
    if (tid == 0) { unsigned long long t; asm volatile("mov.u64 %0, %%clock64;" : "=l"(t)); t0s = t; }
    __syncthreads();
    if (warp < NW && (tid & 31) == 0) {
        constexpr uint32_t idesc = make_idesc(M, N);
        const uint32_t sa = smem_u32(smem);
        const uint64_t da = make_sdesc(sa), db = make_sdesc(sa + M * 128);
        for (int i = 0; i < nmma / NW; ++i)
            tc_mma(tmem + (uint32_t)(warp * 64), da + (uint64_t)((i & 3) * 2), db + (uint64_t)((i & 3) * 2), idesc,
                   i > 0 ? 1u : 0u);
        tc_commit(&bar[warp]);
        mbar_wait(&bar[warp], 0);
    }
    __syncthreads();
    if (tid == 0) {
        unsigned long long t; asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
        out[blockIdx.x * 2 + 0] = 0; out[blockIdx.x * 2 + 1] = t - t0s;
    }
    tc_fence_before();
    __syncthreads();
    if (tid < 32) { tc_fence_after(); tmem_dealloc(tmem, 256); }
}

template <int M, int N, int NW>
void run_mw(int nmma) {
    unsigned long long* d;
    cudaMalloc(&d, 2 * sizeof(unsigned long long));
    const int smem = 1024 + (M + N) * 128;
    cudaFuncSetAttribute(probe_mw<M, N, NW>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int rep = 0; rep < 3; ++rep) probe_mw<M, N, NW><<<1, 128, smem>>>(nmma, d);
    cudaDeviceSynchronize();
    unsigned long long h[2];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("M=%3d N=%3d issuing warps=%d nmma=%3d total  %7llu cyc  = %6.1f cyc/MMA\n", M, N, NW, nmma, h[1],
           (double)h[1] / nmma);
    cudaFree(d);
}

template <int M, int N, int NACC>
void run(int nmma, int grid) {
    static_assert(NACC * N <= 256, "TMEM columns");
    unsigned long long* d;
    cudaMalloc(&d, grid * 2 * sizeof(unsigned long long));
    const int smem = 1024 + (M + N) * 128;
    cudaFuncSetAttribute(probe<M, N, NACC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (int rep = 0; rep < 3; ++rep) probe<M, N, NACC><<<grid, 128, smem>>>(nmma, d);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[2 * 148];
    cudaMemcpy(h, d, grid * 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    double iss = 0, tot = 0;
    for (int b = 0; b < grid; ++b) { iss += h[2 * b]; tot += h[2 * b + 1]; }
    iss /= grid; tot /= grid;
    printf("M=%3d N=%3d acc=%d nmma=%3d grid=%3d  issue %7.0f cyc  done %7.0f cyc  = %6.1f cyc/MMA  %7.0f MAC/cyc %s\n",
           M, N, NACC, nmma, grid, iss, tot, tot / nmma, (double)M * N * 16 * nmma / tot, e ? cudaGetErrorString(e) : "");
    cudaFree(d);
}

int main() {
    run_mw<64, 32, 1>(64); run_mw<64, 32, 2>(64); run_mw<64, 32, 4>(64);
    run_mw<128, 32, 1>(64); run_mw<128, 32, 2>(64); run_mw<128, 32, 4>(64);
    run_mw<128, 64, 1>(64); run_mw<128, 64, 4>(64);
    for (int grid : {1, 148}) {
        run<64, 32, 1>(32, grid);
        run<64, 32, 2>(32, grid);
        run<64, 32, 4>(32, grid);
        run<64, 16, 1>(32, grid);
        run<64, 16, 4>(32, grid);
        run<128, 32, 1>(32, grid);
        run<128, 32, 4>(32, grid);
        run<128, 16, 1>(32, grid);
        run<128, 64, 1>(32, grid);
        run<128, 64, 4>(32, grid);
        run<128, 128, 1>(32, grid);
        run<128, 256, 1>(32, grid);
        run<64, 32, 1>(128, grid);
        run<64, 32, 4>(128, grid);
        run<128, 32, 1>(128, grid);
    }
    return 0;
}
