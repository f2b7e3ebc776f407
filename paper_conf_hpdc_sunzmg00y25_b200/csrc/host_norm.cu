// host_norm.cu -- host-model helper, NOT part of the FT2 method: the
// pre-attention / pre-MLP LayerNorm (OPT) or RMSNorm (Llama) of the decoder
// block that the runner's host model otherwise takes from torch.
//
// Why it exists: in a decode step the critical v_proj GEMM (ft2_protect_fused_gemm)
// is launched right after this norm.  torch's norm kernel never issues
// griddepcontrol.launch_dependents, so the GEMM -- launched with programmatic
// stream serialization -- cannot start its prologue (barrier init, TMEM
// allocation, the first static weight tiles) until the norm has drained.  This
// kernel triggers its dependents on entry; the GEMM's griddepcontrol.wait still
// orders every read of the norm's output after this grid completes.  Grids
// larger than one CTA per SM (prefill-sized) trigger only after their last
// store instead: an early trigger there lets the dependent's CTAs (which
// hold a whole SM's shared memory while they wait) crowd out this kernel's
// later waves (measured: +0.47 ms per OPT-1.3B prefill).
//
// One CTA per row, 256 threads, 16-byte vectors held in registers (n % 8 == 0,
// n <= 8192), fp32 statistics (two-pass mean / variance over the registers).
//
// ft2_host_act does the same for the MLP activation that precedes the
// critical fc2 / down_proj GEMM: ReLU (OPT) or silu(g) * u (Llama), rounded
// like torch (silu in fp32 rounded to the dtype, then the product rounded).
#include <cuda_bf16.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "ft2_internal.h"

namespace ft2impl {
namespace {

constexpr int kNThreads = 256;
constexpr int kNVec = 4;  // 16-byte vectors per thread: n <= 256 * 4 * 8

__device__ __forceinline__ float to_f(uint16_t v, int dt) {
    return dt == 1 ? __half2float(__ushort_as_half(v)) : __bfloat162float(__ushort_as_bfloat16(v));
}
__device__ __forceinline__ uint16_t from_f(float f, int dt) {
    return dt == 1 ? __half_as_ushort(__float2half_rn(f)) : __bfloat16_as_ushort(__float2bfloat16_rn(f));
}

__device__ __forceinline__ float block_sum(float v, float* sh) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    __syncthreads();  // sh reused across calls
    if (lane == 0) sh[warp] = v;
    __syncthreads();
    float t = lane < kNThreads / 32 ? sh[lane] : 0.f;
#pragma unroll
    for (int o = 4; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
    return __shfl_sync(0xffffffffu, t, 0);
}

__global__ void __launch_bounds__(kNThreads) host_norm_kernel(const uint16_t* __restrict__ x, int64_t ldx,
                                                              const uint16_t* __restrict__ w,
                                                              const uint16_t* __restrict__ b, uint16_t* y, int64_t ldy,
                                                              int n, float eps, int rms, int dt, int early) {
    if (early) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    __shared__ float sh[kNThreads / 32];
    const int64_t row = blockIdx.x;
    const int nv = n / 8;
    const uint4* xr = reinterpret_cast<const uint4*>(x + row * ldx);
    float v[kNVec][8];
    float s = 0.f;
#pragma unroll
    for (int u = 0; u < kNVec; ++u) {
        const int i = threadIdx.x + u * kNThreads;
        uint4 d = i < nv ? xr[i] : make_uint4(0, 0, 0, 0);
        const uint32_t q[4] = {d.x, d.y, d.z, d.w};
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            v[u][2 * j] = to_f((uint16_t)(q[j] & 0xFFFFu), dt);
            v[u][2 * j + 1] = to_f((uint16_t)(q[j] >> 16), dt);
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) s += v[u][j];
    }
    float mean = 0.f, var;
    if (rms) {
        float ss = 0.f;
#pragma unroll
        for (int u = 0; u < kNVec; ++u)
#pragma unroll
            for (int j = 0; j < 8; ++j) ss += v[u][j] * v[u][j];
        var = block_sum(ss, sh) / (float)n;
    } else {
        mean = block_sum(s, sh) / (float)n;
        float ss = 0.f;
#pragma unroll
        for (int u = 0; u < kNVec; ++u) {
            if (threadIdx.x + u * kNThreads >= nv) continue;
#pragma unroll
            for (int j = 0; j < 8; ++j) { const float c = v[u][j] - mean; ss += c * c; }
        }
        var = block_sum(ss, sh) / (float)n;
    }
    const float r = rsqrtf(var + eps);
    const uint4* wr = reinterpret_cast<const uint4*>(w);
    const uint4* br = reinterpret_cast<const uint4*>(b);
    uint4* yr = reinterpret_cast<uint4*>(y + row * ldy);
#pragma unroll
    for (int u = 0; u < kNVec; ++u) {
        const int i = threadIdx.x + u * kNThreads;
        if (i >= nv) continue;
        const uint4 wd = wr[i];
        const uint4 bd = b ? br[i] : make_uint4(0, 0, 0, 0);
        const uint32_t wq[4] = {wd.x, wd.y, wd.z, wd.w}, bq[4] = {bd.x, bd.y, bd.z, bd.w};
        uint32_t o[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            float a0 = (v[u][2 * j] - mean) * r * to_f((uint16_t)(wq[j] & 0xFFFFu), dt);
            float a1 = (v[u][2 * j + 1] - mean) * r * to_f((uint16_t)(wq[j] >> 16), dt);
            if (b) {
                a0 += to_f((uint16_t)(bq[j] & 0xFFFFu), dt);
                a1 += to_f((uint16_t)(bq[j] >> 16), dt);
            }
            o[j] = (uint32_t)from_f(a0, dt) | ((uint32_t)from_f(a1, dt) << 16);
        }
        yr[i] = make_uint4(o[0], o[1], o[2], o[3]);
    }
    if (!early) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

constexpr int kAThreads = 256;

__device__ __forceinline__ uint16_t act1(uint16_t a, uint16_t b, int act, int dt) {
    if (act == 0) {  // ReLU: NaN propagates (as torch.relu), negatives and -0 -> +0
        const bool nan = dt == 1 ? ((a & 0x7C00u) == 0x7C00u && (a & 0x03FFu)) : ((a & 0x7F80u) == 0x7F80u && (a & 0x7Fu));
        return (!nan && (a & 0x8000u)) ? (uint16_t)0 : a;
    }
    const float g = to_f(a, dt);
    const float s = to_f(from_f(g / (1.f + expf(-g)), dt), dt);
    return from_f(s * to_f(b, dt), dt);
}

__global__ void __launch_bounds__(kAThreads) host_act_kernel(const uint16_t* a, int64_t lda, const uint16_t* b,
                                                             int64_t ldb, uint16_t* y, int64_t ldy, uint32_t n8,
                                                             uint32_t total, int act, int dt, int early) {
    if (early) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
    for (uint32_t v = blockIdx.x * kAThreads + threadIdx.x; v < total; v += gridDim.x * kAThreads) {
        const uint32_t row = v / n8, c = v - row * n8;
        const uint4 da = reinterpret_cast<const uint4*>(a + (int64_t)row * lda)[c];
        const uint4 db = b ? reinterpret_cast<const uint4*>(b + (int64_t)row * ldb)[c] : make_uint4(0, 0, 0, 0);
        const uint32_t qa[4] = {da.x, da.y, da.z, da.w}, qb[4] = {db.x, db.y, db.z, db.w};
        uint32_t o[4];
#pragma unroll
        for (int j = 0; j < 4; ++j)
            o[j] = (uint32_t)act1((uint16_t)(qa[j] & 0xFFFFu), (uint16_t)(qb[j] & 0xFFFFu), act, dt) |
                   ((uint32_t)act1((uint16_t)(qa[j] >> 16), (uint16_t)(qb[j] >> 16), act, dt) << 16);
        reinterpret_cast<uint4*>(y + (int64_t)row * ldy)[c] = make_uint4(o[0], o[1], o[2], o[3]);
    }
    if (!early) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

}  // namespace
}  // namespace ft2impl

extern "C" ft2_status ft2_host_act(const void* a, int64_t lda, const void* b, int64_t ldb, void* y, int64_t ldy,
                                   int64_t rows, int32_t n, int act, int dtype, void* stream) {
    if (rows < 0 || n <= 0 || (act != 0 && act != 1)) return FT2_ERR_INVALID_ARG;
    if (rows == 0) return FT2_OK;
    if (!a || !y || (act == 1 && !b)) return FT2_ERR_INVALID_ARG;
    if (dtype != FT2_BF16 && dtype != FT2_FP16) return FT2_ERR_UNSUPPORTED;
    if (rows * (int64_t)(n / 8) >= (int64_t)1 << 31) return FT2_ERR_UNSUPPORTED;
    if (act == 0) b = nullptr, ldb = n;
    if (n % 8 || lda < n || ldy < n || ldb < n || lda % 8 || ldy % 8 || ldb % 8 ||
        (reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b) | reinterpret_cast<uintptr_t>(y)) % 16)
        return FT2_ERR_MISALIGNED;
    const uint32_t n8 = (uint32_t)(n / 8), total = (uint32_t)(rows * n8);
    const uint32_t want = (total + ft2impl::kAThreads - 1) / ft2impl::kAThreads;
    const uint32_t cap = (uint32_t)ft2impl::num_sms() * 8, grid = want < cap ? want : cap;
    ft2impl::host_act_kernel<<<grid, ft2impl::kAThreads, 0, static_cast<cudaStream_t>(stream)>>>(
        static_cast<const uint16_t*>(a), lda, static_cast<const uint16_t*>(b), ldb, static_cast<uint16_t*>(y), ldy, n8,
        total, act, dtype, grid <= (uint32_t)ft2impl::num_sms() ? 1 : 0);
    return cudaGetLastError() == cudaSuccess ? FT2_OK : FT2_ERR_CUDA;
}

extern "C" ft2_status ft2_host_norm(const void* x, int64_t ldx, const void* w, const void* b, void* y, int64_t ldy,
                             int64_t rows, int32_t n, float eps, int rms, int dtype, void* stream) {
    if (rows < 0 || n <= 0 || !(eps >= 0.f)) return FT2_ERR_INVALID_ARG;
    if (rows == 0) return FT2_OK;  // (an empty tensor may carry a NULL data pointer)
    if (!x || !w || !y) return FT2_ERR_INVALID_ARG;
    if (dtype != FT2_BF16 && dtype != FT2_FP16) return FT2_ERR_UNSUPPORTED;
    if (n % 8 != 0 || n > ft2impl::kNThreads * ft2impl::kNVec * 8 || rows > 0x7FFFFFFF) return FT2_ERR_UNSUPPORTED;
    if (ldx < n || ldy < n || ldx % 8 || ldy % 8 || (reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(w) |
                                                      reinterpret_cast<uintptr_t>(b) | reinterpret_cast<uintptr_t>(y)) % 16)
        return FT2_ERR_MISALIGNED;
    ft2impl::host_norm_kernel<<<(unsigned)rows, ft2impl::kNThreads, 0, static_cast<cudaStream_t>(stream)>>>(
        static_cast<const uint16_t*>(x), ldx, static_cast<const uint16_t*>(w), static_cast<const uint16_t*>(b),
        static_cast<uint16_t*>(y), ldy, n, eps, rms, dtype, rows <= ft2impl::num_sms() ? 1 : 0);
    return cudaGetLastError() == cudaSuccess ? FT2_OK : FT2_ERR_CUDA;
}
