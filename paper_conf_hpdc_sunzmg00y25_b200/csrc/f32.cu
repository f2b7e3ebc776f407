// f32.cu -- FT2 on binary32 activations: the paper's FP32 study (PAPER.md
// L334, Sec. 6: the method "also applies to FP32 models").  Same steps as the
// 16-bit kernels -- first-token bounds (L150, L221-L233) with non-finite
// correction (L225, L241), check-and-clip (L259-L272), bit-flip injection
// (L84, L90) -- on 32-bit order keys
//     key32(b) = b & 0x80000000 ? ~b : b | 0x80000000
// (total order on non-NaN values; NaN keys fall outside [key(-Inf), key(+Inf)]).
// There is no SWAR here: a 16-byte vector holds 4 values, each one key, one
// IMNMX per min/max.  Still 1 ALU op per byte, far below the HBM budget.
//
// Bound scaling (R3, readings A2/A8/A10): the product / quotient of the fp32
// value and the fp32 scale is formed in fp64 (the product is exact), rounded
// outward to fp32 (__double2float_rd / _ru) and saturated to +-FLT_MAX.
//
// TP keys (keys_out / ft2_bounds_finalize): the MAX-combinable
// int32 encoding for binary32 is (int32)(~key(lo) ^ 0x80000000),
// (int32)(key(hi) ^ 0x80000000); INT32_MIN marks a sequence with no finite value.
#include <cuda_runtime.h>
#include <stdint.h>

#include "ft2_device.cuh"
#include "ft2_internal.h"
#include "sm100_ptx.cuh"
#include "bounds_common.cuh"

namespace ft2impl {
using namespace ft2dev;

namespace {

constexpr int kThreads32 = 256;
constexpr uint32_t kKeyLo32 = 0x00800000u;  // key(-FLT_MAX)
constexpr uint32_t kKeyHi32 = 0xFF7FFFFFu;  // key(+FLT_MAX)

__device__ __forceinline__ uint32_t key32(uint32_t b) { return b ^ ((uint32_t)((int32_t)b >> 31) | 0x80000000u); }
__device__ __forceinline__ uint32_t unkey32(uint32_t k) {
    return k ^ (~(uint32_t)((int32_t)k >> 31) | 0x80000000u);
}
__device__ __forceinline__ bool isnan32(uint32_t b) { return (b & 0x7FFFFFFFu) > 0x7F800000u; }
__device__ __forceinline__ bool nonfinite32(uint32_t b) { return (b & 0x7F800000u) == 0x7F800000u; }

__device__ __forceinline__ uint32_t scale_bound32(uint32_t raw, float c, bool is_hi) {
    const double x = (double)__uint_as_float(raw), cd = (double)c;
    double s;
    if (is_hi) s = (x >= 0.0) ? __dmul_rn(x, cd) : __ddiv_rn(x, cd);
    else       s = (x <= 0.0) ? __dmul_rn(x, cd) : __ddiv_rn(x, cd);
    uint32_t r = __float_as_uint(is_hi ? __double2float_ru(s) : __double2float_rd(s));
    if (r == 0x7F800000u) r = 0x7F7FFFFFu;
    if (r == 0xFF800000u) r = 0xFF7FFFFFu;
    return r;
}

// R5 on one value: NaN -> clamp(+0), else clamp in key space.
__device__ __forceinline__ uint32_t clip32(uint32_t b, uint32_t kL, uint32_t kH) {
    const uint32_t k = isnan32(b) ? 0x80000000u : key32(b);
    return unkey32(max(min(k, kH), kL));
}

struct Bounds32K {
    uint32_t* y;
    int64_t ld;
    uint32_t n4, total_vec, chunk;
    FastDiv div_n4;
    int contiguous;
    const int32_t* seq_offsets;
    int32_t S;
    float scale;
    int32_t finalize, correct;
    uint32_t* bounds_out;
    int32_t* keys_out;
    uint32_t* nonfinite_out;
    uint32_t* nv_out;
    uint32_t* ws;
};

__device__ __forceinline__ uint4* vptr32(const Bounds32K& p, uint32_t v) {
    if (p.contiguous) return reinterpret_cast<uint4*>(p.y) + v;
    const uint32_t row = fdiv(v, p.div_n4), col = v - row * p.n4;
    return reinterpret_cast<uint4*>(p.y + (int64_t)row * p.ld) + col;
}

__device__ __forceinline__ uint32_t nv32(uint32_t b) {   // 1 < |v| < 2
    const uint32_t h = b & 0x7FFFFFFFu;
    return (h > 0x3F800000u && h < 0x40000000u) ? 1u : 0u;
}

template <bool NV>
__global__ void __launch_bounds__(kThreads32) bounds32_kernel(Bounds32K p) {
    __shared__ uint32_t sh_min[kThreads32 / 32], sh_max[kThreads32 / 32], sh_nf[kThreads32 / 32],
        sh_nv[kThreads32 / 32];
    __shared__ int sh_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int S = p.S;
    uint32_t* ws_done = p.ws + 4 * S;
    uint32_t* ws_lc = p.ws + 4 * S + 1;
    uint32_t* ws_ov = p.ws + 4 * S + 2;
    unsigned long long* list = reinterpret_cast<unsigned long long*>(
        reinterpret_cast<char*>(p.ws) + (((size_t)(4 * S + 4) * 4 + 7) & ~(size_t)7));
    constexpr int U = 4;

    uint32_t v = blockIdx.x * p.chunk;
    const uint32_t v_end = min(v + p.chunk, p.total_vec);
    while (v < v_end) {
        int s;
        uint32_t seg_end;
        if (p.seq_offsets == nullptr) {
            s = 0;
            seg_end = v_end;
        } else {
            const uint32_t row = fdiv(v, p.div_n4);
            s = seq_of_row(p.seq_offsets, S, row);
            if (s < 0) { v = min(v_end, (uint32_t)p.seq_offsets[0] * p.n4); continue; }
            if (s >= S) break;
            seg_end = min(v_end, (uint32_t)p.seq_offsets[s + 1] * p.n4);
        }
        uint32_t kmin = 0xFFFFFFFFu, kmax = 0u, nv = 0u;
        for (uint32_t base = v + tid; base < seg_end; base += kThreads32 * U) {
            uint4 d[U];
#pragma unroll
            for (int u = 0; u < U; ++u) {
                const uint32_t vi = base + u * kThreads32;
                d[u] = vi < seg_end ? ld_stream(vptr32(p, vi)) : make_uint4(0x7FC00000u, 0x7FC00000u, 0x7FC00000u, 0x7FC00000u);
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (base + u * kThreads32 >= seg_end) continue;
                const uint32_t k0 = key32(d[u].x), k1 = key32(d[u].y), k2 = key32(d[u].z), k3 = key32(d[u].w);
                kmin = min(kmin, min(min(k0, k1), min(k2, k3)));
                kmax = max(kmax, max(max(k0, k1), max(k2, k3)));
                if (NV) nv += nv32(d[u].x) + nv32(d[u].y) + nv32(d[u].z) + nv32(d[u].w);
            }
        }
        uint32_t nf = 0;
        if (kmin < kKeyLo32 || kmax > kKeyHi32) {
            // a non-finite value: redo this thread's vectors exactly
            kmin = 0xFFFFFFFFu;
            kmax = 0u;
            for (uint32_t vi = v + tid; vi < seg_end; vi += kThreads32) {
                const uint4* q = vptr32(p, vi);
                const uint4 d = *q;
                const uint32_t w[4] = {d.x, d.y, d.z, d.w};
                const uint64_t off = (uint64_t)(reinterpret_cast<const uint32_t*>(q) - p.y);
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    if (nonfinite32(w[j])) {
                        nf++;
                        if (p.correct) {
                            const uint32_t i = atomicAdd(ws_lc, 1u);
                            if (i < (uint32_t)kPatchCap) list[i] = (unsigned long long)((off + j) | ((uint64_t)s << 48));
                            else atomicExch(ws_ov, 1u);
                        }
                    } else {
                        const uint32_t k = key32(w[j]);
                        kmin = min(kmin, k);
                        kmax = max(kmax, k);
                    }
                }
            }
        }
        kmin = __reduce_min_sync(0xFFFFFFFFu, kmin);
        kmax = __reduce_max_sync(0xFFFFFFFFu, kmax);
        nf = __reduce_add_sync(0xFFFFFFFFu, nf);
        if (NV) nv = __reduce_add_sync(0xFFFFFFFFu, nv);
        if (lane == 0) { sh_min[warp] = kmin; sh_max[warp] = kmax; sh_nf[warp] = nf; sh_nv[warp] = nv; }
        __syncthreads();
        if (tid == 0) {
            uint32_t a = sh_min[0], b = sh_max[0], c = sh_nf[0], e = sh_nv[0];
#pragma unroll
            for (int i = 1; i < kThreads32 / 32; ++i) {
                a = min(a, sh_min[i]); b = max(b, sh_max[i]); c += sh_nf[i]; e += sh_nv[i];
            }
            if (NV && e) atomicAdd(&p.ws[4 * s + 3], e);
            if (a <= b) {  // slots: ~min key and max key, both >= 0x00800000 once set
                atomicMax(&p.ws[4 * s + 0], ~a);
                atomicMax(&p.ws[4 * s + 1], b);
            }
            if (c) atomicAdd(&p.ws[4 * s + 2], c);
        }
        __syncthreads();
        v = seg_end;
    }

    __syncthreads();
    if (tid == 0) sh_last = (atom_add_acq_rel_gpu(ws_done, 1u) == gridDim.x - 1);
    __syncthreads();
    if (!sh_last) return;

    // ---- last CTA: scale (R3), keys, counts, R4 fix-up, workspace reset
    const uint32_t lc0 = p.correct ? __ldcg(ws_lc) : 0u, ov0 = p.correct ? __ldcg(ws_ov) : 0u;
    for (int q = tid; q < S; q += kThreads32) {
        const uint2 wa = __ldcg(reinterpret_cast<const uint2*>(p.ws + 4 * q));
        const uint2 wb = __ldcg(reinterpret_cast<const uint2*>(p.ws + 4 * q + 2));
        const bool have = wa.x != 0u && wa.y != 0u;
        const uint32_t kmn = ~wa.x, kmx = wa.y;
        if (p.finalize) {
            uint32_t lo = 0u, hi = 0u;  // reading A9
            if (have) {
                lo = scale_bound32(unkey32(kmn), p.scale, false);
                hi = scale_bound32(unkey32(kmx), p.scale, true);
            }
            p.bounds_out[2 * q] = lo;
            p.bounds_out[2 * q + 1] = hi;
        }
        if (p.keys_out) {
            p.keys_out[2 * q] = have ? (int32_t)(wa.x ^ 0x80000000u) : INT32_MIN;
            p.keys_out[2 * q + 1] = have ? (int32_t)(kmx ^ 0x80000000u) : INT32_MIN;
        }
        if (p.nonfinite_out) p.nonfinite_out[q] = wb.x;
        if (NV) p.nv_out[q] = wb.y;
        *reinterpret_cast<uint2*>(p.ws + 4 * q) = make_uint2(0u, 0u);
        *reinterpret_cast<uint2*>(p.ws + 4 * q + 2) = make_uint2(0u, 0u);
    }
    __syncthreads();
    if (p.correct && lc0 != 0u) {
        if (!ov0) {
            for (uint32_t i = tid; i < lc0; i += kThreads32) {
                const unsigned long long e = __ldcg(list + i);
                const int q = (int)(e >> 48);
                const uint64_t off = e & 0xFFFFFFFFFFFFull;
                const uint32_t lo = p.bounds_out[2 * q], hi = p.bounds_out[2 * q + 1];
                p.y[off] = clip32(p.y[off], key32(lo), key32(hi));
            }
        } else {
            for (uint32_t vi = tid; vi < p.total_vec; vi += kThreads32) {
                int q = 0;
                if (p.seq_offsets) {
                    q = seq_of_row(p.seq_offsets, S, fdiv(vi, p.div_n4));
                    if (q < 0 || q >= S) continue;
                }
                uint32_t* e = reinterpret_cast<uint32_t*>(vptr32(p, vi));
                const uint32_t kL = key32(p.bounds_out[2 * q]), kH = key32(p.bounds_out[2 * q + 1]);
                for (int j = 0; j < 4; ++j)
                    if (nonfinite32(e[j])) e[j] = clip32(e[j], kL, kH);
            }
        }
        __syncthreads();
        const uint32_t used = min(lc0, (uint32_t)kPatchCap);
        for (uint32_t i = tid; i < used; i += kThreads32) list[i] = 0ull;
    }
    if (tid == 0) { *ws_lc = 0u; *ws_ov = 0u; *ws_done = 0u; }
}

__global__ void finalize32_kernel(const int32_t* keys, int32_t S, float scale, uint32_t* out) {
    const int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    const int32_t a = keys[2 * s], b = keys[2 * s + 1];
    uint32_t lo = 0u, hi = 0u;
    if (a != INT32_MIN && b != INT32_MIN) {
        lo = scale_bound32(unkey32(~((uint32_t)a ^ 0x80000000u)), scale, false);
        hi = scale_bound32(unkey32((uint32_t)b ^ 0x80000000u), scale, true);
    }
    out[2 * s] = lo;
    out[2 * s + 1] = hi;
}

struct Protect32K {
    uint32_t* y;
    int64_t ld;
    uint32_t n4, total_vec;
    FastDiv div_n4;
    int contiguous;
    const int32_t* row_to_seq;
    int32_t S, row_mode;
    const uint32_t* bounds;
    uint32_t* counts;
};

__global__ void __launch_bounds__(kThreads32) protect32_kernel(Protect32K p) {
    constexpr int U = 4;
    uint32_t kL = 0, kH = 0;
    if (p.row_mode == 2) { kL = key32(p.bounds[0]); kH = key32(p.bounds[1]); }
    const uint32_t stride = gridDim.x * kThreads32 * U;
    for (uint32_t base = blockIdx.x * kThreads32 * U + threadIdx.x; base < p.total_vec; base += stride) {
        uint4 d[U];
        uint4* q[U];
        uint32_t row[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const uint32_t vi = base + u * kThreads32;
            const uint32_t vv = vi < p.total_vec ? vi : 0u;
            row[u] = fdiv(vv, p.div_n4);
            q[u] = p.contiguous ? reinterpret_cast<uint4*>(p.y) + vv
                                : reinterpret_cast<uint4*>(p.y + (int64_t)row[u] * p.ld) + (vv - row[u] * p.n4);
            if (vi < p.total_vec) d[u] = ld_stream(q[u]);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            if (base + u * kThreads32 >= p.total_vec) continue;
            int s = 0;
            if (p.row_mode != 2) {
                s = p.row_mode == 1 ? (int)row[u] : p.row_to_seq[row[u]];
                if (s < 0 || s >= p.S) continue;
                kL = key32(p.bounds[2 * s]);
                kH = key32(p.bounds[2 * s + 1]);
            }
            uint32_t w[4] = {d[u].x, d[u].y, d[u].z, d[u].w};
            uint32_t diff = 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                const uint32_t k = key32(w[j]);
                diff |= max(min(k, kH), kL) ^ k;   // NaN keys are outside every finite bound
            }
            if (diff) {
                uint32_t cnt = 0;
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t o = clip32(w[j], kL, kH);
                    cnt += (o != w[j]);
                    w[j] = o;
                }
                *q[u] = make_uint4(w[0], w[1], w[2], w[3]);
                if (p.counts && cnt) atomicAdd(&p.counts[s], cnt);
            }
        }
    }
}

__global__ void inject32_kernel(uint32_t* y, int64_t rows, int64_t n, int64_t ld, const ft2_fault_site* sites,
                                int32_t n_sites, int32_t layer, int32_t step, const int32_t* base_row) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_sites) return;
    const ft2_fault_site s = sites[i];
    if ((int32_t)s.step != step || (int32_t)s.layer != layer) return;
    const int64_t row = (base_row ? (int64_t)base_row[i] : (int64_t)i) + (step == 0 ? (int64_t)s.token : 0);
    if (row < 0 || row >= rows || (int64_t)s.col >= n) return;
    y[row * ld + s.col] ^= s.xor_mask;
}

// One full wave of resident CTAs per kernel: the two sweeps differ in register
// count (protect32 holds 4 vectors + their addresses), so each grid is sized
// from its own occupancy -- sizing protect32 from bounds32's 6 CTAs/SM left a
// 20% second wave (measured 84% of HBM peak).
int g_grid32[2] = {0, 0};

template <typename K>
int max_grid32(int which, K kernel) {
    if (g_grid32[which] == 0) {
        int b = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, kernel, kThreads32, 0) != cudaSuccess) b = 1;
        g_grid32[which] = num_sms() * (b > 0 ? b : 1);
    }
    return g_grid32[which];
}

}  // namespace

cudaError_t launch_bounds32(const BoundsArgs& a, cudaStream_t st, int* n_launch) {
    Bounds32K p;
    p.y = reinterpret_cast<uint32_t*>(a.y);
    p.ld = a.ld;
    p.n4 = (uint32_t)(a.n / 4);
    p.total_vec = (uint32_t)(a.rows * (a.n / 4));
    p.div_n4 = make_fastdiv(p.n4);
    p.contiguous = a.ld == a.n;
    p.seq_offsets = a.seq_offsets;
    p.S = a.S;
    p.scale = a.scale;
    p.finalize = a.finalize;
    p.correct = a.correct;
    p.bounds_out = reinterpret_cast<uint32_t*>(a.bounds_out);
    p.keys_out = a.keys_out;
    p.nonfinite_out = a.nonfinite_out;
    p.nv_out = a.nv_out;
    p.ws = a.ws;
    const uint32_t per = kThreads32 * 4, mg = (uint32_t)max_grid32(0, bounds32_kernel<false>);
    uint32_t grid = (p.total_vec + per - 1) / per;
    grid = grid < 1 ? 1 : (grid > mg ? mg : grid);
    p.chunk = (p.total_vec + grid - 1) / grid;
    grid = (p.total_vec + p.chunk - 1) / p.chunk;
    if (grid < 1) grid = 1;
    if (a.nv_out) bounds32_kernel<true><<<grid, kThreads32, 0, st>>>(p);
    else bounds32_kernel<false><<<grid, kThreads32, 0, st>>>(p);
    ++*n_launch;
    return cudaGetLastError();
}

cudaError_t launch_finalize32(const int32_t* keys, int32_t S, float scale, void* out, cudaStream_t st, int* n_launch) {
    finalize32_kernel<<<(S + 127) / 128, 128, 0, st>>>(keys, S, scale, static_cast<uint32_t*>(out));
    ++*n_launch;
    return cudaGetLastError();
}

cudaError_t launch_protect32(const ProtectArgs& a, cudaStream_t st, int* n_launch) {
    Protect32K p;
    p.y = reinterpret_cast<uint32_t*>(a.y);
    p.ld = a.ld;
    p.n4 = (uint32_t)(a.n / 4);
    p.total_vec = (uint32_t)(a.rows * (a.n / 4));
    p.div_n4 = make_fastdiv(p.n4);
    p.contiguous = a.ld == a.n;
    p.row_to_seq = a.row_to_seq;
    p.S = a.S;
    p.row_mode = a.row_to_seq ? 0 : (a.S == 1 ? 2 : 1);
    p.bounds = reinterpret_cast<const uint32_t*>(a.bounds);
    p.counts = a.counts;
    const uint32_t per = kThreads32 * 4, mg = (uint32_t)max_grid32(1, protect32_kernel);
    uint32_t grid = (p.total_vec + per - 1) / per;
    grid = grid < 1 ? 1 : (grid > mg ? mg : grid);
    protect32_kernel<<<grid, kThreads32, 0, st>>>(p);
    ++*n_launch;
    return cudaGetLastError();
}

cudaError_t launch_inject32(void* y, int64_t rows, int64_t n, int64_t ld, const ft2_fault_site* sites, int32_t n_sites,
                            int32_t layer, int32_t step, const int32_t* base_row, cudaStream_t st, int* n_launch) {
    inject32_kernel<<<(n_sites + 127) / 128, 128, 0, st>>>(static_cast<uint32_t*>(y), rows, n, ld, sites, n_sites,
                                                           layer, step, base_row);
    ++*n_launch;
    return cudaGetLastError();
}

}  // namespace ft2impl
