// bounds.cu -- first-token bound profiling as
// one HBM sweep on sm_100a.
//
// Each CTA owns a contiguous range of 16-byte vectors (8 bf16) of the prefill
// output and splits it at sequence boundaries.  Per segment every thread keeps
// a packed-u16x2 min and max of order keys over its 128-bit coalesced loads
// (4-8 loads in flight per thread: PRMT+LOP3 for the keys, VIMNMX.U16x2 for the
// min/max -- 2 ALU ops per element), the warp combines with redux.sync
// (CREDUX), the CTA through shared memory, and the grid through u32 atomicMax
// on a self-cleaning workspace.  The last CTA to finish (threadfence
// reduction) scales the bounds (R3), writes them, patches the few non-finite
// elements it was told about (R4), and zeroes the workspace.
//
// Non-finite values (NaN/Inf) are excluded from the bounds (readings A3/A4).
// The fast loop does not test for them: any non-finite key lies below 0x0080
// or above 0xFF7F, so a thread whose min/max leave [0x0080, 0xFF7F] re-sweeps
// its own vectors in a slow exact path.  In the common all-finite case the
// kernel moves 2 bytes/element and does no extra work.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "ft2_device.cuh"
#include "ft2_internal.h"
#include "sm100_ptx.cuh"
#include "bounds_common.cuh"

namespace ft2impl {
using namespace ft2dev;

constexpr int kThreads = 256;

size_t bounds_ws_bytes(int32_t S) {
    size_t head = (size_t)(4 * S + 4) * 4;
    head = (head + 7) & ~(size_t)7;
    return head + (size_t)kPatchCap * 8;
}

// NaN-vulnerable halves of a packed word (Fig. 7: values in
// (-2,-1) U (1,2), whose exponent-MSB flip gives NaN): |h| strictly between 1
// and 2 <=> (h & 0x7FFF) in [one + 1, two - 1].
template <int DT>
__device__ __forceinline__ uint32_t nv_halves(uint32_t w) {
    constexpr uint32_t one = DT == 1 ? 0x3C00u : 0x3F80u, two = DT == 1 ? 0x4000u : 0x4000u;
    const uint32_t h = w & 0x7FFF7FFFu;
    const uint32_t c = vmax_u16x2(vmin_u16x2(h, (two - 1) * 0x10001u), (one + 1) * 0x10001u);
    return 2u - nonzero_halves(c ^ h);
}

// Slow exact path for one vector: min/max over finite keys, count the rest.
template <int DT>
__device__ __forceinline__ void slow_vec(const BoundsK& p, uint32_t v, int s, uint32_t& kmin, uint32_t& kmax,
                                         uint32_t& nf, uint32_t* lc, uint32_t* ov, unsigned long long* list) {
    const uint4* q = vec_ptr(p, v);
    uint4 d = *q;
    uint32_t w[4] = {d.x, d.y, d.z, d.w};
    uint64_t base = (uint64_t)(reinterpret_cast<const uint16_t*>(q) - p.y);
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        uint16_t b = (uint16_t)(w[j >> 1] >> ((j & 1) * 16));
        if (nonfinite1<DT>(b)) {
            nf++;
            if (p.correct) record_patch(p, lc, ov, list, s, base + j);
        } else {
            uint32_t k = key1(b);
            kmin = min(kmin, k);
            kmax = max(kmax, k);
        }
    }
}

// kUnroll 16-byte loads in flight per thread: 8 for tensors one sweep covers
// (latency-bound, e.g. prefill outputs), 4 for the bandwidth-bound large ones.
template <int DT, bool NV, int kUnroll>
__global__ void __launch_bounds__(kThreads) bounds_kernel(BoundsK p) {
    __shared__ uint32_t sh_min[kThreads / 32], sh_max[kThreads / 32], sh_nf[kThreads / 32], sh_nv[kThreads / 32];
    __shared__ int sh_last;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int S = p.S;
    uint32_t* ws_done = p.ws + 4 * S;
    uint32_t* ws_lc = p.ws + 4 * S + 1;
    uint32_t* ws_ov = p.ws + 4 * S + 2;
    unsigned long long* list = reinterpret_cast<unsigned long long*>(
        reinterpret_cast<char*>(p.ws) + (((size_t)(4 * S + 4) * 4 + 7) & ~(size_t)7));

    uint32_t v = blockIdx.x * p.chunk;
    uint32_t v_end = min(v + p.chunk, p.total_vec);
    while (v < v_end) {
        int s;
        uint32_t seg_end;
        if (p.seq_offsets == nullptr) {
            s = 0;
            seg_end = v_end;
        } else {
            uint32_t row = fdiv(v, p.div_n8);
            s = seq_of_row(p.seq_offsets, S, row);
            if (s < 0) {  // padding rows before the first sequence
                v = min(v_end, (uint32_t)p.seq_offsets[0] * p.n8);
                continue;
            }
            if (s >= S) break;  // padding rows after the last sequence
            seg_end = min(v_end, (uint32_t)p.seq_offsets[s + 1] * p.n8);
        }
        // ---- fast sweep of [v, seg_end): packed key min/max, 4 x 16 B in flight
        uint32_t mn2 = 0xFFFFFFFFu, mx2 = 0u, nv = 0u;
        for (uint32_t base = v + tid; base < seg_end; base += kThreads * kUnroll) {
            uint4 d[kUnroll];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                uint32_t vi = base + u * kThreads;
                d[u] = vi < seg_end ? ld_stream(vec_ptr(p, vi)) : make_uint4(0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu, 0xFFFFFFFFu);
            }
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                uint32_t vi = base + u * kThreads;
                uint32_t k0 = key2(d[u].x), k1 = key2(d[u].y), k2 = key2(d[u].z), k3 = key2(d[u].w);
                uint32_t a = vmin_u16x2(vmin_u16x2(k0, k1), vmin_u16x2(k2, k3));
                uint32_t b = vmax_u16x2(vmax_u16x2(k0, k1), vmax_u16x2(k2, k3));
                if (vi < seg_end) {
                    mn2 = vmin_u16x2(mn2, a);
                    mx2 = vmax_u16x2(mx2, b);
                    if (NV) nv += nv_halves<DT>(d[u].x) + nv_halves<DT>(d[u].y) + nv_halves<DT>(d[u].z) + nv_halves<DT>(d[u].w);
                }
            }
        }
        uint32_t kmin = min(mn2 & 0xFFFFu, mn2 >> 16);
        uint32_t kmax = max(mx2 & 0xFFFFu, mx2 >> 16);
        uint32_t nf = 0;
        if (kmin < Fmt<DT>::kKeyLo || kmax > Fmt<DT>::kKeyHi) {
            // this thread saw a non-finite value: redo its vectors exactly
            kmin = 0xFFFFu;
            kmax = 0u;
            for (uint32_t vi = v + tid; vi < seg_end; vi += kThreads)
                slow_vec<DT>(p, vi, s, kmin, kmax, nf, ws_lc, ws_ov, list);
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
            for (int i = 1; i < kThreads / 32; ++i) {
                a = min(a, sh_min[i]); b = max(b, sh_max[i]); c += sh_nf[i]; e += sh_nv[i];
            }
            if (NV && e) atomicAdd(&p.ws[4 * s + 3], e);
            if (a <= b) {  // at least one finite value in this segment
                atomicMax(&p.ws[4 * s + 0], 0x10000u - a);
                atomicMax(&p.ws[4 * s + 1], b + 1u);
            }
            if (c) atomicAdd(&p.ws[4 * s + 2], c);
        }
        __syncthreads();
        v = seg_end;
    }

    // ---- grid combine: the last CTA finalises.  One acq_rel atomic per CTA
    // (release: cumulative over this CTA's REDs and patch records, which the
    // barrier orders before it; acquire for the last CTA), then every slot is
    // read with independent L2 loads: two L2 round trips on the critical path.
    __syncthreads();
    if (tid == 0) sh_last = (atom_add_acq_rel_gpu(ws_done, 1u) == gridDim.x - 1);
    __syncthreads();
    if (!sh_last) return;

    bounds_finalize_tail<DT, NV>(p, tid, kThreads);
}

template <int DT>
__global__ void finalize_kernel(const int32_t* keys, int32_t S, float scale, uint16_t* out) {
    int s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= S) return;
    int32_t a = keys[2 * s], b = keys[2 * s + 1];
    uint16_t lo = 0, hi = 0;
    if (a >= 0 && b >= 0) {
        lo = scale_bound<DT>(unkey1((uint16_t)(0xFFFF - a)), scale, false);
        hi = scale_bound<DT>(unkey1((uint16_t)b), scale, true);
    }
    out[2 * s] = lo;
    out[2 * s + 1] = hi;
}

static int g_blocks_per_sm = 0;

cudaError_t launch_bounds(const BoundsArgs& a, cudaStream_t st, int* n_launch) {
    BoundsK p;
    p.y = a.y;
    p.ld = a.ld;
    p.n8 = (uint32_t)(a.n / 8);
    p.total_vec = (uint32_t)(a.rows * (a.n / 8));
    p.div_n8 = make_fastdiv(p.n8);
    p.contiguous = (a.ld == a.n);
    p.seq_offsets = a.seq_offsets;
    p.S = a.S;
    p.scale = a.scale;
    p.finalize = a.finalize;
    p.correct = a.correct;
    p.bounds_out = a.bounds_out;
    p.keys_out = a.keys_out;
    p.nonfinite_out = a.nonfinite_out;
    p.nv_out = a.nv_out;
    p.ws = a.ws;
    if (g_blocks_per_sm == 0) {
        int b = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, bounds_kernel<0, false, 4>, kThreads, 0);
        if (e != cudaSuccess) return e;
        g_blocks_per_sm = b > 0 ? b : 1;
    }
    const uint32_t max_grid = (uint32_t)(num_sms() * g_blocks_per_sm);
    const bool one_sweep = p.total_vec <= max_grid * (uint32_t)(kThreads * 8);
    const uint32_t per_iter = kThreads * (one_sweep ? 8 : 4);
    uint32_t want = (p.total_vec + per_iter - 1) / per_iter;  // one sweep per thread if possible
    uint32_t grid = want < 1 ? 1 : (want > max_grid ? max_grid : want);
    static const uint32_t grid_env = [] { const char* e = getenv("FT2_BOUNDS_CTAS"); return e ? (uint32_t)atoi(e) : 0u; }();
    if (grid_env > 0 && grid_env < grid) grid = grid_env;   // experiment: fewer, longer CTAs
    p.chunk = (p.total_vec + grid - 1) / grid;
    grid = (p.total_vec + p.chunk - 1) / p.chunk;
    if (grid < 1) grid = 1;
    void (*kern)(BoundsK);
    const bool fp16 = a.dtype == FT2_FP16, nv = a.nv_out != nullptr;
    if (one_sweep)
        kern = nv ? (fp16 ? bounds_kernel<1, true, 8> : bounds_kernel<0, true, 8>)
                  : (fp16 ? bounds_kernel<1, false, 8> : bounds_kernel<0, false, 8>);
    else
        kern = nv ? (fp16 ? bounds_kernel<1, true, 4> : bounds_kernel<0, true, 4>)
                  : (fp16 ? bounds_kernel<1, false, 4> : bounds_kernel<0, false, 4>);
    kern<<<grid, kThreads, 0, st>>>(p);
    ++*n_launch;
    return cudaGetLastError();
}

cudaError_t launch_finalize(const int32_t* keys, int32_t S, float scale, uint16_t* out, int dtype, cudaStream_t st,
                            int* n_launch) {
    if (dtype == FT2_FP16) finalize_kernel<1><<<(S + 127) / 128, 128, 0, st>>>(keys, S, scale, out);
    else finalize_kernel<0><<<(S + 127) / 128, 128, 0, st>>>(keys, S, scale, out);
    ++*n_launch;
    return cudaGetLastError();
}

}  // namespace ft2impl
