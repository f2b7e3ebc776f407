// protect.cu -- online range restriction (check-and-clip) of one protected
// layer's output, in place (readings A5-A7).
//
// Read-mostly HBM sweep: each thread loads 4 x 16 B (8 bf16 each), maps them
// to order keys and clamps in key space with VIMNMX.U16x2; a vector is written
// back only when some element changed.  NaN keys fall outside every finite
// bound, so the fast path detects them as "changed" for free; the exact slow
// path (NaN -> key(+0), then clamp) and the corrected-neuron count run only on
// vectors that contain a correction.  torch.clamp would write every element;
// this kernel moves 2 B/element plus 16 B per corrected vector.
#include <cuda_runtime.h>

#include "ft2_device.cuh"
#include "ft2_internal.h"

namespace ft2impl {
using namespace ft2dev;

constexpr int kPThreads = 256;
constexpr int kPUnroll = 4;

struct ProtectK {
    uint16_t* y;
    int64_t ld;
    uint32_t n8, total_vec;
    FastDiv div_n8;
    int contiguous;
    const int32_t* row_to_seq;
    int32_t S;
    int32_t row_mode;  // 0: row_to_seq[], 1: row r -> seq r, 2: all rows -> seq 0
    const uint16_t* bounds;
    uint32_t* counts;
};

__device__ __forceinline__ uint4* pvec(const ProtectK& p, uint32_t v, uint32_t& row) {
    row = fdiv(v, p.div_n8);
    if (p.contiguous) return reinterpret_cast<uint4*>(p.y) + v;
    uint32_t col = v - row * p.n8;
    return reinterpret_cast<uint4*>(p.y + (int64_t)row * p.ld) + col;
}

__device__ __forceinline__ int seq_for_row(const ProtectK& p, uint32_t row) {
    if (p.row_mode == 2) return 0;
    if (p.row_mode == 1) return (int)row;
    return p.row_to_seq[row];
}

__device__ __forceinline__ void load_bounds2(const ProtectK& p, int s, uint32_t& kL2, uint32_t& kH2) {
    uint32_t lh = *reinterpret_cast<const uint32_t*>(p.bounds + 2 * s);  // (lo, hi) as one word
    uint32_t k = key2(lh);
    uint32_t kl = k & 0xFFFFu, kh = k >> 16;
    kL2 = kl | (kl << 16);
    kH2 = kh | (kh << 16);
}

template <int DT>
__global__ void __launch_bounds__(kPThreads) protect_kernel(ProtectK p) {
    uint32_t kL2 = 0, kH2 = 0;
    if (p.row_mode == 2) load_bounds2(p, 0, kL2, kH2);
    const uint32_t stride = gridDim.x * kPThreads * kPUnroll;
    for (uint32_t base = blockIdx.x * kPThreads * kPUnroll + threadIdx.x; base < p.total_vec; base += stride) {
        uint4 d[kPUnroll];
        uint4* q[kPUnroll];
        uint32_t row[kPUnroll];
#pragma unroll
        for (int u = 0; u < kPUnroll; ++u) {
            uint32_t vi = base + u * kPThreads;
            q[u] = pvec(p, vi < p.total_vec ? vi : 0, row[u]);
            if (vi < p.total_vec) d[u] = ld_stream(q[u]);
        }
#pragma unroll
        for (int u = 0; u < kPUnroll; ++u) {
            uint32_t vi = base + u * kPThreads;
            if (vi >= p.total_vec) continue;
            int s = 0;
            if (p.row_mode != 2) {
                s = seq_for_row(p, row[u]);
                if (s < 0 || s >= p.S) continue;
                load_bounds2(p, s, kL2, kH2);
            }
            uint32_t w[4] = {d[u].x, d[u].y, d[u].z, d[u].w};
            uint32_t diff = 0;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
                uint32_t k = key2(w[j]);
                diff |= vmax_u16x2(vmin_u16x2(k, kH2), kL2) ^ k;
            }
            if (diff) {  // rare: exact correction of this vector
                uint32_t cnt = 0, c;
#pragma unroll
                for (int j = 0; j < 4; ++j) { w[j] = clip2<DT>(w[j], kL2, kH2, &c); cnt += c; }
                *q[u] = make_uint4(w[0], w[1], w[2], w[3]);
                if (p.counts) atomicAdd(&p.counts[s], cnt);
            }
        }
    }
}

static int g_pblocks_per_sm = 0;

cudaError_t launch_protect(const ProtectArgs& a, cudaStream_t st, int* n_launch) {
    ProtectK p;
    p.y = a.y;
    p.ld = a.ld;
    p.n8 = (uint32_t)(a.n / 8);
    p.total_vec = (uint32_t)(a.rows * (a.n / 8));
    p.div_n8 = make_fastdiv(p.n8);
    p.contiguous = (a.ld == a.n);
    p.row_to_seq = a.row_to_seq;
    p.S = a.S;
    p.row_mode = a.row_to_seq ? 0 : (a.S == 1 ? 2 : 1);
    p.bounds = a.bounds;
    p.counts = a.counts;
    if (g_pblocks_per_sm == 0) {
        int b = 0;
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&b, protect_kernel<0>, kPThreads, 0);
        if (e != cudaSuccess) return e;
        g_pblocks_per_sm = b > 0 ? b : 1;
    }
    const uint32_t per_cta = kPThreads * kPUnroll;
    uint32_t want = (p.total_vec + per_cta - 1) / per_cta;
    uint32_t max_grid = (uint32_t)(num_sms() * g_pblocks_per_sm);
    uint32_t grid = want > max_grid ? max_grid : (want < 1 ? 1 : want);
    if (a.dtype == FT2_FP16) protect_kernel<1><<<grid, kPThreads, 0, st>>>(p);
    else protect_kernel<0><<<grid, kPThreads, 0, st>>>(p);
    ++*n_launch;
    return cudaGetLastError();
}

}  // namespace ft2impl
