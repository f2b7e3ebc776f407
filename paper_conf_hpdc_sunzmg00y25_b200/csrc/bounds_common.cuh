// bounds_common.cuh -- pieces of the first-token bound reduction (PAPER.md
// L150, L221-L241) shared by the standalone sweep (bounds.cu) and the prefill
// GEMM with the reduction fused into its epilogue (gemm_prefill_sm100.cu):
// the workspace protocol (ft2_internal.h), the row -> sequence search, the
// non-finite patch list, and the last-CTA finalisation (R3 scaling, keys,
// counts, R4 correction of the recorded non-finite elements, workspace reset).
#pragma once
#include "ft2_device.cuh"
#include "ft2_internal.h"

namespace ft2impl {
using namespace ft2dev;

struct BoundsK {
    uint16_t* y;
    int64_t ld;
    uint32_t n8;          // vectors per row
    uint32_t total_vec;   // rows * n8
    uint32_t chunk;       // vectors per CTA
    FastDiv div_n8;
    int contiguous;       // ld == n
    const int32_t* seq_offsets;
    int32_t S;
    float scale;
    int32_t finalize, correct;
    uint16_t* bounds_out;
    int32_t* keys_out;
    uint32_t* nonfinite_out;
    uint32_t* nv_out;     // NaN-vulnerable counts or NULL
    uint32_t* ws;
};

__device__ __forceinline__ const uint4* vec_ptr(const BoundsK& p, uint32_t v) {
    if (p.contiguous) return reinterpret_cast<const uint4*>(p.y) + v;
    uint32_t row = fdiv(v, p.div_n8);
    uint32_t col = v - row * p.n8;
    return reinterpret_cast<const uint4*>(p.y + (int64_t)row * p.ld) + col;
}

// largest s in [0, S] with so[s] <= row  (so non-decreasing); -1 if row < so[0]
__device__ __forceinline__ int seq_of_row(const int32_t* so, int S, uint32_t row) {
    if ((int64_t)row < (int64_t)so[0]) return -1;
    int lo = 0, hi = S;  // invariant so[lo] <= row
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if ((int64_t)so[mid] <= (int64_t)row) lo = mid; else hi = mid - 1;
    }
    return lo;
}

__device__ __forceinline__ void record_patch(const BoundsK& p, uint32_t* list_count, uint32_t* overflow,
                                             unsigned long long* list, int s, uint64_t off) {
    uint32_t i = atomicAdd(list_count, 1u);
    if (i < (uint32_t)kPatchCap) list[i] = (unsigned long long)(off | ((uint64_t)s << 48));
    else atomicExch(overflow, 1u);
}

// Last-CTA finalisation, run by all `nthreads` threads of the CTA that saw the
// completion counter reach the grid size (after its acquire).  Every slot is
// read with independent L2 loads; the workspace is left zeroed.
template <int DT, bool NV>
__device__ __forceinline__ void bounds_finalize_tail(const BoundsK& p, int tid, int nthreads) {
    const int S = p.S;
    uint32_t* ws_done = p.ws + 4 * S;
    uint32_t* ws_lc = p.ws + 4 * S + 1;
    uint32_t* ws_ov = p.ws + 4 * S + 2;
    unsigned long long* list = reinterpret_cast<unsigned long long*>(
        reinterpret_cast<char*>(p.ws) + (((size_t)(4 * S + 4) * 4 + 7) & ~(size_t)7));
    const uint32_t lc0 = p.correct ? __ldcg(ws_lc) : 0u, ov0 = p.correct ? __ldcg(ws_ov) : 0u;
    for (int s = tid; s < S; s += nthreads) {
        // lo, hi, non-finite, NaN-vulnerable slots (the workspace is 8-byte aligned)
        const uint2 wa = __ldcg(reinterpret_cast<const uint2*>(p.ws + 4 * s));
        const uint2 wb = __ldcg(reinterpret_cast<const uint2*>(p.ws + 4 * s + 2));
        const uint32_t los = wa.x, his = wa.y, nfc = wb.x;
        bool have = los != 0u && his != 0u;
        uint32_t kmin = 0x10000u - los, kmax = his - 1u;
        if (p.finalize) {
            uint16_t lo = 0, hi = 0;  // reading A9
            if (have) {
                lo = scale_bound<DT>(unkey1((uint16_t)kmin), p.scale, false);
                hi = scale_bound<DT>(unkey1((uint16_t)kmax), p.scale, true);
            }
            p.bounds_out[2 * s] = lo;
            p.bounds_out[2 * s + 1] = hi;
        }
        if (p.keys_out) {
            p.keys_out[2 * s] = have ? (int32_t)(0xFFFFu - kmin) : -1;
            p.keys_out[2 * s + 1] = have ? (int32_t)kmax : -1;
        }
        if (p.nonfinite_out) p.nonfinite_out[s] = nfc;
        if (NV) p.nv_out[s] = wb.y;
        *reinterpret_cast<uint2*>(p.ws + 4 * s) = make_uint2(0u, 0u);
        *reinterpret_cast<uint2*>(p.ws + 4 * s + 2) = make_uint2(0u, 0u);
    }
    __syncthreads();  // bounds_out of every sequence written (read back by the patch fix-up)
    if (p.correct && lc0 != 0u) {
        if (!ov0) {
            for (uint32_t i = tid; i < lc0; i += nthreads) {
                unsigned long long e = __ldcg(list + i);
                int s = (int)(e >> 48);
                uint64_t off = e & 0xFFFFFFFFFFFFull;
                uint16_t b = p.y[off];
                uint16_t lo = p.bounds_out[2 * s], hi = p.bounds_out[2 * s + 1];
                // R5 on a non-finite value: NaN -> clamp(+0), +Inf -> hi, -Inf -> lo
                uint16_t x = isnan1<DT>(b) ? (uint16_t)0 : b;
                uint16_t k = key1(x);
                p.y[off] = k < key1(lo) ? lo : (k > key1(hi) ? hi : x);
            }
        } else {
            // more non-finite values than the patch list holds: this CTA sweeps
            // the whole tensor (only reachable with pathological inputs)
            for (uint32_t vi = tid; vi < p.total_vec; vi += nthreads) {
                uint32_t row = fdiv(vi, p.div_n8);
                int s = 0;
                if (p.seq_offsets) {
                    s = seq_of_row(p.seq_offsets, S, row);
                    if (s < 0 || s >= S) continue;
                }
                uint16_t* q = const_cast<uint16_t*>(reinterpret_cast<const uint16_t*>(vec_ptr(p, vi)));
                uint16_t lo = p.bounds_out[2 * s], hi = p.bounds_out[2 * s + 1];
                for (int j = 0; j < 8; ++j) {
                    uint16_t b = q[j];
                    if (!nonfinite1<DT>(b)) continue;
                    uint16_t x = isnan1<DT>(b) ? (uint16_t)0 : b;
                    uint16_t k = key1(x);
                    q[j] = k < key1(lo) ? lo : (k > key1(hi) ? hi : x);
                }
            }
        }
        __syncthreads();  // leave the patch list zero-filled as well
        const uint32_t used = min(lc0, (uint32_t)kPatchCap);
        for (uint32_t i = tid; i < used; i += nthreads) list[i] = 0ull;
    }
    if (tid == 0) {
        *ws_lc = 0u;
        *ws_ov = 0u;
        *ws_done = 0u;
    }
}

}  // namespace ft2impl
