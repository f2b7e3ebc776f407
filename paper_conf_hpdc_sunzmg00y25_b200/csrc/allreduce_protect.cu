// allreduce_protect.cu -- a tensor-parallel row-parallel critical layer's sum
// all-reduce fused with FT2's check (reading A17:
// row-parallel outputs are checked after their sum all-reduce).
//
// Each of the P ranks holds a partial output [rows x n] of the layer (its
// K-slice of the GEMM, 16-bit, no bias) in a buffer every peer can address
// (CUDA IPC mappings over NVLink/NVSwitch; ft2_ipc_*).  One kernel per rank:
//
//   1. signal: CTA 0 publishes this call's epoch into every peer's flag slot
//      for this rank (fence.sc.sys, then st.release.sys);
//   2. wait: every CTA polls its own P flag slots (ld.acquire.sys) until all
//      ranks reached the epoch -- every partial of this call is complete;
//   3. one-shot reduce of this CTA's contiguous chunk of 16-byte vectors:
//      the P partials are summed in fp32 in rank order 0..P-1 (identical
//      arithmetic on every rank, so every rank ends with the same bits),
//      + bias, rounded to the 16-bit format (RNE), fault XOR, key-space
//      check-and-clip (readings A5-A7, A19, A20),
//      stored to this rank's own output;
//   4. the last CTA bumps the rank's epoch counter (device memory, so the
//      kernel is CUDA-graph replayable).
// P = 1 needs none of 1, 2 and 4 (stream order covers the own partial): the
// kernel is then a plain elementwise pass.  The P partial vectors of an
// output vector are all loaded before the fp32 sum (P NVLink round trips in
// flight at once, not one after another), and a thread owns up to kVecs
// output vectors.
//
// The partial buffers must be double-buffered by the caller (alternate per
// call): a rank reaches call e+1's signal only after its call e finished
// reading, so a buffer written at call e+2 is never read by a late peer.
// Polling is bounded: after 2^24 polls (seconds) the kernel records FT2 status 1 in
// `status` and returns (a dead peer cannot hang the GPU).
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "ft2_device.cuh"
#include "ft2_internal.h"
#include "sm100_ptx.cuh"

namespace ft2impl {
using namespace ft2dev;

namespace {

constexpr int kARThreads = 256;
constexpr int kARSites = 64;
constexpr int kARMaxP = 8;   // ranks whose partials one thread holds in registers at once
constexpr int kVecs = 2;     // output vectors per thread per pass

__device__ __forceinline__ void st_release_sys(uint32_t* p, uint32_t v) {
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
// peer data written during this kernel's lifetime, read after the acquire
// handshake: L2-level loads (never L1, never the non-coherent path)
__device__ __forceinline__ uint4 ld_peer_v4(const void* p) {
    uint4 r;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p) : "memory");
    return r;
}

// w[d / 2] ^= the 16-bit mask in half d % 2 -- by static indices, so w stays
// in registers (a dynamic w[d >> 1] would move it to local memory)
__device__ __forceinline__ void xor_word(uint32_t (&w)[4], uint32_t d, uint32_t mask) {
    const uint32_t m = (mask & 0xFFFFu) << ((d & 1u) * 16), q = d >> 1;
    w[0] ^= q == 0u ? m : 0u;   // branch-free selects (an if would be folded back into w[q])
    w[1] ^= q == 1u ? m : 0u;
    w[2] ^= q == 2u ? m : 0u;
    w[3] ^= q == 3u ? m : 0u;
}

template <int DT>
__device__ __forceinline__ void add8(float (&acc)[8], uint4 v, bool first) {
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int j = 0; j < 8; ++j) {
        const float f = to_f32<DT>((uint16_t)(w[j >> 1] >> ((j & 1) * 16)));
        acc[j] = first ? f : __fadd_rn(acc[j], f);
    }
}

// PB: partials held in registers per output vector (P <= PB, or PB = 8 and the
// ranks beyond 8 are streamed) -- a compile-time bound keeps small P lean
template <int DT, int PB>
__global__ void __launch_bounds__(kARThreads) allreduce_protect_kernel(const AllreduceProtectArgs p, uint32_t chunk,
                                                                       uint32_t n8, uint32_t total_vec, FastDiv div_n8,
                                                                       int row_mode) {
    __shared__ uint32_t sh_e, sh_ok, sh_last, sh_ns;
    __shared__ uint32_t sh_site_e[kARSites], sh_site_m[kARSites];
    const int tid = threadIdx.x;
    const uint32_t v0 = blockIdx.x * chunk, v1 = min(v0 + chunk, total_vec);
    // P = 1 without sites: no handshake, no site list -- straight to the loads
    // (the shared words are only touched on the prologue path)
    const bool prologue = p.P > 1 || p.sites != nullptr;
    // programmatic dependent launch: the grid launches while the producer of
    // the partials (or the previous layer) drains; everything below -- the
    // epoch, the partials, bias, bounds, sites -- may belong to it.  The next
    // kernel may start its own prologue right away (it waits likewise).
    griddep_wait();
    griddep_launch();
    uint32_t e = 0u;
    if (prologue) {
        if (tid == 0) {
            sh_e = p.P > 1 ? *reinterpret_cast<volatile uint32_t*>(p.epoch) + 1u : 0u;
            sh_ok = 1u;
            sh_ns = 0u;
        }
        __syncthreads();
        e = sh_e;
    }
    // ---- 1. signal: my partial (written by the preceding kernel) is ready.
    // P = 1 needs no handshake: stream order already covers my own partial.
    if (p.P > 1 && blockIdx.x == 0 && tid < p.P) {
        __threadfence_system();
        st_release_sys(p.flags[tid] + p.rank, e);
    }
    // ---- 2. wait for every rank's partial of this call
    if (p.P > 1 && tid < p.P) {
        const uint32_t* f = p.flags[p.rank] + tid;
        uint32_t polls = 0;
        while ((int32_t)(ld_acquire_sys(f) - e) < 0) {
            if (++polls > (1u << 24)) { atomicExch(p.status, 1u); sh_ok = 0u; break; }
        }
    }
    // fault sites landing in this CTA's chunk (rare; campaign runs only)
    if (p.sites != nullptr) {
        for (int i = tid; i < p.n_sites; i += kARThreads) {
            const ft2_fault_site s = p.sites[i];
            if ((int)s.step != p.cur_step || (int)s.layer != p.cur_layer) continue;
            const int64_t row = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) +
                                (p.cur_step == 0 ? (int64_t)s.token : 0);
            if (row < 0 || row >= p.rows || (int64_t)s.col >= p.n) continue;
            const uint64_t el = (uint64_t)row * (uint64_t)p.n + s.col;
            const uint64_t vv = el >> 3;
            if (vv < v0 || vv >= v1) continue;
            const uint32_t k = atomicAdd(&sh_ns, 1u);
            if (k < (uint32_t)kARSites) { sh_site_e[k] = (uint32_t)(el - (uint64_t)v0 * 8u); sh_site_m[k] = s.xor_mask; }
        }
    }
    bool ok = true;
    uint32_t nsite = 0u;   // > kARSites: every site is rescanned per vector (none dropped)
    if (prologue) {
        __syncthreads();
        ok = sh_ok != 0u;
        nsite = sh_ns;
    }
    if (ok) {
        const int32_t P = p.P;
        for (uint32_t vb = v0 + tid; vb < v1; vb += kARThreads * kVecs) {
            // every load of this pass is issued before any arithmetic: the
            // read-only operands (bias, the row's bounds word) first, then
            // kVecs vectors x min(P, 8) partials (the peer loads carry a memory
            // clobber, so plain loads placed before them stay before them)
            uint4 part[kVecs][PB], bv[kVecs];
            uint32_t vrow[kVecs], vc8[kVecs], bw[kVecs];
            int vs[kVecs];
#pragma unroll
            for (int q = 0; q < kVecs; ++q) {
                const uint32_t v = vb + q * kARThreads;
                const uint32_t vv = v < v1 ? v : v0;
                vrow[q] = fdiv(vv, div_n8);
                vc8[q] = vv - vrow[q] * n8;
                bv[q] = p.bias ? __ldg(reinterpret_cast<const uint4*>(p.bias + vc8[q] * 8)) : make_uint4(0, 0, 0, 0);
                vs[q] = -1;
                bw[q] = 0u;
                if (p.mode == FT2_GEMM_CHECK) {
                    const int s = row_mode == 2 ? 0 : (row_mode == 1 ? (int)vrow[q] : __ldg(p.row_to_seq + vrow[q]));
                    if (s >= 0 && s < p.S) {
                        vs[q] = s;
                        bw[q] = __ldg(reinterpret_cast<const uint32_t*>(p.bounds + 2 * s));
                    }
                }
            }
#pragma unroll
            for (int q = 0; q < kVecs; ++q) {
                const uint32_t v = vb + q * kARThreads;
#pragma unroll
                for (int t = 0; t < PB; ++t)
                    if (t < P && v < v1)
                        part[q][t] = ld_peer_v4(p.partials[t] + (int64_t)vrow[q] * p.ldp + vc8[q] * 8);
            }
#pragma unroll
            for (int q = 0; q < kVecs; ++q) {
                const uint32_t v = vb + q * kARThreads;
                if (v >= v1) break;
                const uint32_t row = vrow[q], c8 = vc8[q];
                float acc[8];
#pragma unroll
                for (int t = 0; t < PB; ++t)
                    if (t < P) add8<DT>(acc, part[q][t], t == 0);
                for (int t = PB; t < P; ++t)   // rank order continues beyond PB ranks
                    add8<DT>(acc, ld_peer_v4(p.partials[t] + (int64_t)row * p.ldp + c8 * 8), false);
                if (p.bias) {
                    const uint32_t bb[4] = {bv[q].x, bv[q].y, bv[q].z, bv[q].w};
#pragma unroll
                    for (int j = 0; j < 8; ++j)
                        acc[j] = __fadd_rn(acc[j], to_f32<DT>((uint16_t)(bb[j >> 1] >> ((j & 1) * 16))));
                }
                uint32_t w[4];
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    w[j] = (uint32_t)rne16<DT>(acc[2 * j]) | ((uint32_t)rne16<DT>(acc[2 * j + 1]) << 16);
                for (uint32_t i = 0; i < (nsite > (uint32_t)kARSites ? 0u : nsite); ++i) {
                    const uint32_t d = sh_site_e[i] - (v - v0) * 8u;
                    if (d < 8u) xor_word(w, d, sh_site_m[i]);
                }
                if (nsite > (uint32_t)kARSites) {   // rare overflow path: scan every site
                    for (int i = 0; i < p.n_sites; ++i) {
                        const ft2_fault_site st = p.sites[i];
                        if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
                        const int64_t r = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) +
                                          (p.cur_step == 0 ? (int64_t)st.token : 0);
                        if (r != (int64_t)row || (int64_t)st.col >= p.n) continue;
                        const uint32_t d = (uint32_t)((int64_t)st.col - (int64_t)c8 * 8);
                        if (d < 8u) xor_word(w, d, st.xor_mask);
                    }
                }
                if (vs[q] >= 0) {
                    const uint32_t k = key2(bw[q]);
                    const uint32_t kL2 = (k & 0xFFFFu) * 0x10001u, kH2 = (k >> 16) * 0x10001u;
                    uint32_t cnt = 0, c;
#pragma unroll
                    for (int j = 0; j < 4; ++j) { w[j] = clip2<DT>(w[j], kL2, kH2, &c); cnt += c; }
                    if (cnt && p.counts) atomicAdd(&p.counts[vs[q]], cnt);
                }
                uint16_t* const dst = p.y + (int64_t)row * p.ldy + c8 * 8;
                // P = 1 in place (y aliases the partial): like ft2_protect, a
                // vector is written back only when the check changed it
                if (P == 1 && dst == p.partials[0] + (int64_t)row * p.ldp + c8 * 8 && w[0] == part[q][0].x &&
                    w[1] == part[q][0].y && w[2] == part[q][0].z && w[3] == part[q][0].w)
                    continue;
                *reinterpret_cast<uint4*>(dst) = make_uint4(w[0], w[1], w[2], w[3]);
            }
        }
    }
    // ---- 4. last CTA: this rank's call is complete; advance the epoch.
    // P = 1: nobody reads the epoch within a call, so CTA 0 advances it
    // without the completion counter (it stays the call counter)
    if (p.P == 1) {
        if (blockIdx.x == 0 && tid == 0) atomicAdd(p.epoch, 1u);   // fire-and-forget (RED), no round trip
        return;
    }
    __syncthreads();
    if (tid == 0) sh_last = atom_add_acq_rel_gpu(p.done, 1u) == gridDim.x - 1;
    __syncthreads();
    if (sh_last && tid == 0) {
        *p.done = 0u;
        *reinterpret_cast<volatile uint32_t*>(p.epoch) = e;
    }
}

}  // namespace

cudaError_t launch_allreduce_protect(const AllreduceProtectArgs& a, cudaStream_t st, int* n_launch) {
    const uint32_t n8 = (uint32_t)(a.n / 8), total = (uint32_t)(a.rows * (a.n / 8));
    // one vector per thread (kVecs per pass once the grid is capped); at most
    // 2 CTAs per SM (every CTA polls)
    uint32_t grid = (total + kARThreads - 1) / kARThreads;
    const uint32_t cap = (uint32_t)(2 * num_sms());
    grid = grid < 1 ? 1 : (grid > cap ? cap : grid);
    uint32_t chunk = (total + grid - 1) / grid;
    grid = (total + chunk - 1) / chunk;
    const int row_mode = a.row_to_seq ? 0 : (a.S == 1 ? 2 : 1);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kARThreads);
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    static const int pdl = [] { const char* v = getenv("FT2_AR_PDL"); return v ? atoi(v) : 1; }();
    attr[0].val.programmaticStreamSerializationAllowed = pdl;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const FastDiv dv = make_fastdiv(n8);
    cudaError_t e;
#define FT2_AR_LAUNCH(DT_, PB_) cudaLaunchKernelEx(&cfg, allreduce_protect_kernel<DT_, PB_>, a, chunk, n8, total, dv, row_mode)
    if (a.dtype == FT2_FP16)
        e = a.P == 1 ? FT2_AR_LAUNCH(1, 1) : a.P == 2 ? FT2_AR_LAUNCH(1, 2) : a.P <= 4 ? FT2_AR_LAUNCH(1, 4) : FT2_AR_LAUNCH(1, kARMaxP);
    else
        e = a.P == 1 ? FT2_AR_LAUNCH(0, 1) : a.P == 2 ? FT2_AR_LAUNCH(0, 2) : a.P <= 4 ? FT2_AR_LAUNCH(0, 4) : FT2_AR_LAUNCH(0, kARMaxP);
#undef FT2_AR_LAUNCH
    if (e != cudaSuccess) return e;
    ++*n_launch;
    return cudaGetLastError();
}

}  // namespace ft2impl
