// gemm_prefill_sm100.cu -- a critical linear layer at prefill shapes (M = sum
// of prompt lengths > 128 tokens) with FT2's first-token work fused into the
// epilogue, for sm_100a.
//
//   PLAIN   y = inject(bf16_rne(x W^T + b))
//   CHECK   ... then check-and-clip against the row's sequence bounds (R5)
//   DERIVE  ... then the first-token bounds of y: per sequence the min/max
//           order key over the finite outputs (R2), combined across tiles and
//           CTAs, widened x scale by the last CTA (R3), which also corrects the
//           recorded non-finite outputs (R4) -- ft2_bounds_from_prefill on the
//           layer output without reading it back from HBM.
// PAPER.md L150 (bounds from the first token), L221-L233 (min/max, scaling
// factor 2), L225/L237/L241 (NaN in the first token is detected and
// corrected), L259/L272 (check after the critical layer).  Order of the
// epilogue: GEMM -> +bias -> bf16 -> inject -> check / derive (A19, A20).
//
// Persistent, warp-specialised, one CTA per SM (320 threads), normally as a
// CTA pair (cluster of 2, tcgen05.mma.cta_group::2) computing 256 x 256 tiles:
//   warp 0      TMA producer: this CTA's 128 rows of the x box and 128 rows of
//               the W box (128B swizzle) into a 6-stage ring of 32 KB stages;
//               completion is counted on the leader CTA's barrier.
//   warp 1      TMEM allocator (512 columns = two 128x256 fp32 accumulators per
//               CTA); in the leader, the single-thread MMA issuer (M=256 over
//               the pair, N=256, K=16), whose commits are multicast to both CTAs.
//   warps 2-9   epilogue: two warps per TMEM lane quarter (one per 128-column
//               half), tcgen05.ld 32 columns at a time (one TMEM lane = one
//               output row per thread), while the MMA fills the other
//               accumulator with the next tile (TMEM double buffering).
// The pair halves each SM's shared-memory operand traffic (the weight box is
// staged once per 256 rows of x), which the single-CTA 128x256 variant (used
// when there is only one 128-row m-tile) cannot sustain at the MMA rate.
// Tiles are handed out round-robin (tile = cluster + i * clusters).
// DERIVE keeps a per-CTA table of the sequences' key extrema in shared memory
// (warp-reduced when a warp's 32 rows belong to one sequence) and flushes it
// once; the bounds workspace protocol is the one of ft2_bounds_from_prefill
// (bounds_common.cuh), so both produce bit-identical bounds.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdlib.h>

#include "bounds_common.cuh"
#include "ft2_device.cuh"
#include "ft2_internal.h"
#include "sm100_ptx.cuh"

namespace ft2impl {
using namespace ft2dev;

constexpr int kPBM = 128, kPBN = 256, kPBK = 64;
constexpr int kPEpiWarps = 8;                      // two per TMEM lane quarter, one per 128-column half
constexpr int kPThreads = 64 + 32 * kPEpiWarps;    // + producer warp + MMA warp
constexpr int kPABytes = kPBM * kPBK * 2;  // 16 KB: one CTA's 128 rows of x
constexpr int kPTileBytes = 192 * 1024;    // the shared-memory ring
// MC = 1: a CTA loads the whole 256-row weight box (48 KB stages, 4 deep);
// MC = 2: CTA pair, each CTA loads 128 weight rows (32 KB stages, 6 deep)
template <int MC>
struct PCfg {
    static constexpr int kBBytes = kPBN / MC * kPBK * 2;
    static constexpr int kStageBytes = kPABytes + kBBytes;
    static constexpr int kStages = kPTileBytes / kStageBytes;
};
constexpr int kPSeqTab = 512;                        // sequences kept in the per-CTA table
constexpr int kPMaxRowSites = 4;                     // fault sites one row may hold per tile
constexpr int kPMiscBytes = 256;
// split-K staging: per epilogue column half, 128 rows x 16 fp32 (+4 pad: the
// per-row float4 writes of a quarter-warp hit disjoint banks)
constexpr int kSkStride = 20;
constexpr int kSkStageBytes = 2 * kPBM * kSkStride * 4;
constexpr int kPSmemBytes = 1024 + kPTileBytes + kPMiscBytes + 3 * kPSeqTab * 4 + kSkStageBytes;
constexpr int kPGemmDerive = 2;
constexpr int kSplitCounters = 16384;   // split-K arrival counters at the head of the GEMM workspace

struct PrefK {
    int32_t M, N, K, tilesM, ntiles, nkb;
    // split-K for grids the tiles alone cannot fill (small M): `splits` units
    // per tile, all in one wave, fp32 partial slots [half-tile][split][128][256]
    // in skws, two counters per 128 x 256 half-tile in skcnt (partials
    // written / partials read; self-cleaning).  Every split finishes 1/splits
    // of its half-tile's 32-column groups from all the partials.
    int32_t splits;
    float* skws;
    uint32_t* skcnt;
    int32_t mode, col_begin, col_end;
    const uint16_t* bias;
    uint16_t* y;
    int64_t ldy;
    // CHECK: row -> sequence as in ft2_protect
    const int32_t* row_to_seq;
    int32_t S, row_mode;
    const uint16_t* bounds;
    uint32_t* counts;
    // DERIVE: the ft2_bounds_from_prefill arguments (finalize = 1)
    BoundsK bp;
    // faults
    const ft2_fault_site* sites;
    int32_t n_sites, cur_layer, cur_step;
    const int32_t* base_row;
};

__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
constexpr int kMaxSplits = 4;   // K splits the planner picks (partials of all splits held in registers)

__device__ __forceinline__ uint32_t pack_rne2(float a, float b, int dt) {
    return dt == 1 ? ((uint32_t)rne16<1>(a) | ((uint32_t)rne16<1>(b) << 16))
                   : ((uint32_t)rne16<0>(a) | ((uint32_t)rne16<0>(b) << 16));
}

// Tile of the CTA at step i of the persistent loop.  MC == 2: a cluster of two
// CTAs (an SM pair) computes a 256 x 256 tile with tcgen05.mma.cta_group::2:
// CTA r holds rows [128 r, 128 r + 128) of the x box and of the weight box,
// the leader (rank 0) issues the MMA over both, and each CTA's TMEM receives
// its own 128 output rows x 256 columns -- the weight box is read from L2 and
// staged in shared memory once per pair.
template <int MC>
__device__ __forceinline__ bool tile_of(const PrefK& p, int i, int& m0, int& n0, int& ks) {
    // work units (tile, K split), split-major: a tile's splits land on
    // different CTAs (clusters) of the same wave
    if (MC == 1) {
        const int u = blockIdx.x + i * gridDim.x;
        if (u >= p.ntiles * p.splits) return false;
        const int t = u % p.ntiles;
        ks = u / p.ntiles;
        m0 = (t % p.tilesM) * kPBM;
        n0 = (t / p.tilesM) * kPBN;
        return true;
    }
    const int pairsM = (p.tilesM + 1) >> 1;
    const int npairs = pairsM * (p.ntiles / p.tilesM);
    const int u = (int)(blockIdx.x >> 1) + i * (int)(gridDim.x >> 1);
    if (u >= npairs * p.splits) return false;
    const int pr = u % npairs;
    ks = u / npairs;
    m0 = ((pr % pairsM) * 2 + (int)(blockIdx.x & 1)) * kPBM;
    n0 = (pr / pairsM) * kPBN;
    return true;
}

template <int DT, int MC>
__global__ void __launch_bounds__(kPThreads, 1)
    prefill_gemm_kernel(const __grid_constant__ CUtensorMap map_x, const __grid_constant__ CUtensorMap map_w,
                        const __grid_constant__ PrefK p) {
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t* tiles = smem;
    uint8_t* misc = smem + kPTileBytes;
    constexpr int kPStages = PCfg<MC>::kStages, kPStageBytes = PCfg<MC>::kStageBytes;
    uint64_t* full = reinterpret_cast<uint64_t*>(misc);
    uint64_t* empty = full + kPStages;
    uint64_t* tmem_full = empty + kPStages;  // [2]
    uint64_t* tmem_empty = tmem_full + 2;    // [2]
    uint32_t* tmem_base_sh = reinterpret_cast<uint32_t*>(tmem_empty + 2);
    uint32_t* last_sh = tmem_base_sh + 1;
    uint32_t* tab_lo = reinterpret_cast<uint32_t*>(misc + kPMiscBytes);  // 0x10000 - min key (0: none)
    uint32_t* tab_hi = tab_lo + kPSeqTab;                                 // max key + 1 (0: none)
    uint32_t* tab_nf = tab_hi + kPSeqTab;                                 // non-finite count
    float* sk_stage = reinterpret_cast<float*>(tab_nf + kPSeqTab);        // [2][128][kSkStride] (split-K)

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const bool derive = p.mode == kPGemmDerive;
    const bool use_tab = derive && p.bp.S <= kPSeqTab;
    if (warp == 0 && lane == 0) {
        prefetch_tmap(&map_x);
        prefetch_tmap(&map_w);
        // MC = 2: the leader's full[] counts both CTAs' bytes, its tmem_empty[]
        // both CTAs' epilogue warps; empty[] / tmem_full[] are signalled in
        // both CTAs by the leader's multicast commits
        for (int s = 0; s < kPStages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        for (int b = 0; b < 2; ++b) { mbar_init(&tmem_full[b], 1); mbar_init(&tmem_empty[b], kPEpiWarps * MC); }
        fence_mbar_init();
    }
    if (warp == 1) {
        if (MC == 1) tmem_alloc(tmem_base_sh, 512);
        else tmem_alloc2(tmem_base_sh, 512);
    }
    if (use_tab)
        for (int s = tid; s < p.bp.S; s += kPThreads) { tab_lo[s] = 0u; tab_hi[s] = 0u; tab_nf[s] = 0u; }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (MC > 1) {  // the peer's barriers are initialised before anything signals them
        cluster_arrive_relaxed();
        cluster_wait();
    }
    const uint32_t tmem_base = *tmem_base_sh;
    const uint32_t crank = MC > 1 ? cluster_ctarank() : 0u;
    griddep_launch();

    if (warp == 0) {
        if (lane == 0) {
            // ---------------------------------------------------- TMA producer
            griddep_wait();  // x may be the previous kernel's output
            uint32_t stage = 0, phase = 0;
            int m0, n0, ks;
            for (int i = 0; tile_of<MC>(p, i, m0, n0, ks); ++i) {
                const int kb0 = (int)((int64_t)ks * p.nkb / p.splits), kb1 = (int)((int64_t)(ks + 1) * p.nkb / p.splits);
                for (int kb = kb0; kb < kb1; ++kb) {
                    mbar_wait(&empty[stage], phase ^ 1u);
                    uint8_t* st = tiles + stage * kPStageBytes;
                    if (MC == 1) {
                        mbar_expect_tx(&full[stage], kPStageBytes);
                        tma_load_2d(&map_x, &full[stage], st, kb * kPBK, m0);
                        tma_load_2d(&map_w, &full[stage], st + kPABytes, kb * kPBK, n0);
                    } else {  // my 128 rows of x and of the weight box; the leader's barrier counts both CTAs
                        const uint32_t lbar = mapa(smem_u32(&full[stage]), 0u);
                        if (crank == 0) mbar_expect_tx(&full[stage], 2 * kPStageBytes);
                        tma_load_2d_2sm(&map_x, lbar, st, kb * kPBK, m0);
                        tma_load_2d_2sm(&map_w, lbar, st + kPABytes, kb * kPBK, n0 + (int)crank * (kPBN / 2));
                    }
                    if (++stage == kPStages) { stage = 0; phase ^= 1u; }
                }
            }
            if (MC > 1) {  // drain: every stage's release has arrived before the CTA may exit
                for (int s = 0; s < kPStages; ++s) {
                    mbar_wait(&empty[stage], phase ^ 1u);
                    if (++stage == kPStages) { stage = 0; phase ^= 1u; }
                }
            }
        }
    } else if (warp == 1) {
        if (lane == 0 && crank == 0) {
            // ----------------------------------------- MMA issuer (the pair's leader)
            constexpr uint32_t idesc =
                (make_idesc(kPBM * MC, kPBN) & ~((7u << 7) | (7u << 10))) | ((DT == 1 ? 0u : 1u) * ((1u << 7) | (1u << 10)));
            uint32_t stage = 0, phase = 0;
            int tc = 0, m0, n0, ks;
            for (int i = 0; tile_of<MC>(p, i, m0, n0, ks); ++i, ++tc) {
                const int buf = tc & 1;
                mbar_wait(&tmem_empty[buf], ((uint32_t)(tc >> 1) & 1u) ^ 1u);  // the epilogue drained it
                tc_fence_after();
                const uint32_t d = tmem_base + (uint32_t)(buf * kPBN);
                const int kb0 = (int)((int64_t)ks * p.nkb / p.splits), kb1 = (int)((int64_t)(ks + 1) * p.nkb / p.splits);
                for (int kb = kb0; kb < kb1; ++kb) {
                    mbar_wait(&full[stage], phase);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(tiles + stage * kPStageBytes);
                    const uint64_t da = make_sdesc(sa), db = make_sdesc(sa + kPABytes);
#pragma unroll
                    for (int k = 0; k < kPBK / 16; ++k) {
                        if (MC == 1)
                            tc_mma(d, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc, (kb > kb0 || k > 0) ? 1u : 0u);
                        else
                            tc_mma2(d, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc, (kb > kb0 || k > 0) ? 1u : 0u);
                    }
                    if (MC == 1) tc_commit(&empty[stage]);
                    else tc_commit2_mc(&empty[stage], (uint16_t)3u);  // both producers may refill it
                    if (++stage == kPStages) { stage = 0; phase ^= 1u; }
                }
                if (MC == 1) tc_commit(&tmem_full[buf]);
                else tc_commit2_mc(&tmem_full[buf], (uint16_t)3u);  // both CTAs' epilogues
            }
        }
    } else {
        // --------------------------------------------------------- epilogue
        const int q = warp & 3;  // TMEM lane quarter of this warp
        const int e = q * 32 + lane;
        const int h0 = ((warp - 2) >> 2) * (kPBN / 2);  // first column of this warp's half
        griddep_wait();  // bias / bounds / sites / y may belong to the previous kernel
        uint32_t* ws_lc = p.bp.ws + 4 * p.bp.S + 1;
        uint32_t* ws_ov = p.bp.ws + 4 * p.bp.S + 2;
        unsigned long long* list = reinterpret_cast<unsigned long long*>(
            reinterpret_cast<char*>(p.bp.ws) + (((size_t)(4 * p.bp.S + 4) * 4 + 7) & ~(size_t)7));
        int tc = 0, m0, n0, ks;
        for (int i = 0; tile_of<MC>(p, i, m0, n0, ks); ++i, ++tc) {
            const int buf = tc & 1;
            const int m = m0 + e;
            const bool row_ok = m < p.M;
            // row information (independent of the accumulator)
            int seq = -1;
            uint32_t kL2 = 0u, kH2 = 0xFFFFFFFFu;
            if (row_ok) {
                if (derive) {
                    seq = p.bp.seq_offsets ? seq_of_row(p.bp.seq_offsets, p.bp.S, (uint32_t)m) : 0;
                    if (seq >= p.bp.S) seq = -1;  // padding rows after the last sequence (A18)
                } else if (p.mode == FT2_GEMM_CHECK) {
                    const int s = p.row_mode == 2 ? 0 : (p.row_mode == 1 ? m : p.row_to_seq[m]);
                    if (s >= 0 && s < p.S) {
                        const uint32_t k = key2((uint32_t)p.bounds[2 * s] | ((uint32_t)p.bounds[2 * s + 1] << 16));
                        kL2 = (k & 0xFFFFu) * 0x10001u;
                        kH2 = (k >> 16) * 0x10001u;
                        seq = s;
                    }
                }
            }
            // fault sites of this row inside this tile (fault-injection runs only)
            uint32_t site_c[kPMaxRowSites], site_m[kPMaxRowSites];
            int nsite = 0;
            bool site_scan = false;   // more than kPMaxRowSites: rescan every site per chunk (never drop one)
            if (p.sites != nullptr && row_ok) {
                for (int i = 0; i < p.n_sites; ++i) {
                    const ft2_fault_site st = p.sites[i];
                    if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
                    const int64_t r = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) +
                                      (p.cur_step == 0 ? (int64_t)st.token : 0);
                    const int64_t c = (int64_t)st.col - n0;
                    if (r == m && c >= 0 && c < kPBN && (int64_t)st.col < p.N) {
                        if (nsite < kPMaxRowSites) {
                            site_c[nsite] = (uint32_t)c;
                            site_m[nsite] = st.xor_mask & 0xFFFFu;
                            ++nsite;
                        } else {
                            site_scan = true;
                        }
                    }
                }
            }
            uint32_t mn2 = 0xFFFFFFFFu, mx2 = 0u, ncorr = 0u;
            mbar_wait(&tmem_full[buf], (uint32_t)(tc >> 1) & 1u);
            tc_fence_after();
            const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * kPBN);
            uint16_t* yrow = p.y + (int64_t)m * p.ldy;
            const bool split = p.splits > 1;
            // 128 x 256 half-tile id; pairs may cover one phantom m-tile past tilesM
            const int half = m0 / kPBM + (MC == 2 ? ((p.tilesM + 1) & ~1) : p.tilesM) * (n0 / kPBN);
            // split-K slots: [half-tile][split][16 column chunks][128 rows][16],
            // so a chunk is one contiguous 8 KB block (coalesced copies)
            float* const slot0 = split ? p.skws + (size_t)half * p.splits * kPBM * kPBN : nullptr;
            const int grp = (warp - 2) >> 2;  // column half = staging group (4 warps, rows 0..127)
            float* const stg = sk_stage + grp * kPBM * kSkStride;
            if (split) {
                // K split: stage this unit's fp32 partial tile through shared
                // memory into its slot (chunk-major, 16-byte coalesced stores);
                // the last of the tile's splits to arrive sums all slots in
                // split order (deterministic) and runs the epilogue below
                float* mine = slot0 + (size_t)ks * kPBM * kPBN;
#pragma unroll 1
                for (int c0 = h0; c0 < h0 + kPBN / 2; c0 += 32) {
                    uint32_t r[32];
                    tmem_ld32(taddr + (uint32_t)c0, r);
                    tmem_wait_ld();
#pragma unroll
                    for (int sub = 0; sub < 2; ++sub) {
#pragma unroll
                        for (int j = 0; j < 4; ++j)
                            *reinterpret_cast<float4*>(stg + e * kSkStride + 4 * j) =
                                make_float4(__uint_as_float(r[16 * sub + 4 * j]), __uint_as_float(r[16 * sub + 4 * j + 1]),
                                            __uint_as_float(r[16 * sub + 4 * j + 2]), __uint_as_float(r[16 * sub + 4 * j + 3]));
                        named_bar(2 + grp, 128);
                        float* chunk = mine + (size_t)((c0 + 16 * sub) >> 4) * (kPBM * 16);
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            const int i = e + 128 * k;   // float4 index within the chunk
                            __stcg(reinterpret_cast<float4*>(chunk) + i,
                                   *reinterpret_cast<const float4*>(stg + (i >> 2) * kSkStride + 4 * (i & 3)));
                        }
                        named_bar(2 + grp, 128);
                    }
                }
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (MC == 1) mbar_arrive(&tmem_empty[buf]);
                    else mbar_arrive_cluster(mapa(smem_u32(&tmem_empty[buf]), 0u));
                }
                __threadfence();
                named_bar(1, 32 * kPEpiWarps);
                if (tid == 64) {
                    // my partial is written; wait for every split's (they all run in
                    // this one wave -- the host splits only when units * splits <= slots)
                    atom_add_acq_rel_gpu(p.skcnt + 2 * half, 1u);
                    while (ld_acquire_gpu(p.skcnt + 2 * half) < (uint32_t)p.splits) {
                    }
                }
                named_bar(1, 32 * kPEpiWarps);
            }
#pragma unroll 1
            for (int c0 = h0; c0 < h0 + kPBN / 2; c0 += 32) {
                if (split && (c0 >> 5) % p.splits != ks) continue;   // another split finishes these 32 columns
                uint32_t r[32];
                if (!split) {
                    tmem_ld32(taddr + (uint32_t)c0, r);
                    tmem_wait_ld();
                } else {
                    // coalesced chunk sums (split order 0..S-1 per element),
                    // transposed back to one row per thread through shared memory
#pragma unroll
                    for (int sub = 0; sub < 2; ++sub) {
                        const size_t coff = (size_t)((c0 + 16 * sub) >> 4) * (kPBM * 16);
                        // every split's 4 vectors in flight at once (one L2 round trip),
                        // then summed in split order 0..S-1 (deterministic)
                        float4 part[kMaxSplits][4];
#pragma unroll
                        for (int sk = 0; sk < kMaxSplits; ++sk)
                            if (sk < p.splits) {
                                const float4* sl = reinterpret_cast<const float4*>(slot0 + (size_t)sk * kPBM * kPBN + coff);
#pragma unroll
                                for (int k = 0; k < 4; ++k) part[sk][k] = __ldcg(sl + e + 128 * k);
                            }
                        float4 acc[4];
#pragma unroll
                        for (int k = 0; k < 4; ++k) acc[k] = part[0][k];
#pragma unroll
                        for (int sk = 1; sk < kMaxSplits; ++sk)
                            if (sk < p.splits) {
#pragma unroll
                                for (int k = 0; k < 4; ++k) {
                                    acc[k].x += part[sk][k].x; acc[k].y += part[sk][k].y;
                                    acc[k].z += part[sk][k].z; acc[k].w += part[sk][k].w;
                                }
                            }
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            const int i = e + 128 * k;
                            *reinterpret_cast<float4*>(stg + (i >> 2) * kSkStride + 4 * (i & 3)) = acc[k];
                        }
                        named_bar(2 + grp, 128);
#pragma unroll
                        for (int j = 0; j < 4; ++j) {
                            const float4 v = *reinterpret_cast<const float4*>(stg + e * kSkStride + 4 * j);
                            r[16 * sub + 4 * j] = __float_as_uint(v.x);
                            r[16 * sub + 4 * j + 1] = __float_as_uint(v.y);
                            r[16 * sub + 4 * j + 2] = __float_as_uint(v.z);
                            r[16 * sub + 4 * j + 3] = __float_as_uint(v.w);
                        }
                        named_bar(2 + grp, 128);
                    }
                }
                const int nb = n0 + c0;
                if (!row_ok || nb >= p.N) continue;
                const int nvalid = min(32, p.N - nb);
                // bias (the same 32 values for every thread: broadcast loads)
                float bv[32];
                if (p.bias) {
                    const uint4* bq = reinterpret_cast<const uint4*>(p.bias + nb);
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        uint4 u = nvalid == 32 ? __ldg(bq + j) : make_uint4(0u, 0u, 0u, 0u);
                        if (nvalid < 32) {
                            uint32_t tmp[4] = {0u, 0u, 0u, 0u};
                            for (int h = 0; h < 8; ++h)
                                if (j * 8 + h < nvalid) tmp[h >> 1] |= (uint32_t)p.bias[nb + j * 8 + h] << ((h & 1) * 16);
                            u = make_uint4(tmp[0], tmp[1], tmp[2], tmp[3]);
                        }
                        const uint32_t uw[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
                        for (int h = 0; h < 4; ++h) {
                            bv[j * 8 + 2 * h] = to_f32<DT>((uint16_t)(uw[h] & 0xFFFFu));
                            bv[j * 8 + 2 * h + 1] = to_f32<DT>((uint16_t)(uw[h] >> 16));
                        }
                    }
                } else {
#pragma unroll
                    for (int j = 0; j < 32; ++j) bv[j] = 0.f;
                }
                uint32_t w[16];
#pragma unroll
                for (int j = 0; j < 16; ++j)
                    w[j] = pack_rne2(__uint_as_float(r[2 * j]) + bv[2 * j], __uint_as_float(r[2 * j + 1]) + bv[2 * j + 1], DT);
                for (int i = 0; i < (site_scan ? 0 : nsite); ++i) {
                    const uint32_t d = site_c[i] - (uint32_t)c0;
                    if (d < 32u) {
#pragma unroll
                        for (int j = 0; j < 16; ++j)
                            w[j] ^= (d >> 1) == (uint32_t)j ? site_m[i] << ((d & 1u) * 16) : 0u;   // branch-free: w stays in registers
                    }
                }
                if (site_scan) {   // rare overflow path: every site, straight from global memory
                    for (int i = 0; i < p.n_sites; ++i) {
                        const ft2_fault_site st = p.sites[i];
                        if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
                        const int64_t r = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) +
                                          (p.cur_step == 0 ? (int64_t)st.token : 0);
                        const uint32_t d = (uint32_t)((int64_t)st.col - n0 - c0);
                        if (r != m || (int64_t)st.col >= p.N || d >= 32u) continue;
#pragma unroll
                        for (int j = 0; j < 16; ++j)
                            w[j] ^= (d >> 1) == (uint32_t)j ? (st.xor_mask & 0xFFFFu) << ((d & 1u) * 16) : 0u;
                    }
                }
                if (p.mode == FT2_GEMM_CHECK && seq >= 0) {
#pragma unroll
                    for (int j = 0; j < 16; ++j) {
                        const int c = nb + 2 * j;
                        const uint32_t pm = ((c >= p.col_begin && c < p.col_end) ? 0x0000FFFFu : 0u) |
                                            ((c + 1 >= p.col_begin && c + 1 < p.col_end) ? 0xFFFF0000u : 0u);
                        uint32_t ch = 0u;
                        const uint32_t o = clip2<DT>(w[j], kL2, kH2, &ch);
                        const uint32_t nw = (o & pm) | (w[j] & ~pm);
                        ncorr += nonzero_halves(nw ^ w[j]);
                        w[j] = nw;
                    }
                }
                if (derive) {
#pragma unroll
                    for (int j = 0; j < 16; ++j) {
                        // columns beyond N must not contribute: neutral keys
                        const uint32_t k = key2(w[j]);
                        const uint32_t kmn = 2 * j + 1 < nvalid ? k : (2 * j < nvalid ? (k | 0xFFFF0000u) : 0xFFFFFFFFu);
                        const uint32_t kmx = 2 * j + 1 < nvalid ? k : (2 * j < nvalid ? (k & 0x0000FFFFu) : 0u);
                        mn2 = vmin_u16x2(mn2, kmn);
                        mx2 = vmax_u16x2(mx2, kmx);
                    }
                }
                if (nvalid == 32 && ((reinterpret_cast<uintptr_t>(yrow + nb) & 15u) == 0)) {
                    uint4* dst = reinterpret_cast<uint4*>(yrow + nb);
#pragma unroll
                    for (int j = 0; j < 4; ++j) dst[j] = make_uint4(w[4 * j], w[4 * j + 1], w[4 * j + 2], w[4 * j + 3]);
                } else {
#pragma unroll
                    for (int j = 0; j < 32; ++j)   // static indices into w (a runtime bound would spill w to local memory)
                        if (j < nvalid) yrow[nb + j] = (uint16_t)(w[j >> 1] >> ((j & 1) * 16));
                }
            }
            if (split) {   // my reads of the partial slots are done; the last reader resets both counters
                named_bar(1, 32 * kPEpiWarps);
                if (tid == 64 && atom_add_acq_rel_gpu(p.skcnt + 2 * half + 1, 1u) == (uint32_t)(p.splits - 1)) {
                    p.skcnt[2 * half] = 0u;
                    p.skcnt[2 * half + 1] = 0u;
                }
            }
            // accumulator buffer drained: hand it back to the MMA warp (the leader's)
            if (!split) {
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (MC == 1) mbar_arrive(&tmem_empty[buf]);
                    else mbar_arrive_cluster(mapa(smem_u32(&tmem_empty[buf]), 0u));
                }
            }
            if (p.mode == FT2_GEMM_CHECK && ncorr != 0u && p.counts != nullptr && seq >= 0)
                atomicAdd(&p.counts[seq], ncorr);
            if (derive) {
                uint32_t kmin = min(mn2 & 0xFFFFu, mn2 >> 16), kmax = max(mx2 & 0xFFFFu, mx2 >> 16);
                uint32_t nf = 0u;
                if (seq >= 0 && (kmin < Fmt<DT>::kKeyLo || kmax > Fmt<DT>::kKeyHi)) {
                    // a non-finite output in this row segment: exact pass over
                    // what this thread just stored (rare; R2 excludes it, R4 patches it)
                    kmin = 0xFFFFu;
                    kmax = 0u;
                    const int nend = min(p.N, n0 + h0 + kPBN / 2);
                    for (int n = n0 + h0; n < nend; ++n) {
                        if (split && ((n - n0) >> 5) % p.splits != ks) continue;   // columns another split stored
                        const uint16_t b = yrow[n];
                        if (nonfinite1<DT>(b)) {
                            ++nf;
                            if (p.bp.correct)
                                record_patch(p.bp, ws_lc, ws_ov, list, seq, (uint64_t)((int64_t)m * p.ldy + n));
                        } else {
                            const uint32_t k = key1(b);
                            kmin = min(kmin, k);
                            kmax = max(kmax, k);
                        }
                    }
                }
                if (seq < 0) { kmin = 0xFFFFu + 1u; kmax = 0u; }
                // one sequence across the warp's 32 rows (the common case): warp-reduce first
                const int seq0 = __shfl_sync(0xFFFFFFFFu, seq, 0);
                const bool uni = __all_sync(0xFFFFFFFFu, seq == seq0);
                if (uni) {
                    kmin = __reduce_min_sync(0xFFFFFFFFu, kmin);
                    kmax = __reduce_max_sync(0xFFFFFFFFu, kmax);
                    nf = __reduce_add_sync(0xFFFFFFFFu, nf);
                }
                if ((!uni || lane == 0) && seq >= 0) {
                    const bool have = kmin <= kmax;
                    if (use_tab) {
                        if (have) {
                            atomicMax(&tab_lo[seq], 0x10000u - kmin);
                            atomicMax(&tab_hi[seq], kmax + 1u);
                        }
                        if (nf) atomicAdd(&tab_nf[seq], nf);
                    } else {
                        if (have) {
                            atomicMax(&p.bp.ws[4 * seq + 0], 0x10000u - kmin);
                            atomicMax(&p.bp.ws[4 * seq + 1], kmax + 1u);
                        }
                        if (nf) atomicAdd(&p.bp.ws[4 * seq + 2], nf);
                    }
                }
            }
        }
    }

    // ----------------------------------------------------------- teardown
    tc_fence_before();
    __syncthreads();
    if (MC > 1) {  // no CTA leaves while its peer may still signal its barriers
        cluster_arrive_relaxed();
        cluster_wait();
    }
    if (warp == 1) {
        tc_fence_after();
        if (MC == 1) tmem_dealloc(tmem_base, 512);
        else tmem_dealloc2(tmem_base, 512);
    }
    if (!derive) return;
    if (use_tab) {
        for (int s = tid; s < p.bp.S; s += kPThreads) {
            if (tab_lo[s]) atomicMax(&p.bp.ws[4 * s + 0], tab_lo[s]);
            if (tab_hi[s]) atomicMax(&p.bp.ws[4 * s + 1], tab_hi[s]);
            if (tab_nf[s]) atomicAdd(&p.bp.ws[4 * s + 2], tab_nf[s]);
        }
    }
    // grid combine: the last CTA finalises (release covers this CTA's REDs and
    // patch records through the barrier; acquire for the last CTA)
    __syncthreads();
    if (tid == 0) *last_sh = atom_add_acq_rel_gpu(p.bp.ws + 4 * p.bp.S, 1u) == gridDim.x - 1 ? 1u : 0u;
    __syncthreads();
    if (*last_sh) bounds_finalize_tail<DT, false>(p.bp, tid, kPThreads);
}

// ---------------------------------------------------------------- host side
static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = [] {
        void* ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
        return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }();
    return fn;
}

static bool make_map_p(CUtensorMap* m, const void* base, int64_t rows, int64_t K, int64_t ld, int box_rows, int dt) {
    auto enc = encode_fn();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
    cuuint32_t box[2] = {(cuuint32_t)kPBK, (cuuint32_t)box_rows};
    cuuint32_t es[2] = {1, 1};
    return enc(m, dt == FT2_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2,
               const_cast<void*>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
               CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

template <int DT, int MC>
static cudaError_t launch_prefill_dt(const CUtensorMap& mx, const CUtensorMap& mw, const PrefK& p, int grid,
                                     cudaStream_t st) {
    static cudaError_t attr = cudaFuncSetAttribute(prefill_gemm_kernel<DT, MC>,
                                                   cudaFuncAttributeMaxDynamicSharedMemorySize, kPSmemBytes);
    if (attr != cudaSuccess) return attr;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(kPThreads);
    cfg.dynamicSmemBytes = kPSmemBytes;
    cfg.stream = st;
    cudaLaunchAttribute a[2];
    a[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    a[0].val.programmaticStreamSerializationAllowed = 1;
    a[1].id = cudaLaunchAttributeClusterDimension;
    a[1].val.clusterDim.x = MC;
    a[1].val.clusterDim.y = 1;
    a[1].val.clusterDim.z = 1;
    cfg.attrs = a;
    cfg.numAttrs = MC > 1 ? 2 : 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, prefill_gemm_kernel<DT, MC>, mx, mw, p);
    return e != cudaSuccess ? e : cudaGetLastError();
}

// Clusters (MC = 2: CTA pairs) or CTAs (MC = 1) of the persistent kernel that
// can be resident at once.  The split-K path makes the splits of a tile wait
// for each other, so it is planned only when every unit is resident at once.
template <int MC>
static int resident_slots() {
    static int n = [] {
        auto* k = prefill_gemm_kernel<0, MC>;
        if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kPSmemBytes) != cudaSuccess) {
            cudaGetLastError();
            return 0;
        }
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)num_sms());
        cfg.blockDim = dim3(kPThreads);
        cfg.dynamicSmemBytes = kPSmemBytes;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = MC;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        int c = 0;
        if (cudaOccupancyMaxActiveClusters(&c, k, &cfg) != cudaSuccess) {
            cudaGetLastError();
            return 0;
        }
        return c;
    }();
    return n;
}

// K-split plan for the persistent kernel: when the tiles cannot fill the
// machine (small M: e.g. 512 prompt tokens at N = 4096 give 16 pair-tiles for
// 74 SM pairs; a 256-trial decode batch gives 43 at N = 11008), split each
// tile's K range into s units (>= 8 k-blocks each) and pick the s that
// minimises the waves per unit of work, ceil(units * s / slots) / s, by at
// least 10 %.  Partials go through an fp32 workspace (s slots per tile).
PrefillSplit plan_prefill_split(int32_t M, int32_t N, int32_t K, size_t ws_bytes) {
    PrefillSplit r{1, 0, 0};
    const int tilesM = (M + kPBM - 1) / kPBM, tilesN = (N + kPBN - 1) / kPBN, nkb = (K + kPBK - 1) / kPBK;
    const int units = tilesM >= 2 ? ((tilesM + 1) / 2) * tilesN : tilesM * tilesN;
    const int slots = tilesM >= 2 ? num_sms() / 2 : num_sms();
    const int tilesMp = tilesM >= 2 ? ((tilesM + 1) & ~1) : tilesM;  // + the pairs' phantom m-tile
    // the arrival counters sit at a FIXED place (the first kSplitCounters
    // words) whatever the shape, so one launch's partial slots never alias
    // the next launch's counters
    r.cnt_bytes = (size_t)kSplitCounters * 4;
    if ((size_t)tilesMp * tilesN * 2 > (size_t)kSplitCounters) return r;   // two counters per half-tile
    const size_t per_split = (size_t)tilesMp * kPBM * tilesN * kPBN * 4;
    // FT2_PREFILL_SPLITS = s >= 2 forces s, 0 or 1 disables, -1 (default) is
    // the planner: the largest s <= kMaxSplits with units * s <= slots (one
    // wave: the splits of a tile wait for each other) and >= 8 k-blocks each.
    // Round 1 measured the old last-arriver reduction at par with no split
    // (its reads were serialised per split); the distributed one reads every
    // split's vectors at once (profiles/r2_prefill_split.txt).
    const char* ev = getenv("FT2_PREFILL_SPLITS");   // read per call: tests toggle it
    const int env = ev ? atoi(ev) : -1;
    if (env == 0 || env == 1) return r;
    // (a tcgen05.alloc kernel reads as 1 CTA/SM to the occupancy API, which is
    // what this kernel runs at anyway)
    const int resident = tilesM >= 2 ? resident_slots<2>() : resident_slots<1>();
    for (int s = 2; s <= kMaxSplits; ++s) {
        if (nkb < 8 * s || units * s > slots || units * s > resident) break;
        if (env > 0 && s > env) break;
        r.splits = s;
    }
    r.need_bytes = r.splits > 1 ? r.cnt_bytes + (size_t)r.splits * per_split : 0;
    while (r.splits > 1 && r.cnt_bytes + (size_t)r.splits * per_split > ws_bytes) --r.splits;
    return r;
}

cudaError_t launch_prefill_gemm(const GemmArgs& a, const PrefillDerive* d, cudaStream_t st, int* n_launch) {
    CUtensorMap mx, mw;
    if (!make_map_p(&mx, a.x, a.M, a.K, a.ldx, kPBM, a.dtype)) return cudaErrorInvalidValue;
    PrefK p = {};
    p.M = a.M;
    p.N = a.N;
    p.K = a.K;
    p.tilesM = (a.M + kPBM - 1) / kPBM;
    p.ntiles = p.tilesM * ((a.N + kPBN - 1) / kPBN);
    p.nkb = (a.K + kPBK - 1) / kPBK;
    p.mode = d ? kPGemmDerive : a.mode;
    p.col_begin = a.col_begin;
    p.col_end = a.col_end;
    p.bias = a.bias;
    p.y = a.y;
    p.ldy = a.ldy;
    p.row_to_seq = a.row_to_seq;
    p.S = a.S;
    p.row_mode = a.row_to_seq ? 0 : (a.S == 1 ? 2 : 1);
    p.bounds = a.bounds;
    p.counts = a.counts;
    p.sites = a.sites;
    p.n_sites = a.sites ? a.n_sites : 0;
    p.cur_layer = a.cur_layer;
    p.cur_step = a.cur_step;
    p.base_row = a.base_row;
    BoundsK& b = p.bp;
    b.y = a.y;
    b.ld = a.ldy;
    b.n8 = (uint32_t)(a.N / 8);
    b.total_vec = (uint32_t)((int64_t)a.M * (a.N / 8));
    b.chunk = 0;
    b.div_n8 = make_fastdiv(b.n8 > 0 ? b.n8 : 1);
    b.contiguous = a.ldy == a.N;
    if (d) {
        b.seq_offsets = d->seq_offsets;
        b.S = d->S;
        b.scale = d->scale;
        b.finalize = 1;
        b.correct = d->correct;
        b.bounds_out = d->bounds_out;
        b.keys_out = d->keys_out;
        b.nonfinite_out = d->nonfinite_out;
        b.nv_out = nullptr;
        b.ws = d->ws;
    } else {
        b.S = 0;
        b.ws = nullptr;
    }

    static const int mc_env = [] { const char* v = getenv("FT2_PREFILL_MC"); return v ? atoi(v) : 2; }();
    const int mc = (mc_env == 2 && p.tilesM >= 2) ? 2 : 1;  // CTA pairs (cta_group::2) unless one m-tile
    if (!make_map_p(&mw, a.w, a.N, a.K, a.ldw, mc == 2 ? kPBN / 2 : kPBN, a.dtype)) return cudaErrorInvalidValue;
    const int units = mc == 2 ? ((p.tilesM + 1) / 2) * (p.ntiles / p.tilesM) : p.ntiles;
    const int slots = mc == 2 ? num_sms() / 2 : num_sms();
    const PrefillSplit sp = plan_prefill_split(p.M, p.N, p.K, a.ws_bytes);
    p.splits = a.ws != nullptr ? sp.splits : 1;
    p.skcnt = static_cast<uint32_t*>(a.ws);
    p.skws = p.splits > 1 ? reinterpret_cast<float*>(static_cast<char*>(a.ws) + sp.cnt_bytes) : nullptr;
    const int work = units * p.splits;
    int grid = mc * (work < slots ? work : slots);
    cudaError_t e;
    if (mc == 2) e = a.dtype == FT2_FP16 ? launch_prefill_dt<1, 2>(mx, mw, p, grid, st)
                                         : launch_prefill_dt<0, 2>(mx, mw, p, grid, st);
    else e = a.dtype == FT2_FP16 ? launch_prefill_dt<1, 1>(mx, mw, p, grid, st)
                                 : launch_prefill_dt<0, 1>(mx, mw, p, grid, st);
    ++*n_launch;
    return e;
}

}  // namespace ft2impl
