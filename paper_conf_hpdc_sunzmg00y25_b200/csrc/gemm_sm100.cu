// gemm_sm100.cu -- critical linear layer with FT2's check fused into the
// epilogue, for sm_100a (tcgen05 MMA, TMEM accumulators, TMA pipeline).
//
//   y[m, j] = check(inject(bf16_rne(sum_k x[m, k] * w[j, k] + bias[j])))
//
// PAPER.md L259 ("Protection is applied after the execution of each critical
// layer"), L272 (clamp + nan_to_num applied right after the layer).  The
// check operates on the bf16-rounded value after bias (reading A19); a fault
// site is applied before the check (A20).
//
// Structure (one CTA = one 128 x BN output tile x one K slice):
//   warp 0      TMA producer: 128B-swizzled K-major tiles of A and B into a
//               kStages-deep shared-memory ring (mbarrier full/empty).
//   warp 1      TMEM allocator + single-thread tcgen05.mma.cta_group::1.kind::f16
//               issuer (BF16 x BF16 -> FP32 in TMEM); tcgen05.commit frees a
//               stage and finally signals the epilogue.
//   warps 2-5   epilogue: tcgen05.ld (32x32b) TMEM -> registers -> shared memory.
// Split-K runs as a thread-block cluster along K (cluster dims (1, splitk, 1)):
// each CTA's fp32 partial tile is combined through distributed shared memory
// in fixed rank order (deterministic), each CTA then finishes 128/splitk rows:
// bias, RNE to bf16, fault XOR, key-space clamp, corrected count, store.  The
// clip is therefore applied to the complete K reduction (it is non-linear).
//
// Orientation: for decode (M <= 128 tokens) the kernel runs "swap-AB": the
// UMMA M = 128 dimension walks output features (rows of W) and UMMA N = BN
// walks tokens, so skinny activations still fill the tensor core; for prefill
// (M > 128) A = x and B = w.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdio.h>
#include <stdlib.h>

#include <mutex>

#include "ft2_device.cuh"
#include "ft2_internal.h"

namespace ft2impl {
using namespace ft2dev;

constexpr int kBlockA = 128;   // UMMA M
constexpr int kBlockK = 64;    // one 128-byte swizzle atom of bf16
constexpr int kUmmaK = 16;
constexpr int kGemmThreads = 192;
constexpr int kMaxSitesPerCta = 64;
// Split-K tile counters live in a fixed region at the start of the workspace
// (independent of the shape, so one workspace can serve every GEMM); split-K
// is only used when tiles * splitk fits one co-resident wave, i.e. tiles <= 2 x SMs.
constexpr int kMaxSplitTiles = 1024;
constexpr size_t kCounterBytes = (size_t)kMaxSplitTiles * 8;

// ------------------------------------------------------------------ PTX glue
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t a = smem_u32(bar);
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra WAIT_%=;\n}" ::"r"(a),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_2d(const CUtensorMap* map, uint64_t* bar, void* dst, int c0, int c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
            smem_u32(dst)),
        "l"(map), "r"(smem_u32(bar)), "r"(c0), "r"(c1)
        : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(map) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void tc_mma(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "setp.ne.b32 p, %4, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
        "l"(da), "l"(db), "r"(idesc), "r"(acc)
        : "memory");
}
// 32 lanes x 32 consecutive 32-bit columns -> 32 registers per thread
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
        "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 "
        "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa(uint32_t addr, uint32_t rank) {
    uint32_t r;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
    return r;
}
__device__ __forceinline__ float ld_dsmem_f32(uint32_t addr) {
    float v;
    asm volatile("ld.shared::cluster.f32 %0, [%1];" : "=f"(v) : "r"(addr));
    return v;
}

// UMMA shared-memory descriptor: K-major, 128-byte swizzle, 8-row core
// matrix groups 1024 B apart (SBO), sm100 descriptor version 1.
__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr) {
    uint64_t d = 0;
    d |= (uint64_t)((saddr >> 4) & 0x3FFF);
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}

// Instruction descriptor, kind::f16: D fp32, A/B bf16, both K-major.
__host__ __device__ constexpr uint32_t make_idesc(int m, int n) {
    return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}

struct GemmK {
    int32_t M, N, K;
    int32_t swap;          // 1: A = w (features), B = x (tokens)
    int32_t rowsA, rowsB;  // extent of the A / B operands
    int32_t tilesA, tilesB;
    int32_t splitk, nkb;
    int32_t mode, col_begin, col_end;
    const uint16_t* bias;
    uint16_t* y;
    int64_t ldy;
    const int32_t* row_to_seq;
    int32_t S, row_mode;
    const uint16_t* bounds;
    uint32_t* counts;
    const ft2_fault_site* sites;
    int32_t n_sites, cur_layer, cur_step;
    const int32_t* base_row;
    float4* partials;      // [tiles][splitk][BN/4][128] float4 (split-K only)
    uint32_t* tile_ctr;    // [tiles][2] self-resetting arrival / departure counters
    int32_t w_static;      // weights not written by the preceding kernel: prefetch before the PDL wait
};

template <int BN, int STAGES>
struct GemmSmem {
    static constexpr int kABytes = kBlockA * kBlockK * 2;
    static constexpr int kBBytes = BN * kBlockK * 2;
    static constexpr int kStageBytes = kABytes + kBBytes;
    static constexpr int kTileBytes = STAGES * kStageBytes;
    static constexpr int kBytes = 1024 /*align slack*/ + kTileBytes + 1024 /*barriers, site list*/ + (BN + 128) * 20;
};

__device__ __forceinline__ void griddep_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void griddep_launch() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

// Per-row / per-column epilogue context.  In swap-AB mode rows are output
// features (bias, protected-slice flag per row) and columns are tokens (bounds
// per column); otherwise the other way round.  `keys` packs key(lo) | key(hi) << 16;
// seq < 0 means "do not check".
struct EpiSide {
    float bias;
    uint32_t keys;
    int32_t seq;
    int32_t valid;  // index inside [0, M) / [0, N)
};

__device__ __forceinline__ EpiSide make_side(const GemmK& p, bool is_token, int idx) {
    EpiSide e{0.f, 0u, -1, 0};
    if (is_token) {
        e.valid = idx < p.M;
        if (e.valid && p.mode == FT2_GEMM_CHECK) {
            const int s = p.row_mode == 2 ? 0 : (p.row_mode == 1 ? idx : p.row_to_seq[idx]);
            if (s >= 0 && s < p.S) {
                const uint32_t lh = (uint32_t)p.bounds[2 * s] | ((uint32_t)p.bounds[2 * s + 1] << 16);
                e.keys = key2(lh);
                e.seq = s;
            }
        }
    } else {
        e.valid = idx < p.N;
        if (e.valid) {
            if (p.bias) e.bias = __uint_as_float((uint32_t)p.bias[idx] << 16);
            e.seq = (p.mode == FT2_GEMM_CHECK && idx >= p.col_begin && idx < p.col_end) ? 0 : -1;  // flag only
        }
    }
    return e;
}

// Four consecutive columns c..c+3 of one row: all four values are computed
// before any side effect (stores, counter atomics), so the chains overlap.
__device__ __forceinline__ void finish4(const GemmK& p, int ga, int gb0, const EpiSide& rs, const EpiSide* cs,
                                        int la_c0, const float (&acc)[4], const uint32_t* site_e,
                                        const uint32_t* site_m, uint32_t nsite, uint32_t* row_cnt,
                                        uint32_t* col_cnt) {
    uint16_t o[4];
    bool ok[4];
    uint32_t changed = 0;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
        const EpiSide& feat = p.swap ? rs : cs[j];
        const EpiSide& tok = p.swap ? cs[j] : rs;
        ok[j] = feat.valid && tok.valid;
        uint16_t x = bf16_rne(acc[j] + feat.bias);
        for (uint32_t i = 0; i < nsite; ++i)
            if (site_e[i] == (uint32_t)(la_c0 + j)) x ^= (uint16_t)site_m[i];
        const bool chk = feat.seq >= 0 && tok.seq >= 0;
        const uint16_t z = ((x & 0x7FFF) > 0x7F80) ? (uint16_t)0 : x;  // NaN -> +0
        const uint16_t k = key1(z);
        const uint16_t kl = (uint16_t)tok.keys, kh = (uint16_t)(tok.keys >> 16);
        const uint16_t c = k < kl ? unkey1(kl) : (k > kh ? unkey1(kh) : z);
        o[j] = chk ? c : x;
        changed |= (ok[j] && o[j] != x) ? (1u << j) : 0u;
    }
    if (p.swap) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (ok[j]) p.y[(int64_t)(gb0 + j) * p.ldy + ga] = o[j];
    } else {
        uint16_t* dst = p.y + (int64_t)ga * p.ldy + gb0;
        if (ok[0] && ok[3] && ((reinterpret_cast<uintptr_t>(dst) & 7u) == 0)) {
            *reinterpret_cast<uint2*>(dst) = make_uint2((uint32_t)o[0] | ((uint32_t)o[1] << 16),
                                                        (uint32_t)o[2] | ((uint32_t)o[3] << 16));
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (ok[j]) dst[j] = o[j];
        }
    }
    if (changed) {  // corrected neurons, aggregated per CTA in shared memory
        if (p.swap) {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (changed & (1u << j)) atomicAdd_block(&col_cnt[j], 1u);
        } else {
            atomicAdd_block(row_cnt, (uint32_t)__popc(changed));
        }
    }
}

template <int BN, int STAGES>
__global__ void __launch_bounds__(kGemmThreads, 1)
    gemm_kernel(const __grid_constant__ CUtensorMap map_a, const __grid_constant__ CUtensorMap map_b,
                const __grid_constant__ GemmK p) {
    using L = GemmSmem<BN, STAGES>;
    extern __shared__ uint8_t smem_raw[];
    uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~(uintptr_t)1023);
    uint8_t* tiles = smem;
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + L::kTileBytes);
    uint64_t* empty = full + STAGES;
    uint64_t* tmem_full = empty + STAGES;
    uint32_t* tmem_base_sh = reinterpret_cast<uint32_t*>(tmem_full + 1);
    uint32_t* flag_sh = tmem_base_sh + 1;
    uint32_t* site_n = flag_sh + 1;
    uint32_t* site_e = site_n + 1;                 // [kMaxSitesPerCta] local element index (a * BN + c)
    uint32_t* site_m = site_e + kMaxSitesPerCta;   // [kMaxSitesPerCta] xor mask
    EpiSide* col_side = reinterpret_cast<EpiSide*>(site_m + kMaxSitesPerCta);  // [BN] per-column context
    EpiSide* row_side = col_side + BN;                                        // [128] per-row context
    uint32_t* col_cnt = reinterpret_cast<uint32_t*>(row_side + 128);          // [BN] corrected per column
    uint32_t* row_cnt = col_cnt + BN;                                         // [128] corrected per row

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int tileA = blockIdx.x, split = blockIdx.y, tileB = blockIdx.z;
    const int kb0 = (int)((int64_t)split * p.nkb / p.splitk);
    const int kb1 = (int)((int64_t)(split + 1) * p.nkb / p.splitk);
    const int nk = kb1 - kb0;
    constexpr uint32_t kTmemCols = BN < 32 ? 32 : BN;

    if (warp == 0 && lane == 0) {
        prefetch_tmap(&map_a);
        prefetch_tmap(&map_b);
        for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        mbar_init(tmem_full, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        *site_n = 0;
    }
    if (warp == 1) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_sh)),
                     "r"(kTmemCols));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_base_sh;
    // the next kernel in the stream may start its own prologue now (PDL)
    griddep_launch();

    if (warp == 0) {
        if (lane == 0) {
            // ------------------------------------------------ TMA producer
            // The weight operand does not depend on the previous kernel: the
            // first STAGES weight tiles are requested before waiting for it
            // (programmatic dependent launch), the activations after.
            const CUtensorMap* mw = p.swap ? &map_a : &map_b;
            const CUtensorMap* mx = p.swap ? &map_b : &map_a;
            const int w_row = p.swap ? tileA * kBlockA : tileB * BN;
            const int x_row = p.swap ? tileB * BN : tileA * kBlockA;
            const int w_off = p.swap ? 0 : L::kABytes;
            const int x_off = p.swap ? L::kABytes : 0;
            const int pre = nk < STAGES ? nk : STAGES;
            if (!p.w_static) griddep_wait();
            for (int i = 0; i < pre; ++i) {
                uint8_t* st = tiles + i * L::kStageBytes;
                mbar_expect_tx(&full[i], L::kStageBytes);
                tma_load_2d(mw, &full[i], st + w_off, (kb0 + i) * kBlockK, w_row);
            }
            if (p.w_static) griddep_wait();
            for (int i = 0; i < pre; ++i)
                tma_load_2d(mx, &full[i], tiles + i * L::kStageBytes + x_off, (kb0 + i) * kBlockK, x_row);
            for (int i = STAGES; i < nk; ++i) {
                const int s = i % STAGES;
                const uint32_t ph = (uint32_t)(i / STAGES) & 1u;
                mbar_wait(&empty[s], ph ^ 1u);
                uint8_t* st = tiles + s * L::kStageBytes;
                mbar_expect_tx(&full[s], L::kStageBytes);
                const int kc = (kb0 + i) * kBlockK;
                tma_load_2d(mw, &full[s], st + w_off, kc, w_row);
                tma_load_2d(mx, &full[s], st + x_off, kc, x_row);
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ------------------------------------------------ MMA issuer
            constexpr uint32_t idesc = make_idesc(kBlockA, BN);
            for (int i = 0; i < nk; ++i) {
                const int s = i % STAGES;
                const uint32_t ph = (uint32_t)(i / STAGES) & 1u;
                mbar_wait(&full[s], ph);
                tc_fence_after();
                const uint32_t sa = smem_u32(tiles + s * L::kStageBytes);
                const uint32_t sb = sa + L::kABytes;
                const uint64_t da = make_sdesc(sa), db = make_sdesc(sb);
#pragma unroll
                for (int k = 0; k < kBlockK / kUmmaK; ++k)  // 16 elements = 32 B along K per MMA
                    tc_mma(tmem_base, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc,
                           (i > 0 || k > 0) ? 1u : 0u);
                tc_commit(&empty[s]);
            }
            tc_commit(tmem_full);
        }
    } else {
        // ---------------------------------------------------- epilogue warps
        const int q = warp & 3;               // TMEM lane quarter this warp may access
        const int a = q * 32 + lane;          // row of the A tile owned by this thread
        const int et = a;                     // epilogue thread index 0..127
        const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16);
        const int ga = tileA * kBlockA + a;
        const int tile = tileB * p.tilesA + tileA;
        griddep_wait();                       // bias/bounds/y/workspace may belong to the previous kernel
        // rows of the 128-row A tile this CTA finishes: all of them without
        // split-K, else the split's 1/splitk slice (distributed reduction)
        const int r0 = (split * kBlockA) / p.splitk, r1 = ((split + 1) * kBlockA) / p.splitk;
        // epilogue contexts (bias, bound keys) are gathered while the main loop
        // still runs: columns are tokens in swap-AB mode, features otherwise
        for (int c = et; c < BN; c += 128) {
            col_side[c] = make_side(p, p.swap != 0, tileB * BN + c);
            col_cnt[c] = 0u;
        }
        row_side[et] = make_side(p, p.swap == 0, ga);
        row_cnt[et] = 0u;
        // fault sites that land in this CTA's output slice
        if (p.sites != nullptr) {
            for (int i = et; i < p.n_sites; i += 128) {
                ft2_fault_site st = p.sites[i];
                if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
                int64_t m = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) +
                            (p.cur_step == 0 ? (int64_t)st.token : 0);
                int64_t n = st.col;
                if (m < 0 || m >= p.M || n >= p.N) continue;
                int64_t la = (p.swap ? n : m) - (int64_t)tileA * kBlockA;
                int64_t lb = (p.swap ? m : n) - (int64_t)tileB * BN;
                if (la < r0 || la >= r1 || lb < 0 || lb >= BN) continue;
                uint32_t idx = atomicAdd(site_n, 1u);
                if (idx < (uint32_t)kMaxSitesPerCta) {
                    site_e[idx] = (uint32_t)(la * BN + lb);
                    site_m[idx] = st.xor_mask;
                }
            }
        }
        mbar_wait(tmem_full, 0);
        tc_fence_after();
        if (p.splitk == 1) {
            epi_bar();
            const EpiSide rs = row_side[et];
            const uint32_t nsite = min(*site_n, (uint32_t)kMaxSitesPerCta);
#pragma unroll 1
            for (int c0 = 0; c0 < BN; c0 += 16) {
                uint32_t r[16];
                tmem_ld16(taddr + c0, r);
                tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 16; j += 4) {
                    const float acc[4] = {nk > 0 ? __uint_as_float(r[j]) : 0.f, nk > 0 ? __uint_as_float(r[j + 1]) : 0.f,
                                          nk > 0 ? __uint_as_float(r[j + 2]) : 0.f, nk > 0 ? __uint_as_float(r[j + 3]) : 0.f};
                    finish4(p, ga, tileB * BN + c0 + j, rs, col_side + c0 + j, a * BN + c0 + j, acc, site_e, site_m,
                            nsite, row_cnt + et, col_cnt + c0 + j);
                }
            }
        } else {
            // 1. publish this split's fp32 partial tile (coalesced float4 columns)
            float4* tbase = p.partials + (size_t)tile * p.splitk * (BN / 4) * kBlockA;
            float4* mine = tbase + (size_t)split * (BN / 4) * kBlockA;
#pragma unroll 1
            for (int c0 = 0; c0 < BN; c0 += 16) {
                uint32_t r[16];
                tmem_ld16(taddr + c0, r);
                tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 16; j += 4)
                    __stcg(&mine[((c0 + j) / 4) * kBlockA + a],
                           make_float4(__uint_as_float(r[j]), __uint_as_float(r[j + 1]), __uint_as_float(r[j + 2]),
                                       __uint_as_float(r[j + 3])));
            }
            epi_bar();
            // 2. wait until every split of this tile has published.  All split
            // CTAs are co-resident: the grid never exceeds one wave (<= 1 CTA
            // per SM), and PDL dependents launch only after all CTAs started.
            uint32_t* arrive = p.tile_ctr + 2 * tile;
            uint32_t* depart = arrive + 1;
            if (et == 0) {
                // release: the barrier above orders every epilogue thread's partial stores before it
                asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(arrive) : "memory");
                uint32_t seen, ns = 32;
                while (true) {
                    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(seen) : "l"(arrive) : "memory");
                    if (seen >= (uint32_t)p.splitk) break;
                    __nanosleep(ns);
                    if (ns < 256) ns <<= 1;
                }
            }
            epi_bar();  // thread 0's acquire is ordered before everyone's partial loads
            const uint32_t nsite = min(*site_n, (uint32_t)kMaxSitesPerCta);
            // 3. reduce my row slice over all splits in fixed order 0..splitk-1
            const int nrow = r1 - r0;
            const int nvec = nrow * (BN / 4);
            for (int v = et; v < nvec; v += 128) {
                const int la = r0 + v % nrow, c4 = v / nrow;
                float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
                float4 part[16];
#pragma unroll
                for (int rr = 0; rr < 16; ++rr)
                    if (rr < p.splitk) part[rr] = __ldcg(&tbase[((size_t)rr * (BN / 4) + c4) * kBlockA + la]);
#pragma unroll
                for (int rr = 0; rr < 16; ++rr)
                    if (rr < p.splitk) {
                        acc.x += part[rr].x; acc.y += part[rr].y; acc.z += part[rr].z; acc.w += part[rr].w;
                    }
                const int gla = tileA * kBlockA + la;
                const EpiSide rs = row_side[la];
                const float av[4] = {acc.x, acc.y, acc.z, acc.w};
                finish4(p, gla, tileB * BN + c4 * 4, rs, col_side + c4 * 4, la * BN + c4 * 4, av, site_e, site_m,
                        nsite, row_cnt + la, col_cnt + c4 * 4);
            }
            // 4. the last CTA to leave resets the counters for the next launch
            epi_bar();
            if (et == 0) {
                if (atomicAdd(depart, 1u) == (uint32_t)p.splitk - 1) {
                    *arrive = 0u;
                    *depart = 0u;
                }
            }
        }
    }
    if (warp >= 2 && p.counts != nullptr && p.mode == FT2_GEMM_CHECK) {
        epi_bar();  // every finish4 of this CTA has counted
        const int et = (warp & 3) * 32 + lane;
        for (int c = et; c < BN; c += 128)
            if (col_cnt[c] != 0u && col_side[c].seq >= 0 && p.swap) atomicAdd(&p.counts[col_side[c].seq], col_cnt[c]);
        if (!p.swap && row_cnt[et] != 0u && row_side[et].seq >= 0) atomicAdd(&p.counts[row_side[et].seq], row_cnt[et]);
    }
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(kTmemCols));
    }
}

// ---------------------------------------------------------------- host side
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* ptr = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
    });
    return fn;
}

static bool make_map(CUtensorMap* m, const void* base, int64_t rows, int64_t K, int64_t ld, int box_rows) {
    auto enc = get_encode();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
    cuuint32_t box[2] = {(cuuint32_t)kBlockK, (cuuint32_t)box_rows};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// Tiling plan shared by the workspace query and the launch.
struct GemmPlan {
    int swap, bn, tilesA, tilesB, splitk, nkb;
};

// Pipeline depth per BN: BN <= 64 keeps a CTA at <= ~110 KB of shared memory so
// two CTAs fit on an SM (split-K CTAs of one tile must be co-resident).
template <int BN> struct Stages { static constexpr int value = BN <= 16 ? 6 : (BN <= 32 ? 5 : (BN <= 64 ? 4 : 6)); };
static int ctas_per_sm(int bn) {
    static const int deep32 = [] { const char* e = getenv("FT2_GEMM_STAGES32"); return e ? atoi(e) : 0; }();
    if (bn == 32 && deep32 >= 8) return 1;
    return bn <= 64 ? 2 : 1;
}

static GemmPlan plan_gemm(int32_t M, int32_t N, int32_t K) {
    GemmPlan g;
    g.swap = M <= 128 ? 1 : 0;
    g.bn = g.swap ? (M <= 16 ? 16 : (M <= 32 ? 32 : (M <= 64 ? 64 : 128))) : 128;
    const int rowsA = g.swap ? N : M, rowsB = g.swap ? M : N;
    g.tilesA = (rowsA + kBlockA - 1) / kBlockA;
    g.tilesB = (rowsB + g.bn - 1) / g.bn;
    g.nkb = (K + kBlockK - 1) / kBlockK;
    const int tiles = g.tilesA * g.tilesB;
    const int sms = num_sms();
    const int capacity = sms * ctas_per_sm(g.bn);
    // Split K so the busiest SM streams as little of one tile's weights as
    // possible: load(sk) = ceil(tiles*sk / sms) / sk, with a small penalty per
    // split for the partial-tile traffic; all CTAs must be co-resident and keep
    // >= 2 k-blocks each.
    int best = 1;
    double best_cost = 1e30;
    for (int sk = 1; sk <= 16; ++sk) {
        if (sk > 1 && (tiles * sk > capacity || sk * 2 > g.nkb || tiles > kMaxSplitTiles)) break;
        const double load = (double)((tiles * sk + sms - 1) / sms) / sk;
        const double cost = load * (1.0 + 0.03 * sk);
        if (cost < best_cost - 1e-9) { best_cost = cost; best = sk; }
    }
    static const int sk_env = [] { const char* e = getenv("FT2_GEMM_SPLITK"); return e ? atoi(e) : 0; }();
    if (sk_env > 0) {
        best = sk_env < g.nkb ? sk_env : g.nkb;
        while (best > 1 && tiles * best > capacity) --best;
    }
    g.splitk = best;
    return g;
}

size_t gemm_ws_bytes(int32_t M, int32_t N, int32_t K) {
    if (M <= 0 || N <= 0 || K <= 0) return 0;
    GemmPlan g = plan_gemm(M, N, K);
    if (g.splitk <= 1) return 0;
    const size_t tiles = (size_t)g.tilesA * g.tilesB;
    return kCounterBytes + tiles * g.splitk * (size_t)g.bn * kBlockA * 4;
}

template <int BN, int STAGES>
static cudaError_t launch_cfg(const GemmArgs& a, GemmK p, cudaStream_t st, int* n_launch) {
    using L = GemmSmem<BN, STAGES>;
    CUtensorMap ma, mb;
    const void* pa = p.swap ? (const void*)a.w : (const void*)a.x;
    const void* pb = p.swap ? (const void*)a.x : (const void*)a.w;
    int64_t lda = p.swap ? a.ldw : a.ldx, ldb = p.swap ? a.ldx : a.ldw;
    if (!make_map(&ma, pa, p.rowsA, a.K, lda, kBlockA)) return cudaErrorInvalidValue;
    if (!make_map(&mb, pb, p.rowsB, a.K, ldb, BN)) return cudaErrorInvalidValue;
    static bool attr_set = false;  // per template instance
    if (!attr_set) {
        cudaError_t e = cudaFuncSetAttribute(gemm_kernel<BN, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             L::kBytes);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)p.tilesA, (unsigned)p.splitk, (unsigned)p.tilesB);
    cfg.blockDim = dim3(kGemmThreads);
    cfg.dynamicSmemBytes = L::kBytes;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, gemm_kernel<BN, STAGES>, ma, mb, p);
    ++*n_launch;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_gemm(const GemmArgs& a, cudaStream_t st, int* n_launch) {
    GemmPlan g = plan_gemm(a.M, a.N, a.K);
    GemmK p = {};
    p.M = a.M;
    p.N = a.N;
    p.K = a.K;
    p.swap = g.swap;
    p.rowsA = g.swap ? a.N : a.M;
    p.rowsB = g.swap ? a.M : a.N;
    p.tilesA = g.tilesA;
    p.tilesB = g.tilesB;
    p.splitk = g.splitk;
    p.nkb = g.nkb;
    p.mode = a.mode;
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
    p.w_static = a.w_static;
    if (g.splitk > 1) {
        uintptr_t base = reinterpret_cast<uintptr_t>(a.ws);
        p.tile_ctr = reinterpret_cast<uint32_t*>(base);
        uintptr_t part = base + kCounterBytes;
        p.partials = reinterpret_cast<float4*>(part);
    }
    switch (g.bn) {
        case 16: return launch_cfg<16, Stages<16>::value>(a, p, st, n_launch);
        case 32: {
            static const int st_env = [] { const char* e = getenv("FT2_GEMM_STAGES32"); return e ? atoi(e) : 0; }();
            if (st_env == 8) return launch_cfg<32, 8>(a, p, st, n_launch);
            if (st_env == 10) return launch_cfg<32, 10>(a, p, st, n_launch);
            return launch_cfg<32, Stages<32>::value>(a, p, st, n_launch);
        }
        case 64: return launch_cfg<64, Stages<64>::value>(a, p, st, n_launch);
        default: return launch_cfg<128, Stages<128>::value>(a, p, st, n_launch);
    }
}

}  // namespace ft2impl
