// gemm_sm100.cu -- critical linear layer with FT2's check fused into the
// epilogue, for sm_100a (tcgen05 MMA, TMEM accumulators, TMA pipeline).
//
//   y[m, j] = check(inject(bf16_rne(sum_k x[m, k] * w[j, k] + bias[j])))
//
// PAPER.md L259 ("Protection is applied after the execution of each critical
// layer"), L272 (clamp + nan_to_num applied right after the layer).  The check
// operates on the bf16-rounded value after bias (reading A19); a fault site is
// applied before the check (A20).
//
// One CTA = one 128 x BN output tile x one K slice, 192 threads:
//   warp 0     TMA producer: 128B-swizzled K-major tiles of A and B into a
//              STAGES-deep shared-memory ring (mbarrier full/empty).  With
//              programmatic dependent launch the first weight tiles are
//              requested before waiting for the previous kernel (opt-in).
//   warp 1     TMEM allocator + single-thread tcgen05.mma.cta_group::1.kind::f16
//              issuer (BF16 x BF16 -> FP32 in TMEM); tcgen05.commit frees a
//              stage and finally signals the epilogue.
//   warps 2-5  tcgen05.ld the accumulator (32x32b, one TMEM lane per thread)
//              and stage it as fp32 rows in shared memory.
//   all warps  finish the CTA's rows: bias -> RNE bf16 -> fault XOR ->
//              key-space check-and-clip (two values per 32-bit word, the same
//              order-key machinery as ft2_protect) -> store -> count.
// Split-K is a thread-block cluster (1, splitk, 1): CTA r owns rows
// [r0(r), r0(r+1)) of the tile; every CTA pushes each accumulator row into the
// owner's receive slot with st.async over DSMEM (completion counted on the
// owner's mbarrier): no global workspace, no fences, no spinning.  The owner
// sums the slots in fixed order 0..splitk-1 (deterministic) and clips only the
// complete K reduction (clipping is non-linear).
//
// Orientation: decode (M <= 128 tokens) runs "swap-AB": UMMA M = 128 walks
// output features (rows of W), UMMA N = BN walks tokens, so skinny activations
// still fill the tensor core; prefill (M > 128) uses A = x, B = w.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdio.h>
#include <stdlib.h>

#include <mutex>

#include "ft2_device.cuh"
#include "ft2_internal.h"
#include "sm100_ptx.cuh"

namespace ft2impl {
using namespace ft2dev;

constexpr int kBlockA = 128;  // UMMA M
constexpr int kBlockK = 64;   // one 128-byte swizzle atom of bf16
constexpr int kUmmaK = 16;
constexpr int kGemmThreads = 192;
constexpr int kMaxSitesPerCta = 64;
constexpr int kMaxSplitK = 16;        // cluster size along K (non-portable above 8)
constexpr int kMaxSplitPlanned = 12;  // largest split the planner picks (16-CTA clusters schedule slowly)

#ifdef FT2_GEMM_TRACE
// Debug builds only (lib/libft2_trace.so): per-CTA timestamps.
// 256 CTA rows per launch (GemmK::trace_base = 256 * (launch index mod 128))
__device__ unsigned long long g_trace[32768 * 16];
#define FT2_TRACE_ROWS 32768
__device__ __forceinline__ void trace(int slot, int base) {
    unsigned long long t;
#ifdef FT2_TRACE_CLOCK
    asm volatile("mov.u64 %0, %%clock64;" : "=l"(t));
#else
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
#endif
    const int cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
    if (cta < 256 && base + cta < FT2_TRACE_ROWS) g_trace[(base + cta) * 16 + slot] = t;
}
#define FT2_TRACE(slot) trace(slot, p.trace_base)
// slot 10 holds the SM id + 1 of the CTA (CTAs of one launch sharing an SM share its tensor pipe)
__device__ __forceinline__ void trace_smid(int base) {
    uint32_t sm;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    const int cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
    if (cta < 256 && base + cta < FT2_TRACE_ROWS) g_trace[(base + cta) * 16 + 10] = sm + 1u;
}
#define FT2_TRACE_SMID() trace_smid(p.trace_base)
static int g_trace_launch = 0;   // host: launches since the last ft2_debug_trace_reset
#else
#define FT2_TRACE(slot) ((void)0)
#define FT2_TRACE_SMID() ((void)0)
#endif

struct GemmK {
    int32_t M, N, K;
    int32_t rowsA, rowsB;  // extent of the A / B operands
    int32_t tilesA, tilesB;
    int32_t splitk, nkb;
    int32_t mode, col_begin, col_end;
    const uint16_t* bias;
    uint16_t* y;
    int64_t ldy;
    const int32_t* row_to_seq;
    int32_t S, row_mode;  // row_mode 0: row_to_seq[], 1: token m -> seq m, 2: all -> seq 0
    const uint16_t* bounds;
    uint32_t* counts;
    const ft2_fault_site* sites;
    int32_t n_sites, cur_layer, cur_step;
    const int32_t* base_row;
    int32_t w_static;  // weights not written by the preceding kernel: prefetch before the PDL wait
    int32_t trigger;   // where griddepcontrol.launch_dependents is issued (FT2_GEMM_TRIGGER, default 3; see below)
    int32_t w_l2;      // static weights: L2-prefetch the K slice beyond the ring before the PDL wait (FT2_GEMM_W_L2)
    int32_t rows_per_slot;  // ceil(BA / splitk): rows of one split-K receive slot
    uint32_t sk_magic;      // ceil(2^24 / splitk): floor(n / splitk) == (n * sk_magic) >> 24 for n < 2^20
    int32_t trace_base;     // trace builds only: first g_trace row of this launch
    // cA > 1: clusters (cA, splitk, 1) -- cA feature tiles of the same split
    // share each x box through a TMA multicast (whole K slice in the ring only)
    int32_t cA;
    const uint8_t* pf;      // L2 prefetch hint (the next layer's weights) and its size
    uint64_t pf_bytes;
    int32_t pf_at;          // 0: after this CTA issued its last load; 1: after its last stage landed
    // (host-side selector of the MMA2 instantiation; the kernel uses the template flag)
    // 1: two MMA issuers -- warp 1 and, once it has issued every load (whole K
    // slice in the ring), warp 0's producer thread -- each issuing half of
    // every stage's MMAs into its own accumulator (TMEM columns [0, BN) and
    // [cols, cols + BN)), summed in that order by the epilogue.  Measured: one
    // thread issues an M = 64 kind::f16 MMA every ~53 cycles, two warps
    // together one every ~35 (profiles/r2_mma_probe.txt)
    int32_t mma2;
};

// Per-row / per-column epilogue table entry.  Feature side: bias, flags
// bit0 = in range, bit1 = protected column (CHECK and inside [col_begin,
// col_end)).  Token side: keys = key(lo) | key(hi) << 16, seq, flags bit0 =
// in range, bit1 = has bounds (CHECK and a valid sequence).
struct TabE {
    float bias;
    uint32_t keys;
    int32_t seq;
    uint32_t flags;
};

template <int DT>
__device__ __forceinline__ TabE feature_entry(const GemmK& p, int n) {
    TabE e{0.f, 0u, -1, 0u};
    if (n < p.N) {
        e.flags = 1u;
        if (p.bias) e.bias = to_f32<DT>(p.bias[n]);
        if (p.mode == FT2_GEMM_CHECK && n >= p.col_begin && n < p.col_end) e.flags |= 2u;
    }
    return e;
}
__device__ __forceinline__ TabE token_entry(const GemmK& p, int m) {
    TabE e{0.f, 0u, -1, 0u};
    if (m < p.M) {
        e.flags = 1u;
        if (p.mode == FT2_GEMM_CHECK) {
            const int s = p.row_mode == 2 ? 0 : (p.row_mode == 1 ? m : p.row_to_seq[m]);
            if (s >= 0 && s < p.S) {
                e.keys = key2((uint32_t)p.bounds[2 * s] | ((uint32_t)p.bounds[2 * s + 1] << 16));
                e.seq = s;
                e.flags |= 2u;
            }
        }
    }
    return e;
}

// DEEP: one CTA per SM with a ring deep enough (~180 KB) that a CTA's whole K
// slice is in flight at once -- one DRAM round trip for few-tile decode
// shapes.  Otherwise ~105 KB so two CTAs share an SM.
// BA = UMMA M (output features per tile in swap-AB): 128, or 64 for few-tile
// decode shapes -- twice the tiles, so a split keeps a CTA's whole K slice in
// a ring that still fits two CTAs per SM, and half the split-K bytes per CTA.
template <int BA, int BN, bool DEEP = false>
struct Cfg {
    static_assert(BA == 128 || (BA == 64 && BN <= 32 && !DEEP), "BA = 64 serves 16/32-token tiles");
    static constexpr int STAGES = BA == 64 ? (BN <= 16 ? 9 : 8)
                                : DEEP ? (BN <= 16 ? 10 : (BN <= 32 ? 9 : 7))
                                       : (BN <= 16 ? 5 : (BN <= 32 ? 4 : (BN <= 64 ? 3 : 4)));
    static constexpr int kABytes = BA * kBlockK * 2;
    static constexpr int kBBytes = BN * kBlockK * 2;
    static constexpr int kStageBytes = kABytes + kBBytes;
    static constexpr int kTileBytes = STAGES * kStageBytes;
    // fp32 tile staging / split-K receive buffer: splitk slots x ceil(BA/splitk)
    // rows (< BA + 16 in total) x (BN + 4) fp32; the pad keeps float4 row reads
    // bank-conflict free
    static constexpr int kRecvStride = BN + 4;
    static constexpr int kRecvBytes = (BA + 16) * kRecvStride * 4;
    static constexpr int kMiscBytes = 1024;  // mbarriers, TMEM base, site list
    static constexpr int kTabBytes = (BA + BN) * (int)sizeof(TabE) + (BA + BN) * 4;
    static constexpr int kBytes = 1024 /*align slack*/ + kTileBytes + kRecvBytes + kMiscBytes + kTabBytes;
    static constexpr uint32_t kTmemCols = BN < 32 ? 32 : BN;
};

// XOR the fault masks of the sites that hit elements le0..le0+3 (rare: only
// fault-injection runs have sites).  Out of line to keep the epilogue small.
__device__ __noinline__ uint2 xor_sites(uint2 w, uint32_t le0, const uint32_t* site_e, const uint32_t* site_m,
                                        uint32_t nsite) {
    for (uint32_t i = 0; i < nsite; ++i) {
        const uint32_t d = site_e[i] - le0;
        if (d < 4u) {
            const uint32_t m = site_m[i] & 0xFFFFu;
            if (d == 0) w.x ^= m;
            else if (d == 1) w.x ^= m << 16;
            else if (d == 2) w.y ^= m;
            else w.y ^= m << 16;
        }
    }
    return w;
}

// Overflow path (more than kMaxSitesPerCta sites landed in this CTA's slice,
// e.g. a directed campaign): scan every site for the four elements of a quad
// -- slow, but no site is ever dropped.  SWAP: the quad is (feature ga,
// tokens gb0..gb0+3); otherwise (token ga, features gb0..gb0+3).
template <bool SWAP>
__device__ __noinline__ uint2 xor_sites_scan(uint2 w, const GemmK& p, int ga, int gb0) {
    for (int i = 0; i < p.n_sites; ++i) {
        const ft2_fault_site st = p.sites[i];
        if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
        const int64_t m = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) + (p.cur_step == 0 ? (int64_t)st.token : 0);
        const int64_t n = st.col;
        if (m < 0 || m >= p.M || n >= p.N) continue;
        const int64_t d = SWAP ? (n == ga ? m - gb0 : -1) : (m == ga ? n - gb0 : -1);
        if (d < 0 || d >= 4) continue;
        const uint32_t msk = st.xor_mask & 0xFFFFu;
        if (d == 0) w.x ^= msk;
        else if (d == 1) w.x ^= msk << 16;
        else if (d == 2) w.y ^= msk;
        else w.y ^= msk << 16;
    }
    return w;
}

// Sum of the NS split-K slots of one float4 (slot r at src + r * step floats),
// in slot order 0..NS-1 (the same order as the generic loop: bit-identical).
template <int NS>
__device__ __forceinline__ float4 sum_slots(const float* src, int step) {
    float4 part[NS];
#pragma unroll
    for (int r = 0; r < NS; ++r) part[r] = *reinterpret_cast<const float4*>(src + r * step);
    float4 acc = part[0];
#pragma unroll
    for (int r = 1; r < NS; ++r) { acc.x += part[r].x; acc.y += part[r].y; acc.z += part[r].z; acc.w += part[r].w; }
    return acc;
}

// Any other split factor, out of line (kept off the common path's code size).
__device__ __noinline__ float4 sum_slots_any(const float* src, int step, int splitk) {
    float4 part[kMaxSplitK];
#pragma unroll
    for (int r = 0; r < kMaxSplitK; ++r)
        if (r < splitk) part[r] = *reinterpret_cast<const float4*>(src + r * step);
    float4 acc = part[0];
#pragma unroll
    for (int r = 1; r < kMaxSplitK; ++r)
        if (r < splitk) { acc.x += part[r].x; acc.y += part[r].y; acc.z += part[r].z; acc.w += part[r].w; }
    return acc;
}

// The fault sites that land in this CTA's slice (rows [r0, r1) of the tile at
// (a0, b0)), gathered into the shared-memory site list (sites beyond
// kMaxSitesPerCta only raise the count: finish4 then rescans every site).
// Out of line: only fault-injection runs pass sites.
template <bool SWAP>
__device__ __noinline__ void gather_sites(const GemmK& p, int e, int a0, int b0, int BA, int BN, int r0, int r1,
                                          uint32_t* site_n, uint32_t* site_e, uint32_t* site_m) {
    for (int i = e; i < p.n_sites; i += 128) {
        const ft2_fault_site st = p.sites[i];
        if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
        const int64_t m = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) + (p.cur_step == 0 ? (int64_t)st.token : 0);
        const int64_t n = st.col;
        if (m < 0 || m >= p.M || n >= p.N) continue;
        const int64_t la = (SWAP ? n : m) - (int64_t)a0;
        const int64_t lb = (SWAP ? m : n) - (int64_t)b0;
        if (la < r0 || la >= r1 || lb < 0 || lb >= BN) continue;
        const uint32_t idx = atomicAdd(site_n, 1u);
        if (idx < (uint32_t)kMaxSitesPerCta) {
            site_e[idx] = (uint32_t)(la * BN + lb);
            site_m[idx] = st.xor_mask;
        }
    }
}

// Check-and-clip of two packed bf16 (R5): NaN -> key(+0), clamp in key space.
template <int DT>
__device__ __forceinline__ uint32_t clip2_nocount(uint32_t w, uint32_t kL2, uint32_t kH2) {
    const uint32_t k = key2(w);
    const uint32_t nm = half_sign_mask(nan_bits2<DT>(w));
    const uint32_t kz = (k & ~nm) | (0x80008000u & nm);
    return unkey2(vmax_u16x2(vmin_u16x2(kz, kH2), kL2));
}

// Finish four consecutive columns c0..c0+3 of tile row la.
template <bool SWAP, int DT>
__device__ __forceinline__ void finish4(uint16_t* __restrict__ y, int64_t ldy, int ga, int gb0, const TabE& re,
                                        const TabE* __restrict__ ce, uint32_t le0, float4 acc,
                                        const uint32_t* site_e, const uint32_t* site_m, uint32_t nsite,
                                        uint32_t* row_cnt, uint32_t* col_cnt, const GemmK& p) {
    // feature side: SWAP ? the row : the column; token side: the other one
    const float b0 = SWAP ? re.bias : ce[0].bias, b1 = SWAP ? re.bias : ce[1].bias;
    const float b2 = SWAP ? re.bias : ce[2].bias, b3 = SWAP ? re.bias : ce[3].bias;
    uint2 w = make_uint2((uint32_t)rne16<DT>(acc.x + b0) | ((uint32_t)rne16<DT>(acc.y + b1) << 16),
                         (uint32_t)rne16<DT>(acc.z + b2) | ((uint32_t)rne16<DT>(acc.w + b3) << 16));
    if (nsite > (uint32_t)kMaxSitesPerCta) w = xor_sites_scan<SWAP>(w, p, ga, gb0);
    else if (nsite) w = xor_sites(w, le0, site_e, site_m, nsite);
    uint32_t f[4], kL01, kH01, kL23, kH23;
#pragma unroll
    for (int j = 0; j < 4; ++j) f[j] = re.flags & ce[j].flags;  // bit0 valid, bit1 checked
    if (SWAP) {
        kL01 = (ce[0].keys & 0xFFFFu) | (ce[1].keys << 16);
        kH01 = (ce[0].keys >> 16) | (ce[1].keys & 0xFFFF0000u);
        kL23 = (ce[2].keys & 0xFFFFu) | (ce[3].keys << 16);
        kH23 = (ce[2].keys >> 16) | (ce[3].keys & 0xFFFF0000u);
    } else {
        kL01 = kL23 = (re.keys & 0xFFFFu) * 0x10001u;
        kH01 = kH23 = (re.keys >> 16) * 0x10001u;
    }
    const uint32_t m01 = ((f[0] & 2u) ? 0x0000FFFFu : 0u) | ((f[1] & 2u) ? 0xFFFF0000u : 0u);
    const uint32_t m23 = ((f[2] & 2u) ? 0x0000FFFFu : 0u) | ((f[3] & 2u) ? 0xFFFF0000u : 0u);
    const uint32_t o01 = (clip2_nocount<DT>(w.x, kL01, kH01) & m01) | (w.x & ~m01);
    const uint32_t o23 = (clip2_nocount<DT>(w.y, kL23, kH23) & m23) | (w.y & ~m23);
    const uint32_t d01 = o01 ^ w.x, d23 = o23 ^ w.y;
    const uint16_t o[4] = {(uint16_t)o01, (uint16_t)(o01 >> 16), (uint16_t)o23, (uint16_t)(o23 >> 16)};
    if (SWAP) {
        uint16_t* dst = y + (int64_t)gb0 * ldy + ga;
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (f[j] & 1u) dst[(int64_t)j * ldy] = o[j];
    } else {
        uint16_t* dst = y + (int64_t)ga * ldy + gb0;
        if ((f[0] & f[1] & f[2] & f[3] & 1u) && ((reinterpret_cast<uintptr_t>(dst) & 7u) == 0)) {
            *reinterpret_cast<uint2*>(dst) = make_uint2(o01, o23);
        } else {
#pragma unroll
            for (int j = 0; j < 4; ++j)
                if (f[j] & 1u) dst[j] = o[j];
        }
    }
    if (d01 | d23) {  // corrected neurons, aggregated per CTA in shared memory
        const uint32_t ch[4] = {d01 & 0xFFFFu, d01 >> 16, d23 & 0xFFFFu, d23 >> 16};
#pragma unroll
        for (int j = 0; j < 4; ++j)
            if (ch[j] && (f[j] & 1u)) atomicAdd_block(SWAP ? &col_cnt[j] : row_cnt, 1u);
    }
}

template <int BA, int BN, bool SWAP, int DT, bool DEEP, bool MMA2 = false>
__global__ void __launch_bounds__(kGemmThreads, 1)
    gemm_kernel(const __grid_constant__ CUtensorMap map_a, const __grid_constant__ CUtensorMap map_b,
                const __grid_constant__ GemmK p) {
    using C = Cfg<BA, BN, DEEP>;
    constexpr int STAGES = C::STAGES;
    extern __shared__ uint8_t smem_raw[];
    // 1024-byte alignment (128B swizzle) by offset arithmetic on the shared
    // array, so the compiler keeps the shared address space (LDS/STS)
    uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
    uint8_t* tiles = smem;
    float* recv = reinterpret_cast<float*>(smem + C::kTileBytes);
    uint8_t* misc = smem + C::kTileBytes + C::kRecvBytes;
    uint64_t* full = reinterpret_cast<uint64_t*>(misc);
    uint64_t* empty = full + STAGES;
    uint64_t* tmem_full = empty + STAGES;
    uint64_t* recv_bar = tmem_full + 1;
    uint32_t* tmem_base_sh = reinterpret_cast<uint32_t*>(recv_bar + 1);
    uint32_t* site_n = tmem_base_sh + 1;
    uint32_t* site_e = site_n + 1;                // [kMaxSitesPerCta] local element a * BN + b
    uint32_t* site_m = site_e + kMaxSitesPerCta;  // [kMaxSitesPerCta] xor mask
    TabE* row_tab = reinterpret_cast<TabE*>(misc + C::kMiscBytes);  // [BA]
    TabE* col_tab = row_tab + BA;                                     // [BN]
    uint32_t* row_cnt = reinterpret_cast<uint32_t*>(col_tab + BN);    // [BA]
    uint32_t* col_cnt = row_cnt + BA;                                 // [BN]

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int tileA = blockIdx.x, split = blockIdx.y, tileB = blockIdx.z;
    const int splitk = p.splitk;
    const int kb0 = (int)((int64_t)split * p.nkb / splitk);
    const int kb1 = (int)((int64_t)(split + 1) * p.nkb / splitk);
    const int nk = kb1 - kb0;
    // rows of the tile this CTA finishes: all of them, or its split-K slice
    const bool cs = splitk > 1;   // split across the cluster (DSMEM)
    const int r0 = (int)(((uint32_t)(split * BA) * p.sk_magic) >> 24);
    const int r1 = (int)(((uint32_t)((split + 1) * BA) * p.sk_magic) >> 24);

    if (warp == 0 && lane == 0) {
        FT2_TRACE(0);
        FT2_TRACE_SMID();
        prefetch_tmap(&map_a);
        prefetch_tmap(&map_b);
        for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
        mbar_init(tmem_full, MMA2 ? 2u : 1u);
        mbar_init(recv_bar, 1);
        if (cs)  // bytes the other splits will push into my slice
            mbar_expect_tx(recv_bar, (uint32_t)((splitk - 1) * (r1 - r0) * BN * 4));
        fence_mbar_init();
        *site_n = 0;
        if (p.w_static) {
            // static weights: the first stages' weight tiles are requested right
            // here, before the TMEM allocation and the CTA barrier, so the DRAM
            // latency of the first bytes overlaps the prologue (x waits for the
            // PDL wait below; each stage's barrier expects both boxes)
            const int pre = nk < STAGES ? nk : STAGES;
            for (int i = 0; i < pre; ++i) {
                mbar_expect_tx(&full[i], C::kStageBytes);
                tma_load_2d(SWAP ? &map_a : &map_b, &full[i], tiles + i * C::kStageBytes + (SWAP ? 0 : C::kABytes),
                            (kb0 + i) * kBlockK, SWAP ? tileA * BA : tileB * BN);
            }
            // ... and the rest of this CTA's weight slice is pulled into L2
            // right away (no shared memory needed), so the whole layer
            // streams from HBM while this kernel still waits for its
            // activations; the ring's later loads then hit L2
            if (p.w_l2) {   // one more ring's worth (w_l2 1), or the whole slice (w_l2 2: layers that fit L2 easily)
                const int lim = (p.w_l2 >= 2 || nk < pre + STAGES) ? nk : pre + STAGES;
                for (int i = pre; i < lim; ++i)
                    tma_prefetch_l2_2d(SWAP ? &map_a : &map_b, (kb0 + i) * kBlockK, SWAP ? tileA * BA : tileB * BN);
            }
        }
    }
    if (warp == 1) tmem_alloc(tmem_base_sh, (MMA2 ? 2u : 1u) * C::kTmemCols);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    // the next kernel in the stream may start its prologue (PDL): right here
    // (trigger 1), once this CTA's operands are all consumed (trigger 2, by
    // the MMA thread below), or -- the default -- once the MMA thread has
    // issued half of the CTA's k-blocks (trigger 3).  A later trigger keeps the
    // next launch's early weight requests off the L2 -> SM path while this
    // launch's x boxes (its critical path after the wait) stream in; measured
    // back to back (profiles/r2_trigger_ab.txt): OPT graph 6.17 / 6.03 / 5.94 us
    // per launch for 1 / 2 / 3, 2048x2048 4.59 / 4.43 / 4.20; in situ (a host
    // kernel before every critical GEMM) all three equal
    if (p.trigger == 1) griddep_launch();
    // peers may push into my receive buffer once my barrier is initialised
    const int cA = p.cA, rA = (int)(blockIdx.x % (unsigned)cA);
    const bool mc = cA > 1;   // x multicast: every peer's barriers must exist before the first box
    if (mc) {
        cluster_arrive_relaxed();
        cluster_wait();
    } else if (cs) {
        cluster_arrive_relaxed();
    }
    const uint32_t tmem_base = *tmem_base_sh;

    if (warp == 0) {
        if (lane == 0) {
            // ------------------------------------------------ TMA producer
            const CUtensorMap* mw = SWAP ? &map_a : &map_b;
            const CUtensorMap* mx = SWAP ? &map_b : &map_a;
            const int w_row = SWAP ? tileA * BA : tileB * BN;
            const int x_row = SWAP ? tileB * BN : tileA * BA;
            const int w_off = SWAP ? 0 : C::kABytes;
            const int x_off = SWAP ? C::kABytes : 0;
            FT2_TRACE(1);
            const int pre = nk < STAGES ? nk : STAGES;
            if (!p.w_static) {   // (static weights were requested in the prologue)
                griddep_wait();
                for (int i = 0; i < pre; ++i) {
                    mbar_expect_tx(&full[i], C::kStageBytes);
                    tma_load_2d(mw, &full[i], tiles + i * C::kStageBytes + w_off, (kb0 + i) * kBlockK, w_row);
                }
            } else {
                griddep_wait();
            }
            FT2_TRACE(2);
            if (mc) {   // one CTA of each cA group issues a box for all of them (nk <= STAGES)
                const uint16_t mask = (uint16_t)(((1u << cA) - 1u) << (split * cA));
                for (int i = rA; i < pre; i += cA)
                    tma_load_2d_mc(mx, &full[i], tiles + i * C::kStageBytes + x_off, (kb0 + i) * kBlockK, x_row, mask);
            } else {
                for (int i = 0; i < pre; ++i)
                    tma_load_2d(mx, &full[i], tiles + i * C::kStageBytes + x_off, (kb0 + i) * kBlockK, x_row);
            }
            for (int i = STAGES; i < nk; ++i) {
                const int s = i % STAGES;
                mbar_wait(&empty[s], ((uint32_t)(i / STAGES) & 1u) ^ 1u);
                uint8_t* st = tiles + s * C::kStageBytes;
                mbar_expect_tx(&full[s], C::kStageBytes);
                tma_load_2d(mw, &full[s], st + w_off, (kb0 + i) * kBlockK, w_row);
                tma_load_2d(mx, &full[s], st + x_off, (kb0 + i) * kBlockK, x_row);
            }
            if constexpr (MMA2) {
                // second MMA issuer (the host sets mma2 only when nk <= STAGES:
                // no stage is ever refilled, so no stage release is needed):
                // the upper half of every stage's K16 steps into accumulator 1
                constexpr uint32_t idesc2 =
                    (make_idesc(BA, BN) & ~((7u << 7) | (7u << 10))) | ((DT == 1 ? 0u : 1u) * ((1u << 7) | (1u << 10)));
                for (int i = 0; i < nk; ++i) {
                    const int s = i % STAGES;
                    mbar_wait(&full[s], (uint32_t)(i / STAGES) & 1u);
                    tc_fence_after();
                    const uint32_t sa = smem_u32(tiles + s * C::kStageBytes);
                    const uint64_t da = make_sdesc(sa), db = make_sdesc(sa + C::kABytes);
#pragma unroll
                    for (int k = kBlockK / kUmmaK / 2; k < kBlockK / kUmmaK; ++k)
                        tc_mma(tmem_base + C::kTmemCols, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc2,
                               (i > 0 || k > kBlockK / kUmmaK / 2) ? 1u : 0u);
                }
                tc_commit(tmem_full);
            }
            if (p.pf_bytes) {
                // L2 prefetch hint: this CTA's 1/grid share of the next
                // layer's bytes, once its own loads are issued (pf_at 0) or
                // have landed (pf_at 1), so the prefetch does not compete
                // with this kernel's critical-path loads
                if (p.pf_at && nk > 0) {
                    const int last = nk - 1;
                    mbar_wait(&full[last % STAGES], (uint32_t)(last / STAGES) & 1u);
                }
                const uint32_t ncta = gridDim.x * gridDim.y * gridDim.z;
                const uint32_t cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
                const uint64_t chunk = ((p.pf_bytes + ncta - 1) / ncta + 255) & ~(uint64_t)255;
                const uint64_t beg = (uint64_t)cta * chunk;
                const uint64_t end = beg + chunk < p.pf_bytes ? beg + chunk : p.pf_bytes;
                for (uint64_t off = beg; off < end; off += 65536)
                    bulk_prefetch_l2(p.pf + off, (uint32_t)(end - off < 65536 ? end - off : 65536));
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            // ------------------------------------------------ MMA issuer
            // kind::f16 operand format: 0 = F16, 1 = BF16 (bits 7-9 A, 10-12 B)
            constexpr uint32_t idesc =
                (make_idesc(BA, BN) & ~((7u << 7) | (7u << 10))) | ((DT == 1 ? 0u : 1u) * ((1u << 7) | (1u << 10)));
            for (int i = 0; i < nk; ++i) {
                const int s = i % STAGES;
                mbar_wait(&full[s], (uint32_t)(i / STAGES) & 1u);
                if (i == 0) FT2_TRACE(3);
                if (i == 1) FT2_TRACE(12);
                if (i == nk - 1) FT2_TRACE(13);
                tc_fence_after();
                const uint32_t sa = smem_u32(tiles + s * C::kStageBytes);
                const uint64_t da = make_sdesc(sa), db = make_sdesc(sa + C::kABytes);
                if constexpr (MMA2) {   // the lower half of the stage's K16 steps (the producer issues the rest)
#pragma unroll
                    for (int k = 0; k < kBlockK / kUmmaK / 2; ++k)
                        tc_mma(tmem_base, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc, (i > 0 || k > 0) ? 1u : 0u);
                } else {
#pragma unroll
                    for (int k = 0; k < kBlockK / kUmmaK; ++k)  // 16 elements = 32 B along K per MMA
                        tc_mma(tmem_base, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc,
                               (i > 0 || k > 0) ? 1u : 0u);
                }
                if (p.trigger == 3 && i == (nk - 1) / 2) griddep_launch();   // mid-stream trigger (default)
                if (p.trigger >= 10 && i == (nk - 1) * (p.trigger - 10) / 8) griddep_launch();   // experiment: eighths
                // release the stage only if the producer will refill it: a
                // commit costs the issuing thread ~300 cycles (measured), and
                // with the whole K slice in the ring none is ever refilled
                if (i + STAGES < nk) tc_commit(&empty[s]);
            }
            tc_commit(tmem_full);
            if (p.trigger == 2) griddep_launch();
            FT2_TRACE(4);
        }
    } else {
        // ---------------------------------------------------- epilogue warps
        const int q = warp & 3;  // TMEM lane quarter this warp may access
        const int e = tid - 64;  // 0..127
        // Accumulator row a of this thread.  BA = 128: TMEM lane 32q + lane
        // holds row 32q + lane.  BA = 64 (cta_group::1, M = 64): rows 16q..16q+15
        // sit in lanes 32q..32q+15 of the warp's quarter; lanes 16-31 hold none.
        const int a = BA == 128 ? q * 32 + lane : q * 16 + (lane & 15);
        const bool has_row = BA == 128 || lane < 16;
        griddep_wait();  // bias/bounds/sites/y may belong to the previous kernel

        // epilogue tables, gathered while the main loop still streams
        for (int r = e; r < BA; r += 128) {
            row_tab[r] = SWAP ? feature_entry<DT>(p, tileA * BA + r) : token_entry(p, tileA * BA + r);
            row_cnt[r] = 0u;
        }
        for (int c = e; c < BN; c += 128) {
            col_tab[c] = SWAP ? token_entry(p, tileB * BN + c) : feature_entry<DT>(p, tileB * BN + c);
            col_cnt[c] = 0u;
        }
        if (p.sites != nullptr)  // fault sites landing in my slice (out of line: campaign runs only)
            gather_sites<SWAP>(p, e, tileA * BA, tileB * BN, BA, BN, r0, r1, site_n, site_e, site_m);
        // Receive-slot geometry of accumulator row a (independent of the
        // accumulator, so computed while the main loop streams): its owner
        // is the split whose row slice holds a, r0(r) = floor(BA r / splitk)
        // evaluated as (BA r * sk_magic) >> 24 (exact for these ranges).
        const int RS = p.rows_per_slot;
        const int owner = ((a + 1) * splitk - 1) / BA;
        const int own_r0 = (int)(((uint32_t)(owner * BA) * p.sk_magic) >> 24);
        const uint32_t slot_off = (uint32_t)(((split * RS + (a - own_r0)) * C::kRecvStride) * 4);
        const bool local = owner == split;
        const uint32_t owner_rank = (uint32_t)(rA + owner * cA);   // cluster rank of my row's owner
        const uint32_t dst = local ? smem_u32(recv) + slot_off : mapa(smem_u32(recv) + slot_off, owner_rank);
        const uint32_t dbar = local ? 0u : mapa(smem_u32(recv_bar), owner_rank);
        const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16);
        // finish-loop geometry: item v -> (row lr, column quad c4)
        const int nrow = r1 - r0;
        const int nvec = nrow * (BN / 4);
        const uint32_t inv = (uint32_t)((1u << 20) + nrow - 1) / (uint32_t)nrow;  // v / nrow == (v * inv) >> 20
        // kernel parameters the finish needs, loaded while the main loop
        // streams and kept in registers (the empty asm stops the compiler
        // from re-reading them from the constant bank on the critical path)
        uint16_t* y = p.y;
        int64_t ldy = p.ldy;
        uint32_t* counts = (p.counts != nullptr && p.mode == FT2_GEMM_CHECK) ? p.counts : nullptr;
        asm volatile("" : "+l"(y), "+l"(ldy), "+l"(counts));
        if (cs && !mc) cluster_wait();  // every peer's receive barrier is initialised
        mbar_wait(tmem_full, 0);
        if (e == 0) FT2_TRACE(5);
        tc_fence_after();
        // Stage accumulator row a as fp32 in the receive slot of its owner
        // (this CTA without split-K; a cluster peer with it).  The TMEM loads
        // are warp-collective: every lane issues them, rowless lanes drop the data.
        if constexpr (BN == 32) {  // one TMEM load for the whole row, then the pushes back to back
            uint32_t r[32];
            tmem_ld32(taddr, r);
            if constexpr (MMA2) {   // + the second issuer's accumulator (fixed order: deterministic)
                uint32_t r2[32];
                tmem_ld32(taddr + C::kTmemCols, r2);
                tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 32; ++j) r[j] = __float_as_uint(__uint_as_float(r[j]) + __uint_as_float(r2[j]));
            }
            tmem_wait_ld();
            if (e == 0) FT2_TRACE(14);
            if (nk == 0) {
#pragma unroll
                for (int j = 0; j < 32; ++j) r[j] = 0u;
            }
            if (has_row) {
#pragma unroll
                for (int j = 0; j < 32; j += 4) {
                    if (local) st_shared_v4(dst + (uint32_t)(j * 4), r[j], r[j + 1], r[j + 2], r[j + 3]);
                    else st_async_v4(dst + (uint32_t)(j * 4), r[j], r[j + 1], r[j + 2], r[j + 3], dbar);
                }
            }
        } else
#pragma unroll 1
        for (int c0 = 0; c0 < BN; c0 += 16) {
            uint32_t r[16];
            tmem_ld16(taddr + c0, r);
            if constexpr (MMA2) {
                uint32_t r2[16];
                tmem_ld16(taddr + C::kTmemCols + c0, r2);
                tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 16; ++j) r[j] = __float_as_uint(__uint_as_float(r[j]) + __uint_as_float(r2[j]));
            }
            tmem_wait_ld();
            if (e == 0 && c0 == 0) FT2_TRACE(14);
            if (nk == 0) {
#pragma unroll
                for (int j = 0; j < 16; ++j) r[j] = 0u;
            }
            if (has_row) {
#pragma unroll
                for (int j = 0; j < 16; j += 4) {
                    if (local) st_shared_v4(dst + (uint32_t)((c0 + j) * 4), r[j], r[j + 1], r[j + 2], r[j + 3]);
                    else st_async_v4(dst + (uint32_t)((c0 + j) * 4), r[j], r[j + 1], r[j + 2], r[j + 3], dbar);
                }
            }
        }
        if (tid == 64) FT2_TRACE(8);
        // ------------------------------------ finish the slice (epilogue warps)
        named_bar(2, 128);  // tables, site list and my own rows are in shared memory
        if (tid == 64) FT2_TRACE(9);
        if (cs) mbar_wait(recv_bar, 0);  // ... and every peer's rows of my slice
        if (tid == 64) FT2_TRACE(6);
        const uint32_t nsite = *site_n;   // > kMaxSitesPerCta: finish4 scans every site
        if (tid == 64) FT2_TRACE(15);     // (trace builds: the site count read)
#pragma unroll 1
        for (int v = e; v < nvec; v += 128) {
            // consecutive threads take consecutive rows (coalesced stores in swap-AB mode)
            const int c4 = (int)(((uint32_t)v * inv) >> 20), lr = v - c4 * nrow, la = r0 + lr;
            const float* src = recv + lr * C::kRecvStride + c4 * 4;
            float4 acc;
            if (splitk == 4) {   // the common split factors: every slot read issued before the sum
                acc = sum_slots<4>(src, RS * C::kRecvStride);
            } else if (splitk == 8) {
                acc = sum_slots<8>(src, RS * C::kRecvStride);
            } else {
                acc = sum_slots_any(src, RS * C::kRecvStride, splitk);
            }
            if (tid == 64) FT2_TRACE(11);
            finish4<SWAP, DT>(y, ldy, tileA * BA + la, tileB * BN + c4 * 4, row_tab[la], col_tab + c4 * 4,
                              (uint32_t)(la * BN + c4 * 4), acc, site_e, site_m, nsite, row_cnt + la, col_cnt + c4 * 4, p);
        }
        if (tid == 64) FT2_TRACE(7);
        if (counts != nullptr) {
            named_bar(3, 128);  // every finish4 of this CTA has counted
            if (!SWAP && e < BA && row_cnt[e] != 0u) atomicAdd(&counts[row_tab[e].seq], row_cnt[e]);
            for (int c = e; SWAP && c < BN; c += 128)
                if (col_cnt[c] != 0u) atomicAdd(&counts[col_tab[c].seq], col_cnt[c]);
        }
    }
    // warps 0 and 1 pair their prologue cluster arrive (no finish work for them)
    if (cs && !mc && warp < 2) cluster_wait();
    tc_fence_before();
    __syncthreads();
    if (warp == 1) {
        tc_fence_after();
        tmem_dealloc(tmem_base, (MMA2 ? 2u : 1u) * C::kTmemCols);
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

static bool make_map(CUtensorMap* m, const void* base, int64_t rows, int64_t K, int64_t ld, int box_rows,
                     int dtype) {
    auto enc = get_encode();
    if (!enc) return false;
    cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)(ld * 2)};
    cuuint32_t box[2] = {(cuuint32_t)kBlockK, (cuuint32_t)box_rows};
    cuuint32_t es[2] = {1, 1};
    CUresult r = enc(m, dtype == FT2_FP16 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT16 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, es,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

// Experiment knobs (read once): FT2_GEMM_SMEM_PAD adds dynamic shared memory
// (fewer CTAs per SM), FT2_GEMM_SPREAD=1 asks for the spread cluster policy.
static int smem_pad() {
    static const int v = [] { const char* e = getenv("FT2_GEMM_SMEM_PAD"); return e ? atoi(e) : 0; }();
    return v;
}
static int env_int(const char* name, int dflt) {
    const char* e = getenv(name);
    return e ? atoi(e) : dflt;
}
static int spread_policy() {
    static const int v = [] { const char* e = getenv("FT2_GEMM_SPREAD"); return e ? atoi(e) : 0; }();
    return v;
}

template <int BA, int BN, bool SWAP, int DT, bool DEEP, bool MMA2 = false>
static cudaError_t set_attrs() {
    static cudaError_t res = [] {
        auto* k = gemm_kernel<BA, BN, SWAP, DT, DEEP, MMA2>;
        cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                             Cfg<BA, BN, DEEP>::kBytes + smem_pad());
        if (e == cudaSuccess) e = cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        // full shared-memory carveout so two ~105 KB decode CTAs share an SM
        if (e == cudaSuccess && env_int("FT2_GEMM_CARVEOUT", 1))
            e = cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout,
                                     (int)cudaSharedmemCarveoutMaxShared);
        return e;
    }();
    return res;
}

// How many (1, sk, 1) clusters of this instantiation can be resident at once.
template <int BA, int BN, bool SWAP, int DT = 0, bool DEEP = false>
static int max_clusters(int sk) {
    static int cache[kMaxSplitK + 1] = {0};
    if (sk < 1 || sk > kMaxSplitK) return -1;
    if (cache[sk] != 0) return cache[sk];
    if (set_attrs<BA, BN, SWAP, DT, DEEP>() != cudaSuccess) return cache[sk] = -1;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(1, (unsigned)sk, 1);
    cfg.blockDim = dim3(kGemmThreads);
    cfg.dynamicSmemBytes = Cfg<BA, BN, DEEP>::kBytes + smem_pad();
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1;
    attr[0].val.clusterDim.y = (unsigned)sk;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int n = 0;
    if (cudaOccupancyMaxActiveClusters(&n, gemm_kernel<BA, BN, SWAP, DT, DEEP>, &cfg) != cudaSuccess) {
        cudaGetLastError();
        n = -1;
    }
    return cache[sk] = (n > 0 ? n : -1);
}

static int max_clusters_bn(int bn, int sk, bool deep = false) {
    if (deep) {
        switch (bn) {
            case 16: return max_clusters<128, 16, true, 0, true>(sk);
            case 32: return max_clusters<128, 32, true, 0, true>(sk);
            case 64: return max_clusters<128, 64, true, 0, true>(sk);
            default: return -1;
        }
    }
    switch (bn) {
        case 16: return max_clusters<128, 16, true>(sk);
        case 32: return max_clusters<128, 32, true>(sk);
        case 64: return max_clusters<128, 64, true>(sk);
        default: return max_clusters<128, 128, true>(sk);
    }
}
static int deep_stages(int bn) {
    switch (bn) {
        case 16: return Cfg<128, 16, true>::STAGES;
        case 32: return Cfg<128, 32, true>::STAGES;
        case 64: return Cfg<128, 64, true>::STAGES;
        default: return 0;
    }
}

// Tiling plan: orientation, feature-tile height BA, token-tile width, split-K factor.
struct GemmPlan {
    int swap, ba, bn, tilesA, tilesB, splitk, nkb, deep, cA;
};

// 64-row feature tiles (UMMA M = 64) for decode batches of <= 32 tokens:
// FT2_GEMM_BA = 64 / 128 forces the choice; 0 = the planner's rule below.
static bool use_ba64(int32_t M, int32_t N, int32_t K) {
    static const int ba_env = env_int("FT2_GEMM_BA", 0);
    if (M > 32) return false;
    if (ba_env == 64) return true;
    if (ba_env == 128) return false;
    // measured (C3 / OPT shapes, profiles/r2_gemm_ba64.txt): better at
    // N, K <= 4096 (Llama v/o 9.1 -> 8.9 us); worse at N = 11008 (18.2 -> 21.1)
    // (also N <= 2048 at any K, i.e. OPT fc2: back to back 7.06 vs 6.90 us per
    // launch, in situ within noise -- not taken)
    return N <= 4096 && K <= 4096;
}

// Largest token count that runs swap-AB on this kernel (BN = 128 token tiles
// above 64); larger M goes to the persistent prefill kernel.
static int swap_max_m() {
    static const int v = [] { const char* e = getenv("FT2_GEMM_SWAP_MAX"); return e ? atoi(e) : 128; }();
    return v;
}

static GemmPlan plan_gemm_impl(int32_t M, int32_t N, int32_t K, bool force64 = false) {
    GemmPlan g;
    g.swap = M <= swap_max_m() ? 1 : 0;
    g.ba = 128;
    g.cA = 1;
    static const int sk_env0 = env_int("FT2_GEMM_SPLITK", 0);
    if (g.swap && (force64 || use_ba64(M, N, K))) {
        // the smallest split whose K slice fits the ring (one DRAM round trip,
        // weights requested before the PDL wait), at most 2 CTAs per SM and
        // clusters of <= 8; large K keeps streaming at the largest such split
        g.ba = 64;
        g.bn = M <= 16 ? 16 : 32;
        g.deep = 0;
        g.tilesA = (N + 63) / 64;
        g.tilesB = (M + g.bn - 1) / g.bn;
        g.nkb = (K + kBlockK - 1) / kBlockK;
        const int st = g.bn <= 16 ? Cfg<64, 16>::STAGES : Cfg<64, 32>::STAGES;
        const int tiles = g.tilesA * g.tilesB;
        int sk = 1;
        static const int cap64 = env_int("FT2_GEMM_CTA_CAP", 2 * num_sms());   // experiment: CTAs per launch
        while (sk < 8 && (g.nkb + sk - 1) / sk > st && tiles * (sk + 1) <= cap64 && g.nkb >= 2 * (sk + 1)) ++sk;
        if (sk_env0 > 0) sk = sk_env0 < g.nkb ? sk_env0 : g.nkb;
        if (sk > kMaxSplitK) sk = kMaxSplitK;
        g.splitk = sk;
        // x multicast across 2 feature tiles (clusters (2, splitk)) when the
        // whole K slice sits in the ring: measured no faster (the late stages
        // wait for weights, not x; profiles/r2_gemm_ba64.txt) -- FT2_GEMM_XMC=1
        static const int xmc = env_int("FT2_GEMM_XMC", 0);
        g.cA = (xmc && (g.nkb + sk - 1) / sk <= st && g.tilesA % 2 == 0 && 2 * sk <= 8) ? 2 : 1;
        return g;
    }
    g.bn = g.swap ? (M <= 16 ? 16 : (M <= 32 ? 32 : (M <= 64 ? 64 : 128))) : 128;
    static const int bn_env = env_int("FT2_GEMM_BN", 0);   // experiment: force the token-tile width
    if (g.swap && (bn_env == 16 || bn_env == 32 || bn_env == 64)) g.bn = bn_env;
    const int rowsA = g.swap ? N : M, rowsB = g.swap ? M : N;
    g.tilesA = (rowsA + kBlockA - 1) / kBlockA;   // (BA = 128 from here on)
    g.tilesB = (rowsB + g.bn - 1) / g.bn;
    g.nkb = (K + kBlockK - 1) / kBlockK;
    const int tiles = g.tilesA * g.tilesB;
    const int sms = num_sms();
    // Decode (swap-AB) shapes have few tiles (N/128): split K across a cluster
    // so that every SM streams weights.  Measured on B200 (tools/
    // sweep_splitk.sh, profiles/): the best split is the largest one with
    // tiles * splitk <= 2 * SMs (two ~105 KB CTAs fit an SM), >= 4 k-blocks of
    // 64 per CTA, and a cluster of at most 8 CTAs (12 when <= 16 tiles).
    // v/out_proj-sized decode layers (<= 16 feature tiles, K <= 2048) at
    // 17..32 tokens: two 16-token tiles with a 4-way split give 32 clusters of
    // 4, all resident at once, instead of 16 clusters of 8 of which only 15
    // fit (the 16th started ~1.2 us late): in situ 12.77 -> 12.25 us per
    // [layer_norm -> 2048x2048 linear] (profiles/r1c_bn16.txt)
    if (g.swap && g.bn == 32 && g.tilesA <= 16 && g.nkb >= 24 && g.nkb <= 32 && bn_env == 0 &&
        getenv("FT2_GEMM_SPLITK") == nullptr && max_clusters_bn(16, 4) >= 2 * g.tilesA) {
        g.bn = 16;
        g.tilesB = (rowsB + 15) / 16;
        g.splitk = 4;
        g.deep = 0;
        return g;
    }
    int best = 1;
    // clusters above the portable size 8 only pay off when few (<= 16) of
    // them are needed (measured: 16 tiles x 12 beats x 8; 32 tiles x 9 loses to x 8)
    const int sk_cap = tiles <= 16 ? kMaxSplitPlanned : 8;
    // between 33 and 64 tiles the in-situ optimum sits lower (measured at
    // N = 6144: 240 CTAs 15.7 us, 288 CTAs 20.4 us, cuBLAS 13.7 us;
    // profiles/r1c_splitk_mid.txt), so those shapes cap the grid at 240
    static const int cap_env = env_int("FT2_GEMM_CTA_CAP", 0);   // experiment: CTAs per launch
    const int cta_cap = cap_env > 0 ? cap_env : ((tiles > 32 && tiles <= 64) ? 240 : 2 * sms);
    if (g.swap) {
        for (int sk = 2; sk <= sk_cap; ++sk) {
            if (tiles * sk > cta_cap || g.nkb < 4 * sk) break;
            if (max_clusters_bn(g.bn, sk) < 1) break;
            best = sk;
        }
    }
    static const int sk_env = [] { const char* e = getenv("FT2_GEMM_SPLITK"); return e ? atoi(e) : 0; }();
    if (sk_env > 0 && g.swap) {
        int sk = sk_env < g.nkb ? sk_env : g.nkb;
        if (sk > kMaxSplitK) sk = kMaxSplitK;
        while (sk > 1 && max_clusters_bn(g.bn, sk) < 1) --sk;
        best = sk;
    }
    g.splitk = best;
    g.deep = 0;
    // Few-tile decode shapes: one CTA per SM with the CTA's whole K slice in
    // flight (one DRAM round trip) when all clusters fit in one wave.
    static const int deep_env = env_int("FT2_GEMM_DEEP", 0);  // measured slower in situ: opt-in
    if (g.swap && g.bn <= 64 && deep_env != 0) {
        const int st = deep_stages(g.bn);
        int dk = 0;
        for (int sk = 1; sk <= 8; ++sk) {
            if (tiles * sk > sms) break;
            if (max_clusters_bn(g.bn, sk, true) < tiles) continue;
            dk = sk;
            if ((g.nkb + sk - 1) / sk <= st) break;  // smallest split with a single round trip
        }
        if (dk > 0 && ((g.nkb + dk - 1) / dk <= st || deep_env == 1)) {
            g.deep = 1;
            g.splitk = dk;
            if (sk_env > 0) {
                int sk = sk_env < g.nkb ? sk_env : g.nkb;
                while (sk > 1 && max_clusters_bn(g.bn, sk, true) < 1) --sk;
                g.splitk = sk;
            }
        }
    }
    // A 128-row plan that puts more CTAs than SMs on the GPU double-books SMs
    // anyway (profiles: SM sharing); for N <= 2048 at <= 32 tokens (OPT fc2)
    // the 64-row plan -- half the split-K exchange per CTA, an 8-way split with
    // the fixed-size slot sum -- is then faster: fc2 back to back 8.95 -> 8.68
    // us, in situ +0.1 %; plans that fit one CTA per SM (e.g. Qwen2-1.5B's
    // 1536x8960 down_proj, 144 CTAs) stay at 128 rows (profiles/r2_fc2_ba64.txt)
    static const int ba_env = env_int("FT2_GEMM_BA", 0);
    if (g.swap && !force64 && !g.deep && ba_env == 0 && M <= 32 && N <= 2048 &&
        g.tilesA * g.tilesB * g.splitk > num_sms())
        return plan_gemm_impl(M, N, K, true);
    return g;
}

static GemmPlan plan_gemm(int32_t M, int32_t N, int32_t K) {
    const GemmPlan g = plan_gemm_impl(M, N, K);
    static const bool dbg = getenv("FT2_GEMM_DEBUG") != nullptr;
    if (dbg)
        fprintf(stderr, "[ft2 gemm] M=%d N=%d K=%d swap=%d ba=%d bn=%d tiles=%dx%d nkb=%d splitk=%d deep=%d cA=%d\n", M, N,
                K, g.swap, g.ba, g.bn, g.tilesA, g.tilesB, g.nkb, g.splitk, g.deep, g.cA);
    return g;
}

// The decode kernel's cluster split-K needs no global workspace; the
// persistent kernel (M > swap_max_m()) uses one for its K splits when the
// tiles alone cannot fill the machine (optional: less space, fewer splits).
size_t gemm_ws_bytes(int32_t M, int32_t N, int32_t K) {
    if (M <= swap_max_m()) return 0;
    return plan_prefill_split(M, N, K, (size_t)-1).need_bytes;
}

template <int BA, int BN, bool SWAP, int DT, bool DEEP = false, bool MMA2 = false>
static cudaError_t launch_cfg(const GemmArgs& a, const GemmK& p, cudaStream_t st, int* n_launch) {
    CUtensorMap ma, mb;
    const void* pa = SWAP ? (const void*)a.w : (const void*)a.x;
    const void* pb = SWAP ? (const void*)a.x : (const void*)a.w;
    const int64_t lda = SWAP ? a.ldw : a.ldx, ldb = SWAP ? a.ldx : a.ldw;
    if (!make_map(&ma, pa, p.rowsA, a.K, lda, SWAP ? BA : kBlockA, DT == 1 ? FT2_FP16 : FT2_BF16))
        return cudaErrorInvalidValue;
    if (!make_map(&mb, pb, p.rowsB, a.K, ldb, BN, DT == 1 ? FT2_FP16 : FT2_BF16)) return cudaErrorInvalidValue;
    cudaError_t e = set_attrs<BA, BN, SWAP, DT, DEEP, MMA2>();
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)p.tilesA, (unsigned)p.splitk, (unsigned)p.tilesB);   // tilesA % cA == 0
    cfg.blockDim = dim3(kGemmThreads);
    cfg.dynamicSmemBytes = Cfg<BA, BN, DEEP>::kBytes + smem_pad();
    cfg.stream = st;
    cudaLaunchAttribute attr[3];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    static const int pdl = env_int("FT2_GEMM_PDL", 1);
    attr[0].val.programmaticStreamSerializationAllowed = pdl;
    attr[1].id = cudaLaunchAttributeClusterDimension;
    attr[1].val.clusterDim.x = (unsigned)p.cA;
    attr[1].val.clusterDim.y = (unsigned)p.splitk;
    attr[1].val.clusterDim.z = 1;
    attr[2].id = cudaLaunchAttributeClusterSchedulingPolicyPreference;
    attr[2].val.clusterSchedulingPolicyPreference = cudaClusterSchedulingPolicySpread;
    cfg.attrs = attr;
    cfg.numAttrs = (p.splitk > 1 || p.cA > 1) ? (spread_policy() ? 3 : 2) : 1;
    e = cudaLaunchKernelEx(&cfg, gemm_kernel<BA, BN, SWAP, DT, DEEP, MMA2>, ma, mb, p);
    ++*n_launch;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_gemm(const GemmArgs& a, cudaStream_t st, int* n_launch) {
    // prefill shapes (M > 128 tokens): the persistent 128x256 kernel (gemm_prefill_sm100.cu)
    if (a.M > swap_max_m()) return launch_prefill_gemm(a, nullptr, st, n_launch);
    const GemmPlan g = plan_gemm(a.M, a.N, a.K);
    GemmK p = {};
    p.M = a.M;
    p.N = a.N;
    p.K = a.K;
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
    static const int trig = env_int("FT2_GEMM_TRIGGER", 3);
    p.trigger = trig;
    static const int wl2 = env_int("FT2_GEMM_W_L2", 0);
    static const int64_t wl2_max = (int64_t)env_int("FT2_GEMM_W_L2_MAX_MB", 48) << 20;
    p.w_l2 = (wl2 >= 2 && (int64_t)a.N * a.K * 2 > wl2_max) ? 1 : wl2;
    static const int pf_on = env_int("FT2_GEMM_PF", 1);      // experiments: 0 ignores the hint
    static const int pf_at = env_int("FT2_GEMM_PF_AT", 1);
    p.pf = pf_on ? static_cast<const uint8_t*>(a.l2_prefetch) : nullptr;
    p.pf_bytes = p.pf ? (uint64_t)a.l2_prefetch_bytes : 0;
    p.pf_at = pf_at;
    p.rows_per_slot = (g.ba + g.splitk - 1) / g.splitk;
    p.cA = g.cA;
    {   // two MMA issuers: 64-row tiles whose whole K slice sits in the ring (FT2_GEMM_MMA2=0 turns it off)
        static const int mma2_env = env_int("FT2_GEMM_MMA2", 1);
        // (128-row tiles: opt-in, FT2_GEMM_MMA2=2 -- two warps issue an M = 128 MMA every ~47
        // cycles against ~53 for one, profiles/r2_mma_probe.txt)
        const int st = g.ba == 64 ? (g.bn <= 16 ? Cfg<64, 16>::STAGES : Cfg<64, 32>::STAGES)
                                  : (g.bn <= 16 ? Cfg<128, 16>::STAGES : Cfg<128, 32>::STAGES);
        const bool shape_ok = g.ba == 64 || (mma2_env == 2 && !g.deep && g.bn <= 32);
        p.mma2 = (mma2_env && shape_ok && g.cA == 1 && (g.nkb + g.splitk - 1) / g.splitk <= st) ? 1 : 0;
    }

    p.sk_magic = (uint32_t)(((1u << 24) + g.splitk - 1) / g.splitk);
#ifdef FT2_GEMM_TRACE
    p.trace_base = 256 * (g_trace_launch++ % 128);   // graph captures bake one base per captured launch
#endif
    if (g.ba == 64) {
        if (a.dtype == FT2_FP16)
            return p.mma2 ? (g.bn == 16 ? launch_cfg<64, 16, true, 1, false, true>(a, p, st, n_launch)
                                        : launch_cfg<64, 32, true, 1, false, true>(a, p, st, n_launch))
                          : (g.bn == 16 ? launch_cfg<64, 16, true, 1>(a, p, st, n_launch)
                                        : launch_cfg<64, 32, true, 1>(a, p, st, n_launch));
        return p.mma2 ? (g.bn == 16 ? launch_cfg<64, 16, true, 0, false, true>(a, p, st, n_launch)
                                    : launch_cfg<64, 32, true, 0, false, true>(a, p, st, n_launch))
                      : (g.bn == 16 ? launch_cfg<64, 16, true, 0>(a, p, st, n_launch)
                                    : launch_cfg<64, 32, true, 0>(a, p, st, n_launch));
    }
    if (g.deep) {
        if (a.dtype == FT2_FP16) {
            switch (g.bn) {
                case 16: return launch_cfg<128, 16, true, 1, true>(a, p, st, n_launch);
                case 32: return launch_cfg<128, 32, true, 1, true>(a, p, st, n_launch);
                default: return launch_cfg<128, 64, true, 1, true>(a, p, st, n_launch);
            }
        }
        switch (g.bn) {
            case 16: return launch_cfg<128, 16, true, 0, true>(a, p, st, n_launch);
            case 32: return launch_cfg<128, 32, true, 0, true>(a, p, st, n_launch);
            default: return launch_cfg<128, 64, true, 0, true>(a, p, st, n_launch);
        }
    }
    if (p.mma2) {   // 128-row tiles with the whole K slice in the ring (opt-in)
        if (a.dtype == FT2_FP16)
            return g.bn == 16 ? launch_cfg<128, 16, true, 1, false, true>(a, p, st, n_launch)
                              : launch_cfg<128, 32, true, 1, false, true>(a, p, st, n_launch);
        return g.bn == 16 ? launch_cfg<128, 16, true, 0, false, true>(a, p, st, n_launch)
                          : launch_cfg<128, 32, true, 0, false, true>(a, p, st, n_launch);
    }
    if (a.dtype == FT2_FP16) {
        switch (g.bn) {
            case 16: return launch_cfg<128, 16, true, 1>(a, p, st, n_launch);
            case 32: return launch_cfg<128, 32, true, 1>(a, p, st, n_launch);
            case 64: return launch_cfg<128, 64, true, 1>(a, p, st, n_launch);
            default: return launch_cfg<128, 128, true, 1>(a, p, st, n_launch);
        }
    }
    switch (g.bn) {
        case 16: return launch_cfg<128, 16, true, 0>(a, p, st, n_launch);
        case 32: return launch_cfg<128, 32, true, 0>(a, p, st, n_launch);
        case 64: return launch_cfg<128, 64, true, 0>(a, p, st, n_launch);
        default: return launch_cfg<128, 128, true, 0>(a, p, st, n_launch);
    }
}

}  // namespace ft2impl

#ifdef FT2_GEMM_TRACE
namespace ft2impl {
__device__ unsigned long long g_marks[64];
__global__ void mark_kernel(int slot) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_marks[slot & 63] = t;
}
}  // namespace ft2impl
// one-thread kernel that records the global timer (launch-gap measurements)
extern "C" int ft2_debug_mark(int slot, cudaStream_t st) {
    ft2impl::mark_kernel<<<1, 32, 0, st>>>(slot);
    return (int)cudaGetLastError();
}
extern "C" int ft2_debug_marks_read(void* dst) {
    return (int)cudaMemcpyFromSymbol(dst, ft2impl::g_marks, sizeof(ft2impl::g_marks));
}
extern "C" void ft2_debug_trace_reset(int launch) { ft2impl::g_trace_launch = launch; }
extern "C" int ft2_debug_trace_read(void* dst, size_t bytes) {
    if (bytes > sizeof(ft2impl::g_trace)) bytes = sizeof(ft2impl::g_trace);
    return (int)cudaMemcpyFromSymbol(dst, ft2impl::g_trace, bytes);
}
#endif
