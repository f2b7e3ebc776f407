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
    int32_t swap;         // 1: A = w (features), B = x (tokens)
    int32_t rowsA, rowsB; // extent of the A / B operands
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
};

template <int BN, int STAGES>
struct GemmSmem {
    static constexpr int kABytes = kBlockA * kBlockK * 2;
    static constexpr int kBBytes = BN * kBlockK * 2;
    static constexpr int kStageBytes = kABytes + kBBytes;
    static constexpr int kRedStride = BN + 1;  // padded fp32 row (bank-conflict free)
    static constexpr int kRedBytes = kBlockA * kRedStride * 4;
    static constexpr int kTileBytes = STAGES * kStageBytes > kRedBytes ? STAGES * kStageBytes : kRedBytes;
    static constexpr int kBytes = 1024 /*align slack*/ + kTileBytes + 1024 /*barriers etc*/;
};

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
    uint32_t* site_n = tmem_base_sh + 1;
    uint32_t* site_e = site_n + 1;           // [kMaxSitesPerCta] local element index
    uint32_t* site_m = site_e + kMaxSitesPerCta;  // [kMaxSitesPerCta] xor mask
    float* red = reinterpret_cast<float*>(tiles);  // aliases the stage ring after the MMAs

    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int tileA = blockIdx.x, tileB = blockIdx.z;
    const uint32_t rank = p.splitk > 1 ? cluster_rank() : 0u;
    const int kb0 = (int)((int64_t)rank * p.nkb / p.splitk);
    const int kb1 = (int)((int64_t)(rank + 1) * p.nkb / p.splitk);
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

    if (warp == 0) {
        if (lane == 0) {
            // ------------------------------------------------ TMA producer
            for (int i = 0; i < nk; ++i) {
                const int s = i % STAGES;
                const uint32_t ph = (uint32_t)(i / STAGES) & 1u;
                if (i >= STAGES) mbar_wait(&empty[s], ph ^ 1u);
                uint8_t* sa = tiles + s * L::kStageBytes;
                uint8_t* sb = sa + L::kABytes;
                mbar_expect_tx(&full[s], L::kStageBytes);
                const int kc = (kb0 + i) * kBlockK;
                tma_load_2d(&map_a, &full[s], sa, kc, tileA * kBlockA);
                tma_load_2d(&map_b, &full[s], sb, kc, tileB * BN);
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
                for (int k = 0; k < kBlockK / kUmmaK; ++k) {
                    // advance 16 elements (32 B) along K inside the swizzle atom
                    tc_mma(tmem_base, da + (uint64_t)(k * 2), db + (uint64_t)(k * 2), idesc,
                           (i > 0 || k > 0) ? 1u : 0u);
                }
                tc_commit(&empty[s]);
            }
            tc_commit(tmem_full);
        }
    } else {
        // ---------------------------------------------------- epilogue warps
        const int q = warp & 3;  // TMEM lane quarter this warp may access
        mbar_wait(tmem_full, 0);
        tc_fence_after();
        const int row = q * 32 + lane;
        const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16);
        if (BN >= 32) {
#pragma unroll 1
            for (int c = 0; c < BN; c += 32) {
                uint32_t r[32];
                tmem_ld32(taddr + c, r);
                tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 32; ++j) red[row * L::kRedStride + c + j] = nk > 0 ? __uint_as_float(r[j]) : 0.f;
            }
        } else {
            uint32_t r[16];
            tmem_ld16(taddr, r);
            tmem_wait_ld();
#pragma unroll
            for (int j = 0; j < 16; ++j) red[row * L::kRedStride + j] = nk > 0 ? __uint_as_float(r[j]) : 0.f;
        }
    }
    tc_fence_before();
    __syncthreads();

    // --------------------------------------------- fault sites of this CTA
    const int rows_per = kBlockA / p.splitk;
    const int a0 = (int)rank * rows_per;  // my rows of the 128 x BN tile
    if (p.sites != nullptr) {
        for (int i = threadIdx.x; i < p.n_sites; i += kGemmThreads) {
            ft2_fault_site st = p.sites[i];
            if ((int)st.step != p.cur_step || (int)st.layer != p.cur_layer) continue;
            int64_t m = (p.base_row ? (int64_t)p.base_row[i] : (int64_t)i) + (p.cur_step == 0 ? (int64_t)st.token : 0);
            int64_t n = st.col;
            if (m < 0 || m >= p.M || n >= p.N) continue;
            int64_t ga = p.swap ? n : m, gb = p.swap ? m : n;  // global A / B row
            int64_t la = ga - (int64_t)tileA * kBlockA - a0, lb = gb - (int64_t)tileB * BN;
            if (la < 0 || la >= rows_per || lb < 0 || lb >= BN) continue;
            uint32_t idx = atomicAdd(site_n, 1u);
            if (idx < (uint32_t)kMaxSitesPerCta) {
                site_e[idx] = (uint32_t)(la * BN + lb);
                site_m[idx] = st.xor_mask;
            }
        }
    }
    if (p.splitk > 1) cluster_sync_all();
    else __syncthreads();
    const uint32_t nsite = min(*site_n, (uint32_t)kMaxSitesPerCta);

    // ------------------------------------------ split-K combine + epilogue
    const uint32_t red_base = smem_u32(red);
    const int elems = rows_per * BN;
    for (int e = threadIdx.x; e < elems; e += kGemmThreads) {
        int la, lb;
        if (p.swap) { la = e % rows_per; lb = e / rows_per; }   // consecutive threads: consecutive features
        else        { lb = e % BN;       la = e / BN; }
        const int a = a0 + la;
        const int ga = tileA * kBlockA + a, gb = tileB * BN + lb;
        const int m = p.swap ? gb : ga, n = p.swap ? ga : gb;
        float acc;
        const uint32_t off = (uint32_t)(a * L::kRedStride + lb) * 4u;
        if (p.splitk > 1) {
            acc = 0.f;
            for (int r = 0; r < p.splitk; ++r) acc += ld_dsmem_f32(mapa(red_base + off, (uint32_t)r));
        } else {
            acc = red[a * L::kRedStride + lb];
        }
        if (m >= p.M || n >= p.N) continue;
        if (p.bias) acc += __uint_as_float((uint32_t)p.bias[n] << 16);
        uint16_t v = bf16_rne(acc);
        const uint32_t le = (uint32_t)(la * BN + lb);
        for (uint32_t i = 0; i < nsite; ++i)
            if (site_e[i] == le) v ^= (uint16_t)site_m[i];
        if (p.mode == FT2_GEMM_CHECK && n >= p.col_begin && n < p.col_end) {
            int s = p.row_mode == 2 ? 0 : (p.row_mode == 1 ? m : p.row_to_seq[m]);
            if (s >= 0 && s < p.S) {
                uint16_t lo = p.bounds[2 * s], hi = p.bounds[2 * s + 1];
                uint16_t x = ((v & 0x7FFF) > 0x7F80) ? (uint16_t)0 : v;   // NaN -> +0
                uint16_t k = key1(x);
                uint16_t o = k < key1(lo) ? lo : (k > key1(hi) ? hi : x);
                if (o != v) {
                    v = o;
                    if (p.counts) atomicAdd(&p.counts[s], 1u);
                }
            }
        }
        p.y[(int64_t)m * p.ldy + n] = v;
    }
    if (p.splitk > 1) cluster_sync_all();  // peers may still read my partial tile
    if (warp == 1) {
        __syncwarp();
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

size_t gemm_ws_bytes(int32_t, int32_t, int32_t) { return 0; }

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
        e = cudaFuncSetAttribute(gemm_kernel<BN, STAGES>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
        if (e != cudaSuccess) return e;
        attr_set = true;
    }
    const int tilesA = (p.rowsA + kBlockA - 1) / kBlockA;
    const int tilesB = (p.rowsB + BN - 1) / BN;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)tilesA, (unsigned)p.splitk, (unsigned)tilesB);
    cfg.blockDim = dim3(kGemmThreads);
    cfg.dynamicSmemBytes = L::kBytes;
    cfg.stream = st;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 1;
    attr[0].val.clusterDim.y = (unsigned)p.splitk;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, gemm_kernel<BN, STAGES>, ma, mb, p);
    ++*n_launch;
    return e != cudaSuccess ? e : cudaGetLastError();
}

cudaError_t launch_gemm(const GemmArgs& a, cudaStream_t st, int* n_launch) {
    GemmK p = {};
    p.M = a.M;
    p.N = a.N;
    p.K = a.K;
    p.swap = a.M <= 128 ? 1 : 0;
    p.rowsA = p.swap ? a.N : a.M;
    p.rowsB = p.swap ? a.M : a.N;
    p.nkb = (a.K + kBlockK - 1) / kBlockK;
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

    int bn;
    if (p.swap) bn = a.M <= 16 ? 16 : (a.M <= 32 ? 32 : (a.M <= 64 ? 64 : 128));
    else bn = 128;
    const int tiles = ((p.rowsA + kBlockA - 1) / kBlockA) * ((p.rowsB + bn - 1) / bn);
    const int sms = num_sms();
    int sk = 1;
    while (sk < 8 && tiles * sk * 2 <= sms && p.nkb >= sk * 2 * 2) sk *= 2;
    p.splitk = sk;

    switch (bn) {
        case 16: return launch_cfg<16, 8>(a, p, st, n_launch);
        case 32: return launch_cfg<32, 8>(a, p, st, n_launch);
        case 64: return launch_cfg<64, 8>(a, p, st, n_launch);
        default: return launch_cfg<128, 6>(a, p, st, n_launch);
    }
}

}  // namespace ft2impl
