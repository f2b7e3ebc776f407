// ft2_internal.h -- launchers shared between the kernel files and abi.cu.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/ft2.h"

namespace ft2impl {

// Programmatic dependent launch (PDL) contract of this library.  Kernels
// launched with programmaticStreamSerializationAllowed (the decode and prefill
// GEMMs) may start while the previous kernel in the stream still runs: before
// their griddepcontrol.wait they may only touch data no earlier kernel writes
// (their own shared memory and TMEM, tensor-map prefetches, and -- with
// FT2_GEMM_W_STATIC -- the static weight tiles).  Every global read of an
// upstream output (x, bias, bounds, sites, row maps) and EVERY global write
// (y, counters, workspaces) comes after the wait.  Kernels that trigger their
// dependents early (griddepcontrol.launch_dependents: the GEMMs after their
// prologue, ft2_host_norm / ft2_host_act on entry) rely on that rule: a new
// PDL-launched kernel that wrote before its wait would race with them.
// tests/test_gpu_host_norm.py::test_pdl_chain_graph_replay checks the chain
// (norm -> act -> fused GEMM, replayed with changing inputs) bit for bit
// against stream-ordered launches.

// Workspace of the bounds reduction (u32 words unless noted):
//   [4s+0] lo slot  = 0x10000 - min key  (0 = no finite value yet)
//   [4s+1] hi slot  = max key + 1        (0 = none)
//   [4s+2] non-finite count, [4s+3] NaN-vulnerable count
//   [4S+0] CTA completion counter, [4S+1] patch-list count, [4S+2] overflow flag
//   then (8-byte aligned) u64 patch list [kPatchCap]: offset | seq << 48
constexpr int kPatchCap = 4096;
size_t bounds_ws_bytes(int32_t S);

struct BoundsArgs {
    uint16_t* y;
    int64_t ld;
    int64_t rows, n;
    const int32_t* seq_offsets;
    int32_t S;
    float scale;
    int32_t finalize, correct;
    uint16_t* bounds_out;
    int32_t* keys_out;
    uint32_t* nonfinite_out;
    uint32_t* nv_out;  // NaN-vulnerable counts or NULL
    uint32_t* ws;
    int32_t dtype;  // FT2_BF16, FT2_FP16 (bounds.cu) or FT2_FP32 (f32.cu)
};
cudaError_t launch_bounds(const BoundsArgs& a, cudaStream_t st, int* n_launch);
cudaError_t launch_finalize(const int32_t* keys, int32_t S, float scale, uint16_t* out, int dtype,
                            cudaStream_t st, int* n_launch);

struct ProtectArgs {
    uint16_t* y;
    int64_t ld, rows, n;
    const int32_t* row_to_seq;  // or NULL
    int32_t S;
    const uint16_t* bounds;
    uint32_t* counts;
    int32_t dtype;
};
cudaError_t launch_protect(const ProtectArgs& a, cudaStream_t st, int* n_launch);

cudaError_t launch_make_sites(uint64_t seed, uint64_t trial0, int32_t n, int32_t model,
                              int32_t dtype, const ft2_site_geometry& g, ft2_fault_site* out,
                              cudaStream_t st, int* n_launch);
cudaError_t launch_inject(uint16_t* y, int64_t rows, int64_t n, int64_t ld,
                          const ft2_fault_site* sites, int32_t n_sites, int32_t layer,
                          int32_t step, const int32_t* base_row, cudaStream_t st, int* n_launch);

struct GemmArgs {
    const uint16_t* x; int64_t ldx;
    const uint16_t* w; int64_t ldw;
    const uint16_t* bias;
    uint16_t* y; int64_t ldy;
    int32_t M, N, K;
    int32_t mode;
    int32_t col_begin, col_end;
    const int32_t* row_to_seq;
    const uint16_t* bounds;
    int32_t S;
    uint32_t* counts;
    const ft2_fault_site* sites;
    int32_t n_sites, cur_layer, cur_step;
    const int32_t* base_row;
    void* ws; size_t ws_bytes;
    int32_t w_static;
    int32_t dtype;
    const void* l2_prefetch;     // bytes to pull into L2 once this CTA's own operands have landed
    size_t l2_prefetch_bytes;    // (the next layer's weights; multiple of 16, 16-byte aligned)
};
size_t gemm_ws_bytes(int32_t M, int32_t N, int32_t K);
cudaError_t launch_gemm(const GemmArgs& a, cudaStream_t st, int* n_launch);

// First-token bound derivation fused into the prefill GEMM epilogue
// (ft2_prefill_fused_gemm): the ft2_bounds_from_prefill outputs, finalize = 1.
struct PrefillDerive {
    const int32_t* seq_offsets;  // [S + 1] or NULL (one sequence)
    int32_t S;
    float scale;
    int32_t correct;
    uint16_t* bounds_out;
    int32_t* keys_out;
    uint32_t* nonfinite_out;
    uint32_t* ws;  // bounds workspace (bounds_ws_bytes(S))
};
// K-split plan of the persistent kernel (gemm_prefill_sm100.cu): splits that
// fit ws_bytes, the counter-area bytes, and the bytes the best plan needs.
struct PrefillSplit {
    int splits;
    size_t cnt_bytes, need_bytes;
};
PrefillSplit plan_prefill_split(int32_t M, int32_t N, int32_t K, size_t ws_bytes);
// Persistent 128x256-tile tcgen05 GEMM for M > 128 (PLAIN / CHECK, or DERIVE when d != NULL)
cudaError_t launch_prefill_gemm(const GemmArgs& a, const PrefillDerive* d, cudaStream_t st, int* n_launch);

// binary32 variants (f32.cu; the paper's FP32 study).  The
// 16-bit argument structs are reused: y / bounds point at 32-bit elements.
cudaError_t launch_bounds32(const BoundsArgs& a, cudaStream_t st, int* n_launch);
cudaError_t launch_finalize32(const int32_t* keys, int32_t S, float scale, void* out, cudaStream_t st,
                              int* n_launch);
cudaError_t launch_protect32(const ProtectArgs& a, cudaStream_t st, int* n_launch);
cudaError_t launch_inject32(void* y, int64_t rows, int64_t n, int64_t ld, const ft2_fault_site* sites,
                            int32_t n_sites, int32_t layer, int32_t step, const int32_t* base_row,
                            cudaStream_t st, int* n_launch);

// Row-parallel sum all-reduce fused with the check (allreduce_protect.cu).
constexpr int kARMaxRanks = 64;
struct AllreduceProtectArgs {
    // the P (peer-mapped) partial outputs and flag arrays, by value in the
    // kernel parameters: no dependent pointer load before the data loads
    const uint16_t* partials[kARMaxRanks];
    int64_t ldp;
    int32_t P, rank;
    uint32_t* flags[kARMaxRanks];     // rank t's flag array [P]
    uint32_t* epoch;                  // this rank's call counter (device)
    uint32_t* done;                   // this rank's CTA completion counter (device, self-cleaning)
    uint32_t* status;                 // this rank's error word (1 = peer timeout)
    uint16_t* y;
    int64_t ldy, rows, n;
    const uint16_t* bias;
    int32_t mode;
    const int32_t* row_to_seq;
    const uint16_t* bounds;
    int32_t S;
    uint32_t* counts;
    const ft2_fault_site* sites;
    int32_t n_sites, cur_layer, cur_step;
    const int32_t* base_row;
    int32_t dtype;
};
cudaError_t launch_allreduce_protect(const AllreduceProtectArgs& a, cudaStream_t st, int* n_launch);

int num_sms();

}  // namespace ft2impl
