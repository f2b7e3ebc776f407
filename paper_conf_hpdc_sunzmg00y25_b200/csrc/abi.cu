// abi.cu -- the C ABI of libft2.so (include/ft2.h): argument validation,
// status codes, launch bookkeeping.  All compute happens in the kernels of
// bounds.cu, protect.cu, faults.cu and gemm_sm100.cu.
#include <cuda.h>
#include <cuda_runtime.h>

#include <atomic>
#include <cmath>
#include <cstring>

#include "ft2_internal.h"

namespace ft2impl {

int num_sms() {
    static int cached[64] = {0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (dev < 0 || dev >= 64) dev = 0;
    if (cached[dev] == 0) {
        int n = 0;
        cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
        cached[dev] = n > 0 ? n : 148;
    }
    return cached[dev];
}

}  // namespace ft2impl

using namespace ft2impl;

static std::atomic<uint64_t> g_launches{0};

static inline bool al16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

// elements per 16-byte vector: 8 for the 16-bit formats, 4 for binary32
static inline int64_t vec_elems(int32_t dtype) { return dtype == FT2_FP32 ? 4 : 8; }

static ft2_status check_tensor(const ft2_tensor& t, bool allow_null_if_empty = true) {
    if (t.rows < 0 || t.n < 0 || t.ld < t.n) return FT2_ERR_INVALID_ARG;
    if (t.dtype != FT2_BF16 && t.dtype != FT2_FP16 && t.dtype != FT2_FP32) return FT2_ERR_UNSUPPORTED;
    if (t.rows == 0 || t.n == 0) return FT2_OK;
    if (t.data == nullptr) return FT2_ERR_INVALID_ARG;
    const int64_t ve = vec_elems(t.dtype);
    if (!al16(t.data) || (t.n % ve) != 0 || (t.ld % ve) != 0) return FT2_ERR_MISALIGNED;
    (void)allow_null_if_empty;
    return FT2_OK;
}

static inline ft2_status finish(cudaError_t e, int launches) {
    g_launches.fetch_add((uint64_t)launches, std::memory_order_relaxed);
    if (e != cudaSuccess) {
        cudaGetLastError();  // clear the sticky-free launch error
        return FT2_ERR_CUDA;
    }
    return FT2_OK;
}

extern "C" {

size_t ft2_workspace_bytes(int32_t num_seqs) {
    if (num_seqs < 1) num_seqs = 1;
    return bounds_ws_bytes(num_seqs);
}

ft2_status ft2_bounds_from_prefill(ft2_tensor y, const int32_t* seq_offsets, int32_t num_seqs, float scale,
                                   int32_t finalize, int32_t correct_nonfinite, void* bounds_out,
                                   int32_t* keys_out, uint32_t* nonfinite_count, uint32_t* nan_vulnerable_count,
                                   void* workspace, void* stream) {
    ft2_status s = check_tensor(y);
    if (s != FT2_OK) return s;
    if (num_seqs < 1 || num_seqs > FT2_MAX_SEQS) return num_seqs < 1 ? FT2_ERR_INVALID_ARG : FT2_ERR_UNSUPPORTED;
    if (!(std::isfinite(scale)) || scale < 1.0f) return FT2_ERR_INVALID_ARG;
    if (workspace == nullptr) return FT2_ERR_INVALID_ARG;
    if (finalize && bounds_out == nullptr) return FT2_ERR_INVALID_ARG;
    if (!finalize && keys_out == nullptr) return FT2_ERR_INVALID_ARG;
    if (correct_nonfinite && !finalize) return FT2_ERR_INVALID_ARG;
    if (seq_offsets == nullptr && num_seqs != 1) return FT2_ERR_INVALID_ARG;
    if (((uintptr_t)workspace & 7u) != 0 || (bounds_out && ((uintptr_t)bounds_out & (y.dtype == FT2_FP32 ? 7u : 3u)) != 0))
        return FT2_ERR_MISALIGNED;
    if ((y.rows * (y.n / vec_elems(y.dtype))) >= (int64_t(1) << 31)) return FT2_ERR_UNSUPPORTED;
    if (y.rows == 0 || y.n == 0) {
        // nothing to reduce: every sequence is empty (reading A9) -- still a
        // well-defined result, produced by the finalize kernel on "no value" keys
        // would need a buffer; report OK without touching outputs.
        return FT2_OK;
    }
    BoundsArgs a;
    a.y = static_cast<uint16_t*>(y.data);
    a.ld = y.ld;
    a.rows = y.rows;
    a.n = y.n;
    a.seq_offsets = seq_offsets;
    a.S = num_seqs;
    a.scale = scale;
    a.finalize = finalize ? 1 : 0;
    a.correct = correct_nonfinite ? 1 : 0;
    a.bounds_out = static_cast<uint16_t*>(bounds_out);
    a.keys_out = keys_out;
    a.nonfinite_out = nonfinite_count;
    a.nv_out = nan_vulnerable_count;
    a.ws = static_cast<uint32_t*>(workspace);
    a.dtype = y.dtype;
    int nl = 0;
    cudaError_t e = y.dtype == FT2_FP32 ? launch_bounds32(a, static_cast<cudaStream_t>(stream), &nl)
                                        : launch_bounds(a, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_bounds_finalize(const int32_t* keys, int32_t num_seqs, float scale, ft2_dtype dtype,
                               void* bounds_out, void* stream) {
    if (keys == nullptr || bounds_out == nullptr || num_seqs < 1) return FT2_ERR_INVALID_ARG;
    if (!(std::isfinite(scale)) || scale < 1.0f) return FT2_ERR_INVALID_ARG;
    if (dtype != FT2_BF16 && dtype != FT2_FP16 && dtype != FT2_FP32) return FT2_ERR_UNSUPPORTED;
    if (((uintptr_t)bounds_out & (dtype == FT2_FP32 ? 7u : 3u)) != 0) return FT2_ERR_MISALIGNED;
    int nl = 0;
    cudaError_t e = dtype == FT2_FP32
                        ? launch_finalize32(keys, num_seqs, scale, bounds_out, static_cast<cudaStream_t>(stream), &nl)
                        : launch_finalize(keys, num_seqs, scale, static_cast<uint16_t*>(bounds_out), (int)dtype,
                                          static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_protect(ft2_tensor y, const int32_t* row_to_seq, const void* bounds, int32_t num_seqs,
                       uint32_t* corrected_count, void* stream) {
    ft2_status s = check_tensor(y);
    if (s != FT2_OK) return s;
    if (num_seqs < 1 || bounds == nullptr) return FT2_ERR_INVALID_ARG;
    if (row_to_seq == nullptr && num_seqs != 1 && (int64_t)num_seqs != y.rows) return FT2_ERR_INVALID_ARG;
    if (((uintptr_t)bounds & (y.dtype == FT2_FP32 ? 7u : 3u)) != 0) return FT2_ERR_MISALIGNED;
    if ((y.rows * (y.n / vec_elems(y.dtype))) >= (int64_t(1) << 31)) return FT2_ERR_UNSUPPORTED;
    if (y.rows == 0 || y.n == 0) return FT2_OK;
    ProtectArgs a;
    a.y = static_cast<uint16_t*>(y.data);
    a.ld = y.ld;
    a.rows = y.rows;
    a.n = y.n;
    a.row_to_seq = row_to_seq;
    a.S = num_seqs;
    a.bounds = static_cast<const uint16_t*>(bounds);
    a.counts = corrected_count;
    a.dtype = y.dtype;
    int nl = 0;
    cudaError_t e = y.dtype == FT2_FP32 ? launch_protect32(a, static_cast<cudaStream_t>(stream), &nl)
                                        : launch_protect(a, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

size_t ft2_gemm_workspace_bytes(int32_t M, int32_t N, int32_t K) { return gemm_ws_bytes(M, N, K); }

ft2_status ft2_protect_fused_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw, const void* bias,
                                  void* y, int64_t ldy, int32_t M, int32_t N, int32_t K, ft2_gemm_mode mode,
                                  ft2_dtype dtype, int32_t col_begin, int32_t col_end, const int32_t* row_to_seq,
                                  const void* bounds, int32_t num_seqs, uint32_t* corrected_count,
                                  const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer,
                                  int32_t cur_step, const int32_t* base_row, void* workspace, size_t ws_bytes,
                                  void* stream) {
    return ft2_protect_fused_gemm_ex(x, ldx, w, ldw, bias, y, ldy, M, N, K, mode, dtype, col_begin, col_end,
                                     row_to_seq, bounds, num_seqs, corrected_count, sites, n_sites, cur_layer,
                                     cur_step, base_row, workspace, ws_bytes, nullptr, 0, stream);
}

ft2_status ft2_protect_fused_gemm_ex(const void* x, int64_t ldx, const void* w, int64_t ldw, const void* bias,
                                     void* y, int64_t ldy, int32_t M, int32_t N, int32_t K, ft2_gemm_mode mode,
                                     ft2_dtype dtype, int32_t col_begin, int32_t col_end,
                                     const int32_t* row_to_seq, const void* bounds, int32_t num_seqs,
                                     uint32_t* corrected_count, const ft2_fault_site* sites, int32_t n_sites,
                                     int32_t cur_layer, int32_t cur_step, const int32_t* base_row,
                                     void* workspace, size_t ws_bytes, const void* l2_prefetch,
                                     size_t l2_prefetch_bytes, void* stream) {
    if (l2_prefetch_bytes > 0 && (l2_prefetch == nullptr)) return FT2_ERR_INVALID_ARG;
    if (l2_prefetch_bytes > 0 && (!al16(l2_prefetch) || (l2_prefetch_bytes % 16))) return FT2_ERR_MISALIGNED;
    if (M < 0 || N < 0 || K < 0) return FT2_ERR_INVALID_ARG;
    if (dtype != FT2_BF16 && dtype != FT2_FP16) return FT2_ERR_UNSUPPORTED;
    if (M == 0 || N == 0) return FT2_OK;
    if (K == 0) return FT2_ERR_UNSUPPORTED;
    if (x == nullptr || w == nullptr || y == nullptr) return FT2_ERR_INVALID_ARG;
    if (ldx < K || ldw < K || ldy < N) return FT2_ERR_INVALID_ARG;
    const int32_t w_static = (mode & FT2_GEMM_W_STATIC) ? 1 : 0;
    mode = (ft2_gemm_mode)(mode & ~FT2_GEMM_W_STATIC);
    if (mode != FT2_GEMM_PLAIN && mode != FT2_GEMM_CHECK) return FT2_ERR_INVALID_ARG;
    if (!al16(x) || !al16(w) || !al16(y) || (bias && ((uintptr_t)bias & 1u)) || (K % 8) || (ldx % 8) ||
        (ldw % 8) || (ldy % 8))
        return FT2_ERR_MISALIGNED;
    if (mode == FT2_GEMM_CHECK) {
        if (bounds == nullptr || num_seqs < 1) return FT2_ERR_INVALID_ARG;
        if (row_to_seq == nullptr && num_seqs != 1 && num_seqs != M) return FT2_ERR_INVALID_ARG;
        if (col_begin < 0 || col_end > N || col_begin > col_end) return FT2_ERR_INVALID_ARG;
    }
    if (n_sites < 0 || (n_sites > 0 && sites == nullptr)) return FT2_ERR_INVALID_ARG;
    // the workspace is optional (K splits of the persistent M > 128 kernel): a
    // smaller one or none means fewer or no splits
    if (workspace != nullptr && !al16(workspace)) return FT2_ERR_MISALIGNED;
    if (workspace == nullptr) ws_bytes = 0;
    GemmArgs a;
    a.x = static_cast<const uint16_t*>(x);
    a.ldx = ldx;
    a.w = static_cast<const uint16_t*>(w);
    a.ldw = ldw;
    a.bias = static_cast<const uint16_t*>(bias);
    a.y = static_cast<uint16_t*>(y);
    a.ldy = ldy;
    a.M = M;
    a.N = N;
    a.K = K;
    a.mode = mode;
    a.col_begin = (mode == FT2_GEMM_CHECK) ? col_begin : 0;
    a.col_end = (mode == FT2_GEMM_CHECK) ? col_end : N;
    a.row_to_seq = row_to_seq;
    a.bounds = static_cast<const uint16_t*>(bounds);
    a.S = num_seqs;
    a.counts = corrected_count;
    a.sites = n_sites > 0 ? sites : nullptr;
    a.n_sites = n_sites;
    a.cur_layer = cur_layer;
    a.cur_step = cur_step;
    a.base_row = base_row;
    a.ws = workspace;
    a.ws_bytes = ws_bytes;
    a.w_static = w_static;
    a.dtype = dtype;
    a.l2_prefetch = l2_prefetch_bytes ? l2_prefetch : nullptr;
    a.l2_prefetch_bytes = l2_prefetch_bytes;
    int nl = 0;
    cudaError_t e = launch_gemm(a, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_prefill_fused_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw, const void* bias, void* y,
                                  int64_t ldy, int32_t M, int32_t N, int32_t K, ft2_dtype dtype,
                                  const int32_t* seq_offsets, int32_t num_seqs, float scale, int32_t correct_nonfinite,
                                  void* bounds_out, int32_t* keys_out, uint32_t* nonfinite_count,
                                  const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer,
                                  const int32_t* base_row, void* workspace, void* gemm_workspace,
                                  size_t gemm_ws_bytes, void* stream) {
    if (M < 0 || N < 0 || K < 0) return FT2_ERR_INVALID_ARG;
    if (gemm_workspace != nullptr && !al16(gemm_workspace)) return FT2_ERR_MISALIGNED;
    if (dtype != FT2_BF16 && dtype != FT2_FP16) return FT2_ERR_UNSUPPORTED;
    if (num_seqs < 1 || num_seqs > FT2_MAX_SEQS) return num_seqs < 1 ? FT2_ERR_INVALID_ARG : FT2_ERR_UNSUPPORTED;
    if (!(std::isfinite(scale)) || scale < 1.0f) return FT2_ERR_INVALID_ARG;
    if (x == nullptr || w == nullptr || y == nullptr || bounds_out == nullptr || workspace == nullptr)
        return FT2_ERR_INVALID_ARG;
    if (seq_offsets == nullptr && num_seqs != 1) return FT2_ERR_INVALID_ARG;
    if (ldx < K || ldw < K || ldy < N) return FT2_ERR_INVALID_ARG;
    if (n_sites < 0 || (n_sites > 0 && sites == nullptr)) return FT2_ERR_INVALID_ARG;
    if (!al16(x) || !al16(w) || !al16(y) || (bias && ((uintptr_t)bias & 1u)) || (K % 8) || (N % 8) ||
        (ldx % 8) || (ldw % 8) || (ldy % 8) || ((uintptr_t)workspace & 7u) || ((uintptr_t)bounds_out & 3u))
        return FT2_ERR_MISALIGNED;
    if (M == 0 || N == 0) return FT2_OK;  // as ft2_bounds_from_prefill: nothing to reduce
    if (K == 0) return FT2_ERR_UNSUPPORTED;
    if ((int64_t)M * (N / 8) >= (int64_t(1) << 31)) return FT2_ERR_UNSUPPORTED;
    GemmArgs a = {};
    a.x = static_cast<const uint16_t*>(x);
    a.ldx = ldx;
    a.w = static_cast<const uint16_t*>(w);
    a.ldw = ldw;
    a.bias = static_cast<const uint16_t*>(bias);
    a.y = static_cast<uint16_t*>(y);
    a.ldy = ldy;
    a.M = M;
    a.N = N;
    a.K = K;
    a.mode = FT2_GEMM_PLAIN;
    a.col_begin = 0;
    a.col_end = N;
    a.sites = n_sites > 0 ? sites : nullptr;
    a.n_sites = n_sites;
    a.cur_layer = cur_layer;
    a.cur_step = 0;  // the first token (prefill) is step 0 of the fault-site geometry
    a.base_row = base_row;
    a.dtype = dtype;
    a.ws = gemm_workspace;
    a.ws_bytes = gemm_workspace ? gemm_ws_bytes : 0;
    PrefillDerive d;
    d.seq_offsets = seq_offsets;
    d.S = num_seqs;
    d.scale = scale;
    d.correct = correct_nonfinite ? 1 : 0;
    d.bounds_out = static_cast<uint16_t*>(bounds_out);
    d.keys_out = keys_out;
    d.nonfinite_out = nonfinite_count;
    d.ws = static_cast<uint32_t*>(workspace);
    int nl = 0;
    cudaError_t e = launch_prefill_gemm(a, &d, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_make_fault_sites(uint64_t seed, uint64_t trial0, int32_t n_trials, ft2_fault_model model,
                                ft2_dtype dtype, const ft2_site_geometry* geom, ft2_fault_site* sites_out,
                                void* stream) {
    if (geom == nullptr || n_trials < 0) return FT2_ERR_INVALID_ARG;
    if (n_trials == 0) return FT2_OK;
    if (sites_out == nullptr || geom->layer_width == nullptr) return FT2_ERR_INVALID_ARG;
    if (model < FT2_FAULT_1BIT || model > FT2_FAULT_EXP) return FT2_ERR_INVALID_ARG;
    if (dtype < FT2_BF16 || dtype > FT2_FP32) return FT2_ERR_INVALID_ARG;
    if (geom->n_layers < 1 || geom->n_steps < 0 || geom->prompt_len < 1) return FT2_ERR_INVALID_ARG;
    if (geom->step_policy == 1 && geom->n_steps < 1) return FT2_ERR_INVALID_ARG;
    if (geom->n_layers > FT2_MAX_SITE_LAYERS) return FT2_ERR_UNSUPPORTED;
    for (int l = 0; l < geom->n_layers; ++l)
        if (geom->layer_width[l] < 1) return FT2_ERR_INVALID_ARG;
    int nl = 0;
    cudaError_t e = launch_make_sites(seed, trial0, n_trials, (int32_t)model, (int32_t)dtype, *geom, sites_out,
                                      static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_inject_faults(ft2_tensor y, const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer,
                             int32_t cur_step, const int32_t* base_row, void* stream) {
    if (y.rows < 0 || y.n < 0 || y.ld < y.n) return FT2_ERR_INVALID_ARG;
    if (y.dtype != FT2_BF16 && y.dtype != FT2_FP16 && y.dtype != FT2_FP32) return FT2_ERR_UNSUPPORTED;
    if (n_sites < 0) return FT2_ERR_INVALID_ARG;
    if (n_sites == 0 || y.rows == 0 || y.n == 0) return FT2_OK;
    if (sites == nullptr || y.data == nullptr) return FT2_ERR_INVALID_ARG;
    int nl = 0;
    if (y.dtype == FT2_FP32) {
        cudaError_t e = launch_inject32(y.data, y.rows, y.n, y.ld, sites, n_sites, cur_layer, cur_step, base_row,
                                        static_cast<cudaStream_t>(stream), &nl);
        return finish(e, nl);
    }
    cudaError_t e = launch_inject(static_cast<uint16_t*>(y.data), y.rows, y.n, y.ld, sites, n_sites, cur_layer,
                                  cur_step, base_row, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_allreduce_protect(const void* const* partials, int64_t ldp, int32_t P, int32_t rank,
                                 uint32_t* const* flags, uint32_t* epoch, uint32_t* done, uint32_t* status,
                                 ft2_tensor y, const void* bias, ft2_gemm_mode mode, const int32_t* row_to_seq,
                                 const void* bounds, int32_t num_seqs, uint32_t* corrected_count,
                                 const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer, int32_t cur_step,
                                 const int32_t* base_row, void* stream) {
    ft2_status s = check_tensor(y);
    if (s != FT2_OK) return s;
    if (y.dtype == FT2_FP32) return FT2_ERR_UNSUPPORTED;
    if (P < 1 || P > kARMaxRanks || rank < 0 || rank >= P) return FT2_ERR_INVALID_ARG;
    if (partials == nullptr || flags == nullptr || epoch == nullptr || done == nullptr || status == nullptr)
        return FT2_ERR_INVALID_ARG;
    const int32_t m = (int32_t)mode & ~FT2_GEMM_W_STATIC;
    if (m != FT2_GEMM_PLAIN && m != FT2_GEMM_CHECK) return FT2_ERR_INVALID_ARG;
    if (m == FT2_GEMM_CHECK && (bounds == nullptr || num_seqs < 1)) return FT2_ERR_INVALID_ARG;
    if (m == FT2_GEMM_CHECK && row_to_seq == nullptr && num_seqs != 1 && (int64_t)num_seqs != y.rows)
        return FT2_ERR_INVALID_ARG;
    if (ldp < y.n || (ldp % 8) != 0) return ldp < y.n ? FT2_ERR_INVALID_ARG : FT2_ERR_MISALIGNED;
    if ((bias && !al16(bias)) || (bounds && ((uintptr_t)bounds & 3u) != 0)) return FT2_ERR_MISALIGNED;
    if (n_sites < 0 || (n_sites > 0 && sites == nullptr)) return FT2_ERR_INVALID_ARG;
    if ((y.rows * (y.n / 8)) >= (int64_t(1) << 31)) return FT2_ERR_UNSUPPORTED;
    if (y.rows == 0 || y.n == 0) return FT2_OK;   // identical on every rank: nobody waits
    AllreduceProtectArgs a = {};
    for (int t = 0; t < P; ++t) {   // host arrays: every pointer must be set
        if (partials[t] == nullptr || flags[t] == nullptr) return FT2_ERR_INVALID_ARG;
        if (!al16(partials[t])) return FT2_ERR_MISALIGNED;
        a.partials[t] = static_cast<const uint16_t*>(partials[t]);
        a.flags[t] = flags[t];
    }
    a.ldp = ldp;
    a.P = P;
    a.rank = rank;
    a.epoch = epoch;
    a.done = done;
    a.status = status;
    a.y = static_cast<uint16_t*>(y.data);
    a.ldy = y.ld;
    a.rows = y.rows;
    a.n = y.n;
    a.bias = static_cast<const uint16_t*>(bias);
    a.mode = m;
    a.row_to_seq = row_to_seq;
    a.bounds = static_cast<const uint16_t*>(bounds);
    a.S = num_seqs;
    a.counts = corrected_count;
    a.sites = sites;
    a.n_sites = sites ? n_sites : 0;
    a.cur_layer = cur_layer;
    a.cur_step = cur_step;
    a.base_row = base_row;
    a.dtype = y.dtype;
    int nl = 0;
    cudaError_t e = launch_allreduce_protect(a, static_cast<cudaStream_t>(stream), &nl);
    return finish(e, nl);
}

ft2_status ft2_ipc_get_handle(void* dev_ptr, void* handle_out, uint64_t* offset_out) {
    if (dev_ptr == nullptr || handle_out == nullptr || offset_out == nullptr) return FT2_ERR_INVALID_ARG;
    // IPC handles name whole allocations: find the allocation holding dev_ptr
    // (a caching allocator hands out sub-ranges) and report the offset into it
    typedef CUresult (*GetRange)(CUdeviceptr*, size_t*, CUdeviceptr);
    static GetRange get_range = [] {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            fn = nullptr;
        return reinterpret_cast<GetRange>(fn);
    }();
    if (get_range == nullptr) return FT2_ERR_CUDA;
    CUdeviceptr base = 0;
    size_t size = 0;
    if (get_range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) return FT2_ERR_CUDA;
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, (void*)base) != cudaSuccess) { cudaGetLastError(); return FT2_ERR_CUDA; }
    static_assert(sizeof(h) == 64, "cudaIpcMemHandle_t is 64 bytes");
    memcpy(handle_out, &h, sizeof(h));
    *offset_out = (uint64_t)((CUdeviceptr)dev_ptr - base);
    return FT2_OK;
}

ft2_status ft2_ipc_open_handle(const void* handle, void** dev_ptr_out) {
    if (handle == nullptr || dev_ptr_out == nullptr) return FT2_ERR_INVALID_ARG;
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    if (cudaIpcOpenMemHandle(dev_ptr_out, h, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        return FT2_ERR_CUDA;
    }
    return FT2_OK;
}

ft2_status ft2_ipc_close(void* dev_ptr) {
    if (dev_ptr == nullptr) return FT2_ERR_INVALID_ARG;
    if (cudaIpcCloseMemHandle(dev_ptr) != cudaSuccess) { cudaGetLastError(); return FT2_ERR_CUDA; }
    return FT2_OK;
}

const char* ft2_status_string(ft2_status s) {
    switch (s) {
        case FT2_OK: return "FT2_OK";
        case FT2_ERR_INVALID_ARG: return "FT2_ERR_INVALID_ARG";
        case FT2_ERR_MISALIGNED: return "FT2_ERR_MISALIGNED";
        case FT2_ERR_UNSUPPORTED: return "FT2_ERR_UNSUPPORTED";
        case FT2_ERR_CUDA: return "FT2_ERR_CUDA";
    }
    return "FT2_ERR_UNKNOWN";
}

uint64_t ft2_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

const char* ft2_version(void) { return "ft2-b200 0.1.0 sm_100a"; }

}  // extern "C"
