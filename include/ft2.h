/*
 * ft2.h -- C ABI of libft2.so, the B200 (sm_100a) implementation of FT2's
 * online range restriction (Sun et al., "FT2: First-Token-Inspired Online
 * Fault Tolerance on Critical Layers for Generative Large Language Models",
 * HPDC'25).  Citations are to /root/reference/PAPER.md as L<line> (section).
 *
 * The method (Sec. 4): (1) pick the critical linear
 * layers of the model (L149, L212; host-side); (2) while the
 * first token is generated (prefill) reduce each protected layer's output to
 * two bounds, widened by a factor 2 (L150, L221-L233, L332); (3) on every later
 * token check every neuron of each protected layer's output against those
 * bounds: out-of-bound values are clipped to the bound, NaN is corrected to 0
 * (L151, L191, L198, L259-L272).  Faults for evaluation are 1-bit, 2-bit or
 * exponent-bit flips of one neuron of one linear layer's output (L84, L90, L95).
 *
 * Conventions (all entry points):
 *  - Pointers are DEVICE pointers unless stated otherwise.  Every call is
 *    asynchronous on `stream` (a cudaStream_t passed as void*; NULL = legacy
 *    default stream), is CUDA-graph capturable, never allocates device memory,
 *    never synchronises, never throws.
 *  - The caller owns every buffer (tensors, bounds, counters, sites,
 *    workspace).  The library keeps no per-call state; the only global state
 *    is a host-side cache of TMA descriptors (mutex-protected) and a launch
 *    counter.
 *  - Errors are reported synchronously from argument checks:
 *      NULL required pointer, negative sizes, ld < n, num_seqs < 1, a
 *      non-finite or < 1 scale                       -> FT2_ERR_INVALID_ARG
 *      base pointer not 16-byte aligned, or ld % 8 != 0 (bf16)
 *                                                    -> FT2_ERR_MISALIGNED
 *      a dtype the entry point does not implement (see ft2_dtype), shapes
 *      outside the stated limits                     -> FT2_ERR_UNSUPPORTED
 *      kernel launch failure (cudaGetLastError)      -> FT2_ERR_CUDA
 *    A zero-size tensor returns FT2_OK without launching.  Faults inside a
 *    kernel surface at the caller's next synchronisation, as with CUDA.
 *  - Counters accumulate (the caller zeroes them), so one counter can span a
 *    whole request.
 *  - Tensors are row-major: element (r, j) of an ft2_tensor lives at
 *    data + (r * ld + j) * sizeof(dtype).
 *  - Values are compared on the total order of reading A7:
 *    -Inf < ... < -0 < +0 < ... < +Inf; a value equal to a bound is in bounds.
 */
#ifndef FT2_H_
#define FT2_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    FT2_OK = 0,
    FT2_ERR_INVALID_ARG = 1,
    FT2_ERR_MISALIGNED = 2,
    FT2_ERR_UNSUPPORTED = 3,
    FT2_ERR_CUDA = 4
} ft2_status;

/* Activation dtype.  BF16 and FP16 (the paper's main precision, L282) are
 * implemented by every entry point.  FP32 (the paper's FP32 study, L334;
 * SURVEY.md 8(f) NEXT(3)) is implemented by ft2_bounds_from_prefill,
 * ft2_bounds_finalize, ft2_protect, ft2_inject_faults and
 * ft2_make_fault_sites, on 32-bit order keys
 *     key32(b) = b & 0x80000000 ? ~b : b | 0x80000000
 * with bounds stored as fp32 pairs, R3's product/quotient formed in fp64 from
 * the fp32 value and scale and rounded outward to fp32, and keys_out in the
 * MAX-combinable encoding (int32)(~key32(lo_raw) ^ 0x80000000),
 * (int32)(key32(hi_raw) ^ 0x80000000), INT32_MIN = no finite value.  The
 * fused GEMMs (bf16/fp16 tensor-core contractions) return
 * FT2_ERR_UNSUPPORTED for FP32: use a library GEMM + ft2_protect. */
typedef enum { FT2_BF16 = 0, FT2_FP16 = 1, FT2_FP32 = 2 } ft2_dtype;

/* Fault models, PAPER.md L84 (Sec. 2.2): single-bit flip, double-bit flip,
 * single-bit flip in the exponent bits. */
typedef enum { FT2_FAULT_1BIT = 0, FT2_FAULT_2BIT = 1, FT2_FAULT_EXP = 2 } ft2_fault_model;

/* Epilogue of ft2_protect_fused_gemm. */
typedef enum {
    FT2_GEMM_PLAIN = 0, /* y = x W^T + b (+ faults), no check: the unprotected baseline */
    FT2_GEMM_CHECK = 1, /* ... then the check-and-clip of ft2_protect on the bf16 result */
    /* flag, OR-ed into the mode: w is not written by the kernel that precedes
     * this call in the stream (e.g. model weights), so its first tiles may be
     * fetched before the programmatic-dependent-launch wait. */
    FT2_GEMM_W_STATIC = 16
} ft2_gemm_mode;

typedef struct {
    void* data;       /* device pointer, 16-byte aligned */
    int64_t rows;     /* number of rows (tokens) */
    int64_t n;        /* elements per row (output neurons); multiple of 8 (bf16/fp16) or 4 (fp32):
                         one 16-byte vector */
    int64_t ld;       /* row stride in elements, >= n, same multiple as n */
    ft2_dtype dtype;
} ft2_tensor;

/* One fault-injection site: "the location ... is identified by
 * the layer ID, neuron ID, and bit locations"; extended with the trial id, the
 * token step (0 = prefill) and the prompt token for prefill faults. 24 bytes. */
typedef struct {
    uint32_t trial;    /* global trial id */
    uint16_t step;     /* 0 = prefill (first token), s >= 1 = decode step s */
    uint16_t layer;    /* linear-layer id in [0, n_layers) (block-major) */
    uint32_t token;    /* prompt token (row offset) when step == 0, else 0 */
    uint32_t col;      /* output neuron within the layer */
    uint32_t xor_mask; /* bits to flip in the element's bit pattern */
    uint8_t model;     /* ft2_fault_model */
    uint8_t nbits;     /* popcount(xor_mask) */
    uint8_t pad[2];
} ft2_fault_site;

/* Where faults can land (linear layers of the decoder blocks,
 * uniformly distributed locations).  layer_width is a HOST array. */
typedef struct {
    int32_t n_steps;            /* decode steps S; sites draw step in [0, S] */
    int32_t prompt_len;         /* prefill tokens T (token drawn in [0, T) for step 0) */
    int32_t n_layers;           /* linear layers L (<= FT2_MAX_SITE_LAYERS) */
    const int32_t* layer_width; /* host, [n_layers] output neurons per layer */
    int32_t layer_uniform;      /* 1: layer uniform then neuron uniform (reading A11, default);
                                   0: neuron-uniform over all layer outputs */
    int32_t step_policy;        /* 0: step uniform in [0, S] (reading A12);
                                   1: step = 1 + trial mod S (one fault per decode step, config C1) */
} ft2_site_geometry;

#define FT2_MAX_SITE_LAYERS 1024
#define FT2_MAX_SEQS 65535

/* ------------------------------------------------------------------------ */
/* Bytes of workspace ft2_bounds_from_prefill needs for num_seqs sequences.
 * The workspace must be zero-filled once before its first use; every call
 * leaves it zero-filled again (self-cleaning), so it can be reused and
 * captured in CUDA graphs.  One workspace must not be used by two calls that
 * may run concurrently. */
size_t ft2_workspace_bytes(int32_t num_seqs);

/* First-token bound profiling: PAPER.md L150 ("obtain bounds while generating
 * the first token"), L221-L233 (Sec. 4.2; bounds scaled by 2, TA#6), L332 (two
 * bound values per protected layer), L225/L237/L241 (NaN in the first token is
 * detected and corrected).
 *
 * y            [rows x n] prefill output of one protected layer.  Rows
 *              [seq_offsets[s], seq_offsets[s+1]) belong to sequence s
 *              (seq_offsets: device int32 [num_seqs+1], non-decreasing; NULL =
 *              one sequence of all rows).  Rows outside every range (padding)
 *              are ignored (reading A18).  Modified in place only when
 *              correct_nonfinite = 1, and then only its non-finite elements.
 * scale        widening factor c >= 1 (paper: 2).  lo <= 0 is multiplied by c,
 *              lo > 0 divided (symmetrically for hi), in fp32, rounded outward
 *              to bf16 and saturated to +-max finite (readings A2, A8, A10).
 * finalize     1: write bounds_out.  0: only write keys_out (raw order keys for
 *              a tensor-parallel MAX all-reduce, then ft2_bounds_finalize).
 * correct_nonfinite  1 (requires finalize = 1): after the bounds are known,
 *              NaN -> clamp(+0, lo, hi), +Inf -> hi, -Inf -> lo (readings A3-A6).
 * bounds_out   [num_seqs x 2] (lo, hi) per sequence in y.dtype (4-byte aligned; 8 for
 *              fp32), or NULL if finalize = 0.
 *              A sequence without finite values gets lo = hi = +0 (reading A9).
 * keys_out     NULL or int32 [num_seqs x 2]: keys_out[2s] = 0xFFFF - key(lo_raw),
 *              keys_out[2s+1] = key(hi_raw), -1 where the sequence has no finite
 *              value; element-wise MAX of these over shards gives the keys of
 *              the unsharded tensor (min/max are exact and associative).  For
 *              FT2_FP32 the encoding is the 32-bit one given at ft2_dtype.
 * nan_vulnerable_count  NULL or uint32 [num_seqs]: WRITTEN with the number of
 *              NaN-vulnerable values, those in (-2,-1) U (1,2) whose exponent-MSB
 *              flip gives NaN (Fig. 7; L202 reports their share per
 *              layer; L212: the alternative criticality proxy).  Computed in the
 *              same sweep; when NULL the sweep does not count them.
 * nonfinite_count  NULL or uint32 [num_seqs]: WRITTEN with the number of
 *              non-finite elements of each sequence.
 * workspace    ft2_workspace_bytes(num_seqs) bytes, see above.
 * Limits: num_seqs <= FT2_MAX_SEQS, rows * n / (8, fp32: 4) < 2^31. */
ft2_status ft2_bounds_from_prefill(ft2_tensor y, const int32_t* seq_offsets, int32_t num_seqs,
                                   float scale, int32_t finalize, int32_t correct_nonfinite,
                                   void* bounds_out, int32_t* keys_out, uint32_t* nonfinite_count,
                                   uint32_t* nan_vulnerable_count, void* workspace, void* stream);

/* Bounds from (all-reduced) keys in the ft2_bounds_from_prefill keys_out
 * encoding: the second half of the tensor-parallel path. */
ft2_status ft2_bounds_finalize(const int32_t* keys, int32_t num_seqs, float scale,
                               ft2_dtype dtype, void* bounds_out, void* stream);  /* dtype: BF16 / FP16 / FP32 */

/* Online range restriction of one protected layer's output: PAPER.md L151,
 * L259-L261 (Sec. 4.3: check every neuron after each critical layer), L261/L270
 * (TA#8: clip out-of-bound values to the bound), L191/L198 (NaN -> 0), L272
 * (clamp + nan_to_num fused).  In place on y:
 *   y' = clamp(isnan(y) ? +0 : y, lo_s, hi_s),   s = sequence of the row.
 * row_to_seq   device int32 [rows] row -> sequence, or NULL: row r -> sequence
 *              r when num_seqs == rows, every row -> sequence 0 when num_seqs
 *              == 1 (otherwise FT2_ERR_INVALID_ARG).  Rows mapped outside
 *              [0, num_seqs) are left untouched.
 * bounds       [num_seqs x 2] (lo, hi) in y.dtype with key(lo) <= key(hi), finite
 *              (4-byte aligned; 8 for fp32).
 * corrected_count  NULL or uint32 [num_seqs]: += number of elements whose bits
 *              changed (= NaN, +-Inf or out of bounds).
 * Only vectors containing a corrected element are written back. */
ft2_status ft2_protect(ft2_tensor y, const int32_t* row_to_seq, const void* bounds,
                       int32_t num_seqs, uint32_t* corrected_count, void* stream);

/* Critical linear layer with the check fused into the GEMM epilogue (tcgen05
 * MMA, TMEM accumulators, TMA-fed shared-memory pipeline on sm_100a):
 *   y[m, j] = check(inject(bf16_rne(sum_k x[m, k] * w[j, k] + bias[j])))
 * x [M x K] (ldx), w [N x K] (ldw, nn.Linear layout), bias [N] or NULL, y [M x N]
 * (ldy), all of type dtype (FT2_BF16 or FT2_FP16), fp32 accumulation.  The K reduction is complete before the
 * epilogue (split-K partial sums are combined first: clipping is non-linear).
 * mode         FT2_GEMM_PLAIN or FT2_GEMM_CHECK.
 * col_begin/col_end  the protected column slice [col_begin, col_end) (e.g. V of
 *              a fused QKV projection); 0/N = the whole output.
 * row_to_seq, bounds, num_seqs, corrected_count  as in ft2_protect (used by CHECK).
 * sites/n_sites/cur_layer/cur_step/base_row  optional fault injection applied
 *              to the bf16 result before the check (order: GEMM -> bias -> bf16 ->
 *              inject -> check; readings A19, A20), as in ft2_inject_faults.
 *              Any number of sites may land in one output tile: past the
 *              kernel's per-CTA site list (64; the M > 128 kernel: 4 per row
 *              per 256-column tile) it rescans every site for the affected
 *              elements, so no site is ever dropped (only slower).
 * workspace/ws_bytes  optional, 16-byte aligned, zero-filled once before first
 *              use (every call leaves its counters zero again).  Decode shapes
 *              (M <= 128) split K across a thread-block cluster and need none.
 *              The persistent M > 128 kernel splits K through it when its tiles
 *              cannot fill the GPU (small M): ft2_gemm_workspace_bytes(M, N, K)
 *              bytes give the best split, fewer bytes fewer splits, NULL none.
 *              Split partials are summed in split order: results do not depend
 *              on the workspace (only the timing does) -- except that a
 *              different split count changes the fp32 summation order.
 *              A split is planned only when every (tile, split) unit of the
 *              launch fits on the GPU at once (the splits of a tile wait for
 *              each other): do not run such a call concurrently with other
 *              kernels that hold SMs indefinitely (persistent kernels on other
 *              streams); pass NULL, or set FT2_PREFILL_SPLITS=0, to disable it.
 * The kernel is launched with programmatic stream serialization (PDL): its
 * prologue and first weight tiles overlap the previous kernel's tail; it reads
 * x, bias, bounds, sites and writes y, counters, workspace only after the
 * previous kernel has completed.
 * Limits: K % 8 == 0, ldx/ldw/ldy % 8 == 0, 16-byte aligned bases, M, N >= 1. */
size_t ft2_gemm_workspace_bytes(int32_t M, int32_t N, int32_t K);
ft2_status ft2_protect_fused_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw,
                                  const void* bias, void* y, int64_t ldy, int32_t M, int32_t N,
                                  int32_t K, ft2_gemm_mode mode, ft2_dtype dtype, int32_t col_begin, int32_t col_end,
                                  const int32_t* row_to_seq, const void* bounds, int32_t num_seqs,
                                  uint32_t* corrected_count, const ft2_fault_site* sites,
                                  int32_t n_sites, int32_t cur_layer, int32_t cur_step,
                                  const int32_t* base_row, void* workspace, size_t ws_bytes,
                                  void* stream);

/* ft2_protect_fused_gemm plus an L2 prefetch hint for the layer that runs
 * next (e.g. the next critical layer's weights: linear layers
 * are 94% of the compute and, at decode, a pure weight stream).  Decode shapes
 * (M <= 128) only: once a CTA's own operands have landed in shared memory it
 * issues cp.async.bulk.prefetch.L2 for its 1/grid share of
 * [l2_prefetch, l2_prefetch + l2_prefetch_bytes), so HBM keeps streaming
 * through this kernel's epilogue, the kernel boundary and the next kernel's
 * prologue.  A hint only: results are identical with or without it, nothing
 * is written, and the bytes are read-only for this kernel.  M > 128 ignores
 * it.  l2_prefetch == NULL with l2_prefetch_bytes == 0 is
 * ft2_protect_fused_gemm.
 * Errors: l2_prefetch_bytes > 0 with a NULL pointer -> FT2_ERR_INVALID_ARG;
 * pointer not 16-byte aligned or bytes % 16 != 0 -> FT2_ERR_MISALIGNED; else
 * as ft2_protect_fused_gemm. */
ft2_status ft2_protect_fused_gemm_ex(const void* x, int64_t ldx, const void* w, int64_t ldw,
                                     const void* bias, void* y, int64_t ldy, int32_t M, int32_t N,
                                     int32_t K, ft2_gemm_mode mode, ft2_dtype dtype, int32_t col_begin,
                                     int32_t col_end, const int32_t* row_to_seq, const void* bounds,
                                     int32_t num_seqs, uint32_t* corrected_count,
                                     const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer,
                                     int32_t cur_step, const int32_t* base_row, void* workspace,
                                     size_t ws_bytes, const void* l2_prefetch, size_t l2_prefetch_bytes,
                                     void* stream);

/* The critical linear layer during first-token generation (prefill) with the
 * first-token bound derivation fused into its GEMM epilogue (SURVEY.md 8(f)
 * NEXT(1)): PAPER.md L150 (bounds profiled on the first token), L221-L233
 * (min/max of the layer output, scaling factor 2), L225/L237/L241 (NaN/Inf in
 * the first token detected and corrected), L272 (after the critical layer).
 *   y = inject(bf16_rne(x W^T + b))        (as ft2_protect_fused_gemm PLAIN,
 *                                            faults of step 0 = the prefill)
 *   then, on y: exactly ft2_bounds_from_prefill(y, seq_offsets, num_seqs,
 *   scale, finalize = 1, correct_nonfinite, bounds_out, keys_out,
 *   nonfinite_count, NULL, workspace)
 * without reading y back: every output tile's per-row key extrema are reduced
 * per sequence in the epilogue (shared-memory table per CTA, one flush), the
 * last CTA scales the bounds (R3) and patches the recorded non-finite outputs
 * (R4).  Bounds, keys and counts are bit-identical to the two-call sequence
 * (GEMM, then ft2_bounds_from_prefill) on the same inputs.
 * x [M x K], w [N x K], bias [N] or NULL, y [M x N]: as ft2_protect_fused_gemm.
 * seq_offsets [num_seqs + 1] (rows outside [seq_offsets[0], seq_offsets[S]) are
 * padding, reading A18) or NULL for one sequence; scale, correct_nonfinite,
 * bounds_out, keys_out, nonfinite_count, workspace: as ft2_bounds_from_prefill
 * (workspace = ft2_workspace_bytes(num_seqs) bytes, zero-filled once, left zero).
 * gemm_workspace/gemm_ws_bytes: the optional K-split workspace of
 *              ft2_protect_fused_gemm (ft2_gemm_workspace_bytes(M, N, K)).
 * sites/n_sites/cur_layer/base_row: faults of step 0 (base_row = seq_offsets).
 * The GEMM is a persistent 128x256-tile tcgen05 kernel (one CTA per SM, TMEM
 * double-buffered accumulators); it is also what ft2_protect_fused_gemm runs
 * for M > 128.  Limits: N % 8 == 0, K % 8 == 0, ld* % 8 == 0, 16-byte aligned
 * x/w/y, M * N / 8 < 2^31, num_seqs <= FT2_MAX_SEQS.  M == 0: FT2_OK, no launch,
 * outputs untouched. */
ft2_status ft2_prefill_fused_gemm(const void* x, int64_t ldx, const void* w, int64_t ldw,
                                  const void* bias, void* y, int64_t ldy, int32_t M, int32_t N,
                                  int32_t K, ft2_dtype dtype, const int32_t* seq_offsets,
                                  int32_t num_seqs, float scale, int32_t correct_nonfinite,
                                  void* bounds_out, int32_t* keys_out, uint32_t* nonfinite_count,
                                  const ft2_fault_site* sites, int32_t n_sites, int32_t cur_layer,
                                  const int32_t* base_row, void* workspace, void* gemm_workspace,
                                  size_t gemm_ws_bytes, void* stream);

/* Seeded fault sites for trials [trial0, trial0 + n_trials) (reading R6:
 * Philox4x32-10 keyed by seed, counter = trial id; uniform step, layer, neuron
 * and bit position(s) per PAPER.md L84, L90, L95).  Bit-exact with the CPU
 * oracle; any trial range can be generated independently (campaign sharding).
 * geom is a HOST pointer; sites_out is device [n_trials]. */
ft2_status ft2_make_fault_sites(uint64_t seed, uint64_t trial0, int32_t n_trials,
                                ft2_fault_model model, ft2_dtype dtype,
                                const ft2_site_geometry* geom, ft2_fault_site* sites_out,
                                void* stream);

/* Apply the sites whose (step, layer) equals (cur_step, cur_layer) to y:
 * y[row, col] ^= xor_mask with row = (base_row ? base_row[i] : i) +
 * (cur_step == 0 ? token : 0) for site i (site i belongs to batch slot i;
 * pass seq_offsets as base_row during prefill).  Out-of-range sites are
 * ignored.  PAPER.md L90 (hook-based neuron bit flips). */
ft2_status ft2_inject_faults(ft2_tensor y, const ft2_fault_site* sites, int32_t n_sites,
                             int32_t cur_layer, int32_t cur_step, const int32_t* base_row,
                             void* stream);

/* Tensor-parallel row-parallel critical layer (o_proj / down_proj / out_proj /
 * fc2 under Megatron TP): its sum all-reduce fused with the check
 * (reading A17: row-parallel outputs are checked
 * after their sum all-reduce, PAPER.md L259-L272 for the check).  One-shot,
 * over peer memory (NVLink / NVSwitch through CUDA IPC mappings, ft2_ipc_*):
 *   y[r, c] = check(inject(rne(((p_0 + p_1) + ... + p_{P-1}) + bias[c])))
 * summed in fp32 in rank order 0..P-1 (reading A22), so every rank computes
 * the same bits; the check is ft2_protect's (FT2_GEMM_CHECK) or none
 * (FT2_GEMM_PLAIN: a plain one-shot all-reduce).
 * partials     HOST array [P] (P <= 64) of device pointers, 16-byte aligned:
 *              rank t's partial output [rows x n] (16-bit, row stride ldp) as
 *              mapped in THIS process (this rank's own buffer at index rank).
 *              Passed by value to the kernel (a captured graph keeps them).
 *              Double-buffer them: alternate two buffers per call.
 * flags        HOST array [P] of device pointers: rank t's flag array of P
 *              uint32 (zero-filled once, before the first call of any rank).
 * epoch, done, status  this rank's device uint32 words (zero-filled once):
 *              the call counter, a self-cleaning CTA counter, and an error
 *              word set to 1 if a peer did not arrive within 2^24 polls
 *              (the kernel then returns without writing y).
 * y            this rank's output [rows x n] (ld), 16-bit (bf16 / fp16).
 *              It may alias partials[rank] only when P == 1 (peers read the
 *              partials during the call); then, as in ft2_protect, only the
 *              16-byte vectors whose bits change are written back.
 * bias, row_to_seq, bounds, num_seqs, corrected_count, sites, n_sites,
 * cur_layer, cur_step, base_row: as in ft2_protect_fused_gemm / ft2_protect.
 * Sites: as ft2_inject_faults, none dropped (past 64 in one CTA's chunk the
 * kernel rescans every site).
 * Every rank must make the same sequence of calls with the same shapes.
 * Asynchronous on stream; graph-capturable (the epoch lives in device memory).
 * Launched with programmatic dependent launch: the kernel runs
 * griddepcontrol.wait before touching any global memory and releases its own
 * dependents right after it (FT2_AR_PDL=0 launches it plainly). */
ft2_status ft2_allreduce_protect(const void* const* partials, int64_t ldp, int32_t P, int32_t rank,
                                 uint32_t* const* flags, uint32_t* epoch, uint32_t* done, uint32_t* status,
                                 ft2_tensor y, const void* bias, ft2_gemm_mode mode,
                                 const int32_t* row_to_seq, const void* bounds, int32_t num_seqs,
                                 uint32_t* corrected_count, const ft2_fault_site* sites, int32_t n_sites,
                                 int32_t cur_layer, int32_t cur_step, const int32_t* base_row, void* stream);

/* CUDA IPC plumbing for ft2_allreduce_protect's buffers (setup time, not
 * the hot path): export the device allocation holding dev_ptr as a 64-byte
 * handle (host buffer) plus dev_ptr's byte offset inside it; map a peer's
 * handle into this process (the allocation's base; add the offset; peer
 * access is enabled lazily) and unmap it again with ft2_ipc_close(base). */
ft2_status ft2_ipc_get_handle(void* dev_ptr, void* handle_out, uint64_t* offset_out);
ft2_status ft2_ipc_open_handle(const void* handle, void** dev_ptr_out);
ft2_status ft2_ipc_close(void* dev_ptr);

/* Human-readable status. */
const char* ft2_status_string(ft2_status s);

/* Number of kernels this library has launched since it was loaded (host-side
 * counter; launches recorded into a CUDA graph count once, at capture). */
uint64_t ft2_launch_count(void);

/* Library version string ("ft2-b200 <semver> sm_100a"). */
const char* ft2_version(void);

/* ---- Host-model helper (NOT part of the FT2 method; PAPER.md L147-151 put
 * the norms outside the protected linear layers).  The decoder block's norm,
 * y[r, :] = (x[r, :] - mean) * rsqrt(var + eps) * w + b   (rms == 0, LayerNorm)
 * y[r, :] = x[r, :] * rsqrt(mean(x^2) + eps) * w          (rms != 0, RMSNorm; b ignored)
 * over rows x n row-major device tensors (leading dims ldx / ldy elements),
 * dtype FT2_BF16 or FT2_FP16, fp32 statistics, round-to-nearest-even output.
 * b may be NULL.  The kernel issues griddepcontrol.launch_dependents on
 * entry when rows <= the SM count (else after each CTA's last store) so a
 * following PDL launch (ft2_protect_fused_gemm) overlaps its prologue with
 * the norm; it is not counted by ft2_launch_count.
 * Errors: NULL x/w/y, rows < 0, n <= 0, eps < 0 or NaN -> FT2_ERR_INVALID_ARG;
 * n % 8 != 0, n > 8192, other dtypes -> FT2_ERR_UNSUPPORTED; ld < n, ld % 8,
 * pointers not 16-byte aligned -> FT2_ERR_MISALIGNED; launch failure ->
 * FT2_ERR_CUDA.  rows == 0: FT2_OK, no launch (checked before the NULL
 * checks).  Caller owns every buffer. */
ft2_status ft2_host_norm(const void* x, int64_t ldx, const void* w, const void* b, void* y, int64_t ldy,
                         int64_t rows, int32_t n, float eps, int rms, int dtype, void* stream);

/* ---- Host-model helper (NOT part of the FT2 method): the MLP activation
 * feeding the critical fc2 / down_proj layer, elementwise over rows x n
 * row-major device tensors (leading dims in elements):
 *   act == 0: y = relu(a)            (NaN propagates; b ignored, may be NULL)
 *   act == 1: y = round(round(silu(a)) * b), silu(a) = a / (1 + exp(-a)) in fp32
 * dtype FT2_BF16 / FT2_FP16, round-to-nearest-even; y may alias a.  Issues
 * griddepcontrol.launch_dependents as ft2_host_norm does; not counted
 * by ft2_launch_count.  Errors: rows < 0, n <= 0, act not 0/1, NULL a / y,
 * act == 1 with NULL b -> FT2_ERR_INVALID_ARG; other dtypes, rows * n / 8 >=
 * 2^31 -> FT2_ERR_UNSUPPORTED; n % 8, ld < n, ld % 8, pointers not 16-byte
 * aligned -> FT2_ERR_MISALIGNED; launch failure -> FT2_ERR_CUDA.  rows == 0:
 * FT2_OK, no launch. */
ft2_status ft2_host_act(const void* a, int64_t lda, const void* b, int64_t ldb, void* y, int64_t ldy, int64_t rows,
                        int32_t n, int act, int dtype, void* stream);

#ifdef __cplusplus
}
#endif
#endif /* FT2_H_ */
