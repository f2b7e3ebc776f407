/*
 * ft2_oracle.c -- plain, slow, obviously-correct CPU oracle for FT2's hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load this library.  The
 * product path (paper_conf_hpdc_sunzmg00y25_b200/, libft2.so) never links,
 * imports or calls it, and this file shares no code, header, table or
 * constant generator with csrc/.
 *
 * Source of every definition: /root/reference/PAPER.md (FT2, HPDC'25), cited
 * as L<line> plus section; where the paper is silent the reading is the one
 * listed in DESIGN.md "Readings" (A1..A21).
 *
 * Representation (R0): bf16 values are handled as their uint16 bit patterns;
 * every comparison is done on the order key
 *     key(b) = (b & 0x8000) ? (~b & 0xFFFF) : (b | 0x8000)
 * which is a total order on non-NaN values (-Inf < ... < -0 < +0 < ... < +Inf).
 * Floating point appears only in bound scaling (R3, fp32 as the reading fixes)
 * and in the reference GEMM (R8, fp64 accumulation).  Compiled with
 * -O2 -fno-fast-math -ffp-contract=off so every fp op is a single IEEE op.
 */
#include <math.h>
#include <stdint.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

#define EXPORT __attribute__((visibility("default")))

/* ------------------------------------------------------------------ R0 --- */
/* 16-bit floating formats: bf16 1/8/7 (the build's activation type) and the
 * paper's FP16 1/5/10 (PAPER.md L185 describes that layout; L282: FP16 models).
 * dtype 0 = bf16, 1 = fp16.  Both are sign-magnitude, so the order key below
 * is the same function for both; only the exponent field differs. */
typedef struct {
    int mbits;        /* fraction bits */
    int bias;         /* exponent bias */
    uint16_t expmask; /* exponent field */
    uint16_t maxfin;  /* largest finite magnitude */
    uint16_t qnan;    /* canonical NaN */
} ft2o_fmt;
static const ft2o_fmt FMT[2] = {
    {7, 127, 0x7F80, 0x7F7F, 0x7FC0},  /* bf16 */
    {10, 15, 0x7C00, 0x7BFF, 0x7E00},  /* fp16 */
};
static const ft2o_fmt* fmt_of(int dtype) { return &FMT[dtype == 1 ? 1 : 0]; }

EXPORT int ft2o_isnan_dt(uint16_t b, int dtype) { return (b & 0x7FFF) > fmt_of(dtype)->expmask; }
EXPORT int ft2o_isinf_dt(uint16_t b, int dtype) { return (b & 0x7FFF) == fmt_of(dtype)->expmask; }
EXPORT int ft2o_isfinite_dt(uint16_t b, int dtype) {
    const uint16_t e = fmt_of(dtype)->expmask;
    return (b & e) != e;
}
EXPORT int ft2o_isnan(uint16_t b) { return ft2o_isnan_dt(b, 0); }
EXPORT int ft2o_isinf(uint16_t b) { return ft2o_isinf_dt(b, 0); }
EXPORT int ft2o_isfinite(uint16_t b) { return ft2o_isfinite_dt(b, 0); }

EXPORT uint16_t ft2o_key(uint16_t b) {
    return (b & 0x8000) ? (uint16_t)(~b & 0xFFFF) : (uint16_t)(b | 0x8000);
}

EXPORT uint16_t ft2o_unkey(uint16_t k) {
    return (k & 0x8000) ? (uint16_t)(k & 0x7FFF) : (uint16_t)(~k & 0xFFFF);
}

/* Exact value of a 16-bit float (from the definition of the format). */
EXPORT double ft2o_to_f64_dt(uint16_t b, int dtype) {
    const ft2o_fmt* f = fmt_of(dtype);
    const int ebits = (f->expmask >> f->mbits) & 0xFF;  /* all-ones exponent value */
    int e = (b >> f->mbits) & ebits;
    int m = b & ((1 << f->mbits) - 1);
    double s = (b & 0x8000) ? -1.0 : 1.0;
    if (e == ebits) return m ? NAN : s * INFINITY;
    if (e == 0) return s * ldexp((double)m, 1 - f->bias - f->mbits);      /* subnormal */
    return s * ldexp((double)((1 << f->mbits) | m), e - f->bias - f->mbits);
}
EXPORT double ft2o_bf16_to_f64(uint16_t b) { return ft2o_to_f64_dt(b, 0); }

/* Round-to-nearest-even of an arbitrary double to the 16-bit format (NaN ->
 * canonical NaN).  Written from the definition: the representable spacing at
 * the value's binade is 2^(E - mbits) (2^(emin - mbits) below the normal
 * range), and rint() in the default FE_TONEAREST mode is ties-to-even.  Used
 * for R8 (fp64 GEMM -> activation type) and for fp32 inputs (exact promotion
 * to double). */
EXPORT uint16_t ft2o_f64_to_dt_rne(double d, int dtype) {
    const ft2o_fmt* f = fmt_of(dtype);
    const int emin = 1 - f->bias;
    if (isnan(d)) return f->qnan;
    uint16_t sign = signbit(d) ? 0x8000 : 0x0000;
    double a = fabs(d);
    if (isinf(a)) return sign | f->expmask;
    if (a < ldexp(1.0, emin)) {
        /* subnormal range; q == 2^mbits encodes the smallest normal */
        double q = rint(ldexp(a, f->mbits - emin));
        return sign | (uint16_t)q;
    }
    int e;
    double m = frexp(a, &e); /* a = m * 2^e, m in [0.5, 1) */
    double q = rint(ldexp(m, f->mbits + 1)); /* significand, [2^mbits, 2^(mbits+1)] */
    int E = e - 1;
    if (q == ldexp(1.0, f->mbits + 1)) { q = ldexp(1.0, f->mbits); E += 1; }
    if (E + f->bias >= 2 * f->bias + 1) return sign | f->expmask; /* overflow -> Inf */
    return sign | (uint16_t)(((E + f->bias) << f->mbits) | ((int)q - (1 << f->mbits)));
}
EXPORT uint16_t ft2o_f64_to_bf16_rne(double d) { return ft2o_f64_to_dt_rne(d, 0); }

/* Directed rounding of a double: dir = -1 toward -Inf, +1 toward +Inf.  Used
 * by R3 (bounds are rounded outward, reading A10).  Defined from RNE: take
 * the nearest value, and step one ulp outward (in key order) if it lies on
 * the wrong side of d. */
EXPORT uint16_t ft2o_f64_to_dt_dir(double d, int dir, int dtype) {
    uint16_t r = ft2o_f64_to_dt_rne(d, dtype);
    double rv = ft2o_to_f64_dt(r, dtype);
    if (dir < 0 && rv > d) r = ft2o_unkey((uint16_t)(ft2o_key(r) - 1));
    if (dir > 0 && rv < d) r = ft2o_unkey((uint16_t)(ft2o_key(r) + 1));
    return r;
}
EXPORT uint16_t ft2o_f64_to_bf16_dir(double d, int dir) { return ft2o_f64_to_dt_dir(d, dir, 0); }

/* ------------------------------------------------------------------ R3 --- */
/* Bound scaling, PAPER.md L229-L233 (Sec. 4.2.1, TA#6): "the scaling factor is
 * set to 2".  Reading A2: widen away from the interval, i.e. lo <= 0 is
 * multiplied by c and lo > 0 divided by c (and symmetrically for hi).  The
 * product/quotient is formed in fp32 (one IEEE op), then rounded outward to
 * the activation type (A10) and saturated to +-max finite (A8). */
EXPORT uint16_t ft2o_scale_bound_dt(uint16_t raw, float c, int is_hi, int dtype) {
    const ft2o_fmt* f = fmt_of(dtype);
    float x = (float)ft2o_to_f64_dt(raw, dtype);
    volatile float s;
    if (is_hi) s = (x >= 0.0f) ? x * c : x / c;
    else       s = (x <= 0.0f) ? x * c : x / c;
    uint16_t r = ft2o_f64_to_dt_dir((double)s, is_hi ? +1 : -1, dtype);
    if (r == f->expmask) r = f->maxfin;                           /* +Inf -> +max finite */
    if (r == (uint16_t)(0x8000 | f->expmask)) r = 0x8000 | f->maxfin; /* -Inf -> -max finite */
    return r;
}
EXPORT uint16_t ft2o_scale_bound(uint16_t raw, float c, int is_hi) { return ft2o_scale_bound_dt(raw, c, is_hi, 0); }

/* ------------------------------------------------------------------ R5 --- */
/* Check-and-clip of one value, PAPER.md L259-L261 (Sec. 4.3: "FT2 checks all
 * the neuron values within each critical layer"), L261/L270 (TA#8: out-of-bound
 * values are clipped to the bound), L191/L198 (NaN corrected to 0), L272
 * (torch.clamp + torch.nan_to_num).  Reading A5: NaN -> clamp(+0, lo, hi);
 * A6: +-Inf -> hi/lo through the clamp; A7: a value equal to a bound is in
 * bounds, order = key order. Returns the corrected bits. */
EXPORT uint16_t ft2o_clip_value_dt(uint16_t y, uint16_t lo, uint16_t hi, int dtype) {
    uint16_t x = ft2o_isnan_dt(y, dtype) ? 0x0000 : y; /* nan_to_num(nan=0.0) */
    uint16_t k = ft2o_key(x);
    if (k < ft2o_key(lo)) return lo;
    if (k > ft2o_key(hi)) return hi;
    return x;
}
EXPORT uint16_t ft2o_clip_value(uint16_t y, uint16_t lo, uint16_t hi) { return ft2o_clip_value_dt(y, lo, hi, 0); }

/* In-place check-and-clip of y[rows][n] (row stride ld).  Row r belongs to
 * sequence row_to_seq[r]; bounds[2*s] = lo_s, bounds[2*s+1] = hi_s.
 * count[s] += number of elements whose bits changed (R5: corrected <=> y' != y).
 * Rows whose sequence is out of [0, num_seqs) are skipped. */
EXPORT void ft2o_protect_dt(uint16_t* y, int64_t rows, int64_t n, int64_t ld,
                            const int32_t* row_to_seq, const uint16_t* bounds,
                            int32_t num_seqs, uint32_t* count, int dtype) {
    /* rows are independent; a row's corrections are added to its sequence's
     * count once (integer sum: any order gives the same count) */
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < rows; ++r) {
        int32_t s = row_to_seq ? row_to_seq[r] : (num_seqs == 1 ? 0 : (int32_t)r);
        if (s < 0 || s >= num_seqs) continue;
        uint16_t lo = bounds[2 * s], hi = bounds[2 * s + 1];
        uint32_t changed = 0;
        for (int64_t j = 0; j < n; ++j) {
            uint16_t v = y[r * ld + j];
            uint16_t w = ft2o_clip_value_dt(v, lo, hi, dtype);
            if (w != v) {
                y[r * ld + j] = w;
                changed += 1;
            }
        }
        if (count && changed) {
#pragma omp atomic
            count[s] += changed;
        }
    }
}

/* Threads the oracle's loops over independent outputs may use (OpenMP; every
 * result is identical for any count: each output is computed by one thread
 * in the stated order).  n < 1 restores the default. */
EXPORT void ft2o_set_threads(int32_t n) {
#ifdef _OPENMP
    omp_set_num_threads(n >= 1 ? n : omp_get_num_procs());
#else
    (void)n;
#endif
}
EXPORT int32_t ft2o_max_threads(void) {
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
EXPORT void ft2o_protect(uint16_t* y, int64_t rows, int64_t n, int64_t ld, const int32_t* row_to_seq,
                         const uint16_t* bounds, int32_t num_seqs, uint32_t* count) {
    ft2o_protect_dt(y, rows, n, ld, row_to_seq, bounds, num_seqs, count, 0);
}

/* ------------------------------------------------------------- R2/R3/R4 --- */
/* First-token bound profiling, PAPER.md L150 ("obtain bounds while generating
 * the first token"), L221-L233 (Sec. 4.2), L332 ("two bound values are stored
 * for each layer").  Readings A1 (one pair per sequence), A3/A4 (non-finite
 * values excluded from the reduction), A9 (no finite value -> lo = hi = +0),
 * A18 (only rows inside seq_offsets ranges count).
 *
 * y: [rows][n] bits, stride ld.  seq_offsets: [S+1] row offsets (NULL = one
 * sequence covering all rows).  Outputs per sequence s:
 *   raw_keys[2s] = key(min finite) or -1, raw_keys[2s+1] = key(max finite) or -1
 *   bounds[2s], bounds[2s+1] = R3-scaled lo, hi (bits)
 *   nonfinite[s] = number of non-finite elements
 * If correct_nonfinite, R4 applies R5 to the prefill output with the fresh
 * bounds ("NaN can always be detected and
 * corrected" during the first token). */
EXPORT void ft2o_bounds_dt(uint16_t* y, int64_t rows, int64_t n, int64_t ld,
                           const int32_t* seq_offsets, int32_t num_seqs, float scale,
                           int32_t correct_nonfinite, uint16_t* bounds, int32_t* raw_keys,
                           uint32_t* nonfinite, int dtype) {
    /* sequences are independent (one thread each) */
#pragma omp parallel for schedule(dynamic)
    for (int32_t s = 0; s < num_seqs; ++s) {
        int64_t r0 = seq_offsets ? seq_offsets[s] : 0;
        int64_t r1 = seq_offsets ? seq_offsets[s + 1] : rows;
        int have = 0;
        uint16_t kmin = 0, kmax = 0;
        uint32_t nf = 0;
        for (int64_t r = r0; r < r1; ++r) {
            for (int64_t j = 0; j < n; ++j) {
                uint16_t v = y[r * ld + j];
                if (!ft2o_isfinite_dt(v, dtype)) { nf++; continue; }
                uint16_t k = ft2o_key(v);
                if (!have || k < kmin) kmin = k;
                if (!have || k > kmax) kmax = k;
                have = 1;
            }
        }
        uint16_t lo, hi;
        if (have) {
            lo = ft2o_scale_bound_dt(ft2o_unkey(kmin), scale, 0, dtype);
            hi = ft2o_scale_bound_dt(ft2o_unkey(kmax), scale, 1, dtype);
        } else {
            lo = hi = 0x0000; /* A9 */
        }
        if (raw_keys) {
            raw_keys[2 * s] = have ? (int32_t)kmin : -1;
            raw_keys[2 * s + 1] = have ? (int32_t)kmax : -1;
        }
        if (bounds) { bounds[2 * s] = lo; bounds[2 * s + 1] = hi; }
        if (nonfinite) nonfinite[s] = nf;
        if (correct_nonfinite) {
            for (int64_t r = r0; r < r1; ++r)
                for (int64_t j = 0; j < n; ++j)
                    y[r * ld + j] = ft2o_clip_value_dt(y[r * ld + j], lo, hi, dtype);
        }
    }
}
EXPORT void ft2o_bounds(uint16_t* y, int64_t rows, int64_t n, int64_t ld, const int32_t* seq_offsets,
                        int32_t num_seqs, float scale, int32_t correct_nonfinite, uint16_t* bounds,
                        int32_t* raw_keys, uint32_t* nonfinite) {
    ft2o_bounds_dt(y, rows, n, ld, seq_offsets, num_seqs, scale, correct_nonfinite, bounds, raw_keys, nonfinite, 0);
}

/* Bounds from raw keys (the TP path): raw_keys as produced by
 * ft2o_bounds (-1 = no finite value). */
EXPORT void ft2o_bounds_from_keys_dt(const int32_t* raw_keys, int32_t num_seqs, float scale,
                                     uint16_t* bounds, int dtype) {
    for (int32_t s = 0; s < num_seqs; ++s) {
        int32_t a = raw_keys[2 * s], b = raw_keys[2 * s + 1];
        if (a < 0 || b < 0) { bounds[2 * s] = bounds[2 * s + 1] = 0; continue; }
        bounds[2 * s] = ft2o_scale_bound_dt(ft2o_unkey((uint16_t)a), scale, 0, dtype);
        bounds[2 * s + 1] = ft2o_scale_bound_dt(ft2o_unkey((uint16_t)b), scale, 1, dtype);
    }
}
EXPORT void ft2o_bounds_from_keys(const int32_t* raw_keys, int32_t num_seqs, float scale, uint16_t* bounds) {
    ft2o_bounds_from_keys_dt(raw_keys, num_seqs, scale, bounds, 0);
}

/* NaN-vulnerable values, PAPER.md L185 (Sec. 4.1.1, Fig. 7): "Values with
 * specific exponent bits can become NaN after a single-bit flip, and most of
 * them are in the intervals (-2, -1) or (1, 2) ... the NaN-vulnerable area";
 * L202/L212: their share is the alternative criticality proxy.  Count, per
 * sequence, the elements whose value v satisfies 1 < |v| < 2. */
EXPORT void ft2o_nan_vulnerable_count(const uint16_t* y, int64_t rows, int64_t n, int64_t ld,
                                      const int32_t* seq_offsets, int32_t num_seqs, uint32_t* out, int dtype) {
    for (int32_t s = 0; s < num_seqs; ++s) {
        int64_t r0 = seq_offsets ? seq_offsets[s] : 0;
        int64_t r1 = seq_offsets ? seq_offsets[s + 1] : rows;
        uint32_t c = 0;
        for (int64_t r = r0; r < r1; ++r)
            for (int64_t j = 0; j < n; ++j) {
                double v = fabs(ft2o_to_f64_dt(y[r * ld + j], dtype));
                if (v > 1.0 && v < 2.0) c++;
            }
        out[s] = c;
    }
}

/* --------------------------------------------------------------- Philox --- */
/* Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11), the counter-based
 * generator the fault-site reading R6 uses. */
static void mulhilo32(uint32_t a, uint32_t b, uint32_t* hi, uint32_t* lo) {
    uint64_t p = (uint64_t)a * (uint64_t)b;
    *hi = (uint32_t)(p >> 32);
    *lo = (uint32_t)p;
}
EXPORT void ft2o_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
    uint32_t c[4] = {ctr_in[0], ctr_in[1], ctr_in[2], ctr_in[3]};
    uint32_t k0 = key_in[0], k1 = key_in[1];
    for (int r = 0; r < 10; ++r) {
        if (r > 0) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
        uint32_t hi0, lo0, hi1, lo1;
        mulhilo32(0xD2511F53u, c[0], &hi0, &lo0);
        mulhilo32(0xCD9E8D57u, c[2], &hi1, &lo1);
        uint32_t n0 = hi1 ^ c[1] ^ k0, n1 = lo1, n2 = hi0 ^ c[3] ^ k1, n3 = lo0;
        c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
    }
    out[0] = c[0]; out[1] = c[1]; out[2] = c[2]; out[3] = c[3];
}

/* --------------------------------------------------------------- R6 ------ */
/* Fault sites, PAPER.md L84 (Sec. 2.2: 1-bit, 2-bit, EXP fault models), L88
 * ("only one error occurs per inference"), L90 ("the location ... is
 * identified by the layer ID, neuron ID, and bit locations"), L95 (uniformly
 * distributed location; linear layers of the decoder blocks).  Readings A11
 * (layer-then-neuron uniform, or size-weighted neuron-uniform), A12 (step
 * uniform over 0..S, 0 = prefill with a uniform prompt token), A13 (2-bit =
 * two distinct uniform positions; EXP = uniform over the exponent field).
 *
 * Site layout matches include/ft2.h's ft2_fault_site bit for bit, but the
 * struct is restated here (no shared header). */
typedef struct {
    uint32_t trial;
    uint16_t step, layer;
    uint32_t token, col;
    uint32_t xor_mask;
    uint8_t model, nbits, pad[2];
} ft2o_site;

static uint32_t draw_below(uint32_t u, uint32_t n) { /* floor(u * n / 2^32) */
    return (uint32_t)(((uint64_t)u * (uint64_t)n) >> 32);
}

/* dtype: 0 bf16 (16 bits, exponent bits 7..14), 1 fp16 (10..14), 2 fp32 (23..30) */
EXPORT void ft2o_make_sites(uint64_t seed, uint64_t trial0, int32_t n_trials, int32_t model,
                            int32_t dtype, int32_t n_steps, int32_t prompt_len, int32_t n_layers,
                            const int32_t* layer_width, int32_t layer_uniform, int32_t step_policy,
                            ft2o_site* out) {
    uint32_t width_bits = (dtype == 2) ? 32u : 16u;
    uint32_t exp_lo = (dtype == 0) ? 7u : (dtype == 1) ? 10u : 23u;
    uint32_t exp_n = (dtype == 0) ? 8u : (dtype == 1) ? 5u : 8u;
    uint64_t total_neurons = 0;
    for (int32_t l = 0; l < n_layers; ++l) total_neurons += (uint64_t)layer_width[l];
    for (int32_t i = 0; i < n_trials; ++i) {
        uint64_t t = trial0 + (uint64_t)i;
        uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
        uint32_t c0[4] = {(uint32_t)t, (uint32_t)(t >> 32), 0u, 0x46543200u};
        uint32_t c1[4] = {(uint32_t)t, (uint32_t)(t >> 32), 1u, 0x46543200u};
        uint32_t u[4], v[4];
        ft2o_philox4x32_10(c0, key, u);
        ft2o_philox4x32_10(c1, key, v);
        ft2o_site s;
        memset(&s, 0, sizeof(s));
        s.trial = (uint32_t)t;
        uint32_t step;
        if (step_policy == 1) step = 1u + (uint32_t)(t % (uint64_t)n_steps); /* one per decode step */
        else step = draw_below(u[0], (uint32_t)n_steps + 1u);               /* A12 */
        s.step = (uint16_t)step;
        uint32_t layer, col;
        if (layer_uniform) {
            layer = draw_below(u[1], (uint32_t)n_layers);
            col = draw_below(u[2], (uint32_t)layer_width[layer]);
        } else {
            /* neuron-uniform over all layers' outputs: one draw in [0, total) */
            uint64_t g = ((uint64_t)u[1] * total_neurons) >> 32;
            layer = 0;
            while (g >= (uint64_t)layer_width[layer]) { g -= (uint64_t)layer_width[layer]; layer++; }
            col = (uint32_t)g;
        }
        s.layer = (uint16_t)layer;
        s.col = col;
        s.token = (step == 0) ? draw_below(v[0], (uint32_t)prompt_len) : 0u;
        uint32_t mask;
        if (model == 0) {        /* 1-bit */
            mask = 1u << draw_below(u[3], width_bits);
            s.nbits = 1;
        } else if (model == 1) { /* 2-bit: two distinct positions */
            uint32_t b1 = draw_below(u[3], width_bits);
            uint32_t b2p = draw_below(v[1], width_bits - 1u);
            uint32_t b2 = b2p + (b2p >= b1 ? 1u : 0u);
            mask = (1u << b1) | (1u << b2);
            s.nbits = 2;
        } else {                 /* EXP: one bit of the exponent field */
            mask = 1u << (exp_lo + draw_below(u[3], exp_n));
            s.nbits = 1;
        }
        s.xor_mask = mask;
        s.model = (uint8_t)model;
        out[i] = s;
    }
}

/* --------------------------------------------------------------- R7 ------ */
/* Injection, PAPER.md L90 (hook flips bits of the selected neuron in the
 * layer output).  Site i belongs to batch slot i; its row is
 * base_row[i] (or i if base_row is NULL) plus the prompt token when the
 * current step is the prefill (step 0).  Sites that do not match
 * (cur_step, cur_layer) or fall outside y are ignored. */
EXPORT void ft2o_inject(uint16_t* y, int64_t rows, int64_t n, int64_t ld, const ft2o_site* sites,
                        int32_t n_sites, int32_t cur_layer, int32_t cur_step, const int32_t* base_row) {
    for (int32_t i = 0; i < n_sites; ++i) {
        const ft2o_site* s = &sites[i];
        if ((int32_t)s->step != cur_step || (int32_t)s->layer != cur_layer) continue;
        int64_t row = (base_row ? base_row[i] : i) + (cur_step == 0 ? (int64_t)s->token : 0);
        if (row < 0 || row >= rows || (int64_t)s->col >= n) continue;
        y[row * ld + s->col] ^= (uint16_t)s->xor_mask;
    }
}

/* --------------------------------------------------------------- R8 ------ */
/* Reference linear layer for the fused path: y = x W^T + b (nn.Linear),
 * accumulated in fp64 (independent of summation order), rounded once to bf16.
 * x: [M][K] (ldx), w: [N][K] (ldw), bias: [N] or NULL, y: [M][N] (ldy). */
EXPORT void ft2o_linear_f64_dt(const uint16_t* x, int64_t ldx, const uint16_t* w, int64_t ldw,
                               const uint16_t* bias, int32_t M, int32_t N, int32_t K,
                               double* y_f64, uint16_t* y_out, int64_t ldy, int dtype) {
    /* every output element is one thread's sequential k = 0..K-1 sum */
#pragma omp parallel for collapse(2) schedule(static)
    for (int32_t m = 0; m < M; ++m) {
        for (int32_t j = 0; j < N; ++j) {
            double acc = 0.0;
            for (int32_t k = 0; k < K; ++k)
                acc += ft2o_to_f64_dt(x[(int64_t)m * ldx + k], dtype) * ft2o_to_f64_dt(w[(int64_t)j * ldw + k], dtype);
            if (bias) acc += ft2o_to_f64_dt(bias[j], dtype);
            if (y_f64) y_f64[(int64_t)m * ldy + j] = acc;
            if (y_out) y_out[(int64_t)m * ldy + j] = ft2o_f64_to_dt_rne(acc, dtype);
        }
    }
}
EXPORT void ft2o_linear_f64(const uint16_t* x, int64_t ldx, const uint16_t* w, int64_t ldw,
                            const uint16_t* bias, int32_t M, int32_t N, int32_t K,
                            double* y_f64, uint16_t* y_bf16, int64_t ldy) {
    ft2o_linear_f64_dt(x, ldx, w, ldw, bias, M, N, K, y_f64, y_bf16, ldy, 0);
}

/* Full oracle layer (R8 then R7 then R5): linear -> bf16 -> inject -> check. */
EXPORT void ft2o_protected_linear(const uint16_t* x, int64_t ldx, const uint16_t* w, int64_t ldw,
                                  const uint16_t* bias, int32_t M, int32_t N, int32_t K,
                                  uint16_t* y, int64_t ldy, const int32_t* row_to_seq,
                                  const uint16_t* bounds, int32_t num_seqs, uint32_t* count,
                                  const ft2o_site* sites, int32_t n_sites, int32_t cur_layer,
                                  int32_t cur_step, const int32_t* base_row) {
    ft2o_linear_f64(x, ldx, w, ldw, bias, M, N, K, 0, y, ldy);
    if (sites && n_sites > 0) ft2o_inject(y, M, N, ldy, sites, n_sites, cur_layer, cur_step, base_row);
    if (bounds) ft2o_protect(y, M, N, ldy, row_to_seq, bounds, num_seqs, count);
}

EXPORT void ft2o_protected_linear_dt(const uint16_t* x, int64_t ldx, const uint16_t* w, int64_t ldw,
                                     const uint16_t* bias, int32_t M, int32_t N, int32_t K,
                                     uint16_t* y, int64_t ldy, const int32_t* row_to_seq,
                                     const uint16_t* bounds, int32_t num_seqs, uint32_t* count,
                                     const ft2o_site* sites, int32_t n_sites, int32_t cur_layer,
                                     int32_t cur_step, const int32_t* base_row, int dtype) {
    ft2o_linear_f64_dt(x, ldx, w, ldw, bias, M, N, K, 0, y, ldy, dtype);
    if (sites && n_sites > 0) ft2o_inject(y, M, N, ldy, sites, n_sites, cur_layer, cur_step, base_row);
    if (bounds) ft2o_protect_dt(y, M, N, ldy, row_to_seq, bounds, num_seqs, count, dtype);
}


/* ------------------------------------------------------------ FP32 --- */
/* The paper's FP32 study (Sec. 6: FT2 "also applies to FP32
 * models") runs the same method on 32-bit activations.  R0 for binary32:
 * values are uint32 bit patterns, ordered by the 32-bit key
 *     key32(b) = (b & 0x80000000) ? ~b : (b | 0x80000000)
 * (total order on non-NaN values: -Inf = 0x007FFFFF < ... < -0 = 0x7FFFFFFF
 * < +0 = 0x80000000 < ... < +Inf = 0xFF800000; NaN keys lie outside).
 * Readings A2-A10 carry over unchanged; R3's product / quotient is formed in
 * fp64 from the fp32 value and the fp32 scale (the product is exact; the
 * quotient is one IEEE division), then rounded outward to fp32 and saturated
 * to +-FLT_MAX. */
EXPORT int ft2o_isnan32(uint32_t b) { return (b & 0x7FFFFFFFu) > 0x7F800000u; }
EXPORT int ft2o_isfinite32(uint32_t b) { return (b & 0x7F800000u) != 0x7F800000u; }
EXPORT uint32_t ft2o_key32(uint32_t b) { return (b & 0x80000000u) ? ~b : (b | 0x80000000u); }
EXPORT uint32_t ft2o_unkey32(uint32_t k) { return (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k; }

static float f32_of(uint32_t b) { float f; memcpy(&f, &b, 4); return f; }
static uint32_t bits_of(float f) { uint32_t b; memcpy(&b, &f, 4); return b; }

/* Outward rounding of a double to fp32 (dir -1 toward -Inf, +1 toward +Inf):
 * the nearest fp32 (the C conversion, round-to-nearest-even), then one step
 * outward in key order if it lies on the wrong side of d. */
static uint32_t f64_to_f32_dir(double d, int dir) {
    uint32_t r = bits_of((float)d);
    double rv = (double)f32_of(r);
    if (dir < 0 && rv > d) r = ft2o_unkey32(ft2o_key32(r) - 1u);
    if (dir > 0 && rv < d) r = ft2o_unkey32(ft2o_key32(r) + 1u);
    return r;
}

EXPORT uint32_t ft2o_scale_bound32(uint32_t raw, float c32, int is_hi) {
    double x = (double)f32_of(raw), c = (double)c32;   /* the ABI's fp32 scale, exact in fp64 */
    volatile double s;
    if (is_hi) s = (x >= 0.0) ? x * c : x / c;
    else       s = (x <= 0.0) ? x * c : x / c;
    uint32_t r = f64_to_f32_dir((double)s, is_hi ? +1 : -1);
    if (r == 0x7F800000u) r = 0x7F7FFFFFu;   /* +Inf -> +FLT_MAX (A8) */
    if (r == 0xFF800000u) r = 0xFF7FFFFFu;   /* -Inf -> -FLT_MAX */
    return r;
}

/* R5 for binary32 (A5-A7 as for the 16-bit formats). */
EXPORT uint32_t ft2o_clip_value32(uint32_t y, uint32_t lo, uint32_t hi) {
    uint32_t x = ft2o_isnan32(y) ? 0u : y;
    uint32_t k = ft2o_key32(x);
    if (k < ft2o_key32(lo)) return lo;
    if (k > ft2o_key32(hi)) return hi;
    return x;
}

EXPORT void ft2o_protect32(uint32_t* y, int64_t rows, int64_t n, int64_t ld, const int32_t* row_to_seq,
                           const uint32_t* bounds, int32_t num_seqs, uint32_t* count) {
    for (int64_t r = 0; r < rows; ++r) {
        int32_t s = row_to_seq ? row_to_seq[r] : (num_seqs == 1 ? 0 : (int32_t)r);
        if (s < 0 || s >= num_seqs) continue;
        for (int64_t j = 0; j < n; ++j) {
            uint32_t v = y[r * ld + j];
            uint32_t w = ft2o_clip_value32(v, bounds[2 * s], bounds[2 * s + 1]);
            if (w != v) {
                y[r * ld + j] = w;
                if (count) count[s] += 1;
            }
        }
    }
}

/* R2-R4 for binary32.  raw_keys[2s], raw_keys[2s+1] = key32 of the finite
 * min / max as uint32, have[s] = 0 when the sequence has no finite value (A9). */
EXPORT void ft2o_bounds32(uint32_t* y, int64_t rows, int64_t n, int64_t ld, const int32_t* seq_offsets,
                          int32_t num_seqs, float scale, int32_t correct_nonfinite, uint32_t* bounds,
                          uint32_t* raw_keys, int32_t* have_out, uint32_t* nonfinite) {
    for (int32_t s = 0; s < num_seqs; ++s) {
        int64_t r0 = seq_offsets ? seq_offsets[s] : 0;
        int64_t r1 = seq_offsets ? seq_offsets[s + 1] : rows;
        int have = 0;
        uint32_t kmin = 0, kmax = 0, nf = 0;
        for (int64_t r = r0; r < r1; ++r)
            for (int64_t j = 0; j < n; ++j) {
                uint32_t v = y[r * ld + j];
                if (!ft2o_isfinite32(v)) { nf++; continue; }
                uint32_t k = ft2o_key32(v);
                if (!have || k < kmin) kmin = k;
                if (!have || k > kmax) kmax = k;
                have = 1;
            }
        uint32_t lo = 0u, hi = 0u;
        if (have) {
            lo = ft2o_scale_bound32(ft2o_unkey32(kmin), scale, 0);
            hi = ft2o_scale_bound32(ft2o_unkey32(kmax), scale, 1);
        }
        if (raw_keys) { raw_keys[2 * s] = kmin; raw_keys[2 * s + 1] = kmax; }
        if (have_out) have_out[s] = have;
        if (bounds) { bounds[2 * s] = lo; bounds[2 * s + 1] = hi; }
        if (nonfinite) nonfinite[s] = nf;
        if (correct_nonfinite)
            for (int64_t r = r0; r < r1; ++r)
                for (int64_t j = 0; j < n; ++j)
                    y[r * ld + j] = ft2o_clip_value32(y[r * ld + j], lo, hi);
    }
}

/* R7 for binary32: the 32-bit mask of the site (dtype 2 in ft2o_make_sites). */
EXPORT void ft2o_inject32(uint32_t* y, int64_t rows, int64_t n, int64_t ld, const ft2o_site* sites,
                          int32_t n_sites, int32_t cur_layer, int32_t cur_step, const int32_t* base_row) {
    for (int32_t i = 0; i < n_sites; ++i) {
        const ft2o_site* s = &sites[i];
        if ((int32_t)s->step != cur_step || (int32_t)s->layer != cur_layer) continue;
        int64_t row = (base_row ? base_row[i] : i) + (cur_step == 0 ? (int64_t)s->token : 0);
        if (row < 0 || row >= rows || (int64_t)s->col >= n) continue;
        y[row * ld + s->col] ^= s->xor_mask;
    }
}


/* ------------------------------------------------------ NEXT(2) / A22 --- */
/* Row-parallel critical layer under tensor parallelism: the sum all-reduce of
 * the P ranks' partial outputs followed by the check (reading A17: check after
 * the sum all-reduce).  Reading A22 fixes the reduction:
 * the partials (16-bit) are summed in fp32 in rank order,
 *     acc = f32(p_0); acc = fl32(acc + f32(p_t)) for t = 1..P-1;
 *     acc = fl32(acc + f32(bias[c]))  (if bias),
 * then rounded once to the 16-bit format (RNE), then R7 (inject), then R5.
 * partials: [P][rows][n] contiguous. */
EXPORT void ft2o_allreduce_protect(const uint16_t* partials, int32_t P, int64_t rows, int64_t n,
                                   const uint16_t* bias, int32_t check, const int32_t* row_to_seq,
                                   const uint16_t* bounds, int32_t num_seqs, uint32_t* count,
                                   const ft2o_site* sites, int32_t n_sites, int32_t cur_layer, int32_t cur_step,
                                   const int32_t* base_row, uint16_t* y, int dtype) {
    for (int64_t r = 0; r < rows; ++r)
        for (int64_t c = 0; c < n; ++c) {
            volatile float acc = (float)ft2o_to_f64_dt(partials[r * n + c], dtype);
            for (int32_t t = 1; t < P; ++t)
                acc = acc + (float)ft2o_to_f64_dt(partials[((int64_t)t * rows + r) * n + c], dtype);
            if (bias) acc = acc + (float)ft2o_to_f64_dt(bias[c], dtype);
            y[r * n + c] = ft2o_f64_to_dt_rne((double)acc, dtype);
        }
    if (sites && n_sites > 0) ft2o_inject(y, rows, n, n, sites, n_sites, cur_layer, cur_step, base_row);
    if (check) ft2o_protect_dt(y, rows, n, n, row_to_seq, bounds, num_seqs, count, dtype);
}

EXPORT int32_t ft2o_site_size(void) { return (int32_t)sizeof(ft2o_site); }
