// ft2_device.cuh -- device primitives for the FT2 kernels (sm_100a).
//
// Order keys: a bf16 bit pattern b maps to the
// 16-bit key  b & 0x8000 ? ~b : b | 0x8000,  monotone in the value on all
// non-NaN inputs (-Inf = 0x007F ... -0 = 0x7FFF < +0 = 0x8000 ... +Inf = 0xFF80;
// NaN keys lie outside [0x007F, 0xFF80]).  All of FT2's bounds, checks and
// clips become unsigned 16-bit min/max/compare, done two at a time on packed
// 32-bit words (PRMT sign replicate + LOP3 for the key, VIMNMX.U16x2 for
// min/max), which makes every result bit-exact and independent of reduction
// order.
#pragma once
#include <cuda_fp16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace ft2dev {

// 0xFFFF in each 16-bit half whose bit 15 is set, else 0 (PRMT sign replicate).
__device__ __forceinline__ uint32_t half_sign_mask(uint32_t w) {
    uint32_t m;
    asm("prmt.b32 %0, %1, 0, 0xBB99;" : "=r"(m) : "r"(w));
    return m;
}

// Two packed bf16 -> two packed order keys.
__device__ __forceinline__ uint32_t key2(uint32_t w) {
    return w ^ (half_sign_mask(w) | 0x80008000u);
}

// Two packed keys -> two packed bf16.
__device__ __forceinline__ uint32_t unkey2(uint32_t k) {
    return k ^ (~half_sign_mask(k) | 0x80008000u);
}

__device__ __forceinline__ uint32_t vmin_u16x2(uint32_t a, uint32_t b) {
    uint32_t d;
    asm("min.u16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
    return d;
}
__device__ __forceinline__ uint32_t vmax_u16x2(uint32_t a, uint32_t b) {
    uint32_t d;
    asm("max.u16x2 %0, %1, %2;" : "=r"(d) : "r"(a), "r"(b));
    return d;
}

// 16-bit activation formats: DT 0 = bf16 (1/8/7), DT 1 = fp16 (1/5/10, the
// paper's precision).  Both are sign-magnitude, so the order
// key is the same; only the exponent field (and so NaN/Inf) differs.
template <int DT> struct Fmt;
template <> struct Fmt<0> {
    static constexpr uint32_t kExp = 0x7F80u;     // exponent field = +Inf pattern
    static constexpr uint32_t kMaxFin = 0x7F7Fu;  // largest finite magnitude
    static constexpr uint32_t kKeyLo = 0x0080u;   // key(-max finite)
    static constexpr uint32_t kKeyHi = 0xFF7Fu;   // key(+max finite)
};
template <> struct Fmt<1> {
    static constexpr uint32_t kExp = 0x7C00u;
    static constexpr uint32_t kMaxFin = 0x7BFFu;
    static constexpr uint32_t kKeyLo = 0x0400u;
    static constexpr uint32_t kKeyHi = 0xFBFFu;
};

// Bit 15 of each half set iff that half is NaN: (h & 0x7FFF) > kExp.
template <int DT = 0>
__device__ __forceinline__ uint32_t nan_bits2(uint32_t w) {
    constexpr uint32_t add = (0x7FFFu - Fmt<DT>::kExp) * 0x10001u;
    return ((w & 0x7FFF7FFFu) + add) & 0x80008000u;
}

// Bit 15 of each half set iff that half is non-finite (exponent all ones).
template <int DT = 0>
__device__ __forceinline__ uint32_t nonfinite_bits2(uint32_t w) {
    constexpr uint32_t e = Fmt<DT>::kExp * 0x10001u, one = (0x8000u - Fmt<DT>::kExp) * 0x10001u;
    return ((w & e) + one) & 0x80008000u;
}
template <int DT = 0>
__device__ __forceinline__ bool isnan1(uint16_t b) { return (b & 0x7FFFu) > Fmt<DT>::kExp; }
template <int DT = 0>
__device__ __forceinline__ bool nonfinite1(uint16_t b) { return (b & Fmt<DT>::kExp) == Fmt<DT>::kExp; }

// Number of 16-bit halves of d that are non-zero (0, 1 or 2).
__device__ __forceinline__ uint32_t nonzero_halves(uint32_t d) {
    return (uint32_t)((d & 0xFFFFu) != 0) + (uint32_t)((d >> 16) != 0);
}

__device__ __forceinline__ uint16_t key1(uint16_t b) {
    return (b & 0x8000) ? (uint16_t)~b : (uint16_t)(b | 0x8000);
}
__device__ __forceinline__ uint16_t unkey1(uint16_t k) {
    return (k & 0x8000) ? (uint16_t)(k & 0x7FFF) : (uint16_t)~k;
}

// Check-and-clip of two packed bf16 against packed keys (kL2 = kL|kL<<16 ...).
// NaN halves are first replaced by +0 (key 0x8000), then clamped in key space.
// Returns the corrected packed bf16; *changed = number of halves whose bits changed.
template <int DT = 0>
__device__ __forceinline__ uint32_t clip2(uint32_t w, uint32_t kL2, uint32_t kH2, uint32_t* changed) {
    uint32_t k = key2(w);
    uint32_t nm = half_sign_mask(nan_bits2<DT>(w));       // 0xFFFF on NaN halves
    uint32_t kz = (k & ~nm) | (0x80008000u & nm);          // NaN -> key(+0)
    uint32_t kc = vmax_u16x2(vmin_u16x2(kz, kH2), kL2);
    *changed = nonzero_halves(kc ^ k);
    return unkey2(kc);
}

// ------------------------------------------------------------------ scaling
// R3 / readings A2, A8, A10: widen the raw bound by c in fp32, round outward
// to bf16, saturate to +-max finite.  With c = 2 every step is exact.
__device__ __forceinline__ uint16_t bf16_from_f32_dir(float s, bool up) {
    uint32_t u = __float_as_uint(s);
    uint32_t t = u >> 16;                  // truncation toward zero
    bool inexact = (u & 0xFFFFu) != 0;
    bool neg = (u >> 31) != 0;
    if ((u & 0x7FFFFFFFu) > 0x7F800000u) return 0x7FC0;   // not reachable (no NaN input)
    // toward +Inf: positive inexact values move away from zero; toward -Inf:
    // negative inexact values move away from zero.
    if (inexact && (up ? !neg : neg)) t += 1;
    return (uint16_t)t;
}

template <int DT = 0>
__device__ __forceinline__ float to_f32(uint16_t b) {
    if (DT == 0) return __uint_as_float((uint32_t)b << 16);
    return __half2float(__ushort_as_half(b));
}

template <int DT = 0>
__device__ __forceinline__ uint16_t scale_bound(uint16_t raw, float c, bool is_hi) {
    const float x = to_f32<DT>(raw);
    float s;
    if (is_hi) s = (x >= 0.0f) ? __fmul_rn(x, c) : __fdiv_rn(x, c);
    else       s = (x <= 0.0f) ? __fmul_rn(x, c) : __fdiv_rn(x, c);
    uint16_t r;
    if (DT == 0) r = bf16_from_f32_dir(s, is_hi);
    else r = __half_as_ushort(is_hi ? __float2half_ru(s) : __float2half_rd(s));
    if (r == Fmt<DT>::kExp) r = (uint16_t)Fmt<DT>::kMaxFin;
    if (r == (0x8000u | Fmt<DT>::kExp)) r = (uint16_t)(0x8000u | Fmt<DT>::kMaxFin);
    return r;
}

// fp32 -> bf16 round-to-nearest-even (NaN -> canonical 0x7FC0).
__device__ __forceinline__ uint16_t bf16_rne(float f) {
    uint32_t u = __float_as_uint(f);
    if ((u & 0x7FFFFFFFu) > 0x7F800000u) return 0x7FC0;
    u += 0x7FFFu + ((u >> 16) & 1u);
    return (uint16_t)(u >> 16);
}
// fp32 -> activation format, round-to-nearest-even; NaN -> the canonical
// quiet NaN of the format (bf16 0x7FC0, fp16 0x7E00), as the oracle's R0.
template <int DT = 0>
__device__ __forceinline__ uint16_t rne16(float f) {
    if (DT == 0) return bf16_rne(f);
    if (f != f) return 0x7E00;
    return __half_as_ushort(__float2half_rn(f));
}

// ------------------------------------------------------------------ Philox
struct u32x4 { uint32_t x, y, z, w; };

__device__ __forceinline__ u32x4 philox4x32_10(u32x4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        if (r) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
        uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
        uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
        c = u32x4{hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0};
    }
    return c;
}

__device__ __forceinline__ uint32_t draw_below(uint32_t u, uint32_t n) {
    return (uint32_t)(((uint64_t)u * (uint64_t)n) >> 32);
}

// ------------------------------------------------------------------ loads
// Streaming 16-byte load that does not allocate in L1.  Deliberately NOT
// .nc: the protect kernels write back (and the bounds kernel's last CTA
// patches) the very tensor they stream, and the non-coherent path is only
// defined for data that is read-only for the kernel's whole lifetime.
__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
    uint4 r;
    asm volatile("ld.global.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p) : "memory");
    return r;
}

// Fast unsigned division by a runtime constant d (n < 2^31).
struct FastDiv {
    uint32_t d, m, s;
};
static inline FastDiv make_fastdiv(uint32_t d) {
    FastDiv f{d, 0, 0};
    if (d <= 1) return f;
    uint32_t l = 0;
    while ((1u << l) < d) ++l;             // ceil(log2 d)
    uint32_t p = 31 + l;
    f.m = (uint32_t)(((1ull << p) + d - 1) / d);
    f.s = p - 32;
    return f;
}
__device__ __forceinline__ uint32_t fdiv(uint32_t n, const FastDiv& f) {
    return f.d <= 1 ? n : (__umulhi(n, f.m) >> f.s);
}

}  // namespace ft2dev
