// pfpl_device.cuh -- sm_100a device building blocks of the PFPL hot path.
//
// Quantizers, portable log2/pow2 (reading R5), bit-plane
// transposes, warp/block scans and look-back
// (Merrill & Garland).  Compiled with -fmad=false, IEEE division and
// no FTZ, so every floating-point operation is one correctly rounded IEEE
// operation, as P:110 requires for CPU/GPU bit-identity.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "pfpl_internal.h"

namespace pfpl {

#define PFPL_FULL 0xFFFFFFFFu
#define PFPL_HD __host__ __device__ __forceinline__

// ------------------------------------------------------------------------
// traits: one thread owns 32 consecutive elements; a chunk is 16384 bytes
// ------------------------------------------------------------------------
template <typename T> struct Tr;
template <> struct Tr<float> {
    typedef uint32_t W;
    static constexpr int B = 32, CW = 4096, NT = 128, NW = 4, S = 4, MANT = 23;
};
template <> struct Tr<double> {
    typedef uint64_t W;
    static constexpr int B = 64, CW = 2048, NT = 64, NW = 2, S = 8, MANT = 52;
};

PFPL_HD uint32_t f2u(float x) { union { float f; uint32_t u; } v; v.f = x; return v.u; }
PFPL_HD float u2f(uint32_t x) { union { float f; uint32_t u; } v; v.u = x; return v.f; }
PFPL_HD uint64_t d2u(double x) { union { double f; uint64_t u; } v; v.f = x; return v.u; }
PFPL_HD double u2d(uint64_t x) { union { double f; uint64_t u; } v; v.u = x; return v.f; }

// [stage] quantize (ABS/REL/NOA + verify)
// ------------------------------------------------------------------------
// portable log2 / pow2.  Format-version-1 constants: nearest binary32 /
// binary64 to 2/(k ln 2) (atanh series of log2) and ln2^j/j! (Taylor of 2^f).
// Plain operators: -fmad=false (device) / -ffp-contract=off (host) keep every
// operation separately rounded.
// ------------------------------------------------------------------------
PFPL_HD float log2p_f32(float a) {
    uint32_t u = f2u(a);
    int e = (int)((u >> 23) & 0xFFu) - 127;
    float m = u2f((u & 0x007FFFFFu) | 0x3F800000u);
    if (m > u2f(0x3FB504F3u)) { m = m * 0.5f; e = e + 1; }
    float t = (m - 1.0f) / (m + 1.0f);
    float t2 = t * t;
    float p = u2f(0x3ED30BB1u);
    p = p * t2; p = p + u2f(0x3F13BB63u);
    p = p * t2; p = p + u2f(0x3F76384Fu);
    p = p * t2; p = p + u2f(0x4038AA3Bu);
    float r = t * p;
    return (float)e + r;
}

PFPL_HD float pow2p_f32(float y) {
    float k = rintf(y);
    float f = y - k;
    float p = u2f(0x377FE5FEu);
    p = p * f; p = p + u2f(0x39218489u);
    p = p * f; p = p + u2f(0x3AAEC3FFu);
    p = p * f; p = p + u2f(0x3C1D955Bu);
    p = p * f; p = p + u2f(0x3D635847u);
    p = p * f; p = p + u2f(0x3E75FDF0u);
    p = p * f; p = p + u2f(0x3F317218u);
    p = p * f; p = p + 1.0f;
    if (!(k <= 127.0f)) return u2f(0x7F800000u);
    if (k < -126.0f) return 0.0f;
    int ki = (int)k;
    return p * u2f((uint32_t)(ki + 127) << 23);
}

PFPL_HD double log2p_f64(double a) {
    uint64_t u = d2u(a);
    int e = (int)((u >> 52) & 0x7FFu) - 1023;
    double m = u2d((u & 0x000FFFFFFFFFFFFFull) | 0x3FF0000000000000ull);
    if (m > u2d(0x3FF6A09E667F3BCDull)) { m = m * 0.5; e = e + 1; }
    double t = (m - 1.0) / (m + 1.0);
    double t2 = t * t;
    double p = u2d(0x3FC1964EC6FC9491ull);                         // c21
    p = p * t2; p = p + u2d(0x3FC3703C1F4D0FFEull);                 // c19
    p = p * t2; p = p + u2d(0x3FC5B9AC9B743F0Dull);                 // c17
    p = p * t2; p = p + u2d(0x3FC89F3B1694CFFEull);                 // c15
    p = p * t2; p = p + u2d(0x3FCC68F568D31760ull);                 // c13
    p = p * t2; p = p + u2d(0x3FD0C9A84994022Dull);                 // c11
    p = p * t2; p = p + u2d(0x3FD484B13D7C02A9ull);                 // c9
    p = p * t2; p = p + u2d(0x3FDA61762A7ADED9ull);                 // c7
    p = p * t2; p = p + u2d(0x3FE2776C50EF9BFEull);                 // c5
    p = p * t2; p = p + u2d(0x3FEEC709DC3A03FDull);                 // c3
    p = p * t2; p = p + u2d(0x40071547652B82FEull);                 // c1
    double r = t * p;
    return (double)e + r;
}

PFPL_HD double pow2p_f64(double y) {
    double k = rint(y);
    double f = y - k;
    double p = u2d(0x3D7816193166D0F9ull);                          // ln2^13/13!
    p = p * f; p = p + u2d(0x3DBC3BD650FC2986ull);
    p = p * f; p = p + u2d(0x3DFE8CAC7351BB25ull);
    p = p * f; p = p + u2d(0x3E3E4CF5158B8ECAull);
    p = p * f; p = p + u2d(0x3E7B5253D395E7C4ull);
    p = p * f; p = p + u2d(0x3EB62C0223A5C824ull);
    p = p * f; p = p + u2d(0x3EEFFCBFC588B0C7ull);
    p = p * f; p = p + u2d(0x3F2430912F86C787ull);
    p = p * f; p = p + u2d(0x3F55D87FE78A6731ull);
    p = p * f; p = p + u2d(0x3F83B2AB6FBA4E77ull);
    p = p * f; p = p + u2d(0x3FAC6B08D704A0C0ull);
    p = p * f; p = p + u2d(0x3FCEBFBDFF82C58Full);
    p = p * f; p = p + u2d(0x3FE62E42FEFA39EFull);
    p = p * f; p = p + 1.0;
    if (!(k <= 1023.0)) return u2d(0x7FF0000000000000ull);
    if (k < -1022.0) return 0.0;
    long long ki = (long long)k;
    return p * u2d((uint64_t)(ki + 1023) << 52);
}

// Device forms of log2p_f32 / pow2p_f32 with the same bits and no XU-pipe
// conversions: for an integer-valued float or int |x| < 2^22, x + 1.5*2^23 has bits
// 0x4B400000 + x, which replaces (float)e, rintf and (int)k exactly.
// pow2p: for |y| >= 2^22 both forms of k are beyond +-127 (or NaN/inf), so both
// return the same inf / 0.
__device__ __forceinline__ float i2f_small(int e) { return u2f(0x4B400000u + (uint32_t)e) - 12582912.0f; }
__device__ __forceinline__ float log2p_f32_d(float a) {
    uint32_t u = f2u(a);
    int e = (int)((u >> 23) & 0xFFu) - 127;
    float m = u2f((u & 0x007FFFFFu) | 0x3F800000u);
    if (m > u2f(0x3FB504F3u)) { m = m * 0.5f; e = e + 1; }
    float t = (m - 1.0f) / (m + 1.0f);
    float t2 = t * t;
    float p = u2f(0x3ED30BB1u);
    p = p * t2; p = p + u2f(0x3F13BB63u);
    p = p * t2; p = p + u2f(0x3F76384Fu);
    p = p * t2; p = p + u2f(0x4038AA3Bu);
    float r = t * p;
    return i2f_small(e) + r;
}
__device__ __forceinline__ float pow2p_f32_d(float y) {
    const float tk = y + 12582912.0f;
    float k = tk - 12582912.0f;
    float f = y - k;
    float p = u2f(0x377FE5FEu);
    p = p * f; p = p + u2f(0x39218489u);
    p = p * f; p = p + u2f(0x3AAEC3FFu);
    p = p * f; p = p + u2f(0x3C1D955Bu);
    p = p * f; p = p + u2f(0x3D635847u);
    p = p * f; p = p + u2f(0x3E75FDF0u);
    p = p * f; p = p + u2f(0x3F317218u);
    p = p * f; p = p + 1.0f;
    if (!(k <= 127.0f)) return u2f(0x7F800000u);
    if (k < -126.0f) return 0.0f;
    const int ki = (int)(f2u(tk) - 0x4B400000u);
    return p * u2f((uint32_t)(ki + 127) << 23);
}

// f64 forms: x + 1.5*2^52 has bits 0x4338000000000000 + x for integer |x| < 2^51
__device__ __forceinline__ double i2d_small(long long e) {
    return u2d(0x4338000000000000ull + (uint64_t)e) - 6755399441055744.0;
}
__device__ __forceinline__ double log2p_f64_d(double a) {
    uint64_t u = d2u(a);
    int e = (int)((u >> 52) & 0x7FFu) - 1023;
    double m = u2d((u & 0x000FFFFFFFFFFFFFull) | 0x3FF0000000000000ull);
    if (m > u2d(0x3FF6A09E667F3BCDull)) { m = m * 0.5; e = e + 1; }
    double t = (m - 1.0) / (m + 1.0);
    double t2 = t * t;
    double p = u2d(0x3FC1964EC6FC9491ull);
    p = p * t2; p = p + u2d(0x3FC3703C1F4D0FFEull);
    p = p * t2; p = p + u2d(0x3FC5B9AC9B743F0Dull);
    p = p * t2; p = p + u2d(0x3FC89F3B1694CFFEull);
    p = p * t2; p = p + u2d(0x3FCC68F568D31760ull);
    p = p * t2; p = p + u2d(0x3FD0C9A84994022Dull);
    p = p * t2; p = p + u2d(0x3FD484B13D7C02A9ull);
    p = p * t2; p = p + u2d(0x3FDA61762A7ADED9ull);
    p = p * t2; p = p + u2d(0x3FE2776C50EF9BFEull);
    p = p * t2; p = p + u2d(0x3FEEC709DC3A03FDull);
    p = p * t2; p = p + u2d(0x40071547652B82FEull);
    double r = t * p;
    return i2d_small(e) + r;
}
__device__ __forceinline__ double pow2p_f64_d(double y) {
    const double tk = y + 6755399441055744.0;
    double k = tk - 6755399441055744.0;
    double f = y - k;
    double p = u2d(0x3D7816193166D0F9ull);
    p = p * f; p = p + u2d(0x3DBC3BD650FC2986ull);
    p = p * f; p = p + u2d(0x3DFE8CAC7351BB25ull);
    p = p * f; p = p + u2d(0x3E3E4CF5158B8ECAull);
    p = p * f; p = p + u2d(0x3E7B5253D395E7C4ull);
    p = p * f; p = p + u2d(0x3EB62C0223A5C824ull);
    p = p * f; p = p + u2d(0x3EEFFCBFC588B0C7ull);
    p = p * f; p = p + u2d(0x3F2430912F86C787ull);
    p = p * f; p = p + u2d(0x3F55D87FE78A6731ull);
    p = p * f; p = p + u2d(0x3F83B2AB6FBA4E77ull);
    p = p * f; p = p + u2d(0x3FAC6B08D704A0C0ull);
    p = p * f; p = p + u2d(0x3FCEBFBDFF82C58Full);
    p = p * f; p = p + u2d(0x3FE62E42FEFA39EFull);
    p = p * f; p = p + 1.0;
    if (!(k <= 1023.0)) return u2d(0x7FF0000000000000ull);
    if (k < -1022.0) return 0.0;
    const long long ki = (long long)(d2u(tk) - 0x4338000000000000ull);
    return p * u2d((uint64_t)(ki + 1023) << 52);
}

// [stage] quantize (ABS/REL/NOA + verify)
// ------------------------------------------------------------------------
// packed binary32 pairs (FFMA2 / FADD2, sm_100): two IEEE operations per instruction,
// each lane rounded on its own.  ptxas contracts mul.rn.f32x2 + add.rn.f32x2 into
// one FFMA2 (a single rounding) even with -fmad=false, so a product is formed as
// fma(a, b, nz2) with nz2 = (-0, -0) supplied at run time: a*b + (-0) = a*b exactly
// (also for a*b = -0), and ptxas cannot fold an unknown addend into the next add.
// ------------------------------------------------------------------------
__device__ __forceinline__ uint64_t pk(float lo, float hi) {
    return ((uint64_t)f2u(hi) << 32) | f2u(lo);
}
__device__ __forceinline__ float pk_lo(uint64_t x) { return u2f((uint32_t)x); }
__device__ __forceinline__ float pk_hi(uint64_t x) { return u2f((uint32_t)(x >> 32)); }
__device__ __forceinline__ uint64_t pk_mul(uint64_t a, uint64_t b, uint64_t nz2) {
    uint64_t r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(nz2));
    return r;
}
__device__ __forceinline__ uint64_t pk_fma(uint64_t a, uint64_t b, uint64_t c) {   // exact cases only
    uint64_t r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ uint64_t pk_add(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ uint64_t pk_sub(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}

// predicated select that the compiler cannot turn into a branch
__device__ __forceinline__ uint32_t selp_u32(uint32_t a, uint32_t b, bool p) {
    uint32_t r;
    asm("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\tselp.b32 %0, %1, %2, q;\n\t}"
        : "=r"(r) : "r"(a), "r"(b), "r"((uint32_t)p));
    return r;
}

// [stage] quantize (ABS/REL/NOA + verify)
// ------------------------------------------------------------------------
// quantizers: value -> word (bin code or raw bits)
// ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t zz(int32_t b) { return ((uint32_t)b << 1) ^ (uint32_t)(b >> 31); }
__device__ __forceinline__ uint64_t zz(int64_t b) { return ((uint64_t)b << 1) ^ (uint64_t)(b >> 63); }
__device__ __forceinline__ int32_t unzz(uint32_t z) { return (int32_t)((z >> 1) ^ (0u - (z & 1u))); }
__device__ __forceinline__ int64_t unzz(uint64_t z) { return (int64_t)((z >> 1) ^ (0ull - (z & 1ull))); }

template <typename T> struct QF;
template <> struct QF<float> {
    float a, b, c, m1, m2;
    float limc;     // REL fast path: 0.5 - (m1 * 125.5 + m2) rounded down, the margin at the largest |L|
    float lmax;     // REL fast path: largest certified |L|: 125.5, and |L| * c <= 2^20 so |k| < 2^21
    __device__ __forceinline__ void load(const QConst& q) {
        a = u2f((uint32_t)q.a); b = u2f((uint32_t)q.b); c = u2f((uint32_t)q.c);
        m1 = u2f((uint32_t)q.m1); m2 = u2f((uint32_t)q.m2);
        limc = __fsub_rd(0.5f, __fmaf_ru(125.5f, m1, m2));
        lmax = fminf(125.5f, __fdiv_rd(1048576.0f, c));
    }
    // ABS/NOA: a = eps_eff, b = inv, c = eb2.  Bin = rint(v*inv); decode
    // immediately and keep the bin only if |v - bin*2eps| <= eps (R7);
    // |bin| < 2^22 so the zigzag code stays in the denormal range (R8).
    //
    // rint without the XU pipe: t = s + 1.5*2^23 rounds s to the nearest integer
    // (ties to even) for |s| < 2^22 and bits(t) = 0x4B400000 + rint(s); for
    // |s| >= 2^22 (or inf/NaN) the recovered rb has |rb| >= 2^22 (or is NaN) and
    // the value is stored losslessly, exactly as with rint.
    __device__ __forceinline__ uint32_t abs_q(float v) const {
        float s = v * b;
        float t = s + 12582912.0f;
        float rb = t - 12582912.0f;
        float vr = rb * c;
        float diff = fabsf(v - vr);
        bool ok = (fabsf(rb) < 4194304.0f) && (diff <= a);
        // zigzag(rb) = 2|rb| - (rb < 0) = |2rb + 0.5| - 0.5, exact for |rb| < 2^22
        const float w2 = __fmaf_rn(rb, 2.0f, 0.5f);
        const uint32_t z = f2u(fabsf(w2) + 8388607.5f) - 0x4B000000u;
        return ok ? z : f2u(v);
    }
    // biased word: abs_q(v) + 0x4B000000 (mod 2^32).  The bias cancels in the
    // residuals q[i] - q[i-1], so the encoder can skip the integer subtraction:
    // bits(|2rb + 0.5| + (2^23 - 0.5)) = 0x4B000000 + zigzag(rb) (two FMA-pipe ops)
    __device__ __forceinline__ uint32_t abs_qb(float v) const {
        float s = v * b;
        float t = s + 12582912.0f;
        float rb = t - 12582912.0f;
        float vr = rb * c;
        float diff = fabsf(v - vr);
        bool ok = (fabsf(rb) < 4194304.0f) && (diff <= a);
        const float w2 = __fmaf_rn(rb, 2.0f, 0.5f);
        const uint32_t z = f2u(fabsf(w2) + 8388607.5f);
        uint32_t rawb;
        asm("mad.lo.u32 %0, %1, 1, 0x4B000000;" : "=r"(rawb) : "r"(f2u(v)));
        return ok ? z : rawb;
    }
    // fast-path biased word: same as abs_qb(v) whenever the value is quantizable;
    // `ok` accumulates both checks of abs_qb (two chained FSETP.AND, no select and
    // no raw word); if it ends false the caller redoes the words with abs_qb.
    __device__ __forceinline__ uint32_t abs_qf(float v, bool& ok) const {
        float s = v * b;
        float t = s + 12582912.0f;
        float rb = t - 12582912.0f;
        float vr = rb * c;
        float diff = fabsf(v - vr);
        ok = ok && (fabsf(rb) < 4194304.0f) && (diff <= a);
        const float w2 = __fmaf_rn(rb, 2.0f, 0.5f);
        return f2u(fabsf(w2) + 8388607.5f);
    }
    // abs_qf on a packed pair (v = values 2i, 2i+1): the same IEEE operations in the same
    // order, two per instruction (s = v*inv, t = s + 1.5*2^23, rb = t - 1.5*2^23,
    // vr = rb*eb2, v - vr, and the exact 2*rb + 0.5)
    __device__ __forceinline__ void abs_qf2(uint64_t v, bool& ok0, bool& ok1, uint32_t& z0, uint32_t& z1,
                                            uint64_t nz2) const {
        const uint64_t s = pk_mul(v, pk(b, b), nz2);
        const uint64_t t = pk_add(s, pk(12582912.0f, 12582912.0f));
        const uint64_t rb = pk_add(t, pk(-12582912.0f, -12582912.0f));
        const uint64_t vr = pk_mul(rb, pk(c, c), nz2);
        const uint64_t d = pk_sub(v, vr);
        ok0 = ok0 && (fabsf(pk_lo(rb)) < 4194304.0f) && (fabsf(pk_lo(d)) <= a);
        ok1 = ok1 && (fabsf(pk_hi(rb)) < 4194304.0f) && (fabsf(pk_hi(d)) <= a);
        const uint64_t w2 = pk_fma(rb, pk(2.0f, 2.0f), pk(0.5f, 0.5f));     // exact for |rb| < 2^22
        z0 = f2u(fabsf(pk_lo(w2)) + 8388607.5f);
        z1 = f2u(fabsf(pk_hi(w2)) + 8388607.5f);
    }
    __device__ __forceinline__ float abs_dq(uint32_t w) const {
        return w < 0x00800000u ? __int2float_rn(unzz(w)) * c : u2f(w);
    }
    // same value without the XU pipe: |b| = (z+1)>>1, bits(2^23 + |b|) = (z + 0x96000001) >> 1,
    // fl(|b| * eb2) = fma(2^23 + |b|, eb2, -2^23*eb2) (one rounding of the exact product;
    // c23 = 2^23*eb2 must be finite), sign from the zigzag LSB.
    __device__ __forceinline__ float abs_dq_fast(uint32_t w, float c23) const {
        const float f = u2f((w + 0x96000001u) >> 1);
        const float mag = __fmaf_rn(f, c, -c23);
        return u2f(selp_u32(f2u(mag) ^ (w * 0x80000000u), w, w < 0x00800000u));
    }
    // abs_dq_fast for a word known to be a bin (w < 2^23)
    __device__ __forceinline__ float abs_dq_bins(uint32_t w, float c23) const {
        const float f = u2f((w + 0x96000001u) >> 1);
        const float mag = __fmaf_rn(f, c, -c23);
        return u2f(f2u(mag) ^ (w * 0x80000000u));
    }
    // REL: a = c_lo, b = w, c = inv_w.  log-space bin (R5), conservative
    // 1-ulp-shrunk check (R7), sign+bin in the negative-NaN payload (R10),
    // sign and exponent bits of every word inverted (R11).
    __device__ __forceinline__ uint32_t rel_q(float v) const {
        uint32_t u = f2u(v);
        uint32_t sign = u >> 31;
        uint32_t au = u & 0x7FFFFFFFu;
        uint32_t q0 = au > 0x7F800000u ? au : u;
        if (au >= 0x00800000u && au < 0x7F800000u) {
            float av = u2f(au);
            float L = log2p_f32_d(av);
            float s = L * c;
            // rb = rint(s) whenever |s| < 2^22; otherwise |rb| >= 2^21 and the value
            // is stored losslessly, as with rint
            const float ts = s + 12582912.0f;
            float rb = ts - 12582912.0f;
            if (fabsf(rb) < 2097152.0f) {
                float y = rb * b;
                float r = pow2p_f32_d(y);
                float lo = u2f(f2u(av / a) + 1u);
                float hi = u2f(f2u(av * a) - 1u);
                if (lo <= r && r <= hi)
                    q0 = 0xFF800000u | (1u + ((zz((int32_t)(f2u(ts) - 0x4B400000u)) << 1) | sign));
            }
        }
        return q0 ^ 0xFF800000u;
    }
    // REL fast path: the bin decision of rel_q taken from lg2.approx when it is certain.
    // s_exact = fl(log2p(a) * c) and s_fast = fl(lg2.approx(a) * c) differ by less than
    // margin(L) = m1*|L| + m2 (host: bounds of both log approximations and of the
    // roundings of s, y = bin*w and the R7 window, with headroom), so when
    // |s_fast - rint(s_fast)| <= 0.5 - margin, rint(s_exact) = rint(s_fast) = k, and the
    // reconstruction 2^(k w) lies inside [a/c_lo, a*c_lo] by at least the same margin:
    // rel_q accepts.  |L| <= 125.5 keeps pow2p away from its inf/0 clamps.  Otherwise
    // `slow` is set and the caller runs rel_q (same bits either way).
    __device__ __forceinline__ uint32_t rel_q_fast(float v, bool& slow) const {
        bool bin;
        return rel_q_fast(v, slow, bin);
    }
    // also reports whether the word is a bin (false: raw, or slow)
    __device__ __forceinline__ uint32_t rel_q_fast(float v, bool& slow, bool& bin) const {
        // branch-free: every quantity is computed, the word is selected at the end
        const uint32_t u = f2u(v), sign = u >> 31, au = u & 0x7FFFFFFFu;
        const bool normal = au - 0x00800000u < 0x7F800000u - 0x00800000u;   // finite, not denormal/0
        float L;
        asm("lg2.approx.f32 %0, %1;" : "=f"(L) : "f"(u2f(au)));
        const float s = L * c;
        const float ts = s + 12582912.0f;
        const float k = ts - 12582912.0f;
        const float aL = fabsf(L);
        // margin test |s - k| <= 0.5 - (m1 |L| + m2) (m2 >= 0.5 disables the path); the
        // FMA is margin arithmetic only, outside the format's operations
        const float lim = __fmaf_rn(-m1, aL, 0.5f - m2);
        const bool certain = (fabsf(s - k) <= lim) & (aL <= 125.5f);
        // bin word (R10, R11): payload 1 + (zigzag(k) << 1 | sign) = |4k + 1| + sign,
        // exact as a float for |k| < 2^21; the sign+exponent inversion cancels the NaN tag
        const uint32_t binw = f2u(fabsf(__fmaf_rn(k, 4.0f, 1.0f)) + 8388608.0f) - 0x4B000000u + sign;
        const uint32_t lossw = (au > 0x7F800000u ? au : u) ^ 0xFF800000u;
        bin = normal & certain & (fabsf(k) < 2097152.0f);
        slow = normal & !certain;
        return bin ? binw : lossw;
    }
    // rel_q_fast in the form the encoder's REL loop uses: the word of a certain bin, the
    // lossless word of a zero / denormal / inf / NaN, and the input bits of an uncertain
    // (slow) value, which sets `slow`; `nraw` counts the lossless ones.  |L| <= lmax also keeps |k| < 2^21, so one compare replaces rel_q_fast's |k|
    // test (the margin stays m1 |L| + m2: the constant bound at |L| = 125.5 sends ~18% of
    // the values of a 1E-3 field to the exact pass).  lg2.approx.ftz: L of a zero / denormal is -inf, of inf +inf,
    // of NaN NaN, so `certain` implies a normal input.
    __device__ __forceinline__ uint32_t rel_q_fast_w(float v, bool& slow, uint32_t& nraw) const {
        const uint32_t u = f2u(v), au = u & 0x7FFFFFFFu;
        const bool normal = au - 0x00800000u < 0x7F800000u - 0x00800000u;
        float L;
        asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(L) : "f"(u2f(au)));
        const float s = L * c;
        const float ts = s + 12582912.0f;
        const float k = ts - 12582912.0f;
        const float aL = fabsf(L);
        const float lim = __fmaf_rn(-m1, aL, 0.5f - m2);      // margin arithmetic only
        const bool certain = (fabsf(s - k) <= lim) & (aL <= lmax);
        const uint32_t binw = f2u(fabsf(__fmaf_rn(k, 4.0f, 1.0f)) + 8388608.0f) - 0x4B000000u + (u >> 31);
        const uint32_t lossw = (au > 0x7F800000u ? au : u) ^ 0xFF800000u;
        slow = normal & !certain;
        nraw += normal ? 0u : 1u;
        return certain ? binw : (normal ? u : lossw);
    }
    // rel_q_fast on a pair (u0, u1 the input bits): s = L*c and rint(s) on FP32x2 (the same
    // IEEE operations as rel_q_fast); the margin is the constant limc (the bound at the
    // largest |L|).  A slow value's word is its input bits (for the exact pass).
    __device__ __forceinline__ uint64_t rel_q_fast2(uint32_t u0, uint32_t u1, uint64_t nz2, uint32_t& slow2,
                                                   uint32_t& raw2) const {
        const uint32_t au0 = u0 & 0x7FFFFFFFu, au1 = u1 & 0x7FFFFFFFu;
        float L0, L1;
        asm("lg2.approx.f32 %0, %1;" : "=f"(L0) : "f"(u2f(au0)));
        asm("lg2.approx.f32 %0, %1;" : "=f"(L1) : "f"(u2f(au1)));
        const uint64_t s = pk_mul(pk(L0, L1), pk(c, c), nz2);
        const uint64_t ts = pk_add(s, pk(12582912.0f, 12582912.0f));
        const uint64_t k = pk_add(ts, pk(-12582912.0f, -12582912.0f));
        const uint64_t d = pk_sub(s, k);
        auto one = [&](uint32_t u, uint32_t au, float L, float kf, float df, uint32_t& sl, uint32_t& rw) -> uint32_t {
            const bool normal = au - 0x00800000u < 0x7F800000u - 0x00800000u;
            const bool certain = (fabsf(df) <= limc) & (fabsf(L) <= 125.5f);
            const uint32_t binw = f2u(fabsf(__fmaf_rn(kf, 4.0f, 1.0f)) + 8388608.0f) - 0x4B000000u + (u >> 31);
            const uint32_t lossw = (au > 0x7F800000u ? au : u) ^ 0xFF800000u;
            const bool bin = normal & certain & (fabsf(kf) < 2097152.0f);
            const bool slw = normal & !certain;
            sl = slw ? 1u : 0u;
            rw = (bin | slw) ? 0u : 1u;
            return slw ? u : (bin ? binw : lossw);
        };
        uint32_t sl0, sl1, rw0, rw1;
        const uint32_t w0 = one(u0, au0, L0, pk_lo(k), pk_lo(d), sl0, rw0);
        const uint32_t w1 = one(u1, au1, L1, pk_hi(k), pk_hi(d), sl1, rw1);
        slow2 = sl0 | (sl1 << 1);
        raw2 = rw0 | (rw1 << 1);
        return ((uint64_t)w1 << 32) | w0;
    }
    // rel_dq on a pair of words: the same IEEE operations (bin*w, rint by 1.5*2^23, f, the
    // degree-7 Horner of pow2p, the power-of-two scale), two per instruction
    __device__ __forceinline__ uint64_t rel_dq2(uint32_t w0, uint32_t w1, uint64_t nz2) const {
        const uint32_t u0 = w0 ^ 0xFF800000u, u1 = w1 ^ 0xFF800000u;
        const uint32_t t0 = (u0 & 0x007FFFFFu) - 1u, t1 = (u1 & 0x007FFFFFu) - 1u;
        const uint64_t bin = pk(i2f_small(unzz(t0 >> 1)), i2f_small(unzz(t1 >> 1)));   // exact, |bin| < 2^21
        const uint64_t y = pk_mul(bin, pk(b, b), nz2);
        const uint64_t tk = pk_add(y, pk(12582912.0f, 12582912.0f));
        const uint64_t k = pk_add(tk, pk(-12582912.0f, -12582912.0f));
        const uint64_t f = pk_sub(y, k);
        uint64_t p = pk(u2f(0x377FE5FEu), u2f(0x377FE5FEu));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x39218489u), u2f(0x39218489u)));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x3AAEC3FFu), u2f(0x3AAEC3FFu)));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x3C1D955Bu), u2f(0x3C1D955Bu)));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x3D635847u), u2f(0x3D635847u)));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x3E75FDF0u), u2f(0x3E75FDF0u)));
        p = pk_add(pk_mul(p, f, nz2), pk(u2f(0x3F317218u), u2f(0x3F317218u)));
        p = pk_add(pk_mul(p, f, nz2), pk(1.0f, 1.0f));
        // scale 2^k (k in [-126, 127]; the clamps below replace out-of-range results)
        const int ki0 = (int)((uint32_t)tk - 0x4B400000u), ki1 = (int)((uint32_t)(tk >> 32) - 0x4B400000u);
        const int c0 = ki0 < -126 ? -126 : (ki0 > 127 ? 127 : ki0), c1 = ki1 < -126 ? -126 : (ki1 > 127 ? 127 : ki1);
        const uint64_t mag = pk_mul(p, pk(u2f((uint32_t)(c0 + 127) << 23), u2f((uint32_t)(c1 + 127) << 23)), nz2);
        auto fin = [&](uint32_t u, uint32_t t, float kf, float m) -> uint32_t {
            float r = m;
            if (!(kf <= 127.0f)) r = u2f(0x7F800000u);
            else if (kf < -126.0f) r = 0.0f;
            const uint32_t rb = f2u(r) | ((t & 1u) << 31);
            return ((u & 0xFF800000u) == 0xFF800000u && (u & 0x007FFFFFu) != 0) ? rb : u;
        };
        return ((uint64_t)fin(u1, t1, pk_hi(k), pk_hi(mag)) << 32) | fin(u0, t0, pk_lo(k), pk_lo(mag));
    }
    __device__ __forceinline__ float rel_dq(uint32_t w) const {
        uint32_t u = w ^ 0xFF800000u;
        if ((u & 0xFF800000u) == 0xFF800000u && (u & 0x007FFFFFu) != 0) {
            uint32_t t = (u & 0x007FFFFFu) - 1u;
            float mag = pow2p_f32_d(i2f_small(unzz(t >> 1)) * b);     // |bin| < 2^21 (R10)
            return (t & 1u) ? -mag : mag;
        }
        return u2f(u);
    }
};
template <> struct QF<double> {
    double a, b, c, m1, m2;
    double limc;    // REL fast path: 0.5 - (m1 * 1021.5 + m2) rounded down
    double lmax;    // REL fast path: largest certified |L|: 1021.5, and |L| * c <= 2^49 so |k| < 2^50
    __device__ __forceinline__ void load(const QConst& q) {
        a = u2d(q.a); b = u2d(q.b); c = u2d(q.c); m1 = u2d(q.m1); m2 = u2d(q.m2);
        limc = __dsub_rd(0.5, __fma_ru(1021.5, m1, m2));
        lmax = fmin(1021.5, __ddiv_rd(562949953421312.0, c));
    }
    __device__ __forceinline__ uint64_t abs_q(double v) const {
        double s = v * b;
        double t = s + 6755399441055744.0;          // 1.5 * 2^52
        double rb = t - 6755399441055744.0;
        double vr = rb * c;
        double diff = fabs(v - vr);
        bool ok = (fabs(rb) < 2251799813685248.0) && (diff <= a);
        int64_t bi = (int64_t)(d2u(t) - 0x4338000000000000ull);
        return ok ? zz(bi) : d2u(v);
    }
    __device__ __forceinline__ uint64_t abs_qb(double v) const { return abs_q(v); }
    __device__ __forceinline__ double abs_dq_fast(uint32_t, float) const { return 0.0; }   // f32 only
    __device__ __forceinline__ double abs_dq(uint64_t w) const {
        return w < 0x0010000000000000ull ? __ll2double_rn((long long)unzz(w)) * c : u2d(w);
    }
    __device__ __forceinline__ uint64_t rel_q(double v) const {
        uint64_t u = d2u(v);
        uint64_t sign = u >> 63;
        uint64_t au = u & 0x7FFFFFFFFFFFFFFFull;
        uint64_t q0 = au > 0x7FF0000000000000ull ? au : u;
        if (au >= 0x0010000000000000ull && au < 0x7FF0000000000000ull) {
            double av = u2d(au);
            double L = log2p_f64_d(av);
            double s = L * c;
            const double ts = s + 6755399441055744.0;     // rint(s) for |s| < 2^51 (see f32)
            double rb = ts - 6755399441055744.0;
            if (fabs(rb) < 1125899906842624.0) {
                double y = rb * b;
                double r = pow2p_f64_d(y);
                double lo = u2d(d2u(av / a) + 1u);
                double hi = u2d(d2u(av * a) - 1u);
                if (lo <= r && r <= hi)
                    q0 = 0xFFF0000000000000ull | (1ull + ((zz((int64_t)(d2u(ts) - 0x4338000000000000ull)) << 1) | sign));
            }
        }
        return q0 ^ 0xFFF0000000000000ull;
    }
    // f64 form of QF<float>::rel_q_fast: L = exponent (exact) + lg2.approx.f32 of the
    // mantissa truncated to binary32; |L| <= 1021.5 keeps pow2p away from its clamps
    __device__ __forceinline__ uint64_t rel_q_fast(double v, bool& slow) const {
        bool bin;
        return rel_q_fast(v, slow, bin);
    }
    __device__ __forceinline__ uint64_t rel_q_fast(double v, bool& slow, bool& bin) const {
        const uint64_t u = d2u(v), sign = u >> 63, au = u & 0x7FFFFFFFFFFFFFFFull;
        const bool normal = au - 0x0010000000000000ull < 0x7FF0000000000000ull - 0x0010000000000000ull;
        const int e = (int)(au >> 52) - 1023;
        float lm;
        asm("lg2.approx.f32 %0, %1;" : "=f"(lm) : "f"(u2f(0x3F800000u | (uint32_t)((au >> 29) & 0x7FFFFFu))));
        const double L = i2d_small(e) + (double)lm;
        const double s = L * c;
        const double ts = s + 6755399441055744.0;
        const double k = ts - 6755399441055744.0;
        // the margin at |L| = 1021.5 bounds every smaller |L| (m1 >= 0): one compare
        const bool certain = (fabs(s - k) <= limc) & (fabs(L) <= 1021.5);
        // payload 1 + (zigzag(k) << 1 | sign) = |4k + 1| + sign, exact for |k| < 2^50
        const uint64_t binw = d2u(fabs(__fma_rn(k, 4.0, 1.0)) + 4503599627370496.0) - 0x4330000000000000ull + sign;
        const uint64_t lossw = (au > 0x7FF0000000000000ull ? au : u) ^ 0xFFF0000000000000ull;
        bin = normal & certain & (fabs(k) < 1125899906842624.0);
        slow = normal & !certain;
        return bin ? binw : lossw;
    }
    // f64 form of QF<float>::rel_q_fast_w (L of a zero / denormal has |L| >= 1022, of an
    // inf / NaN >= 1024, so `certain` implies a normal input)
    __device__ __forceinline__ uint64_t rel_q_fast_w(double v, bool& slow, uint32_t& nraw) const {
        const uint64_t u = d2u(v), au = u & 0x7FFFFFFFFFFFFFFFull;
        const bool normal = au - 0x0010000000000000ull < 0x7FF0000000000000ull - 0x0010000000000000ull;
        const int e = (int)(au >> 52) - 1023;
        float lm;
        asm("lg2.approx.f32 %0, %1;" : "=f"(lm) : "f"(u2f(0x3F800000u | (uint32_t)((au >> 29) & 0x7FFFFFu))));
        const double L = i2d_small(e) + (double)lm;
        const double s = L * c;
        const double ts = s + 6755399441055744.0;
        const double k = ts - 6755399441055744.0;
        const bool certain = (fabs(s - k) <= limc) & (fabs(L) <= lmax);
        const uint64_t binw = d2u(fabs(__fma_rn(k, 4.0, 1.0)) + 4503599627370496.0) - 0x4330000000000000ull + (u >> 63);
        const uint64_t lossw = (au > 0x7FF0000000000000ull ? au : u) ^ 0xFFF0000000000000ull;
        slow = normal & !certain;
        nraw += normal ? 0u : 1u;
        return certain ? binw : (normal ? u : lossw);
    }
    // rel_dq without branches (the same IEEE operations; non-bin words compute a
    // discarded value), so the decoder can interleave the 26-operation Horner chains
    // of several words
    __device__ __forceinline__ double rel_dq_bf(uint64_t w) const {
        const uint64_t u = w ^ 0xFFF0000000000000ull;
        const bool isbin = (u & 0xFFF0000000000000ull) == 0xFFF0000000000000ull && (u & 0x000FFFFFFFFFFFFFull) != 0;
        const uint64_t t = (u & 0x000FFFFFFFFFFFFFull) - 1u;
        const double y = i2d_small((long long)unzz(t >> 1)) * b;
        const double tk = y + 6755399441055744.0;
        const double k = tk - 6755399441055744.0;
        const double f = y - k;
        double p = u2d(0x3D7816193166D0F9ull);
        p = p * f; p = p + u2d(0x3DBC3BD650FC2986ull);
        p = p * f; p = p + u2d(0x3DFE8CAC7351BB25ull);
        p = p * f; p = p + u2d(0x3E3E4CF5158B8ECAull);
        p = p * f; p = p + u2d(0x3E7B5253D395E7C4ull);
        p = p * f; p = p + u2d(0x3EB62C0223A5C824ull);
        p = p * f; p = p + u2d(0x3EEFFCBFC588B0C7ull);
        p = p * f; p = p + u2d(0x3F2430912F86C787ull);
        p = p * f; p = p + u2d(0x3F55D87FE78A6731ull);
        p = p * f; p = p + u2d(0x3F83B2AB6FBA4E77ull);
        p = p * f; p = p + u2d(0x3FAC6B08D704A0C0ull);
        p = p * f; p = p + u2d(0x3FCEBFBDFF82C58Full);
        p = p * f; p = p + u2d(0x3FE62E42FEFA39EFull);
        p = p * f; p = p + 1.0;
        long long ki = (long long)(d2u(tk) - 0x4338000000000000ull);
        ki = ki < -1022 ? -1022 : (ki > 1023 ? 1023 : ki);       // in range: ki == k
        double mag = p * u2d((uint64_t)(ki + 1023) << 52);
        if (!(k <= 1023.0)) mag = u2d(0x7FF0000000000000ull);
        else if (k < -1022.0) mag = 0.0;
        return isbin ? u2d(d2u(mag) | (t << 63)) : u2d(u);
    }
    __device__ __forceinline__ double rel_dq(uint64_t w) const {
        uint64_t u = w ^ 0xFFF0000000000000ull;
        if ((u & 0xFFF0000000000000ull) == 0xFFF0000000000000ull &&
            (u & 0x000FFFFFFFFFFFFFull) != 0) {
            uint64_t t = (u & 0x000FFFFFFFFFFFFFull) - 1u;
            double mag = pow2p_f64_d(i2d_small((long long)unzz(t >> 1)) * b);   // |bin| < 2^50 (R10)
            return (t & 1u) ? -mag : mag;
        }
        return u2d(u);
    }
};

template <typename T, int MODE>
__device__ __forceinline__ typename Tr<T>::W quantize(const QF<T>& q, T v, bool raw) {
    if (MODE == MODE_RAW) return sizeof(T) == 4 ? (typename Tr<T>::W)f2u((float)v) : (typename Tr<T>::W)d2u((double)v);
    if (MODE == MODE_NOA && raw) {
        if (sizeof(T) == 4) return (typename Tr<T>::W)f2u((float)v);
        return (typename Tr<T>::W)d2u((double)v);
    }
    if (MODE == MODE_REL) return q.rel_q(v);
    return q.abs_q(v);
}

// encoder form: a word that differs from quantize() by a per-type constant
// (QBIAS), which cancels in the delta coding
template <typename T, int MODE>
__device__ __forceinline__ typename Tr<T>::W quantize_b(const QF<T>& q, T v, bool raw) {
    if (MODE == MODE_ABS || (MODE == MODE_NOA && !raw)) {
        if (sizeof(T) == 4) return q.abs_qb(v);
    }
    return quantize<T, MODE>(q, v, raw);
}

template <typename T, int MODE>
__device__ __forceinline__ T dequantize(const QF<T>& q, typename Tr<T>::W w, bool raw);
template <> __device__ __forceinline__ float dequantize<float, MODE_ABS>(const QF<float>& q, uint32_t w, bool) { return q.abs_dq(w); }
template <> __device__ __forceinline__ float dequantize<float, MODE_NOA>(const QF<float>& q, uint32_t w, bool raw) { return raw ? u2f(w) : q.abs_dq(w); }
template <> __device__ __forceinline__ float dequantize<float, MODE_REL>(const QF<float>& q, uint32_t w, bool) { return q.rel_dq(w); }
template <> __device__ __forceinline__ float dequantize<float, MODE_RAW>(const QF<float>&, uint32_t w, bool) { return u2f(w); }
template <> __device__ __forceinline__ double dequantize<double, MODE_ABS>(const QF<double>& q, uint64_t w, bool) { return q.abs_dq(w); }
template <> __device__ __forceinline__ double dequantize<double, MODE_NOA>(const QF<double>& q, uint64_t w, bool raw) { return raw ? u2d(w) : q.abs_dq(w); }
template <> __device__ __forceinline__ double dequantize<double, MODE_REL>(const QF<double>& q, uint64_t w, bool) { return q.rel_dq(w); }
template <> __device__ __forceinline__ double dequantize<double, MODE_RAW>(const QF<double>&, uint64_t w, bool) { return u2d(w); }

// [stage] delta + residual code
// ------------------------------------------------------------------------
// residual codes: negabinary (default) or zigzag (flag A1)
// ------------------------------------------------------------------------
template <bool MS> __device__ __forceinline__ uint32_t rcode(uint32_t d) {
    return MS ? ((d << 1) ^ (uint32_t)((int32_t)d >> 31)) : ((d + 0xAAAAAAAAu) ^ 0xAAAAAAAAu);
}
template <bool MS> __device__ __forceinline__ uint64_t rcode(uint64_t d) {
    return MS ? ((d << 1) ^ (uint64_t)((int64_t)d >> 63))
              : ((d + 0xAAAAAAAAAAAAAAAAull) ^ 0xAAAAAAAAAAAAAAAAull);
}
template <bool MS> __device__ __forceinline__ uint32_t rdecode(uint32_t r) {
    return MS ? ((r >> 1) ^ (0u - (r & 1u))) : ((r ^ 0xAAAAAAAAu) - 0xAAAAAAAAu);
}
template <bool MS> __device__ __forceinline__ uint64_t rdecode(uint64_t r) {
    return MS ? ((r >> 1) ^ (0ull - (r & 1ull)))
              : ((r ^ 0xAAAAAAAAAAAAAAAAull) - 0xAAAAAAAAAAAAAAAAull);
}

// [stage] bit-plane transpose
// ------------------------------------------------------------------------
// bit-plane transpose of 32 words with values < 2^K (K in {4,8,16,32}):
// out[b] bit j = bit b of in[j].  Pack 32/K elements per word (element j at
// word j%K, position K*(j/K)+bit), then exchange word-index bit i with
// position bit i for i < log2 K (delta swaps).  The exchanges are involutions,
// so the inverse is: same exchanges, then unpack.
// ------------------------------------------------------------------------
template <int I> __device__ __forceinline__ void xchg(uint32_t& a, uint32_t& b) {
    if (I == 4) {
        uint32_t na = __byte_perm(a, b, 0x5410), nb = __byte_perm(a, b, 0x7632);
        a = na; b = nb;
    } else if (I == 3) {
        uint32_t na = __byte_perm(a, b, 0x6240), nb = __byte_perm(a, b, 0x7351);
        a = na; b = nb;
    } else {
        // mask form: 2 LOP3 + 1 SHF on the ALU pipe, 1 IMAD.SHL on the FMA pipe
        constexpr uint32_t M = I == 0 ? 0x55555555u : I == 1 ? 0x33333333u : 0x0F0F0F0Fu;
        constexpr int s = 1 << I;
        const uint32_t na = (a & M) | ((b * (1u << s)) & ~M);
        const uint32_t nb = ((a >> s) & M) | (b & ~M);
        a = na; b = nb;
    }
}

template <int K> __device__ __forceinline__ void xchg_all(uint32_t* o) {
#pragma unroll
    for (int i = 0; (1 << i) < K; ++i) {
#pragma unroll
        for (int a = 0; a < K; ++a) {
            if (a & (1 << i)) continue;
            const int b = a | (1 << i);
            switch (i) {
                case 0: xchg<0>(o[a], o[b]); break;
                case 1: xchg<1>(o[a], o[b]); break;
                case 2: xchg<2>(o[a], o[b]); break;
                case 3: xchg<3>(o[a], o[b]); break;
                default: xchg<4>(o[a], o[b]); break;
            }
        }
    }
}

// in place: r[0..K-1] receive the K plane words (bit b of the 32 values)
template <int K> __device__ __forceinline__ void transpose_fwd(uint32_t (&r)[32]) {
    constexpr int H = 32 / K;
#pragma unroll
    for (int w = 0; w < K; ++w) {
        uint32_t x = r[w];
#pragma unroll
        for (int h = 1; h < H; ++h) x += r[w + K * h] * (1u << (K * h));   // disjoint fields
        r[w] = x;
    }
    xchg_all<K>(r);
}

// in place inverse: r[0..K-1] hold plane words; on return r[0..31] hold values < 2^K
template <int K> __device__ __forceinline__ void transpose_inv(uint32_t (&r)[32]) {
    constexpr int H = 32 / K;
    xchg_all<K>(r);
#pragma unroll
    for (int w = 0; w < K; ++w) {
#pragma unroll
        for (int h = H - 1; h >= 0; --h) {
            if (K == 32) r[w + K * h] = r[w];
            else if (K == 8) r[w + K * h] = __byte_perm(r[w], 0, 0x4440 + h);            // 1 PRMT
            else if (K == 16) r[w + K * h] = __byte_perm(r[w], 0, h ? 0x4432 : 0x4410);
            else r[w + K * h] = (r[w] >> (K * h)) & ((1u << (K & 31)) - 1u);
        }
    }
}

// [stage] byte masks (zero/repeat elimination)
// ------------------------------------------------------------------------
// byte helpers
// ------------------------------------------------------------------------
// 0x01 in every non-zero byte of x
__device__ __forceinline__ uint32_t nzbytes(uint32_t x) {
    return (((x & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | x) >> 7 & 0x01010101u;
}
// 0x80 in every non-zero byte of x
__device__ __forceinline__ uint32_t nzmark(uint32_t x) {
    return (((x & 0x7F7F7F7Fu) + 0x7F7F7F7Fu) | x) & 0x80808080u;
}
// H = nzmark(x): returns (lo, hi) of H * 0x02020202, i.e. lo byte k = number of
// marked bytes below k (exclusive rank), hi byte 0 = number of marked bytes
__device__ __forceinline__ uint64_t rankcount(uint32_t H) {
    return (uint64_t)H * 0x02020202ull;
}
// gather the low bits of the 4 bytes of h (values 0/1) into a nibble
__device__ __forceinline__ uint32_t nib(uint32_t h) { return (h * 0x10204080u) >> 28; }

// [stage] warp scans / sums
// ------------------------------------------------------------------------
// scans
// ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t warp_incl_scan(uint32_t v, int lane) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint32_t t = __shfl_up_sync(PFPL_FULL, v, d);
        if (lane >= d) v += t;
    }
    return v;
}
__device__ __forceinline__ uint64_t warp_incl_scan64(uint64_t v, int lane) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        uint64_t t = __shfl_up_sync(PFPL_FULL, v, d);
        if (lane >= d) v += t;
    }
    return v;
}
__device__ __forceinline__ uint64_t warp_sum64(uint64_t v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(PFPL_FULL, v, d);
    return v;
}

// [stage] look-back descriptors
// ------------------------------------------------------------------------
// look-back descriptors: [63:48] epoch | [47:46] flag | [45:0] value
// ------------------------------------------------------------------------
constexpr uint64_t LB_A = 1, LB_P = 2;
constexpr uint64_t LB_VAL = (1ull << 46) - 1;

__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint4 ldg_nc_v4(const void* p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

// [stage] mbarrier / TMA / watchdog waits
// ------------------------------------------------------------------------
// sm_90+/sm_100 asynchronous primitives: mbarrier, TMA, named barriers
// ------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t a, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(a), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint32_t a, uint32_t tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(a), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t a) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(a) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t a, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred P1;\n"
        "LAB_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@P1 bra DONE;\n\t"
        "bra LAB_WAIT;\n"
        "DONE:\n\t}" ::"r"(a), "r"(parity) : "memory");
}
__device__ __forceinline__ bool mbar_test(uint32_t a, uint32_t parity) {
    uint32_t r;
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P1;\n\t}" : "=r"(r) : "r"(a), "r"(parity) : "memory");
    return r != 0;
}
// ---- watchdog: every spin loop of the library is bounded in time.  On expiry
// the site code, block and a detail word go to mapped host memory (readable
// even after the context dies) and the kernel traps: a protocol bug becomes an
// error (PFPL_ERR_CUDA) instead of a hung caller.
static __device__ unsigned int* g_pfpl_wd;   // per TU; set from the kernel parameters
constexpr uint64_t kWatchdogNs = 5000000000ull;   // 5 s
__device__ __forceinline__ uint64_t globaltimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
    return t;
}
static __device__ __noinline__ void watchdog_fire(uint32_t site, uint32_t detail) {
    unsigned int* h = g_pfpl_wd;
    if (h) {
        h[1] = blockIdx.x;
        h[2] = threadIdx.x;
        h[3] = detail;
        __threadfence_system();
        atomicExch(h, site);
        __threadfence_system();
    }
    __trap();
}
__device__ __forceinline__ bool mbar_try(uint32_t a, uint32_t parity) {
    uint32_t r;
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, P1;\n\t}" : "=r"(r) : "r"(a), "r"(parity) : "memory");
    return r != 0;
}
// try_wait with a suspend-time hint: the thread is parked by the hardware until
// the phase completes (or the hint expires), so waiting does not spin on the
// issue port
__device__ __forceinline__ bool mbar_try_hint(uint32_t a, uint32_t parity, uint32_t ns) {
    uint32_t r;
    asm volatile(
        "{\n\t.reg .pred P1;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, P1;\n\t}" : "=r"(r) : "r"(a), "r"(parity), "r"(ns) : "memory");
    return r != 0;
}
#ifndef PFPL_WAIT_NOINLINE
#define PFPL_WAIT_NOINLINE 1     // +1.5-2% NYX compress (less hot code)
#endif
#if PFPL_WAIT_NOINLINE
// the slow path out of line: every wait site keeps only one try_wait inline (less hot code)
static __device__ __noinline__ void mbar_wait_slow(uint32_t a, uint32_t parity, uint32_t site,
                                                   uint32_t hint_ns) {
    const uint64_t t0 = globaltimer();
    for (;;) {
        if (mbar_try_hint(a, parity, hint_ns)) return;
        if (globaltimer() - t0 > kWatchdogNs) watchdog_fire(site, parity);
    }
}
__device__ __forceinline__ void mbar_wait_wd(uint32_t a, uint32_t parity, uint32_t site,
                                             uint32_t hint_ns = 20000) {
    if (mbar_try(a, parity)) return;
    mbar_wait_slow(a, parity, site, hint_ns);
}
#else
__device__ __forceinline__ void mbar_wait_wd(uint32_t a, uint32_t parity, uint32_t site,
                                             uint32_t hint_ns = 20000) {
    if (mbar_try(a, parity)) return;
    const uint64_t t0 = globaltimer();
    for (;;) {
        if (mbar_try_hint(a, parity, hint_ns)) return;
        if (globaltimer() - t0 > kWatchdogNs) watchdog_fire(site, parity);
    }
}
#endif
// poll with a sleep between tries: for waits that are the common case and whose
// latency does not matter (a producer running ahead of its consumers)
__device__ __forceinline__ void mbar_wait_sleep(uint32_t a, uint32_t parity, uint32_t site,
                                                uint32_t ns = 256) {
    if (mbar_try(a, parity)) return;
    const uint64_t t0 = globaltimer();
    for (;;) {
        __nanosleep(ns);
        if (mbar_try(a, parity)) return;
        if (globaltimer() - t0 > kWatchdogNs) watchdog_fire(site, parity);
    }
}
__device__ __forceinline__ void fence_barrier_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
// 2-D tiled TMA load into shared memory, completion counted on an mbarrier
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const void* tmap, int x, int y, uint32_t mbar) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
        " [%0], [%1, {%2, %3}], [%4];" ::"r"(dst), "l"(tmap), "r"(x), "r"(y), "r"(mbar) : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const void* tmap) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(tmap) : "memory");
}
__device__ __forceinline__ void named_sync(int id, int n) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void named_arrive(int id, int n) {
    asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory");
}

}  // namespace pfpl
