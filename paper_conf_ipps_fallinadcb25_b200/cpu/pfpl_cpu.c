/*
 * pfpl_cpu.c -- multi-core CPU PFPL codec (include/pfpl_cpu.h).
 *
 * The paper's PFPL_OMP design for the host CPU of a B200 node:
 *   - 16 KiB chunks, handed to OpenMP threads dynamically by an atomic counter
 *     (P:141);
 *   - all stages fused per chunk: quantize + verify, delta +
 *     negabinary, bit shuffle, zero / repeat elimination
 *     (P:129-131), in two 16 KiB buffers per thread that stay in L1;
 *   - the chunks' output placed through a shared carry array with atomic reads
 *     and writes: chunk c waits for carry[c-1], publishes
 *     carry[c] = carry[c-1] + size, then copies its bytes.
 * AVX2 for the quantizer, the 32-element bit transposes (movemask) and the
 * byte compactions (pshufb tables).  Every floating-point step is one IEEE
 * operation (-ffp-contract=off, no fast-math, explicit mul/sub intrinsics), so
 * the stream is byte-identical to the GPU's.
 * Product code: shares no code with the CPU test reference or the CUDA sources.
 */
#include "../../include/pfpl_cpu.h"

#include <float.h>
#include <immintrin.h>
#include <math.h>
#include <omp.h>
#include <stdatomic.h>
#include <stdlib.h>
#include <string.h>

#define CHUNK 16384u
#define HDR 48u
enum { F32 = 0, F64 = 1 };
enum { ABS = 0, REL = 1, NOA = 2 };
enum { FL_RAWWORDS = 1, FL_MS = 2 };
enum { E_ARG = -1, E_BOUND = -2, E_CAP = -3, E_CORRUPT = -4 };

static uint32_t fbits(float x) { uint32_t u; memcpy(&u, &x, 4); return u; }
static float ffrom(uint32_t u) { float x; memcpy(&x, &u, 4); return x; }
static uint64_t dbits(double x) { uint64_t u; memcpy(&u, &x, 8); return u; }
static double dfrom(uint64_t u) { double x; memcpy(&x, &u, 8); return x; }

/* ---------------------------------------------------------------------- */
/* portable log2 / pow2 (reading R5): format-version-1 constants    */
/* ---------------------------------------------------------------------- */
static float lg2_f(float a) {
    uint32_t u = fbits(a);
    int e = (int)((u >> 23) & 0xFFu) - 127;
    float m = ffrom((u & 0x007FFFFFu) | 0x3F800000u);
    if (m > ffrom(0x3FB504F3u)) { m = m * 0.5f; e = e + 1; }
    const float t = (m - 1.0f) / (m + 1.0f), t2 = t * t;
    float p = ffrom(0x3ED30BB1u);
    p = p * t2 + ffrom(0x3F13BB63u);
    p = p * t2 + ffrom(0x3F76384Fu);
    p = p * t2 + ffrom(0x4038AA3Bu);
    return (float)e + t * p;
}
static float pw2_f(float y) {
    const float k = rintf(y), f = y - k;
    static const uint32_t C[8] = {0x3F800000u, 0x3F317218u, 0x3E75FDF0u, 0x3D635847u,
                                  0x3C1D955Bu, 0x3AAEC3FFu, 0x39218489u, 0x377FE5FEu};
    float p = ffrom(C[7]);
    for (int j = 6; j >= 0; --j) p = p * f + ffrom(C[j]);
    if (!(k <= 127.0f)) return ffrom(0x7F800000u);
    if (k < -126.0f) return 0.0f;
    return p * ffrom((uint32_t)((int)k + 127) << 23);
}
static double lg2_d(double a) {
    uint64_t u = dbits(a);
    int e = (int)((u >> 52) & 0x7FFu) - 1023;
    double m = dfrom((u & 0x000FFFFFFFFFFFFFull) | 0x3FF0000000000000ull);
    if (m > dfrom(0x3FF6A09E667F3BCDull)) { m = m * 0.5; e = e + 1; }
    const double t = (m - 1.0) / (m + 1.0), t2 = t * t;
    static const uint64_t C[11] = {0x40071547652B82FEull, 0x3FEEC709DC3A03FDull, 0x3FE2776C50EF9BFEull,
                                   0x3FDA61762A7ADED9ull, 0x3FD484B13D7C02A9ull, 0x3FD0C9A84994022Dull,
                                   0x3FCC68F568D31760ull, 0x3FC89F3B1694CFFEull, 0x3FC5B9AC9B743F0Dull,
                                   0x3FC3703C1F4D0FFEull, 0x3FC1964EC6FC9491ull};
    double p = dfrom(C[10]);
    for (int j = 9; j >= 0; --j) p = p * t2 + dfrom(C[j]);
    return (double)e + t * p;
}
static double pw2_d(double y) {
    const double k = rint(y), f = y - k;
    static const uint64_t C[14] = {0x3FF0000000000000ull, 0x3FE62E42FEFA39EFull, 0x3FCEBFBDFF82C58Full,
                                   0x3FAC6B08D704A0C0ull, 0x3F83B2AB6FBA4E77ull, 0x3F55D87FE78A6731ull,
                                   0x3F2430912F86C787ull, 0x3EEFFCBFC588B0C7ull, 0x3EB62C0223A5C824ull,
                                   0x3E7B5253D395E7C4ull, 0x3E3E4CF5158B8ECAull, 0x3DFE8CAC7351BB25ull,
                                   0x3DBC3BD650FC2986ull, 0x3D7816193166D0F9ull};
    double p = dfrom(C[13]);
    for (int j = 12; j >= 0; --j) p = p * f + dfrom(C[j]);
    if (!(k <= 1023.0)) return dfrom(0x7FF0000000000000ull);
    if (k < -1022.0) return 0.0;
    return p * dfrom((uint64_t)((long long)k + 1023) << 52);
}

/* ---------------------------------------------------------------------- */
/* quantizer constants (R1, R3, R4, R5)                       */
/* ---------------------------------------------------------------------- */
typedef struct {
    int dtype, bound, mode;          /* mode: ABS (also NOA), REL, or -1 raw words */
    unsigned flags;
    uint64_t qconst;
    double eps, range;
    float fa, fb, fc;                /* ABS: eps_eff, inv, eb2;  REL: c_lo, w, inv_w */
    double da, db, dc;
} qk_t;

static float down_f32(double x) {    /* largest binary32 <= x (x > 0, R1) */
    float f = (float)x;
    if (isinf(f)) f = FLT_MAX;
    while ((double)f > x) f = nextafterf(f, 0.0f);
    return f;
}

static int abs_consts(qk_t* q, double e) {   /* 0, or -2 when below the normal range */
    if (q->dtype == F32) {
        float ee = e > 0.0 ? down_f32(e) : 0.0f;
        if (ee > FLT_MAX / 2) ee = FLT_MAX / 2;
        if (!(ee >= FLT_MIN)) return E_BOUND;
        q->fa = ee; q->fb = 0.5f / ee; q->fc = 2.0f * ee; q->qconst = fbits(ee);
    } else {
        double ee = e;
        if (ee > DBL_MAX / 2) ee = DBL_MAX / 2;
        if (!(ee >= DBL_MIN)) return E_BOUND;
        q->da = ee; q->db = 0.5 / ee; q->dc = 2.0 * ee; q->qconst = dbits(ee);
    }
    q->mode = ABS;
    return 0;
}

/* NOA: min/max over the finite values (-0 as +0, R2), in parallel */
static void minmax(const void* in, uint64_t n, int dtype, int nt, double* mn_out, double* mx_out) {
    double mn = INFINITY, mx = -INFINITY;
#pragma omp parallel for num_threads(nt) reduction(min : mn) reduction(max : mx) schedule(static)
    for (long long i = 0; i < (long long)n; ++i) {
        const double v = dtype == F32 ? (double)((const float*)in)[i] : ((const double*)in)[i];
        if (!isfinite(v)) continue;
        const double w = v == 0.0 ? 0.0 : v;
        if (w < mn) mn = w;
        if (w > mx) mx = w;
    }
    *mn_out = mn;
    *mx_out = mx;
}

static int make_consts(qk_t* q, const void* in, uint64_t n, int dtype, int bound, double eps,
                       unsigned opts, int nt) {
    memset(q, 0, sizeof(*q));
    q->dtype = dtype; q->bound = bound; q->eps = eps;
    q->flags = (opts & FL_MS) ? FL_MS : 0u;
    if (!(eps > 0.0) || isinf(eps)) return E_BOUND;
    if (bound == ABS) return abs_consts(q, eps);
    if (bound == NOA) {
        double mn, mx;
        minmax(in, n, dtype, nt, &mn, &mx);
        const double d = mx >= mn ? mx - mn : 0.0;          /* no finite value: 0 */
        q->range = d;
        const double rlo = d > 0.0 ? nextafter(d, 0.0) : 0.0;     /* R3: two round-downs */
        const double e = eps * rlo;
        const double ea = e > 0.0 ? nextafter(e, 0.0) : 0.0;
        if (abs_consts(q, ea) != 0) {                       /* R4: degenerate -> raw words */
            q->flags |= FL_RAWWORDS; q->mode = -1; q->qconst = 0;
        }
        return 0;
    }
    /* REL (R5): c_lo = largest T <= 1 + eps; w = 2 log2p(c_lo) */
    if (dtype == F32) {
        float c;
        if (eps < 4503599627370496.0) {
            c = (float)(1.0 + eps);
            if (isinf(c)) c = FLT_MAX;
            while ((double)c - 1.0 > eps) c = nextafterf(c, 0.0f);
        } else {
            c = down_f32(eps);
        }
        const float lw = lg2_f(c), w = 2.0f * lw;
        if (!(w > 0.0f) || isinf(w)) { q->flags |= FL_RAWWORDS; q->mode = -1; return 0; }
        q->fa = c; q->fb = w; q->fc = 0.5f / lw; q->qconst = fbits(w);
    } else {
        double c;
        if (eps < 4503599627370496.0) {
            c = 1.0 + eps;
            if (c - 1.0 > eps) c = nextafter(c, 0.0);
        } else {
            c = isinf(eps) ? DBL_MAX : eps;
        }
        const double lw = lg2_d(c), w = 2.0 * lw;
        if (!(w > 0.0) || isinf(w)) { q->flags |= FL_RAWWORDS; q->mode = -1; return 0; }
        q->da = c; q->db = w; q->dc = 0.5 / lw; q->qconst = dbits(w);
    }
    q->mode = REL;
    return 0;
}

/* ---------------------------------------------------------------------- */
/* quantizers: value -> word                                   */
/* ---------------------------------------------------------------------- */
static uint32_t zz32(int32_t b) { return ((uint32_t)b << 1) ^ (uint32_t)(b >> 31); }
static uint64_t zz64(int64_t b) { return ((uint64_t)b << 1) ^ (uint64_t)(b >> 63); }

static uint32_t rel_word_f(const qk_t* q, float v) {
    const uint32_t u = fbits(v), sign = u >> 31, au = u & 0x7FFFFFFFu;
    if (au >= 0x00800000u && au < 0x7F800000u) {            /* R9: 0, denormals, inf, NaN exact */
        const float a = ffrom(au), rb = rintf(lg2_f(a) * q->fc);
        if (fabsf(rb) < 2097152.0f) {
            const float r = pw2_f(rb * q->fb);
            const float lo = ffrom(fbits(a / q->fa) + 1u), hi = ffrom(fbits(a * q->fa) - 1u);   /* R7 */
            if (lo <= r && r <= hi) return (0xFF800000u | (1u + ((zz32((int32_t)rb) << 1) | sign))) ^ 0xFF800000u;
        }
    }
    return (au > 0x7F800000u ? au : u) ^ 0xFF800000u;      /* P:104, R10, R11 */
}
static uint64_t rel_word_d(const qk_t* q, double v) {
    const uint64_t u = dbits(v), sign = u >> 63, au = u & 0x7FFFFFFFFFFFFFFFull;
    if (au >= 0x0010000000000000ull && au < 0x7FF0000000000000ull) {
        const double a = dfrom(au), rb = rint(lg2_d(a) * q->dc);
        if (fabs(rb) < 1125899906842624.0) {
            const double r = pw2_d(rb * q->db);
            const double lo = dfrom(dbits(a / q->da) + 1u), hi = dfrom(dbits(a * q->da) - 1u);
            if (lo <= r && r <= hi)
                return (0xFFF0000000000000ull | (1u + ((zz64((int64_t)rb) << 1) | sign))) ^ 0xFFF0000000000000ull;
        }
    }
    return (au > 0x7FF0000000000000ull ? au : u) ^ 0xFFF0000000000000ull;
}

/* f32 ABS, 8 at a time: rint(v*inv); keep the bin iff |bin| < 2^22 and
 * |v - bin*eb2| <= eps_eff (R7), else the raw bits (R8) */
static void quant_f32(const qk_t* q, const float* x, uint32_t* w, uint32_t m) {
    uint32_t i = 0;
    if (q->mode == ABS) {
        const __m256 inv = _mm256_set1_ps(q->fb), eb2 = _mm256_set1_ps(q->fc), ea = _mm256_set1_ps(q->fa);
        const __m256 lim = _mm256_set1_ps(4194304.0f), am = _mm256_castsi256_ps(_mm256_set1_epi32(0x7FFFFFFF));
        for (; i + 8 <= m; i += 8) {
            const __m256 v = _mm256_loadu_ps(x + i);
            const __m256 rb = _mm256_round_ps(_mm256_mul_ps(v, inv), _MM_FROUND_TO_NEAREST_INT | _MM_FROUND_NO_EXC);
            const __m256 diff = _mm256_and_ps(_mm256_sub_ps(v, _mm256_mul_ps(rb, eb2)), am);
            const __m256 ok = _mm256_and_ps(_mm256_cmp_ps(_mm256_and_ps(rb, am), lim, _CMP_LT_OQ),
                                            _mm256_cmp_ps(diff, ea, _CMP_LE_OQ));
            const __m256i b = _mm256_cvtps_epi32(rb);
            const __m256i z = _mm256_xor_si256(_mm256_slli_epi32(b, 1), _mm256_srai_epi32(b, 31));
            _mm256_storeu_si256((__m256i*)(w + i),
                                _mm256_blendv_epi8(_mm256_castps_si256(v), z, _mm256_castps_si256(ok)));
        }
        for (; i < m; ++i) {
            const float v = x[i], rb = rintf(v * q->fb);
            const int ok = fabsf(rb) < 4194304.0f && fabsf(v - rb * q->fc) <= q->fa;
            w[i] = ok ? zz32((int32_t)rb) : fbits(v);
        }
    } else if (q->mode == REL) {
        for (; i < m; ++i) w[i] = rel_word_f(q, x[i]);
    } else {
        memcpy(w, x, (size_t)m * 4);
    }
}

static void quant_f64(const qk_t* q, const double* x, uint64_t* w, uint32_t m) {
    uint32_t i = 0;
    if (q->mode == ABS) {
        const __m256d inv = _mm256_set1_pd(q->db), eb2 = _mm256_set1_pd(q->dc), ea = _mm256_set1_pd(q->da);
        const __m256d lim = _mm256_set1_pd(2251799813685248.0), mg = _mm256_set1_pd(6755399441055744.0);
        const __m256d am = _mm256_castsi256_pd(_mm256_set1_epi64x(0x7FFFFFFFFFFFFFFFll));
        const __m256i mgb = _mm256_set1_epi64x(0x4338000000000000ll);
        for (; i + 4 <= m; i += 4) {
            const __m256d v = _mm256_loadu_pd(x + i);
            const __m256d rb = _mm256_round_pd(_mm256_mul_pd(v, inv), _MM_FROUND_TO_NEAREST_INT | _MM_FROUND_NO_EXC);
            const __m256d diff = _mm256_and_pd(_mm256_sub_pd(v, _mm256_mul_pd(rb, eb2)), am);
            const __m256d ok = _mm256_and_pd(_mm256_cmp_pd(_mm256_and_pd(rb, am), lim, _CMP_LT_OQ),
                                             _mm256_cmp_pd(diff, ea, _CMP_LE_OQ));
            /* integer bin: bits(rb + 1.5*2^52) - bits(1.5*2^52), exact for |rb| < 2^51 */
            const __m256i b = _mm256_sub_epi64(_mm256_castpd_si256(_mm256_add_pd(rb, mg)), mgb);
            const __m256i sg = _mm256_cmpgt_epi64(_mm256_setzero_si256(), b);
            const __m256i z = _mm256_xor_si256(_mm256_slli_epi64(b, 1), sg);
            _mm256_storeu_si256((__m256i*)(w + i),
                                _mm256_blendv_epi8(_mm256_castpd_si256(v), z, _mm256_castpd_si256(ok)));
        }
        for (; i < m; ++i) {
            const double v = x[i], rb = rint(v * q->db);
            const int ok = fabs(rb) < 2251799813685248.0 && fabs(v - rb * q->dc) <= q->da;
            w[i] = ok ? zz64((int64_t)rb) : dbits(v);
        }
    } else if (q->mode == REL) {
        for (; i < m; ++i) w[i] = rel_word_d(q, x[i]);
    } else {
        memcpy(w, x, (size_t)m * 8);
    }
}

/* ---------------------------------------------------------------------- */
/* byte compaction tables (zero / repeat elimination)                      */
/* ---------------------------------------------------------------------- */
static uint64_t g_comp[256];          /* pshufb control: set bytes of the mask to the front */
static uint64_t g_expd[256];          /* inverse: the first popc bytes to the set positions */
__attribute__((constructor)) static void init_tables(void) {
    for (int m = 0; m < 256; ++m) {
        uint64_t c = 0x8080808080808080ull, e = 0x8080808080808080ull;
        int k = 0;
        for (int j = 0; j < 8; ++j)
            if ((m >> j) & 1) {
                c = (c & ~(0xFFull << (8 * k))) | ((uint64_t)j << (8 * k));
                e = (e & ~(0xFFull << (8 * j))) | ((uint64_t)k << (8 * j));
                ++k;
            }
        g_comp[m] = c;
        g_expd[m] = e;
    }
}

/* append the bytes of src[0..32) flagged in mask to dst (writes up to 8 bytes past) */
static inline uint8_t* compact32(uint8_t* dst, const uint8_t* src, uint32_t mask) {
    for (int g = 0; g < 4; ++g) {
        const uint32_t m8 = (mask >> (8 * g)) & 0xFFu;
        if (!m8) continue;
        const __m128i x = _mm_loadl_epi64((const __m128i*)(src + 8 * g));
        _mm_storel_epi64((__m128i*)dst, _mm_shuffle_epi8(x, _mm_cvtsi64_si128((long long)g_comp[m8])));
        dst += __builtin_popcount(m8);
    }
    return dst;
}

/* 32-bit mask of the non-zero bytes of src[0..32) */
static inline uint32_t nz32(const uint8_t* src) {
    const __m256i v = _mm256_loadu_si256((const __m256i*)src);
    return ~(uint32_t)_mm256_movemask_epi8(_mm256_cmpeq_epi8(v, _mm256_setzero_si256()));
}
/* 32-bit mask of the bytes of src[0..32) that differ from their predecessor src[-1..31) */
static inline uint32_t rep32(const uint8_t* src) {
    const __m256i v = _mm256_loadu_si256((const __m256i*)src);
    const __m256i p = _mm256_loadu_si256((const __m256i*)(src - 1));
    return ~(uint32_t)_mm256_movemask_epi8(_mm256_cmpeq_epi8(v, p));
}

/* repeated-byte elimination of X[0..len) (len % 32 == 0, X[-1] readable and 0, R15):
 * bitmap M (len/8 bytes) and the non-repeating bytes; returns their count */
static uint32_t repeat_level(const uint8_t* X, uint32_t len, uint8_t* M, uint8_t* Z) {
    uint8_t* z = Z;
    for (uint32_t o = 0; o < len; o += 32) {
        const uint32_t mk = rep32(X + o);
        memcpy(M + o / 8, &mk, 4);
        if (mk) z = compact32(z, X + o, mk);
    }
    return (uint32_t)(z - Z);
}

/* ---------------------------------------------------------------------- */
/* bit shuffle (R13) of 32 consecutive 32-bit residuals: plane b's */
/* 32 bits (bit i = element i) for b = 0..31, via a 4x32 byte transpose   */
/* and movemask on the bytes shifted left one bit at a time               */
/* ---------------------------------------------------------------------- */
static inline void bytes_of_32(const uint32_t* r, __m256i B[4]) {
    const __m256i sh = _mm256_setr_epi8(0, 4, 8, 12, 1, 5, 9, 13, 2, 6, 10, 14, 3, 7, 11, 15,
                                        0, 4, 8, 12, 1, 5, 9, 13, 2, 6, 10, 14, 3, 7, 11, 15);
    const __m256i pm = _mm256_setr_epi32(0, 4, 1, 5, 2, 6, 3, 7);
    __m256i V[4];
    for (int j = 0; j < 4; ++j)
        V[j] = _mm256_permutevar8x32_epi32(_mm256_shuffle_epi8(_mm256_loadu_si256((const __m256i*)(r + 8 * j)), sh), pm);
    /* V[j] = 64-bit pairs P(j,k) = byte k of elements 8j..8j+7, k = 0..3 */
    const __m256i t0 = _mm256_unpacklo_epi64(V[0], V[1]), t1 = _mm256_unpackhi_epi64(V[0], V[1]);
    const __m256i t2 = _mm256_unpacklo_epi64(V[2], V[3]), t3 = _mm256_unpackhi_epi64(V[2], V[3]);
    B[0] = _mm256_permute2x128_si256(t0, t2, 0x20);
    B[1] = _mm256_permute2x128_si256(t1, t3, 0x20);
    B[2] = _mm256_permute2x128_si256(t0, t2, 0x31);
    B[3] = _mm256_permute2x128_si256(t1, t3, 0x31);
}
/* planes b < P of the 32 residuals r[0..32) -> S[(B-1-b-off)*ps + 4g] */
static inline void shuffle32(const uint32_t* r, int P, uint8_t* S, int B, int boff, uint32_t ps, uint32_t g) {
    __m256i Bk[4];
    bytes_of_32(r, Bk);
    for (int k = 0; k < 4 && 8 * k < P; ++k) {
        __m256i x = Bk[k];
        for (int j = 7; j >= 0; --j) {
            const int b = 8 * k + j;
            if (b < P) {
                const uint32_t m = (uint32_t)_mm256_movemask_epi8(x);
                memcpy(S + (size_t)(B - 1 - (b + boff)) * ps + 4 * g, &m, 4);
            }
            x = _mm256_add_epi8(x, x);
        }
    }
}

/* ---------------------------------------------------------------------- */
/* one chunk: encode                                                       */
/* ---------------------------------------------------------------------- */
typedef struct {
    uint32_t size, raw, n1, n2, n3, n4;
    uint8_t* z1;                 /* Z1 in the thread's buffer B */
    uint8_t m4[4];
} enc_t;

typedef struct {                 /* per-thread working set (two 16 KiB buffers) */
    uint8_t A[CHUNK + 64] __attribute__((aligned(64)));   /* words / residuals -> shuffled bytes */
    uint8_t B[CHUNK + 64] __attribute__((aligned(64)));   /* residuals, then Z1 */
    uint8_t m1[2048 + 64] __attribute__((aligned(64)));   /* [32] = M1[0], M1[-1] = 0 */
    uint8_t m2[256 + 64] __attribute__((aligned(64)));
    uint8_t m3[32 + 64] __attribute__((aligned(64)));
    uint8_t z2[2048 + 16], z3[256 + 16], z4[32 + 16];
} work_t;

/* words w[0..m) (padded to cw with the last word, R12) -> residuals r */
static uint32_t delta32(const uint32_t* w, uint32_t m, uint32_t* r, int ms) {
    const uint32_t cw = CHUNK / 4, last = w[m - 1];
    uint32_t prev = 0, orv = 0;
    for (uint32_t i = 0; i < cw; ++i) {
        const uint32_t cur = i < m ? w[i] : last;
        const uint32_t d = cur - prev;
        const uint32_t x = ms ? ((d << 1) ^ (uint32_t)((int32_t)d >> 31)) : ((d + 0xAAAAAAAAu) ^ 0xAAAAAAAAu);
        r[i] = x;
        orv |= x;
        prev = cur;
    }
    return orv;
}
static uint64_t delta64(const uint64_t* w, uint32_t m, uint64_t* r, int ms) {
    const uint32_t cw = CHUNK / 8;
    const uint64_t last = w[m - 1];
    uint64_t prev = 0, orv = 0;
    for (uint32_t i = 0; i < cw; ++i) {
        const uint64_t cur = i < m ? w[i] : last;
        const uint64_t d = cur - prev;
        const uint64_t x = ms ? ((d << 1) ^ (uint64_t)((int64_t)d >> 63))
                              : ((d + 0xAAAAAAAAAAAAAAAAull) ^ 0xAAAAAAAAAAAAAAAAull);
        r[i] = x;
        orv |= x;
        prev = cur;
    }
    return orv;
}

static void encode_chunk(const qk_t* q, const void* in, uint32_t m, work_t* W, enc_t* e) {
    const int f32 = q->dtype == F32;
    const uint32_t s = f32 ? 4u : 8u, cw = CHUNK / s, B = 8 * s, ps = cw / 8;   /* plane bytes */
    const int ms = (q->flags & FL_MS) != 0;
    int P;
    /* O1 quantize -> A; O3 delta -> B (residuals) */
    if (f32) {
        quant_f32(q, (const float*)in, (uint32_t*)W->A, m);
        const uint32_t o = delta32((const uint32_t*)W->A, m, (uint32_t*)W->B, ms);
        P = o ? 32 - __builtin_clz(o) : 0;
    } else {
        quant_f64(q, (const double*)in, (uint64_t*)W->A, m);
        const uint64_t o = delta64((const uint64_t*)W->A, m, (uint64_t*)W->B, ms);
        P = o ? 64 - __builtin_clzll(o) : 0;
    }
    /* O4 shuffle -> A (only the P active planes: the others are zero) */
    uint8_t* const S = W->A;
    if (f32) {
        const uint32_t* r = (const uint32_t*)W->B;
        for (uint32_t g = 0; g < cw / 32; ++g) shuffle32(r + 32 * g, P, S, 32, 0, ps, g);
    } else {
        const uint64_t* r = (const uint64_t*)W->B;
        uint32_t lo[32], hi[32];
        for (uint32_t g = 0; g < cw / 32; ++g) {
            for (int i = 0; i < 32; ++i) { lo[i] = (uint32_t)r[32 * g + i]; hi[i] = (uint32_t)(r[32 * g + i] >> 32); }
            shuffle32(lo, P < 32 ? P : 32, S, 64, 0, ps, g);
            if (P > 32) shuffle32(hi, P - 32, S, 64, 32, ps, g);
        }
    }
    /* O5 level 1: zero-byte elimination of the active planes -> Z1 in B */
    uint8_t* const m1 = W->m1 + 32;
    const uint32_t first = (uint32_t)(B - P);              /* first active plane */
    memset(m1, 0, (size_t)first * ps / 8);
    uint8_t* z = W->B;
    for (uint32_t pl = first; pl < B; ++pl)
        for (uint32_t o = 0; o < ps; o += 32) {
            const uint8_t* src = S + (size_t)pl * ps + o;
            const uint32_t mk = nz32(src);
            memcpy(m1 + (pl * ps + o) / 8, &mk, 4);
            if (mk) z = compact32(z, src, mk);
        }
    e->z1 = W->B;
    e->n1 = (uint32_t)(z - W->B);
    /* levels 2-4: repeated-byte elimination (R14, R15) */
    uint8_t* const m2 = W->m2 + 32;
    uint8_t* const m3 = W->m3 + 32;
    e->n2 = repeat_level(m1, 2048, m2, W->z2);
    e->n3 = repeat_level(m2, 256, m3, W->z3);
    e->n4 = repeat_level(m3, 32, e->m4, W->z4);
    const uint32_t size = 4 + e->n4 + e->n3 + e->n2 + e->n1;
    e->raw = size >= m * s;                                  /* P:158, R17 */
    e->size = e->raw ? m * s : size;
}

/* ---------------------------------------------------------------------- */
/* stream                                                                  */
/* ---------------------------------------------------------------------- */
static void put64(uint8_t* p, uint64_t v) { for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i)); }
static uint64_t get64(const uint8_t* p) { uint64_t v = 0; for (int i = 7; i >= 0; --i) v = (v << 8) | p[i]; return v; }

uint64_t pfpl_cpu_max_compressed_bytes(uint64_t n, int dtype) {
    if (dtype != F32 && dtype != F64) return 0;
    const uint64_t s = dtype == F32 ? 4 : 8;
    return HDR + 4 * ((n * s + CHUNK - 1) / CHUNK) + n * s;
}

int pfpl_cpu_max_threads(void) { return omp_get_max_threads(); }

int pfpl_cpu_compress(const void* in, uint64_t n, int dtype, int bound, double eps, unsigned opts,
                      void* out, uint64_t* out_bytes, int nthreads) {
    if (dtype != F32 && dtype != F64) return E_ARG;
    if (bound != ABS && bound != REL && bound != NOA) return E_ARG;
    if (!out || !out_bytes || (n && !in) || n > (1ull << 40)) return E_ARG;
    const int nt = nthreads > 0 ? nthreads : omp_get_max_threads();
    const uint64_t s = dtype == F32 ? 4 : 8, cw = CHUNK / s, C = (n + cw - 1) / cw;
    const uint64_t cap = *out_bytes, base = HDR + 4 * C;
    if (cap < base) return E_CAP;
    qk_t q;
    const int st = make_consts(&q, in, n, dtype, bound, eps, opts, nt);
    if (st) return st;
    uint8_t* const o = (uint8_t*)out;
    memset(o, 0, HDR);
    o[0] = 'P'; o[1] = 'F'; o[2] = 'P'; o[3] = 'L'; o[4] = 1;
    o[5] = (uint8_t)dtype; o[6] = (uint8_t)bound; o[7] = (uint8_t)q.flags;
    put64(o + 8, n); put64(o + 16, dbits(eps)); put64(o + 24, q.qconst); put64(o + 32, dbits(q.range));
    put64(o + 40, CHUNK);
    /* shared carry array: carry[c] = payload bytes of chunks 0..c; ~0 = not yet */
    _Atomic uint64_t* carry = (_Atomic uint64_t*)malloc((C ? C : 1) * sizeof(uint64_t));
    if (!carry) return E_ARG;
    for (uint64_t c = 0; c < C; ++c) atomic_init(&carry[c], ~0ull);
    _Atomic uint64_t next;
    atomic_init(&next, 0);
    _Atomic int overflow;
    atomic_init(&overflow, 0);
#pragma omp parallel num_threads(nt)
    {
        work_t* W = (work_t*)aligned_alloc(64, sizeof(work_t));
        if (W) {
            memset(W->m1, 0, 32); memset(W->m2, 0, 32); memset(W->m3, 0, 32);   /* X[-1] = 0 */
            for (;;) {
                const uint64_t c = atomic_fetch_add_explicit(&next, 1, memory_order_relaxed);
                if (c >= C) break;
                const uint32_t m = (uint32_t)(c + 1 < C ? cw : n - c * cw);
                const uint8_t* src = (const uint8_t*)in + c * cw * s;
                enc_t e;
                encode_chunk(&q, src, m, W, &e);
                uint64_t off = 0;
                if (c > 0)
                    while ((off = atomic_load_explicit(&carry[c - 1], memory_order_acquire)) == ~0ull) _mm_pause();
                atomic_store_explicit(&carry[c], off + e.size, memory_order_release);
                const uint32_t sz = e.size;
                memcpy(o + HDR + 4 * c, &sz, 4);
                uint8_t* d = o + base + off;
                if (base + off + e.size > cap) {
                    atomic_store(&overflow, 1);
                } else if (e.raw) {
                    memcpy(d, src, e.size);
                } else {                                 /* R16: M4 | Z4 | Z3 | Z2 | Z1 */
                    memcpy(d, e.m4, 4); d += 4;
                    memcpy(d, W->z4, e.n4); d += e.n4;
                    memcpy(d, W->z3, e.n3); d += e.n3;
                    memcpy(d, W->z2, e.n2); d += e.n2;
                    memcpy(d, e.z1, e.n1);
                }
            }
            free(W);
        } else {
            atomic_store(&overflow, 2);
        }
    }
    const uint64_t total = base + (C ? atomic_load(&carry[C - 1]) : 0);
    const int of = atomic_load(&overflow);
    free(carry);
    if (of == 2) return E_ARG;
    if (of || total > cap) return E_CAP;
    *out_bytes = total;
    return 0;
}

/* ---------------------------------------------------------------------- */
/* one chunk: decode (the exact inverse)                             */
/* ---------------------------------------------------------------------- */
/* inverse of repeat_level: X[i] = next Z byte if bit i of M is set, else X[i-1]
 * (X[-1] = 0); returns the Z bytes consumed, or -1 if Z is shorter than needed */
static long unrepeat(const uint8_t* M, uint32_t len, const uint8_t* Z, uint64_t zavail, uint8_t* X) {
    uint64_t k = 0;
    uint8_t prev = 0;
    for (uint32_t i = 0; i < len; i += 8) {
        const uint32_t m8 = M[i / 8];
        if (!m8) { memset(X + i, prev, 8); continue; }
        for (int j = 0; j < 8; ++j) {
            if ((m8 >> j) & 1) {
                if (k >= zavail) return -1;
                prev = Z[k++];
            }
            X[i + j] = prev;
        }
    }
    return (long)k;
}

/* inverse bit shuffle of 32 consecutive residuals: r[i] bit b = bit i of plane b's word */
static inline void unshuffle32(const uint8_t* S, int P, int B, int boff, uint32_t ps, uint32_t g, uint32_t* r) {
    const __m256i bytesel = _mm256_setr_epi8(0, 0, 0, 0, 0, 0, 0, 0, 1, 1, 1, 1, 1, 1, 1, 1,
                                             2, 2, 2, 2, 2, 2, 2, 2, 3, 3, 3, 3, 3, 3, 3, 3);
    const __m256i bitsel = _mm256_set1_epi64x(0x8040201008040201ll);
    __m256i Bk[4] = {_mm256_setzero_si256(), _mm256_setzero_si256(), _mm256_setzero_si256(), _mm256_setzero_si256()};
    for (int b = 0; b < P; ++b) {
        uint32_t m;
        memcpy(&m, S + (size_t)(B - 1 - (b + boff)) * ps + 4 * g, 4);
        if (!m) continue;
        /* byte i = 0xFF iff bit i of m (element i has bit b) */
        const __m256i x = _mm256_shuffle_epi8(_mm256_set1_epi32((int)m), bytesel);
        const __m256i e = _mm256_cmpeq_epi8(_mm256_and_si256(x, bitsel), bitsel);
        Bk[b >> 3] = _mm256_or_si256(Bk[b >> 3], _mm256_and_si256(e, _mm256_set1_epi8((char)(1 << (b & 7)))));
    }
    /* inverse of bytes_of_32: Bk = byte k of elements 0..31 -> 32 words */
    const __m256i t0 = _mm256_permute2x128_si256(Bk[0], Bk[2], 0x20);   /* P00 P10 | P02 P12 */
    const __m256i t2 = _mm256_permute2x128_si256(Bk[0], Bk[2], 0x31);   /* P20 P30 | P22 P32 */
    const __m256i t1 = _mm256_permute2x128_si256(Bk[1], Bk[3], 0x20);
    const __m256i t3 = _mm256_permute2x128_si256(Bk[1], Bk[3], 0x31);
    __m256i V[4];
    V[0] = _mm256_unpacklo_epi64(t0, t1);
    V[1] = _mm256_unpackhi_epi64(t0, t1);
    V[2] = _mm256_unpacklo_epi64(t2, t3);
    V[3] = _mm256_unpackhi_epi64(t2, t3);
    const __m256i ipm = _mm256_setr_epi32(0, 2, 4, 6, 1, 3, 5, 7);
    const __m256i ish = _mm256_setr_epi8(0, 4, 8, 12, 1, 5, 9, 13, 2, 6, 10, 14, 3, 7, 11, 15,
                                         0, 4, 8, 12, 1, 5, 9, 13, 2, 6, 10, 14, 3, 7, 11, 15);
    for (int j = 0; j < 4; ++j)
        _mm256_storeu_si256((__m256i*)(r + 8 * j), _mm256_shuffle_epi8(_mm256_permutevar8x32_epi32(V[j], ipm), ish));
}

static int decode_chunk(const qk_t* q, const uint8_t* in, uint32_t size, uint32_t m, uint8_t* out,
                        work_t* W) {
    const int f32 = q->dtype == F32;
    const uint32_t s = f32 ? 4u : 8u, cw = CHUNK / s, B = 8 * s, ps = cw / 8;
    if (size == m * s) { memcpy(out, in, size); return 0; }   /* raw chunk */
    if (size > m * s || size < 4) return E_CORRUPT;
    /* RZE levels 4 -> 1, every read bounded by `size` */
    uint8_t* const m3 = W->m3 + 32;
    uint8_t* const m2 = W->m2 + 32;
    uint8_t* const m1 = W->m1 + 32;
    uint64_t o = 4;
    long k = unrepeat(in, 32, in + o, size - o, m3);
    if (k < 0) return E_CORRUPT;
    o += (uint64_t)k;
    if ((k = unrepeat(m3, 256, in + o, size - o, m2)) < 0) return E_CORRUPT;
    o += (uint64_t)k;
    if ((k = unrepeat(m2, 2048, in + o, size - o, m1)) < 0) return E_CORRUPT;
    o += (uint64_t)k;
    /* level 1: Z1 bytes to the flagged positions of the shuffled chunk (A) */
    const uint8_t* z1 = in + o;
    const uint64_t n1 = size - o;
    uint64_t used = 0;
    /* the first plane (M1 order) with a non-zero byte: planes before it are all zero
     * and are never read (P = the number of active bit planes from bit 0 up) */
    uint32_t i0 = 0;
    while (i0 < CHUNK / 8 && !m1[i0]) ++i0;
    const uint32_t pfirst = i0 < CHUNK / 8 ? 8 * i0 / ps : B;
    const int P = (int)(B - pfirst);
    uint8_t* const S = W->A;
    for (uint32_t i = pfirst * ps / 8; i < CHUNK / 8; ++i) {
        const uint32_t m8 = m1[i];
        uint64_t x = 0;
        if (m8) {
            const uint32_t c = (uint32_t)__builtin_popcount(m8);
            if (used + c > n1) return E_CORRUPT;
            uint64_t raw8 = 0;
            memcpy(&raw8, z1 + used, c);
            const __m128i v = _mm_shuffle_epi8(_mm_cvtsi64_si128((long long)raw8), _mm_cvtsi64_si128((long long)g_expd[m8]));
            x = (uint64_t)_mm_cvtsi128_si64(v);
            used += c;
        }
        memcpy(S + 8 * i, &x, 8);
    }
    if (used != n1) return E_CORRUPT;
    /* inverse shuffle -> residuals (B), NB^-1 + prefix sum -> words, dequantize */
    const int ms = (q->flags & FL_MS) != 0;
    if (f32) {
        uint32_t* r = (uint32_t*)W->B;
        for (uint32_t g = 0; g < cw / 32; ++g) unshuffle32(S, P, 32, 0, ps, g, r + 32 * g);
        uint32_t acc = 0;
        float* y = (float*)out;
        uint32_t* wq = (uint32_t*)W->A;          /* words (the shuffled bytes are consumed) */
        if (ms) for (uint32_t i = 0; i < m; ++i) { const uint32_t x = r[i]; acc += (x >> 1) ^ (0u - (x & 1u)); wq[i] = acc; }
        else for (uint32_t i = 0; i < m; ++i) { acc += (r[i] ^ 0xAAAAAAAAu) - 0xAAAAAAAAu; wq[i] = acc; }
        if (q->mode == ABS) {
            /* bins below 2^23 (R8): unzz(w) * eb2, else the raw bits; 8 at a time */
            const __m256 eb2 = _mm256_set1_ps(q->fc);
            const __m256i lim = _mm256_set1_epi32(0x00800000), one = _mm256_set1_epi32(1);
            uint32_t i = 0;
            for (; i + 8 <= m; i += 8) {
                const __m256i w = _mm256_loadu_si256((const __m256i*)(wq + i));
                const __m256i b = _mm256_xor_si256(_mm256_srli_epi32(w, 1), _mm256_sub_epi32(_mm256_setzero_si256(), _mm256_and_si256(w, one)));
                const __m256 v = _mm256_mul_ps(_mm256_cvtepi32_ps(b), eb2);
                const __m256i isbin = _mm256_cmpgt_epi32(lim, w);        /* w < 2^23 (w >= 0 as int: < 2^31) */
                const __m256i big = _mm256_srai_epi32(w, 31);             /* w >= 2^31: never a bin */
                _mm256_storeu_si256((__m256i*)(y + i),
                                    _mm256_blendv_epi8(w, _mm256_castps_si256(v), _mm256_andnot_si256(big, isbin)));
            }
            for (; i < m; ++i) {
                const uint32_t w = wq[i];
                y[i] = w < 0x00800000u ? (float)(int32_t)((w >> 1) ^ (0u - (w & 1u))) * q->fc : ffrom(w);
            }
        } else for (uint32_t i = 0; i < m; ++i) {
            const uint32_t w = wq[i];
            if (q->mode == REL) {
                const uint32_t u = w ^ 0xFF800000u;
                if ((u & 0xFF800000u) == 0xFF800000u && (u & 0x007FFFFFu)) {
                    const uint32_t t = (u & 0x007FFFFFu) - 1u;
                    const float mag = pw2_f((float)(int32_t)((t >> 2) ^ (0u - ((t >> 1) & 1u))) * q->fb);
                    y[i] = (t & 1u) ? -mag : mag;
                } else {
                    y[i] = ffrom(u);
                }
            } else {
                y[i] = ffrom(w);
            }
        }
    } else {
        uint64_t* r = (uint64_t*)W->B;
        uint32_t lo[32], hi[32];
        for (uint32_t g = 0; g < cw / 32; ++g) {
            unshuffle32(S, P < 32 ? P : 32, 64, 0, ps, g, lo);
            if (P > 32) unshuffle32(S, P - 32, 64, 32, ps, g, hi);
            else memset(hi, 0, sizeof(hi));
            for (int i = 0; i < 32; ++i) r[32 * g + i] = ((uint64_t)hi[i] << 32) | lo[i];
        }
        uint64_t acc = 0;
        double* y = (double*)out;
        for (uint32_t i = 0; i < m; ++i) {
            const uint64_t x = r[i];
            acc += ms ? ((x >> 1) ^ (0ull - (x & 1u))) : ((x ^ 0xAAAAAAAAAAAAAAAAull) - 0xAAAAAAAAAAAAAAAAull);
            const uint64_t w = acc;
            if (q->mode == ABS) {
                y[i] = w < 0x0010000000000000ull ? (double)(int64_t)((w >> 1) ^ (0ull - (w & 1u))) * q->dc : dfrom(w);
            } else if (q->mode == REL) {
                const uint64_t u = w ^ 0xFFF0000000000000ull;
                if ((u & 0xFFF0000000000000ull) == 0xFFF0000000000000ull && (u & 0x000FFFFFFFFFFFFFull)) {
                    const uint64_t t = (u & 0x000FFFFFFFFFFFFFull) - 1u;
                    const double mag = pw2_d((double)(int64_t)((t >> 2) ^ (0ull - ((t >> 1) & 1u))) * q->db);
                    y[i] = (t & 1u) ? -mag : mag;
                } else {
                    y[i] = dfrom(u);
                }
            } else {
                y[i] = dfrom(w);
            }
        }
    }
    return 0;
}

int pfpl_cpu_decompress(const void* in_, uint64_t in_bytes, void* out, uint64_t* out_bytes, int nthreads) {
    const uint8_t* in = (const uint8_t*)in_;
    if (!in || !out_bytes) return E_ARG;
    if (in_bytes < HDR) return E_CORRUPT;
    if (in[0] != 'P' || in[1] != 'F' || in[2] != 'P' || in[3] != 'L' || in[4] != 1) return E_CORRUPT;
    if (in[5] > 1 || in[6] > 2 || (in[7] & ~3u)) return E_CORRUPT;
    if (get64(in + 40) != CHUNK) return E_CORRUPT;
    qk_t q;
    memset(&q, 0, sizeof(q));
    q.dtype = in[5]; q.bound = in[6]; q.flags = in[7];
    const uint64_t n = get64(in + 8), qc = get64(in + 24);
    if (n > (1ull << 40)) return E_CORRUPT;
    const uint64_t s = q.dtype == F32 ? 4 : 8, cw = CHUNK / s, C = (n + cw - 1) / cw;
    if (q.flags & FL_RAWWORDS) {
        q.mode = -1;
    } else if (q.dtype == F32) {
        if (qc >> 32) return E_CORRUPT;
        const float c = ffrom((uint32_t)qc);
        if (q.bound == REL) {
            if (!(c > 0.0f) || isinf(c)) return E_CORRUPT;
            q.mode = REL; q.fb = c;
        } else {
            if (!(c >= FLT_MIN && c <= FLT_MAX / 2)) return E_CORRUPT;
            q.mode = ABS; q.fa = c; q.fc = 2.0f * c;
        }
    } else {
        const double c = dfrom(qc);
        if (q.bound == REL) {
            if (!(c > 0.0) || isinf(c)) return E_CORRUPT;
            q.mode = REL; q.db = c;
        } else {
            if (!(c >= DBL_MIN && c <= DBL_MAX / 2)) return E_CORRUPT;
            q.mode = ABS; q.da = c; q.dc = 2.0 * c;
        }
    }
    if (*out_bytes < n * s) return E_CAP;
    if (!out && n) return E_ARG;
    if (in_bytes < HDR + 4 * C) return E_CORRUPT;
    /* the decoder's prefix sum over the stored chunk sizes */
    uint64_t* offs = (uint64_t*)malloc((C + 1) * sizeof(uint64_t));
    if (!offs) return E_ARG;
    offs[0] = HDR + 4 * C;
    for (uint64_t c = 0; c < C; ++c) {
        uint32_t sz;
        memcpy(&sz, in + HDR + 4 * c, 4);
        const uint64_t m = c + 1 < C ? cw : n - c * cw;
        if (sz > m * s || (sz < 4 && sz != m * s)) { free(offs); return E_CORRUPT; }
        offs[c + 1] = offs[c] + sz;
    }
    if (offs[C] != in_bytes) { free(offs); return E_CORRUPT; }
    const int nt = nthreads > 0 ? nthreads : omp_get_max_threads();
    _Atomic int bad;
    atomic_init(&bad, 0);
#pragma omp parallel num_threads(nt)
    {
        work_t* W = (work_t*)aligned_alloc(64, sizeof(work_t));
        if (!W) {
            atomic_store(&bad, E_ARG);
        } else {
            memset(W->m1, 0, 32); memset(W->m2, 0, 32); memset(W->m3, 0, 32);
#pragma omp for schedule(dynamic, 4)
            for (long long c = 0; c < (long long)C; ++c) {
                const uint64_t m = (uint64_t)c + 1 < C ? cw : n - (uint64_t)c * cw;
                const int st = decode_chunk(&q, in + offs[c], (uint32_t)(offs[c + 1] - offs[c]), (uint32_t)m,
                                            (uint8_t*)out + (uint64_t)c * cw * s, W);
                if (st) atomic_store(&bad, st);
            }
            free(W);
        }
    }
    free(offs);
    const int b = atomic_load(&bad);
    if (b) return b;
    *out_bytes = n * s;
    return 0;
}
