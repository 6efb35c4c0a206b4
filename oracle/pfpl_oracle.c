/*
 * pfpl_oracle.c -- plain CPU oracle of the PFPL codec (TEST INFRASTRUCTURE).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this.  It shares no code with the CUDA
 * path.  Written step by step from PAPER.md (P:NNN) in the paper's order;
 * where the paper is silent the reading id (R#) from DESIGN.md section 3 is
 * cited.  One chunk at a time, obvious loops, IEEE binary32/binary64
 * arithmetic with round-to-nearest-even, no FMA contraction
 * (compiled with -ffp-contract=off -fno-fast-math).
 */
#include "pfpl_oracle.h"
#include <math.h>
#include <float.h>
#include <string.h>
#include <stdlib.h>

/* ------------------------------------------------------------------ */
/* bit casts                                                          */
/* ------------------------------------------------------------------ */
static uint32_t bits_f(float x) { uint32_t u; memcpy(&u, &x, 4); return u; }
static float flt_f(uint32_t u) { float x; memcpy(&x, &u, 4); return x; }
static uint64_t bits_d(double x) { uint64_t u; memcpy(&u, &x, 8); return u; }
static double flt_d(uint64_t u) { double x; memcpy(&x, &u, 8); return x; }

/* R1: largest binary32 value <= x (x > 0, may be +inf) */
static float round_down_f32(double x) {
    float f = (float)x;
    if (isinf(f) && f > 0) f = FLT_MAX;
    while ((double)f > x) f = nextafterf(f, 0.0f);
    return f;
}

/* zigzag ("magnitude-sign" with the sign in the LSB, reading R8) */
static uint32_t zz32(int32_t b) { return ((uint32_t)b << 1) ^ (uint32_t)(b >> 31); }
static int32_t unzz32(uint32_t z) { return (int32_t)((z >> 1) ^ (0u - (z & 1u))); }
static uint64_t zz64(int64_t b) { return ((uint64_t)b << 1) ^ (uint64_t)(b >> 63); }
static int64_t unzz64(uint64_t z) { return (int64_t)((z >> 1) ^ (0ull - (z & 1ull))); }

/* ------------------------------------------------------------------ */
/* A11: portable log2 / pow2 using only IEEE +,-,*,/ and integer ops  */
/* ("we wrote approximations for both functions that use only   */
/* IEEE-compliant operations"; the formulas are reading R5).          */
/* log2(m) = 2/ln2 * atanh(t), t=(m-1)/(m+1): odd series in t.        */
/* 2^f = sum (f ln2)^j / j!  (Taylor, Horner form).                   */
/* Constants are binary32/binary64 nearest to 2/(k ln 2), ln2^j/j!.  */
/* ------------------------------------------------------------------ */
float orc_log2p_f32(float a) {
    uint32_t u = bits_f(a);
    int e = (int)((u >> 23) & 0xFFu) - 127;
    float m = flt_f((u & 0x007FFFFFu) | 0x3F800000u);     /* m in [1,2) */
    const float SQRT2 = flt_f(0x3FB504F3u);
    if (m > SQRT2) { m = m * 0.5f; e = e + 1; }
    float t = (m - 1.0f) / (m + 1.0f);
    float t2 = t * t;
    const float C1 = flt_f(0x4038AA3Bu), C3 = flt_f(0x3F76384Fu),
                C5 = flt_f(0x3F13BB63u), C7 = flt_f(0x3ED30BB1u);
    float p = C7;
    p = p * t2; p = p + C5;
    p = p * t2; p = p + C3;
    p = p * t2; p = p + C1;
    float r = t * p;
    return (float)e + r;
}

float orc_pow2p_f32(float y) {
    float k = rintf(y);
    float f = y - k;                                      /* f in [-0.5, 0.5] */
    const uint32_t PC[8] = {0x3F800000u, 0x3F317218u, 0x3E75FDF0u, 0x3D635847u,
                            0x3C1D955Bu, 0x3AAEC3FFu, 0x39218489u, 0x377FE5FEu};
    float p = flt_f(PC[7]);
    for (int j = 6; j >= 0; --j) { p = p * f; p = p + flt_f(PC[j]); }
    if (!(k <= 127.0f)) return INFINITY;                  /* also NaN input */
    if (k < -126.0f) return 0.0f;
    int ki = (int)k;
    float scale = flt_f((uint32_t)(ki + 127) << 23);
    return p * scale;
}

double orc_log2p_f64(double a) {
    uint64_t u = bits_d(a);
    int e = (int)((u >> 52) & 0x7FFu) - 1023;
    double m = flt_d((u & 0x000FFFFFFFFFFFFFull) | 0x3FF0000000000000ull);
    const double SQRT2 = flt_d(0x3FF6A09E667F3BCDull);
    if (m > SQRT2) { m = m * 0.5; e = e + 1; }
    double t = (m - 1.0) / (m + 1.0);
    double t2 = t * t;
    const uint64_t CK[11] = {0x40071547652B82FEull, 0x3FEEC709DC3A03FDull,
                             0x3FE2776C50EF9BFEull, 0x3FDA61762A7ADED9ull,
                             0x3FD484B13D7C02A9ull, 0x3FD0C9A84994022Dull,
                             0x3FCC68F568D31760ull, 0x3FC89F3B1694CFFEull,
                             0x3FC5B9AC9B743F0Dull, 0x3FC3703C1F4D0FFEull,
                             0x3FC1964EC6FC9491ull};            /* c_1, c_3, ..., c_21 */
    double p = flt_d(CK[10]);
    for (int j = 9; j >= 0; --j) { p = p * t2; p = p + flt_d(CK[j]); }
    double r = t * p;
    return (double)e + r;
}

double orc_pow2p_f64(double y) {
    double k = rint(y);
    double f = y - k;
    const uint64_t PC[14] = {0x3FF0000000000000ull, 0x3FE62E42FEFA39EFull,
                             0x3FCEBFBDFF82C58Full, 0x3FAC6B08D704A0C0ull,
                             0x3F83B2AB6FBA4E77ull, 0x3F55D87FE78A6731ull,
                             0x3F2430912F86C787ull, 0x3EEFFCBFC588B0C7ull,
                             0x3EB62C0223A5C824ull, 0x3E7B5253D395E7C4ull,
                             0x3E3E4CF5158B8ECAull, 0x3DFE8CAC7351BB25ull,
                             0x3DBC3BD650FC2986ull, 0x3D7816193166D0F9ull};
    double p = flt_d(PC[13]);
    for (int j = 12; j >= 0; --j) { p = p * f; p = p + flt_d(PC[j]); }
    if (!(k <= 1023.0)) return INFINITY;
    if (k < -1022.0) return 0.0;
    long long ki = (long long)k;
    double scale = flt_d((uint64_t)(ki + 1023) << 52);
    return p * scale;
}

/* ------------------------------------------------------------------ */
/* O0: constants                                                      */
/* ------------------------------------------------------------------ */
int orc_params_init(orc_params* P, const void* in, uint64_t n, int dtype, int bound,
                    double eps, int ms) {
    memset(P, 0, sizeof(*P));
    if (dtype != ORC_F32 && dtype != ORC_F64) return ORC_ERR_ARG;
    if (bound != ORC_ABS && bound != ORC_REL && bound != ORC_NOA) return ORC_ERR_ARG;
    P->dtype = dtype; P->bound = bound; P->eps = eps;
    P->flags = ms ? ORC_FLAG_MS : 0;
    if (!(eps > 0.0) || isinf(eps)) return ORC_ERR_BOUND;  /* NaN, <=0, inf */

    double eps_abs = eps;
    if (bound == ORC_NOA) {
        /* P:92 "first determines the minimum and maximum values in the input";
         * reading R2: over finite values only, -0 canonicalised to +0. */
        int have = 0; double mn = 0.0, mx = 0.0;
        for (uint64_t i = 0; i < n; ++i) {
            double v = dtype == ORC_F32 ? (double)((const float*)in)[i]
                                        : ((const double*)in)[i];
            if (!isfinite(v)) continue;
            if (v == 0.0) v = 0.0;
            if (!have) { mn = mx = v; have = 1; }
            else { if (v < mn) mn = v; if (v > mx) mx = v; }
        }
        /* P:92 abs = eps * (max - min); reading R3: two round-downs so the
         * derived bound never exceeds the exact eps*(max-min). */
        double d = have ? mx - mn : 0.0;
        P->range = d;
        double r_lo = d > 0.0 ? nextafter(d, 0.0) : 0.0;
        double e = eps * r_lo;
        eps_abs = e > 0.0 ? nextafter(e, 0.0) : 0.0;
    }

    if (bound == ORC_ABS || bound == ORC_NOA) {
        /* R1: eps_eff = largest T <= eps; R4: clamp to T_MAX/2 */
        if (dtype == ORC_F32) {
            float ee = eps_abs > 0.0 ? round_down_f32(eps_abs) : 0.0f;
            if (ee > FLT_MAX / 2) ee = FLT_MAX / 2;
            if (!(ee >= FLT_MIN)) {   /* bound cannot be below the smallest normal */
                if (bound == ORC_ABS) return ORC_ERR_BOUND;
                P->flags |= ORC_FLAG_RAWWORDS;              /* R4 */
                return ORC_OK;
            }
            P->eps_eff_f = ee;
            P->inv_f = 0.5f / ee;                           /* P:88 "multiplying by 0.5/eps" */
            P->eb2_f = 2.0f * ee;                           /* bin center spacing 2 eps */
            P->qconst = bits_f(ee);
        } else {
            double ee = eps_abs;
            if (ee > DBL_MAX / 2) ee = DBL_MAX / 2;
            if (!(ee >= DBL_MIN)) {
                if (bound == ORC_ABS) return ORC_ERR_BOUND;
                P->flags |= ORC_FLAG_RAWWORDS;
                return ORC_OK;
            }
            P->eps_eff_d = ee;
            P->inv_d = 0.5 / ee;
            P->eb2_d = 2.0 * ee;
            P->qconst = bits_d(ee);
        }
        return ORC_OK;
    }

    /* REL, P:90 with reading R5: bin = round(log2|v| * 0.5/log2(1+eps)).
     * R1: c_lo = largest T <= 1+eps (exactly). */
    if (dtype == ORC_F32) {
        float c;
        if (eps < 4503599627370496.0) {                    /* 2^52: c-1 exact below */
            c = (float)(1.0 + eps);
            if (isinf(c)) c = FLT_MAX;
            while ((double)c - 1.0 > eps) c = nextafterf(c, 0.0f);
        } else {
            c = round_down_f32(eps);
        }
        P->c_lo_f = c;
        float lw = orc_log2p_f32(c);
        float w = 2.0f * lw;
        if (!(w > 0.0f) || isinf(w)) { P->flags |= ORC_FLAG_RAWWORDS; return ORC_OK; }
        P->w_f = w;
        P->inv_w_f = 0.5f / lw;
        P->qconst = bits_f(w);
    } else {
        double c;
        if (eps < 4503599627370496.0) {
            c = 1.0 + eps;
            if (c - 1.0 > eps) c = nextafter(c, 0.0);
        } else {
            c = eps;
            if (isinf(c)) c = DBL_MAX;
        }
        P->c_lo_d = c;
        double lw = orc_log2p_f64(c);
        double w = 2.0 * lw;
        if (!(w > 0.0) || isinf(w)) { P->flags |= ORC_FLAG_RAWWORDS; return ORC_OK; }
        P->w_d = w;
        P->inv_w_d = 0.5 / lw;
        P->qconst = bits_d(w);
    }
    return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* O1: quantize + immediate verify                         */
/* ------------------------------------------------------------------ */
static uint32_t quant_abs_f32(const orc_params* P, float v) {
    float s = v * P->inv_f;                  /* P:88 multiply by 0.5/eps */
    float rb = rintf(s);                     /* round to nearest (R6: ties-to-even) */
    if (!(fabsf(rb) < 4194304.0f))           /* bin too large, NaN/inf too */
        return bits_f(v);
    float vr = rb * P->eb2_f;                /* decode immediately ... */
    float diff = fabsf(v - vr);
    if (!(diff <= P->eps_eff_f))             /* ... and check the bound (R7) */
        return bits_f(v);                    /* emit the unmodified value */
    return zz32((int32_t)rb);                /* bin in the denormal range */
}

static uint64_t quant_abs_f64(const orc_params* P, double v) {
    double s = v * P->inv_d;
    double rb = rint(s);
    if (!(fabs(rb) < 2251799813685248.0))    /* 2^51 */
        return bits_d(v);
    double vr = rb * P->eb2_d;
    double diff = fabs(v - vr);
    if (!(diff <= P->eps_eff_d))
        return bits_d(v);
    return zz64((int64_t)rb);
}

static uint32_t quant_rel_f32(const orc_params* P, float v) {
    uint32_t u = bits_f(v);
    uint32_t sign = u >> 31;
    uint32_t au = u & 0x7FFFFFFFu;
    uint32_t q0;
    int lossless = 1;
    if (au >= 0x00800000u && au < 0x7F800000u) {   /* R9: 0, denormal, inf, NaN lossless */
        float a = flt_f(au);
        float L = orc_log2p_f32(a);            /* P:90 logarithm of the absolute value */
        float s = L * P->inv_w_f;
        float rb = rintf(s);
        if (fabsf(rb) < 2097152.0f) {          /* 2^(23-2) */
            float y = rb * P->w_f;
            float r = orc_pow2p_f32(y);         /* reconstruction magnitude */
            /* R7: conservative check |v|/(1+eps) <= |v'| <= |v|(1+eps) */
            float lo = flt_f(bits_f(a / P->c_lo_f) + 1u);    /* nextup   (>0) */
            float hi = flt_f(bits_f(a * P->c_lo_f) - 1u);    /* nextdown (>0) */
            if (lo <= r && r <= hi) lossless = 0;
            if (!lossless) {
                uint32_t payload = 1u + ((zz32((int32_t)rb) << 1) | sign);   /* R10 */
                q0 = 0xFF800000u | payload;    /* negative-NaN range */
            }
        }
    }
    if (lossless) {
        q0 = u;
        if (au > 0x7F800000u) q0 = au;        /* P:104 make all negative NaNs positive */
    }
    return q0 ^ 0xFF800000u;                   /* P:104 invert the leading bits (R11) */
}

static uint64_t quant_rel_f64(const orc_params* P, double v) {
    uint64_t u = bits_d(v);
    uint64_t sign = u >> 63;
    uint64_t au = u & 0x7FFFFFFFFFFFFFFFull;
    uint64_t q0 = 0;
    int lossless = 1;
    if (au >= 0x0010000000000000ull && au < 0x7FF0000000000000ull) {
        double a = flt_d(au);
        double L = orc_log2p_f64(a);
        double s = L * P->inv_w_d;
        double rb = rint(s);
        if (fabs(rb) < 1125899906842624.0) {   /* 2^(52-2) */
            double y = rb * P->w_d;
            double r = orc_pow2p_f64(y);
            double lo = flt_d(bits_d(a / P->c_lo_d) + 1u);
            double hi = flt_d(bits_d(a * P->c_lo_d) - 1u);
            if (lo <= r && r <= hi) {
                lossless = 0;
                uint64_t payload = 1u + ((zz64((int64_t)rb) << 1) | sign);
                q0 = 0xFFF0000000000000ull | payload;
            }
        }
    }
    if (lossless) {
        q0 = u;
        if (au > 0x7FF0000000000000ull) q0 = au;
    }
    return q0 ^ 0xFFF0000000000000ull;
}

void orc_quantize(const orc_params* P, const void* in, uint64_t n, void* words) {
    if (P->dtype == ORC_F32) {
        const float* x = (const float*)in; uint32_t* q = (uint32_t*)words;
        for (uint64_t i = 0; i < n; ++i) {
            if (P->flags & ORC_FLAG_RAWWORDS) q[i] = bits_f(x[i]);
            else if (P->bound == ORC_REL) q[i] = quant_rel_f32(P, x[i]);
            else q[i] = quant_abs_f32(P, x[i]);
        }
    } else {
        const double* x = (const double*)in; uint64_t* q = (uint64_t*)words;
        for (uint64_t i = 0; i < n; ++i) {
            if (P->flags & ORC_FLAG_RAWWORDS) q[i] = bits_d(x[i]);
            else if (P->bound == ORC_REL) q[i] = quant_rel_f64(P, x[i]);
            else q[i] = quant_abs_f64(P, x[i]);
        }
    }
}

void orc_dequantize(const orc_params* P, const void* words, uint64_t n, void* out) {
    if (P->dtype == ORC_F32) {
        const uint32_t* q = (const uint32_t*)words; float* y = (float*)out;
        for (uint64_t i = 0; i < n; ++i) {
            uint32_t w = q[i];
            if (P->flags & ORC_FLAG_RAWWORDS) { y[i] = flt_f(w); continue; }
            if (P->bound == ORC_REL) {
                uint32_t u = w ^ 0xFF800000u;
                if ((u & 0xFF800000u) == 0xFF800000u && (u & 0x007FFFFFu) != 0) {
                    uint32_t t = (u & 0x007FFFFFu) - 1u;
                    int32_t b = unzz32(t >> 1);
                    float mag = orc_pow2p_f32((float)b * P->w_f);
                    y[i] = (t & 1u) ? -mag : mag;
                } else {
                    y[i] = flt_f(u);
                }
            } else {
                if (w < 0x00800000u) y[i] = (float)unzz32(w) * P->eb2_f;
                else y[i] = flt_f(w);
            }
        }
    } else {
        const uint64_t* q = (const uint64_t*)words; double* y = (double*)out;
        for (uint64_t i = 0; i < n; ++i) {
            uint64_t w = q[i];
            if (P->flags & ORC_FLAG_RAWWORDS) { y[i] = flt_d(w); continue; }
            if (P->bound == ORC_REL) {
                uint64_t u = w ^ 0xFFF0000000000000ull;
                if ((u & 0xFFF0000000000000ull) == 0xFFF0000000000000ull &&
                    (u & 0x000FFFFFFFFFFFFFull) != 0) {
                    uint64_t t = (u & 0x000FFFFFFFFFFFFFull) - 1u;
                    int64_t b = unzz64(t >> 1);
                    double mag = orc_pow2p_f64((double)b * P->w_d);
                    y[i] = (t & 1u) ? -mag : mag;
                } else {
                    y[i] = flt_d(u);
                }
            } else {
                if (w < 0x0010000000000000ull) y[i] = (double)unzz64(w) * P->eb2_d;
                else y[i] = flt_d(w);
            }
        }
    }
}

/* ------------------------------------------------------------------ */
/* O3: difference coding (delta modulation) + negabinary       */
/* ------------------------------------------------------------------ */
static uint64_t wmask(int bits) { return bits == 64 ? ~0ull : ((1ull << bits) - 1ull); }

void orc_delta_encode(const uint64_t* q, uint64_t* r, size_t cw, int bits, int ms) {
    const uint64_t M = wmask(bits);
    const uint64_t K = 0xAAAAAAAAAAAAAAAAull & M;
    uint64_t prev = 0;                                  /* predecessor of the first value is 0 */
    for (size_t i = 0; i < cw; ++i) {
        uint64_t d = (q[i] - prev) & M;                 /* "itself minus the previous value" */
        if (!ms) {
            r[i] = ((d + K) & M) ^ K;                   /* two's complement -> base -2 */
        } else {
            uint64_t sgn = (d >> (bits - 1)) & 1u;      /* A1: magnitude-sign (zigzag) */
            r[i] = ((d << 1) & M) ^ (sgn ? M : 0);
        }
        prev = q[i];
    }
}

void orc_delta_decode(const uint64_t* r, uint64_t* q, size_t cw, int bits, int ms) {
    const uint64_t M = wmask(bits);
    const uint64_t K = 0xAAAAAAAAAAAAAAAAull & M;
    uint64_t prev = 0;
    for (size_t i = 0; i < cw; ++i) {
        uint64_t d;
        if (!ms) d = ((r[i] ^ K) - K) & M;
        else d = ((r[i] >> 1) ^ (0ull - (r[i] & 1u))) & M;
        prev = (prev + d) & M;
        q[i] = prev;
    }
}

/* ------------------------------------------------------------------ */
/* O4: bit shuffle -- "MSB of all residuals, then the second MSB ..." */
/* (P:127). Plane p (p=0 is the MSB) occupies bytes [p*cw/8, (p+1)*cw/8); */
/* element i is bit (i%8) of byte i/8 of its plane (R13).             */
/* ------------------------------------------------------------------ */
void orc_shuffle(const uint64_t* r, size_t cw, int bits, uint8_t* S) {
    memset(S, 0, cw * (size_t)bits / 8);
    for (int p = 0; p < bits; ++p) {
        int b = bits - 1 - p;
        for (size_t i = 0; i < cw; ++i) {
            uint64_t bit = (r[i] >> b) & 1u;
            S[(size_t)p * (cw / 8) + i / 8] |= (uint8_t)(bit << (i % 8));
        }
    }
}

void orc_unshuffle(const uint8_t* S, size_t cw, int bits, uint64_t* r) {
    for (size_t i = 0; i < cw; ++i) r[i] = 0;
    for (int p = 0; p < bits; ++p) {
        int b = bits - 1 - p;
        for (size_t i = 0; i < cw; ++i) {
            uint64_t bit = (S[(size_t)p * (cw / 8) + i / 8] >> (i % 8)) & 1u;
            r[i] |= bit << b;
        }
    }
}

/* ------------------------------------------------------------------ */
/* O5: zero-byte elimination + 3 levels of repeated-byte elimination  */
/* (readings R14-R16). Output: M4 | Z4 | Z3 | Z2 | Z1.     */
/* ------------------------------------------------------------------ */
/* level 1 (zeros): M bit j of byte k set iff X[8k+j] != 0 */
static size_t elim_zero(const uint8_t* X, size_t len, uint8_t* M, uint8_t* Z) {
    size_t nz = 0;
    memset(M, 0, len / 8);
    for (size_t i = 0; i < len; ++i)
        if (X[i] != 0) { M[i / 8] |= (uint8_t)(1u << (i % 8)); Z[nz++] = X[i]; }
    return nz;
}
/* levels 2..4 (repeats): bit set iff the byte differs from the previous
 * one ("a cleared bit means the byte repeats"); X[-1] = 0 (R15) */
static size_t elim_repeat(const uint8_t* X, size_t len, uint8_t* M, uint8_t* Z) {
    size_t nz = 0;
    uint8_t prev = 0;
    memset(M, 0, len / 8);
    for (size_t i = 0; i < len; ++i) {
        if (X[i] != prev) { M[i / 8] |= (uint8_t)(1u << (i % 8)); Z[nz++] = X[i]; }
        prev = X[i];
    }
    return nz;
}

size_t orc_rze_encode(const uint8_t* X1, uint8_t* out) {
    uint8_t M1[2048], M2[256], M3[32], M4[4];
    uint8_t Z1[16384], Z2[2048], Z3[256], Z4[32];
    size_t n1 = elim_zero(X1, 16384, M1, Z1);
    size_t n2 = elim_repeat(M1, 2048, M2, Z2);
    size_t n3 = elim_repeat(M2, 256, M3, Z3);
    size_t n4 = elim_repeat(M3, 32, M4, Z4);
    size_t o = 0;
    memcpy(out + o, M4, 4); o += 4;
    memcpy(out + o, Z4, n4); o += n4;
    memcpy(out + o, Z3, n3); o += n3;
    memcpy(out + o, Z2, n2); o += n2;
    memcpy(out + o, Z1, n1); o += n1;
    return o;
}

static int popcount8(uint8_t x) { int c = 0; while (x) { c += x & 1u; x >>= 1; } return c; }

/* inverse of one level; returns bytes of Z consumed or -1 */
static long undo_level(const uint8_t* M, size_t len, const uint8_t* Z, size_t zavail,
                       int repeat, uint8_t* X) {
    size_t nz = 0;
    uint8_t prev = 0;
    for (size_t i = 0; i < len; ++i) {
        if ((M[i / 8] >> (i % 8)) & 1u) {
            if (nz >= zavail) return -1;
            X[i] = Z[nz++];
        } else {
            X[i] = repeat ? prev : 0;
        }
        prev = X[i];
    }
    return (long)nz;
}

long orc_rze_decode(const uint8_t* in, size_t in_len, uint8_t* X1) {
    uint8_t M1[2048], M2[256], M3[32];
    size_t o = 0;
    if (in_len < 4) return -1;
    const uint8_t* M4 = in; o = 4;
    long k;
    k = undo_level(M4, 32, in + o, in_len - o, 1, M3); if (k < 0) return -1; o += (size_t)k;
    k = undo_level(M3, 256, in + o, in_len - o, 1, M2); if (k < 0) return -1; o += (size_t)k;
    k = undo_level(M2, 2048, in + o, in_len - o, 1, M1); if (k < 0) return -1; o += (size_t)k;
    k = undo_level(M1, 16384, in + o, in_len - o, 0, X1); if (k < 0) return -1; o += (size_t)k;
    (void)popcount8;
    return (long)o;
}

/* ------------------------------------------------------------------ */
/* O2-O6: one chunk                                                   */
/* ------------------------------------------------------------------ */
static size_t tsize(int dtype) { return dtype == ORC_F32 ? 4u : 8u; }

size_t orc_encode_chunk(const orc_params* P, const void* in, size_t m, uint8_t* out) {
    const size_t s = tsize(P->dtype);
    const size_t cw = ORC_CHUNK_BYTES / s;
    const int bits = (int)(8 * s);
    uint64_t q[4096], r[4096];
    uint8_t S[16384];
    uint8_t tmp[4 + 32 + 256 + 2048 + 16384];
    /* O1 */
    if (P->dtype == ORC_F32) {
        uint32_t w[4096];
        orc_quantize(P, in, m, w);
        for (size_t i = 0; i < m; ++i) q[i] = w[i];
    } else {
        orc_quantize(P, in, m, q);
    }
    /* O2 (R12): pad a short chunk with its last word -> zero residuals */
    for (size_t i = m; i < cw; ++i) q[i] = q[m - 1];
    orc_delta_encode(q, r, cw, bits, (P->flags & ORC_FLAG_MS) != 0);   /* O3 */
    orc_shuffle(r, cw, bits, S);                                        /* O4 */
    size_t sz = orc_rze_encode(S, tmp);                                 /* O5 */
    if (sz >= m * s) {                  /* O6: incompressible -> raw, flagged */
        memcpy(out, in, m * s);
        return m * s;
    }
    memcpy(out, tmp, sz);
    return sz;
}

int orc_decode_chunk(const orc_params* P, const uint8_t* in, size_t size, size_t m,
                     void* out) {
    const size_t s = tsize(P->dtype);
    const size_t cw = ORC_CHUNK_BYTES / s;
    const int bits = (int)(8 * s);
    if (size == m * s) { memcpy(out, in, m * s); return ORC_OK; }      /* raw chunk */
    if (size > m * s) return ORC_ERR_CORRUPT;
    uint8_t S[16384];
    uint64_t r[4096], q[4096];
    long used = orc_rze_decode(in, size, S);
    if (used < 0 || (size_t)used != size) return ORC_ERR_CORRUPT;
    orc_unshuffle(S, cw, bits, r);
    orc_delta_decode(r, q, cw, bits, (P->flags & ORC_FLAG_MS) != 0);
    if (P->dtype == ORC_F32) {
        uint32_t w[4096];
        for (size_t i = 0; i < m; ++i) w[i] = (uint32_t)q[i];
        orc_dequantize(P, w, m, out);
    } else {
        orc_dequantize(P, q, m, out);
    }
    return ORC_OK;
}

/* ------------------------------------------------------------------ */
/* O7/O8: stream = header(48) | u32 size[C] | payload_0 | ... (R18)   */
/* ------------------------------------------------------------------ */
static void put_u32(uint8_t* p, uint32_t v) { for (int i = 0; i < 4; ++i) p[i] = (uint8_t)(v >> (8 * i)); }
static void put_u64(uint8_t* p, uint64_t v) { for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i)); }
static uint32_t get_u32(const uint8_t* p) { uint32_t v = 0; for (int i = 3; i >= 0; --i) v = (v << 8) | p[i]; return v; }
static uint64_t get_u64(const uint8_t* p) { uint64_t v = 0; for (int i = 7; i >= 0; --i) v = (v << 8) | p[i]; return v; }

uint64_t orc_max_compressed_bytes(uint64_t n, int dtype) {
    uint64_t s = tsize(dtype);
    uint64_t C = (n * s + ORC_CHUNK_BYTES - 1) / ORC_CHUNK_BYTES;
    return ORC_HEADER_BYTES + 4 * C + n * s;
}

int64_t orc_compress(const void* in, uint64_t n, int dtype, int bound, double eps, int ms,
                     uint8_t* out, uint64_t cap, int nthreads) {
    orc_params P;
    int st = orc_params_init(&P, in, n, dtype, bound, eps, ms);
    if (st != ORC_OK) return st;
    const uint64_t s = tsize(dtype);
    const uint64_t cw = ORC_CHUNK_BYTES / s;
    const uint64_t C = (n + cw - 1) / cw;
    if (cap < ORC_HEADER_BYTES + 4 * C) return ORC_ERR_CAPACITY;
    /* header */
    uint8_t* h = out;
    memset(h, 0, ORC_HEADER_BYTES);
    h[0] = 'P'; h[1] = 'F'; h[2] = 'P'; h[3] = 'L';
    h[4] = 1; h[5] = (uint8_t)dtype; h[6] = (uint8_t)bound; h[7] = (uint8_t)P.flags;
    put_u64(h + 8, n);
    put_u64(h + 16, bits_d(eps));
    put_u64(h + 24, P.qconst);
    put_u64(h + 32, bits_d(P.range));
    put_u32(h + 40, ORC_CHUNK_BYTES);
    put_u32(h + 44, 0);
    /* chunks are independent, encoded into private buffers, then
     * concatenated in order by a serial prefix over their sizes */
    uint8_t* tmp = (uint8_t*)malloc((size_t)C * ORC_CHUNK_BYTES + 1);
    uint32_t* sizes = (uint32_t*)malloc((size_t)C * 4 + 4);
    if (!tmp || !sizes) { free(tmp); free(sizes); return ORC_ERR_ARG; }
    const char* base = (const char*)in;
#ifdef _OPENMP
    #pragma omp parallel for schedule(dynamic, 16) num_threads(nthreads > 0 ? nthreads : 1)
#endif
    for (long long c = 0; c < (long long)C; ++c) {
        uint64_t m = (uint64_t)c + 1 < C ? cw : n - (uint64_t)c * cw;
        sizes[c] = (uint32_t)orc_encode_chunk(&P, base + (uint64_t)c * cw * s, (size_t)m,
                                              tmp + (uint64_t)c * ORC_CHUNK_BYTES);
    }
    uint64_t off = ORC_HEADER_BYTES + 4 * C;
    int64_t result = 0;
    for (uint64_t c = 0; c < C; ++c) {
        put_u32(out + ORC_HEADER_BYTES + 4 * c, sizes[c]);
        if (off + sizes[c] > cap) { result = ORC_ERR_CAPACITY; break; }
        memcpy(out + off, tmp + c * ORC_CHUNK_BYTES, sizes[c]);
        off += sizes[c];
    }
    free(tmp); free(sizes);
    return result < 0 ? result : (int64_t)off;
}

int orc_decompress(const uint8_t* in, uint64_t in_bytes, void* out, uint64_t out_cap,
                   uint64_t* n_out, int nthreads) {
    if (in_bytes < ORC_HEADER_BYTES) return ORC_ERR_CORRUPT;
    if (in[0] != 'P' || in[1] != 'F' || in[2] != 'P' || in[3] != 'L' || in[4] != 1)
        return ORC_ERR_CORRUPT;
    orc_params P;
    memset(&P, 0, sizeof(P));
    P.dtype = in[5]; P.bound = in[6]; P.flags = in[7];
    if (P.dtype > ORC_F64 || P.bound > ORC_NOA || (P.flags & ~3) != 0) return ORC_ERR_CORRUPT;
    if (get_u32(in + 40) != ORC_CHUNK_BYTES || get_u32(in + 44) != 0) return ORC_ERR_CORRUPT;
    uint64_t n = get_u64(in + 8);
    P.eps = flt_d(get_u64(in + 16));
    P.range = flt_d(get_u64(in + 32));
    uint64_t qc = get_u64(in + 24);
    const uint64_t s = tsize(P.dtype);
    if (n > (1ull << 60) / s) return ORC_ERR_CORRUPT;
    if (n_out) *n_out = n;
    if (!(P.flags & ORC_FLAG_RAWWORDS)) {
        if (P.dtype == ORC_F32) {
            if (qc >> 32) return ORC_ERR_CORRUPT;
            float c = flt_f((uint32_t)qc);
            if (P.bound == ORC_REL) {
                if (!(c > 0.0f) || isinf(c)) return ORC_ERR_CORRUPT;
                P.w_f = c;
            } else {
                if (!(c >= FLT_MIN && c <= FLT_MAX / 2)) return ORC_ERR_CORRUPT;
                P.eps_eff_f = c; P.eb2_f = 2.0f * c;
            }
        } else {
            double c = flt_d(qc);
            if (P.bound == ORC_REL) {
                if (!(c > 0.0) || isinf(c)) return ORC_ERR_CORRUPT;
                P.w_d = c;
            } else {
                if (!(c >= DBL_MIN && c <= DBL_MAX / 2)) return ORC_ERR_CORRUPT;
                P.eps_eff_d = c; P.eb2_d = 2.0 * c;
            }
        }
    }
    if (out_cap < n * s) return ORC_ERR_CAPACITY;
    const uint64_t cw = ORC_CHUNK_BYTES / s;
    const uint64_t C = (n + cw - 1) / cw;
    if (in_bytes < ORC_HEADER_BYTES + 4 * C) return ORC_ERR_CORRUPT;
    /* P:160 "the decoder computes a prefix sum over the stored chunk sizes" */
    uint64_t* offs = (uint64_t*)malloc((size_t)(C + 1) * 8);
    if (!offs) return ORC_ERR_ARG;
    offs[0] = ORC_HEADER_BYTES + 4 * C;
    for (uint64_t c = 0; c < C; ++c) {
        uint64_t m = c + 1 < C ? cw : n - c * cw;
        uint32_t sz = get_u32(in + ORC_HEADER_BYTES + 4 * c);
        if (sz > m * s) { free(offs); return ORC_ERR_CORRUPT; }
        offs[c + 1] = offs[c] + sz;
    }
    if (offs[C] != in_bytes) { free(offs); return ORC_ERR_CORRUPT; }
    int bad = 0;
    char* obase = (char*)out;
#ifdef _OPENMP
    #pragma omp parallel for schedule(dynamic, 16) num_threads(nthreads > 0 ? nthreads : 1)
#endif
    for (long long c = 0; c < (long long)C; ++c) {
        uint64_t m = (uint64_t)c + 1 < C ? cw : n - (uint64_t)c * cw;
        int st = orc_decode_chunk(&P, in + offs[c], (size_t)(offs[c + 1] - offs[c]),
                                  (size_t)m, obase + (uint64_t)c * cw * s);
        if (st != ORC_OK) bad = 1;
    }
    free(offs);
    (void)nthreads;
    return bad ? ORC_ERR_CORRUPT : ORC_OK;
}
