/*
 * pfpl_oracle.h -- plain, slow, CPU reference ("oracle") of the PFPL codec.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * The product path (paper_conf_ipps_fallinadcb25_b200/ + include/pfpl.h)
 * never links, imports or executes it, and the two share no code, headers,
 * tables or constant generators.  Both are written from the paper:
 *   Fallin, Azami, Di, Cappello, Burtscher, "Fast and Effective Lossy
 *   Compression on GPUs and CPUs with Guaranteed Error Bounds", IPDPS 2025
 *   (/root/reference/PAPER.md; "P:NNN" = line NNN of that file)
 * and the readings R1..R20/A1 recorded in DESIGN.md section 3.
 *
 * Parity status per function (see DESIGN.md section 4 for the pins):
 *   every function below is pinned by tests/test_oracle_*.py, except the
 *   log2p/pow2p *accuracy constants*, which are pinned only by accuracy
 *   bounds (their exact bits are a format constant, not a paper value).
 */
#ifndef PFPL_ORACLE_H
#define PFPL_ORACLE_H
#include <stdint.h>
#include <stddef.h>

#ifdef __cplusplus
extern "C" {
#endif

/* enums mirror the stream header byte values */
enum { ORC_F32 = 0, ORC_F64 = 1 };
enum { ORC_ABS = 0, ORC_REL = 1, ORC_NOA = 2 };
enum { ORC_FLAG_RAWWORDS = 1, ORC_FLAG_MS = 2 };
enum { ORC_OK = 0, ORC_ERR_ARG = -1, ORC_ERR_BOUND = -2, ORC_ERR_CAPACITY = -3,
       ORC_ERR_CORRUPT = -4 };

#define ORC_CHUNK_BYTES 16384u
#define ORC_HEADER_BYTES 48u

/* ---- O0: constants (readings R1, R3, R4, R5) ---- */
typedef struct {
    int dtype, bound, flags;       /* flags: ORC_FLAG_* */
    double eps;                    /* as given by the user */
    double range;                  /* NOA: d = fl64(max-min) over finite values, else 0 */
    /* ABS/NOA (f32 uses the *_f fields, f64 the *_d fields) */
    float eps_eff_f, inv_f, eb2_f;
    double eps_eff_d, inv_d, eb2_d;
    /* REL */
    float c_lo_f, w_f, inv_w_f;
    double c_lo_d, w_d, inv_w_d;
    uint64_t qconst;               /* header field at offset 24 */
} orc_params;

/* Derive constants. For NOA, `in`/`n` are scanned for finite min/max.
 * Returns ORC_OK or ORC_ERR_BOUND / ORC_ERR_ARG. */
int orc_params_init(orc_params* P, const void* in, uint64_t n, int dtype, int bound,
                    double eps, int ms);

/* ---- A11 portable log2/pow2 (reading R5) ---- */
float  orc_log2p_f32(float a);
float  orc_pow2p_f32(float y);
double orc_log2p_f64(double a);
double orc_pow2p_f64(double y);

/* ---- O1: quantize n values into words (u32 for f32, u64 for f64) ---- */
void orc_quantize(const orc_params* P, const void* in, uint64_t n, void* words);
/* inverse of O1 (decoder side, O8 step 3) */
void orc_dequantize(const orc_params* P, const void* words, uint64_t n, void* out);

/* ---- O3: delta + negabinary or magnitude-sign (flag A1) ---- */
void orc_delta_encode(const uint64_t* q, uint64_t* r, size_t cw, int bits, int ms);
void orc_delta_decode(const uint64_t* r, uint64_t* q, size_t cw, int bits, int ms);

/* ---- O4: bit shuffle ---- */
void orc_shuffle(const uint64_t* r, size_t cw, int bits, uint8_t* S /* cw*bits/8 */);
void orc_unshuffle(const uint8_t* S, size_t cw, int bits, uint64_t* r);

/* ---- O5: zero / repeat elimination, 4 bitmap levels ---- */
/* encodes 16384 bytes; returns payload length (<= 4+32+256+2048+16384) */
size_t orc_rze_encode(const uint8_t* X1, uint8_t* out);
/* decodes; returns bytes consumed, or -1 if malformed / would exceed in_len */
long   orc_rze_decode(const uint8_t* in, size_t in_len, uint8_t* X1);

/* ---- O2..O6: one chunk. Returns stored size (raw fallback = m*s). ---- */
size_t orc_encode_chunk(const orc_params* P, const void* in, size_t m, uint8_t* out);
int    orc_decode_chunk(const orc_params* P, const uint8_t* in, size_t size, size_t m,
                        void* out);

/* ---- O7/O8: whole stream ---- */
uint64_t orc_max_compressed_bytes(uint64_t n, int dtype);
/* returns stream bytes (>0) or a negative ORC_ERR_*; nthreads<=1 = serial */
int64_t orc_compress(const void* in, uint64_t n, int dtype, int bound, double eps, int ms,
                     uint8_t* out, uint64_t cap, int nthreads);
/* returns 0 or ORC_ERR_*; *n_out receives the element count */
int orc_decompress(const uint8_t* in, uint64_t in_bytes, void* out, uint64_t out_cap,
                   uint64_t* n_out, int nthreads);

#ifdef __cplusplus
}
#endif
#endif
