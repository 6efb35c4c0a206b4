/*
 * pfpl.h -- C ABI of the B200-native PFPL hot path (libpfpl.so).
 *
 * PFPL = the error-bounded lossy floating-point compressor of Fallin, Azami,
 * Di, Cappello, Burtscher, "Fast and Effective Lossy Compression on GPUs and
 * CPUs with Guaranteed Error Bounds", IPDPS 2025 (/root/reference/PAPER.md;
 * "P:NNN" below = line NNN of that file).  The stream format and every reading
 * of the paper (R1..R20, A1) are specified in DESIGN.md sections 3 and 5.
 *
 * Conventions for every entry point:
 *  - Pointers named *_dev are CUDA global memory on the *current* device;
 *    pointers named *_host are host memory.  `in`/`out` of the codec calls
 *    are device pointers, must not overlap, and must be 16-byte aligned
 *    (else PFPL_ERR_ALIGN).
 *  - All work is enqueued on `stream` (cudaStream_t passed as void*; NULL =
 *    legacy default stream).  Functions that return a size through a host
 *    pointer synchronise `stream` before returning; the *_async variants never
 *    synchronise.
 *  - The caller owns all buffers.  The library owns per-(device, stream)
 *    scratch (look-back descriptors, tickets, NOA constants), allocated on
 *    first use and kept until pfpl_release_scratch().  Calls that share a
 *    stream are ordered by the stream; calls on different streams use
 *    different scratch and may run concurrently.
 *  - Errors are returned as negative pfpl_status values; nothing aborts.
 *    pfpl_strerror() maps a status to text; pfpl_last_cuda_error() returns the
 *    last cudaError_t the library observed.
 *  - Element counts are 64-bit: n up to 2^40 elements.
 */
#ifndef PFPL_H
#define PFPL_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { PFPL_F32 = 0, PFPL_F64 = 1 } pfpl_dtype;

/* error-bound types:
 *   ABS |x - x'| <= eps
 *   REL same sign and |x|/(1+eps) <= |x'| <= |x|(1+eps)
 *   NOA |x - x'| <= eps * (max - min) over finite x */
typedef enum { PFPL_ABS = 0, PFPL_REL = 1, PFPL_NOA = 2 } pfpl_bound;

typedef enum {
    PFPL_OK = 0,
    PFPL_ERR_ARG = -1,       /* bad dtype/bound/pointer/count                     */
    PFPL_ERR_BOUND = -2,     /* eps NaN, <= 0 or inf; ABS eps below the smallest
                                normal after rounding down                 */
    PFPL_ERR_CAPACITY = -3,  /* *out_bytes on entry smaller than needed           */
    PFPL_ERR_CORRUPT = -4,   /* malformed stream (header, size table, chunk data) */
    PFPL_ERR_ALIGN = -5,     /* in/out not 16-byte aligned                        */
    PFPL_ERR_CUDA = -6       /* a CUDA runtime call failed                        */
} pfpl_status;

/* stream option bits for pfpl_compress_ex (header byte 7) */
#define PFPL_OPT_MS_RESIDUALS 2u   /* A1: zigzag residuals instead of negabinary */

#define PFPL_HEADER_BYTES 48u
#define PFPL_CHUNK_BYTES 16384u    /* P:141 "16 kB chunks" (reading R19) */

/* Upper bound of a stream for n elements: header + u32 size table + n*s,
 * reached when every chunk is stored raw (P:158 caps the expansion). */
uint64_t pfpl_max_compressed_bytes(uint64_t n, int dtype);

/* Compress n elements of `dtype` at in_dev into out_dev.
 *   *out_bytes (host, in/out): capacity of out_dev on entry, stream size on
 *   return.  Synchronises `stream`.  The stream is byte-identical to the
 *   CPU oracle's (P:43 CPU/GPU compatibility). */
int pfpl_compress(const void* in_dev, uint64_t n, int dtype, int bound, double eps,
                  void* out_dev, uint64_t* out_bytes, void* stream);

/* Same, with option bits (PFPL_OPT_*). */
int pfpl_compress_ex(const void* in_dev, uint64_t n, int dtype, int bound, double eps,
                     unsigned opts, void* out_dev, uint64_t* out_bytes, void* stream);

/* Asynchronous form: never synchronises.  The stream size (u64) and a status
 * word (i32, 0 = OK or a pfpl_status) are written to result_dev[0] and
 * ((int32_t*)result_dev)[2] when the stream reaches them.  `cap` is the
 * capacity of out_dev.  Argument errors detectable on the host are returned
 * immediately.  Safe to capture in a CUDA graph. */
int pfpl_compress_async(const void* in_dev, uint64_t n, int dtype, int bound, double eps,
                        unsigned opts, void* out_dev, uint64_t cap, uint64_t* result_dev,
                        void* stream);

/* Decompress the stream in_dev[0..in_bytes) into out_dev (O8 = exact inverse,
 * P:86 "Decompression employs the inverse of these transformations").
 *   *out_bytes (host, in/out): capacity of out_dev on entry, n*s on return.
 *   Reads the 48-byte header with one device->host copy; synchronises. */
int pfpl_decompress(const void* in_dev, uint64_t in_bytes, void* out_dev,
                    uint64_t* out_bytes, void* stream);

/* Asynchronous form for callers that already hold the header on the host
 * (hdr_host = first 48 bytes of the stream).  Corruption found on the device
 * is reported in ((int32_t*)result_dev)[2]; never synchronises. */
int pfpl_decompress_async(const void* in_dev, uint64_t in_bytes, const void* hdr_host,
                          void* out_dev, uint64_t cap, uint64_t* result_dev, void* stream);

/* Parse a header (host memory, >= 48 bytes).  Any output pointer may be NULL. */
int pfpl_peek_header(const void* hdr_host, uint64_t bytes, uint64_t* n, int* dtype,
                     int* bound, double* eps, unsigned* flags);

/* ---- multi-GPU building blocks (not in the paper) ---- */

/* NOA step a1: min and max over the finite elements of in_dev,
 * written as two doubles {min, max} to mnmx_dev.  If there is no finite
 * element, min = +inf and max = -inf.  Asynchronous. */
int pfpl_minmax(const void* in_dev, uint64_t n, int dtype, double* mnmx_dev, void* stream);

/* Compress the chunk-aligned shard in_dev = elements [first_chunk*CW,
 * first_chunk*CW + n_local) of a global array of n_total elements, so that
 * the shard's size-table slice and payload are exactly the bytes the
 * single-device call would produce for those chunks (chunks are
 * independent).  n_local must be a multiple of CW = 16384/s unless the shard
 * holds the global tail.  For NOA, mnmx_dev holds the *global* {min, max}
 * (e.g. after an all-reduce); ignored otherwise.
 * Output layout in out_dev: u32 size[n_chunks] followed by the payload.  When
 * hdr_out_host != NULL the 48-byte global header is also produced there
 * (identical on every rank).  *payload_bytes (host) receives the payload size.
 * `cap` = capacity of out_dev.  Synchronises. */
int pfpl_compress_shard(const void* in_dev, uint64_t n_local, uint64_t first_chunk,
                        uint64_t n_total, int dtype, int bound, double eps, unsigned opts,
                        const double* mnmx_dev, void* out_dev, uint64_t cap,
                        uint64_t* payload_bytes, void* hdr_out_host, void* stream);

/* Decompress a run of consecutive chunks: table_host = their u32 sizes,
 * payload_dev = their concatenated payloads, hdr_host = the stream header,
 * output = elements [first_chunk*CW, ...) of the array, written to out_dev.
 * Synchronises. */
int pfpl_decompress_chunks(const void* hdr_host, const uint32_t* table_host,
                           uint64_t first_chunk, uint64_t n_chunks, const void* payload_dev,
                           uint64_t payload_bytes, void* out_dev, uint64_t cap, void* stream);

/* ---- host-resident (out-of-core) arrays ----
 * The array and the stream live in HOST memory (pinned for full PCIe rate;
 * pageable works, slower) and may exceed HBM.  They are streamed through two
 * device segment buffers of seg_chunks chunks each (0 = default 2048 chunks =
 * 32 MiB): segment k+1's H2D and segment k-1's D2H (two library-owned copy
 * streams) overlap segment k's kernel on `stream`.  Chunks are independent
 * and payload offsets are a prefix sum of the chunk sizes,
 * carried across segments on the host, so the stream is byte-identical to
 * pfpl_compress of the same array on the device.  NOA makes one extra
 * streaming pass for the global {min, max}.  The copy streams, events
 * and about 4 * seg_chunks * 16 KiB of segment buffers are library-owned,
 * cached per (device, stream) and grow-only.
 * pfpl_compress_host: *out_bytes = capacity of out_host on entry (use
 * pfpl_max_compressed_bytes), stream size on return; PFPL_ERR_CAPACITY if the
 * stream would overflow (nothing is written past the capacity).
 * pfpl_decompress_host: *out_bytes = capacity of out_host on entry, n*s on
 * return; PFPL_ERR_CORRUPT for a table whose sizes exceed in_bytes.
 * Both synchronise and return only after every copy has landed. */
int pfpl_compress_host(const void* in_host, uint64_t n, int dtype, int bound, double eps,
                       unsigned opts, void* out_host, uint64_t* out_bytes, uint64_t seg_chunks,
                       void* stream);
int pfpl_decompress_host(const void* in_host, uint64_t in_bytes, void* out_host,
                         uint64_t* out_bytes, uint64_t seg_chunks, void* stream);

/* ---- multi-field batches (e.g. CESM's 33 fields) ----
 * Compresses `count` independent device arrays (same dtype, bound and eps)
 * into `count` independent streams, each byte-identical to pfpl_compress of
 * that array.  The fields are forked over 4 library-owned non-blocking
 * streams (cached per (device, stream)) so consecutive small fields overlap
 * each other's launch ramp-up and drain, and joined back onto `stream`.
 * in[f], out[f]: device pointers, 16-B aligned; out_bytes[f] (host array):
 * capacity of out[f] on entry, stream size on return.  Synchronises once.
 * Returns the first error (argument errors before anything is enqueued;
 * PFPL_ERR_CAPACITY if any field overflowed -- its out_bytes entry is then
 * left at its capacity). */
int pfpl_compress_batch(int count, const void* const* in, const uint64_t* n, int dtype, int bound,
                        double eps, unsigned opts, void* const* out, uint64_t* out_bytes,
                        void* stream);
/* Decompresses `count` independent streams (device pointers in[f], in_bytes[f]
 * bytes each) into out[f] (device, 16-B aligned; out_bytes[f] = capacity on
 * entry, n*s on return).  The headers come back in one round trip, the fields
 * are forked over the same 4 streams; each output equals pfpl_decompress's.
 * Synchronises twice.  Returns the first error (PFPL_ERR_CORRUPT for a stream
 * shorter than its header or a corrupt table/payload). */
int pfpl_decompress_batch(int count, const void* const* in, const uint64_t* in_bytes,
                          void* const* out, uint64_t* out_bytes, void* stream);

/* ---- misc ---- */
const char* pfpl_strerror(int status);
int pfpl_last_cuda_error(void);
/* If a kernel's bounded wait expired (a protocol error; the kernel traps and
 * the call returns PFPL_ERR_CUDA), copies {site, block, thread, detail} to
 * out4 and returns 1; otherwise returns 0. */
int pfpl_watchdog_report(unsigned int* out4);
/* Frees the library's cached scratch for the current device: per-stream
 * look-back/result scratch, the host-pipeline buffers and copy streams, and
 * the batch lanes.  Synchronises the device; later calls re-create them. */
int pfpl_release_scratch(void);
/* Reconstruction-quality metrics of a decompression against the original values
 * (the paper's Fig. 16 analogue), accumulated in the
 * decoder's epilogue in f64 arithmetic (exact differences for f32 data).  Finite
 * originals only, except `violations`, which also counts non-finite originals that
 * did not come back bit-identical (REL: NaN sign cleared). */
typedef struct {
    uint64_t n;             /* values decoded */
    uint64_t n_finite;      /* finite original values */
    double max_abs_err;     /* max |x - y| */
    double max_rel_err;     /* max |x - y| / |x| over x != 0 */
    double sum_sq_err;      /* sum (x - y)^2 (summation order is unspecified) */
    double mse;             /* sum_sq_err / n_finite */
    double psnr;            /* 20 log10(value_max - value_min) - 10 log10(mse); +inf if mse == 0 */
    double value_min, value_max;   /* range of the finite originals */
    uint64_t violations;    /* values outside the stream's bound (ABS eps, REL eps*|x|,
                               NOA eps*range) -- must be 0 */
} pfpl_metrics;

/* pfpl_decompress plus verification: `orig` (device, 16-byte aligned, n values of the
 * stream's dtype, as given to pfpl_compress) is read once, alongside the decode, and
 * *m is filled on return.  Same arguments, ownership, sync and errors as
 * pfpl_decompress; PFPL_ERR_ARG if orig or m is null, PFPL_ERR_ALIGN if orig is
 * misaligned.  Costs one extra read of n values. */
int pfpl_decompress_verify(const void* in, uint64_t in_bytes, const void* orig, void* out,
                           uint64_t* out_bytes, pfpl_metrics* m, void* stream);

/* Statistics of the most recent compression enqueued on `stream` (current
 * device), counted inside the encoder at no cost on chunks without them:
 *   *unquantizable = values whose bin failed the reconstruct-and-verify check
 *                    (or all values in raw-words mode) and were stored
 *                    losslessly -- the paper's "unquantizable values";
 *   *raw_chunks    = chunks stored as raw bytes because the encoded chunk was not
 *                    smaller.
 * Synchronizes `stream`.  Zeros if nothing was compressed on it yet.  A later
 * compression on the same stream overwrites them.  Returns PFPL_OK,
 * PFPL_ERR_ARG (null output) or PFPL_ERR_CUDA. */
int pfpl_last_stats(void* stream, uint64_t* unquantizable, uint64_t* raw_chunks);
/* Number of kernel launches issued by the library since load (for bench's
 * gpu_launches claim). */
uint64_t pfpl_launch_count(void);
/* The form the next f32 compression with bound `bound` (PFPL_ABS or PFPL_NOA) will run
 * (both forms write the same bytes): 1 = the encoder that stores a chunk's first
 * residual (taken against q[-1] = 0) in single-byte extra planes instead of widening
 * warp 0's bit-plane tier, 0 = the plain encoder.  Every f32 ABS / NOA launch leaves this
 * hint for the next one of its bound from 8 samples of its input (large first bins on a
 * smooth field -> 1).  pfpl_decompress* picks its f32 decoder form from the same word of
 * the stream's bound (both decoder forms decode every stream).  Host-only read of mapped
 * memory; no sync.  Returns 0 for any other bound. */
int pfpl_f32_encoder_form(int bound);
/* Build identification string ("pfpl-b200 sm_100a ..."). */
const char* pfpl_version(void);

#ifdef __cplusplus
}
#endif
#endif
