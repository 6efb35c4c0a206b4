// pfpl_internal.h -- structures shared by the host API and the sm_100a kernels
// of libpfpl.so.  Product code only; shares nothing with the CPU test reference.
// Stream format and readings: DESIGN.md sections 3 and 5.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace pfpl {

constexpr uint32_t kChunkBytes = 16384;   // P:141 "16 kB chunks" (R19: 16384 for both dtypes)
constexpr uint32_t kHeaderBytes = 48;     // R18
constexpr uint64_t kFusedScanChunks = 8192;   // decoder: d1 inside the IO warps up to 128 MiB streams
constexpr int kEPT = 32;                  // elements per thread (one 32-bit plane word)

enum Mode : int { MODE_ABS = 0, MODE_REL = 1, MODE_RAW = 2, MODE_NOA = 3 };
enum HdrFlags : uint32_t { HF_RAWWORDS = 1, HF_MS = 2 };

// Quantizer constants.  Bit patterns of T values (f32 in the low 32 bits).
//   ABS/NOA: a = eps_eff, b = inv = 0.5/eps_eff, c = eb2 = 2*eps_eff
//   REL    : a = c_lo (largest T <= 1+eps), b = w = 2*log2p(c_lo), c = inv_w = 0.5/log2p(c_lo)
struct QConst {
    uint64_t a, b, c;
    uint64_t qconst;   // header offset 24
    double range;      // header offset 32 (NOA)
    uint32_t flags;    // header byte 7
    uint32_t pad;
    // REL encoder fast path: margin(L) = m1*|L| + m2 in bin units, bits of
    // T; 0 = always the exact path
    uint64_t m1, m2;
};

struct EncParams {
    const void* in;          // local elements (16B aligned)
    uint64_t n;              // local element count
    uint64_t C;              // local chunk count
    uint8_t* out;            // stream base
    uint64_t cap;            // capacity of out (bytes)
    uint32_t* table;         // size table (local slice)
    uint64_t payload_off;    // payload start relative to out
    unsigned long long* status;   // look-back descriptors, one per chunk [C]
    unsigned long long* ticket;   // monotone ticket counter
    uint64_t ticket_base;
    uint32_t epoch;
    int write_header;
    QConst qc;               // ABS/REL/RAW constants
    const QConst* qc_dev;    // NOA: constants derived on the device
    uint64_t* result;        // result[0] = stream bytes (payload_off + payload)
    uint64_t n_total;        // header n
    double eps;              // header eps
    uint32_t dtype, bound;   // header bytes 5, 6
    unsigned int* wd;        // watchdog report (mapped host memory) or null
    unsigned long long* stats;       // [0] unquantizable values, [1] raw chunks (this call)
    unsigned long long* stats_next;  // the other slot: zeroed for the next call
    uint64_t nz2;            // two binary32 -0.0 (0x8000000080000000), opaque to ptxas: see pk_mul
    unsigned int* x0_hint;   // f32 ABS: mapped host word, 1 = the next call should use the split form
};

struct DecParams {
    const uint8_t* in;       // payload base (first chunk's payload)
    uint64_t in_bytes;       // bytes available from `in`
    const uint32_t* table;   // size table (device)
    uint64_t n;              // elements to produce
    uint64_t C;              // chunks
    void* out;
    unsigned long long* status;
    unsigned long long* ticket;
    uint64_t ticket_base;
    uint32_t epoch;
    QConst qc;               // a/b/c as in QConst; decoder uses eb2 (ABS/NOA) or w (REL)
    int* err;                // set to PFPL_ERR_CORRUPT on malformed chunks
    uint64_t c23;            // f32 ABS: bits of 2^23 * eb2 (inf if it overflows)
    const uint64_t* offs;    // offs[c] = byte offset of chunk c's payload (size_scan_kernel), or
                             // null: the IO warp sums the size table itself (small streams)
    unsigned int* wd;        // watchdog report (mapped host memory) or null
    // verify mode (pfpl_decompress_verify): original values and the metric accumulators
    // vm[0] max |x-y| (f64 bits), [1] max |x-y|/|x| (f64 bits), [2] sum (x-y)^2 (f64),
    // [3] bound violations, [4] finite values, [5] / [6] order-mapped min / max of x
    const void* orig;
    unsigned long long* vm;
    int vbound;              // bound of the stream (header byte 6)
    double veps, vrange;     // user eps and the NOA range d (header fields)
    uint64_t nz2;            // two binary32 -0.0, opaque to ptxas (pfpl_device.cuh pk_mul)
};

// kernel launchers (pfpl_kernels.cu)
cudaError_t launch_encode(int dtype, int mode, bool ms, bool x0, const EncParams& p, int grid,
                          cudaStream_t s);
cudaError_t launch_decode(int dtype, int mode, bool ms, bool x0, const DecParams& p, int grid,
                          cudaStream_t s);   // p.orig != null selects the verify kernel
int scan_grid(uint64_t C);
cudaError_t launch_size_scan(const uint32_t* table, uint64_t C, uint64_t n, uint32_t cw,
                             uint32_t s_bytes, uint64_t in_bytes, uint64_t* offs,
                             unsigned long long* status, uint32_t epoch,
                             unsigned long long* ticket, uint64_t tbase, int* err,
                             unsigned int* wd, cudaStream_t s);
cudaError_t launch_minmax(int dtype, const void* in, uint64_t n, double* partial,
                          int blocks, cudaStream_t s);
cudaError_t launch_minmax_final(const double* partial, int blocks, double* mnmx,
                                cudaStream_t s);
cudaError_t launch_noa_derive(int dtype, const double* mnmx, double eps, uint32_t ms_flag,
                              QConst* qc_out, cudaStream_t s);
cudaError_t launch_header_only(uint8_t* out, uint64_t n, int dtype, int bound, double eps,
                               const QConst qc, const QConst* qc_dev, uint64_t* result,
                               cudaStream_t s);
// test knob: PFPL_GRID_LIMIT=k caps the persistent encoder/decoder grids at k CTAs, so
// small inputs exercise the many-chunks-per-CTA paths (arena and ring wrap-around)
// quickly, e.g. under compute-sanitizer.  Unset (the default) = full occupancy.
int grid_limit();
int encode_grid(int dtype, int mode, bool ms, uint64_t C);
int encode_tickets_per_cta(int dtype);   // tickets a persistent encoder CTA draws beyond its chunks
int decode_grid(int dtype, int mode, bool ms, uint64_t C);
int decode_tickets_per_cta();

// host-side portable log2 (same operation sequence as the device code)
float log2p_host_f32(float a);
double log2p_host_f64(double a);

// the host-side argument checks of pfpl_compress_async (pfpl_batch.cu validates every
// field with it before anything is enqueued)
int check_compress_args(const void* in, uint64_t n, int dtype, int bound, double eps,
                        unsigned opts, const void* out, uint64_t cap);
// records e as the last CUDA error (pfpl_last_cuda_error) and returns PFPL_ERR_CUDA
int record_cuda_error(int e);
// free the host-pipeline (pfpl_pipeline.cu) and batch-lane (pfpl_batch.cu) caches of device dev
void release_pipes(int dev);
void release_lanes(int dev);

}  // namespace pfpl
