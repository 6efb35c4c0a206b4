/*
 * pfpl_cpu.h -- C ABI of the multi-core CPU PFPL codec (libpfpl_cpu.so).
 *
 * The paper's second implementation (PFPL_OMP),
 * re-built for the host CPU of a B200 node: OpenMP threads take 16 KiB chunks
 * dynamically ("we dynamically assign the chunks to the threads"),
 * run all four stages fused on one chunk in two L1-resident 16 KiB buffers
 * (P:166-168), and place their output through a shared carry array read and
 * written atomically.  Streams are byte-identical to libpfpl.so's and
 * the CPU test reference's (P:43 CPU/GPU compatibility): same format, same
 * readings R1..R20.  x86-64-v3 (AVX2, BMI2) host code; no GPU.
 *
 * Conventions: `in`/`out` are HOST pointers (any alignment), owned by the caller.
 * nthreads <= 0 means all cores (omp_get_max_threads()).  Errors are the
 * negative pfpl_status codes of pfpl.h (same values); nothing aborts.
 */
#ifndef PFPL_CPU_H
#define PFPL_CPU_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Upper bound of a stream for n elements of dtype (0 f32, 1 f64): header + u32
 * size table + n*s (every chunk stored raw).  0 for a bad dtype. */
uint64_t pfpl_cpu_max_compressed_bytes(uint64_t n, int dtype);

/* Compress n elements (dtype 0 f32 / 1 f64) at in with bound 0 ABS / 1 REL / 2 NOA
 * and eps into out.  *out_bytes: capacity on entry, stream size on
 * return.  opts: bit 1 = zigzag residuals (reading A1, pfpl.h PFPL_OPT_MS_RESIDUALS).
 * Returns 0, -1 (argument), -2 (eps: NaN, <= 0, inf, or ABS below the smallest
 * normal after rounding down) or -3 (capacity; nothing is written past it). */
int pfpl_cpu_compress(const void* in, uint64_t n, int dtype, int bound, double eps,
                      unsigned opts, void* out, uint64_t* out_bytes, int nthreads);

/* Decompress the stream in[0..in_bytes) into out.  *out_bytes: capacity on entry,
 * n*s on return.  Returns 0, -1, -3 (capacity) or -4 (corrupt header, size table
 * or chunk data; never reads outside in[0..in_bytes)). */
int pfpl_cpu_decompress(const void* in, uint64_t in_bytes, void* out, uint64_t* out_bytes,
                        int nthreads);

/* Threads an nthreads <= 0 call uses. */
int pfpl_cpu_max_threads(void);

#ifdef __cplusplus
}
#endif
#endif
