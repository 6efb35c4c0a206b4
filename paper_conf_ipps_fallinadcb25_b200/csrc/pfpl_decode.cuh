// pfpl_decode.cu -- fused PFPL chunk decoder for sm_100a.
//
// The exact inverse of pfpl_encode.cu ("Decompression employs the inverse
// of these transformations in the opposite order").  Persistent,
// warp-specialised CTAs:
//
//   IO warp                                   compute warps (4 for f32, 2 for f64)
//   -------                                   ------------------------------------
//   chunk c; its offset from the prefix sum    wait for chunk k's payload; repeat
//   of the stored sizes (size_scan_     levels 4 -> 2 rebuilt top-down
//   kernel, or the IO warp's own sums);        with popcount prefix ranks --
//   validate; load the payload into a byte     every warp derives M3/M2 itself, no
//   ring with cp.async.bulk, up to 8 chunks    barrier; zero level: gather the
//   ahead                                      plane words from Z1, inverse shuffle in
//                                              registers, negabinary^-1 and
//                                              the delta decoder's inclusive scan
//                                              (the decode bottleneck P:302),
//                                              dequantize into swizzled
//                                              rows; one thread stores the chunk with
//                                              a TMA 2-D tensor store
#pragma once
#include <cuda.h>
#include <type_traits>
#include "pfpl_device.cuh"

namespace pfpl {

#ifndef PFPL_TP_UNROLL_D
#define PFPL_TP_UNROLL_D 1
#endif
#ifndef PFPL_DQ64_BF
#define PFPL_DQ64_BF 1        // f64 REL dequantize without branches (interleaved Horner chains)
#endif
constexpr int kTpUnrollD = PFPL_TP_UNROLL_D;
#ifndef PFPL_DEC_LUT
#define PFPL_DEC_LUT 1     // PRMT-selector gathers (+8% NYX, +17% rough decode)
#endif
#ifndef PFPL_DEC_WORCHK
#define PFPL_DEC_WORCHK 0
#endif
#ifndef PFPL_DEC_IO_HINT
#define PFPL_DEC_IO_HINT 0
#endif
#ifndef PFPL_DEC_IO_NS
#define PFPL_DEC_IO_NS 1024       // the IO warp runs up to 8 chunks ahead: poll rarely
#endif
#ifndef PFPL_DEC_LANE_ARRIVE
#define PFPL_DEC_LANE_ARRIVE 1    // every IO lane arrives on full[] (else lane 0 after __syncwarp)
#endif
constexpr int NQD = 8;                 // chunks in flight per CTA (payload queue depth)
#ifndef PFPL_DEC_RING
#define PFPL_DEC_RING 24576
#endif
#ifndef PFPL_DEC_MINB
#define PFPL_DEC_MINB 5
#endif
// f64: 4 CTAs per SM fit 168 registers; REL/NOA gain from a 5th CTA (128 registers,
// a few spills; Miranda REL +4%, NOA +9%), ABS loses 1.5%
#ifndef PFPL_DEC_MINB64
#define PFPL_DEC_MINB64(MODE) ((MODE) == MODE_ABS ? 4 : 5)
#endif
constexpr int RING = PFPL_DEC_RING;    // circular payload ring (bytes, multiple of 16)

struct DecEntry {
    unsigned long long c;
    uint32_t pos, size, delta, bad, rend, pad;
};

struct DecShared {
    uint8_t m1[2048];
    uint8_t act[128];                  // non-zero flag per 16-byte M1 segment
    uint8_t wcnt[4][64];
    unsigned long long wtot[4];        // per-warp totals of the delta scan
    DecEntry q[NQD];
    unsigned long long full[NQD], empty[NQD];
    uint32_t sel[16];                  // PRMT selector spreading popc(n) packed bytes to mask n
    uint32_t selr[16];                 // same, unset bits repeating the previous byte (carry = 4)
    unsigned long long vacc[8];        // verify mode: the CTA's metric accumulators (layout of p.vm)
};
constexpr int DOUT = 0;                // swizzled output staging (1024-aligned)
constexpr int DRING = 16384;
constexpr int DSH_OFF = DRING + RING + 64;
constexpr int DEC_SMEM = DSH_OFF + (int)sizeof(DecShared);
static_assert(DEC_SMEM <= 233472 / PFPL_DEC_MINB - 1024, "PFPL_DEC_MINB CTAs per SM must fit in shared memory");

__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t mbar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(dst), "l"(src), "r"(bytes), "r"(mbar) : "memory");
}
__device__ __forceinline__ void tma_store_2d(const void* tmap, int x, int y, uint32_t src) {
    asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                 ::"l"(tmap), "r"(x), "r"(y), "r"(src) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

// ---- level 1 inverse, phase A: nibbles of this thread's plane words, counts
template <typename T, int KL, int KH>
__device__ __forceinline__ void dec1_count(const uint8_t* m1, DecShared& S, int tid, int lane,
                                          int warp, uint32_t (&nb)[64], uint32_t (&ex)[16]) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW;
    constexpr int NP = KL + KH, NG = NP / 4;
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const int b = j < KL ? j : 32 + j - KL;
        const int pl = B - 1 - b;
        nb[j] = (m1[pl * (CW / 64) + (tid >> 1)] >> (4 * (tid & 1))) & 0xFu;
    }
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        uint32_t v = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) v |= (uint32_t)__popc(nb[4 * g + i]) << (8 * i);
        uint32_t inc = 0;
        if (__any_sync(PFPL_FULL, v != 0)) inc = warp_incl_scan(v, lane);
        ex[g] = inc - v;
        const int b0 = 4 * g < KL ? 4 * g : 32 + 4 * g - KL;
        if (lane == 31) *(uint32_t*)&S.wcnt[warp][b0] = inc;
    }
    if (lane == 31) {
#pragma unroll
        for (int b0 = KL; b0 < 32; b0 += 4) *(uint32_t*)&S.wcnt[warp][b0] = 0u;
#pragma unroll
        for (int b0 = 32 + KH; b0 < B; b0 += 4) *(uint32_t*)&S.wcnt[warp][b0] = 0u;
    }
}

// ---- level 1 inverse, phase B: gather the plane words from Z1, inverse transpose
template <typename T, int KL, int KH>
__device__ __forceinline__ void dec1_gather(uint32_t (&lo)[32], uint32_t (&hi)[32], const uint8_t* z1,
                                           int lane, const uint32_t (&nb)[64],
                                           const uint32_t (&ex)[16], uint32_t offl, uint32_t offh,
                                           const uint32_t* sel) {
    constexpr int NP = KL + KH;
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const int b = j < KL ? j : 32 + j - KL;
        const uint32_t o = __shfl_sync(PFPL_FULL, j < KL ? offl : offh, b & 31) +
                           __byte_perm(ex[j / 4], 0, 0x4440 + (j % 4));
        const uint32_t n = nb[j];
        uint32_t w = 0, r = o;
        if (!__any_sync(PFPL_FULL, n != 0)) {              // plane empty in this warp
            if (j < KL) lo[j] = 0; else hi[j - KL] = 0;
            continue;
        }
#if PFPL_DEC_LUT
        // the lane's popc(n) bytes are contiguous at z1 + o: one unaligned 4-byte read
        // (two aligned words; the ring keeps >= 16 bytes of slack after a payload) and
        // one PRMT that spreads them to the byte positions set in n (selector from sel[])
        {
            const uint8_t* pz = z1 + o;
            const uint32_t mis = smem_u32(pz) & 3u;
            const uint32_t* wp = (const uint32_t*)(pz - mis);
            w = __byte_perm(__funnelshift_r(wp[0], wp[1], 8u * mis), 0u, sel[n]);
        }
        (void)r;
#else
        if (n & 1u) w |= (uint32_t)z1[r++];
        if (n & 2u) w |= (uint32_t)z1[r++] << 8;
        if (n & 4u) w |= (uint32_t)z1[r++] << 16;
        if (n & 8u) w |= (uint32_t)z1[r] << 24;
#endif
        if (j < KL) lo[j] = w; else hi[j - KL] = w;
    }
    if constexpr (KL > 0) transpose_inv<KL>(lo);
    else {
#pragma unroll
        for (int i = 0; i < 32; ++i) lo[i] = 0;
    }
    if constexpr (KH > 0) transpose_inv<KH>(hi);
    else {
#pragma unroll
        for (int i = 0; i < 32; ++i) hi[i] = 0;
    }
}

#define PFPL_DEC_TIER(FN, ...)                                                          \
    do {                                                                                \
        if (P == 0) FN<T, 0, 0>(__VA_ARGS__);                                           \
        else if (B == 32 || P <= 32) {                                                  \
            if (P <= 4) FN<T, 4, 0>(__VA_ARGS__);                                       \
            else if (P <= 8) FN<T, 8, 0>(__VA_ARGS__);                                  \
            else if (P <= 16) FN<T, 16, 0>(__VA_ARGS__);                                \
            else FN<T, 32, 0>(__VA_ARGS__);                                             \
        } else {                                                                        \
            if (P <= 36) FN<T, 32, 4>(__VA_ARGS__);                                     \
            else if (P <= 40) FN<T, 32, 8>(__VA_ARGS__);                                \
            else if (P <= 48) FN<T, 32, 16>(__VA_ARGS__);                               \
            else FN<T, 32, 32>(__VA_ARGS__);                                            \
        }                                                                               \
    } while (0)

__device__ __forceinline__ void set_err(int* err) { atomicExch(err, -4); }

// order-preserving map of a double to u64 (for atomicMin / atomicMax)
__device__ __forceinline__ unsigned long long ord_u64(double v) {
    const uint64_t u = d2u(v);
    return (u >> 63) ? ~u : (u | 0x8000000000000000ull);
}

// Verify mode: reconstruction-quality metrics of the decoded values y
// against the originals x, accumulated in the decode epilogue (Fig. 16), and a
// count of values outside the stream's bound -- in f64 arithmetic, exact for f32
// data.  Non-finite x must come back bit-identical (REL: NaN sign cleared).
template <typename T>
struct VerAcc {
    double mabs = 0.0, mrel = 0.0, ssq = 0.0, vmin = INFINITY, vmax = -INFINITY;
    unsigned long long nviol = 0, nfin = 0;
    __device__ __forceinline__ void add(T x, T y, const DecParams& p) {
        const double xd = (double)x, yd = (double)y;
        if (isfinite(xd)) {
            const double d = fabs(xd - yd);
            mabs = fmax(mabs, d);
            ssq += d * d;
            // divide only for candidates: q > mrel implies d > mrel*|x|*(1 - 2^-40), so the
            // filter never drops a new maximum (the quotient itself is exact IEEE)
            const double ax = fabs(xd);
            if (ax != 0.0 && d > mrel * ax * 0.9999999999990905) mrel = fmax(mrel, d / ax);
            vmin = fmin(vmin, xd);
            vmax = fmax(vmax, xd);
            nfin += 1;
            const double lim = p.vbound == 1 ? p.veps * fabs(xd) : p.vbound == 2 ? p.veps * p.vrange : p.veps;
            if (!(d <= lim)) nviol += 1;
        } else if (!((isnan(xd) && isnan(yd)) || xd == yd)) {
            nviol += 1;
        }
    }
    // per chunk: warp-reduce into the CTA's shared accumulators and restart, so nothing
    // stays live across the chunk loop (the kernel is register-bound)
    __device__ __forceinline__ void flush_chunk(unsigned long long* sv) {
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) {
            mabs = fmax(mabs, __shfl_xor_sync(PFPL_FULL, mabs, d));
            mrel = fmax(mrel, __shfl_xor_sync(PFPL_FULL, mrel, d));
            ssq += __shfl_xor_sync(PFPL_FULL, ssq, d);
            vmin = fmin(vmin, __shfl_xor_sync(PFPL_FULL, vmin, d));
            vmax = fmax(vmax, __shfl_xor_sync(PFPL_FULL, vmax, d));
            nviol += __shfl_xor_sync(PFPL_FULL, nviol, d);
            nfin += __shfl_xor_sync(PFPL_FULL, nfin, d);
        }
        if ((threadIdx.x & 31) == 0 && nfin + nviol) {
            atomicMax(&sv[0], (unsigned long long)d2u(mabs));
            atomicMax(&sv[1], (unsigned long long)d2u(mrel));
            atomicAdd((double*)&sv[2], ssq);
            atomicAdd(&sv[3], nviol);
            atomicAdd(&sv[4], nfin);
            if (nfin) {
                atomicMin(&sv[5], ord_u64(vmin));
                atomicMax(&sv[6], ord_u64(vmax));
            }
        }
        mabs = mrel = ssq = 0.0;
        vmin = INFINITY;
        vmax = -INFINITY;
        nviol = nfin = 0;
    }
    // once per CTA: shared accumulators -> global
    static __device__ __forceinline__ void flush_cta(const unsigned long long* sv, const DecParams& p) {
        if (sv[4] + sv[3] == 0) return;
        atomicMax(&p.vm[0], sv[0]);
        atomicMax(&p.vm[1], sv[1]);
        atomicAdd((double*)&p.vm[2], u2d(sv[2]));
        if (sv[3]) atomicAdd(&p.vm[3], sv[3]);
        atomicAdd(&p.vm[4], sv[4]);
        if (sv[4]) {
            atomicMin(&p.vm[5], sv[5]);
            atomicMax(&p.vm[6], sv[6]);
        }
    }
    __device__ __forceinline__ void flush(const DecParams& p) {
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) {
            mabs = fmax(mabs, __shfl_xor_sync(PFPL_FULL, mabs, d));
            mrel = fmax(mrel, __shfl_xor_sync(PFPL_FULL, mrel, d));
            ssq += __shfl_xor_sync(PFPL_FULL, ssq, d);
            vmin = fmin(vmin, __shfl_xor_sync(PFPL_FULL, vmin, d));
            vmax = fmax(vmax, __shfl_xor_sync(PFPL_FULL, vmax, d));
            nviol += __shfl_xor_sync(PFPL_FULL, nviol, d);
            nfin += __shfl_xor_sync(PFPL_FULL, nfin, d);
        }
        if ((threadIdx.x & 31) == 0) {
            atomicMax(&p.vm[0], (unsigned long long)d2u(mabs));      // non-negative: bits order
            atomicMax(&p.vm[1], (unsigned long long)d2u(mrel));
            atomicAdd((double*)&p.vm[2], ssq);
            if (nviol) atomicAdd(&p.vm[3], nviol);
            atomicAdd(&p.vm[4], nfin);
            if (nfin) {
                atomicMin(&p.vm[5], ord_u64(vmin));
                atomicMax(&p.vm[6], ord_u64(vmax));
            }
        }
    }
};
template <typename T>
struct VerNone {
    __device__ __forceinline__ void add(T, T, const DecParams&) {}
    __device__ __forceinline__ void flush_chunk(unsigned long long*) {}
    static __device__ __forceinline__ void flush_cta(const unsigned long long*, const DecParams&) {}
};

// X0: the decoder form for streams whose chunks start with a large first residual (the
// encoder's X0 form writes them, and so does any encoder on such fields): a warp's top planes
// in which only its first byte is non-zero are folded into thread 0 of the warp after the
// inverse transpose instead of widening its tier.  Both forms decode every stream.
template <typename T, int MODE, bool MSR, bool VER = false, bool X0 = false>
__global__ void __launch_bounds__(Tr<T>::NT + 32, sizeof(T) == 4 ? PFPL_DEC_MINB : PFPL_DEC_MINB64(MODE))
decode_kernel(const DecParams p, const __grid_constant__ CUtensorMap tmap) {
    typedef typename Tr<T>::W W;
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NTC = Tr<T>::NT, NWC = Tr<T>::NW, S_ = Tr<T>::S;
    constexpr int NB2 = 2048 / NTC;          // M1 bytes per compute thread (16 or 32)

    extern __shared__ __align__(1024) uint8_t smem[];
    DecShared& S = *reinterpret_cast<DecShared*>(smem + DSH_OFF);
    uint8_t* const stage_out = smem + DOUT;
    uint8_t* const ring = smem + DRING;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t C = p.C;

    if (tid == 0) {
        g_pfpl_wd = p.wd;
        if (smem_u32(smem) & 1023u) __trap();
        for (int k = 0; k < NQD; ++k) {
            mbar_init(smem_u32(&S.full[k]), PFPL_DEC_LANE_ARRIVE ? 32 : 1);   // IO lanes (+ the bulk bytes)
            mbar_init(smem_u32(&S.empty[k]), 1);
        }
        fence_barrier_init();
    }
    if (tid < 16) {
        // selector nibble j: rank of byte j among the set bits of n, or 4 (a zero byte)
        uint32_t v = 0, k = 0;
        for (int j = 0; j < 4; ++j) v |= (((uint32_t)tid >> j) & 1u ? k++ : 4u) << (4 * j);
        S.sel[tid] = v;
        // repeat form: byte j = the last new byte at or before j, else the carry (byte 4)
        uint32_t vr = 0, last = 4u;
        k = 0;
        for (int j = 0; j < 4; ++j) {
            if (((uint32_t)tid >> j) & 1u) last = k++;
            vr |= last << (4 * j);
        }
        S.selr[tid] = vr;
        if (tid < 8)   // zeros; min = order(+inf), max = order(-inf)
            S.vacc[tid] = tid == 5 ? 0xFFF0000000000000ull : tid == 6 ? ~0xFFF0000000000000ull : 0ull;
    }
    if (tid == 0) {
        prefetch_tmap(&tmap);
    }
    __syncthreads();

    if (warp == NWC) {
        // =========================== IO warp ===========================
        // static round-robin assignment (chunk c = blockIdx.x + k * gridDim.x), so no
        // ticket atomics sit on the IO warp's critical path.
        // d1 (the prefix sum over the stored sizes), fused: the IO warp keeps the
        // inclusive prefix of its own previous chunk c - G and adds the G - 1 table
        // entries in between (first chunk: the entries before it) -- independent
        // coalesced loads of the L2-resident table, no cross-CTA dependency and no
        // separate scan launch.  The last chunk checks the total against the payload.
        uint32_t head = 0, rel = 0;     // ring: next free byte / released up to (monotone)
        const uint64_t G = gridDim.x;
        uint64_t c = blockIdx.x;
        // Large streams (p.offs set) take the offsets from size_scan_kernel instead, loaded
        // one chunk ahead: there the window sums would sit on the IO warp's critical
        // path every chunk, while the scan launch is small against the decode.
        const bool fused = p.offs == nullptr;
        uint64_t incl_prev = 0, from = 0;   // excl(c) = incl_prev + sum(table[from .. c))
        uint32_t size_n = 0;
        uint64_t excl_n = 0;
        if (c < C) { size_n = p.table[c]; if (!fused) excl_n = p.offs[c]; }
        for (uint32_t k = 0;; ++k, c += G) {
            const int slot = k % NQD;
            if (c >= C) {
                mbar_wait_sleep(smem_u32(&S.empty[slot]), ((k / NQD) & 1u) ^ 1u, 0x21);
                if (lane == 0) S.q[slot].c = c;
                __syncwarp();
                if (PFPL_DEC_LANE_ARRIVE || lane == 0) mbar_arrive(smem_u32(&S.full[slot]));
                break;
            }
            const uint32_t size = size_n;
            uint64_t excl = excl_n;
            if (c + G < C) { size_n = p.table[c + G]; if (!fused) excl_n = p.offs[c + G]; }
            if (fused) {
                // up to 24 x 32 entries (a 740-CTA grid) in one round of independent loads
                uint64_t part = 0;
                for (uint64_t i0 = from + lane; i0 < c; i0 += 32 * 24) {
#pragma unroll
                    for (int j = 0; j < 24; ++j)
                        if (i0 + 32 * j < c) part += p.table[i0 + 32 * j];
                }
                excl = incl_prev + warp_sum64(part);
                incl_prev = excl + size;
                from = c + 1;
            }
            const uint32_t m = (uint32_t)min((uint64_t)CW, (uint64_t)(p.n - c * (uint64_t)CW));
            const uint32_t rawb = m * S_;
            uint32_t bad = 0;
            if (size > rawb || excl + size > p.in_bytes || (size < 4 && size != rawb)) bad = 1;
            if (c == C - 1 && excl + size != p.in_bytes) bad = 1;    // sizes must add up to the payload
            // reserve a ring slice for the 16-byte aligned superset of the payload
            const uint8_t* g = p.in + excl;
            const uint32_t delta = (uint32_t)((uintptr_t)g & 15u);
            const uint32_t R = bad ? 16u : ((delta + size + 15u) & ~15u) + 16u;
            const uint32_t head0 = head;
            if (head % RING + R > (uint32_t)RING) head += RING - head % RING;   // never wrap a slice
            // Ring release protocol (as the encoder's arena): the compute warps arrive on
            // empty[j % NQD] once chunk j's payload is consumed; the IO warp waits on the
            // phase of every chunk whose ring bytes it reuses, so each reuse is ordered by
            // an mbarrier.  First the queue slot (chunk k - NQD), whose ring end `rel`
            // the IO warp recorded itself; then, if the slice still does not fit (live
            // bytes [rel, head0) plus the slice span more than RING, and the ring is not
            // empty), the chunks after it, oldest first.  The IO warp runs up to NQD
            // chunks ahead: waiting is the common case, so it sleeps between polls.
#if PFPL_DEC_IO_HINT
            mbar_wait_wd(smem_u32(&S.empty[slot]), ((k / NQD) & 1u) ^ 1u, 0x21);
#else
            mbar_wait_sleep(smem_u32(&S.empty[slot]), ((k / NQD) & 1u) ^ 1u, 0x21, PFPL_DEC_IO_NS);
#endif
            if (k >= (uint32_t)NQD) rel = __shfl_sync(PFPL_FULL, S.q[slot].rend, 0);
            auto fits = [&](uint32_t r) { return r == head0 || head + R - r <= (uint32_t)RING; };
            if (!fits(rel)) {
                for (uint32_t j = k >= (uint32_t)NQD ? k - NQD + 1 : 0; j < k; ++j) {
                    mbar_wait_sleep(smem_u32(&S.empty[j % NQD]), (j / NQD) & 1u, 0x23, 64);
                    rel = __shfl_sync(PFPL_FULL, S.q[j % NQD].rend, 0);
                    if (fits(rel)) break;
                }
            }
            const uint32_t pos = head % RING;
            head += R;
            // bulk copy of the aligned superset, never past the last 16-byte
            // boundary of the stream; the remainder by the lanes
            const uint8_t* a0 = g - delta;
            const uint8_t* want = g + size;
            const uint8_t* a1 = (const uint8_t*)(((uintptr_t)want + 15u) & ~(uintptr_t)15u);
            const uint8_t* lim = (const uint8_t*)((uintptr_t)(p.in + p.in_bytes) & ~(uintptr_t)15u);
            if (a1 > lim) a1 = lim;
            if (a1 < a0) a1 = a0;
            const uint32_t bulk = bad ? 0u : (uint32_t)(a1 - a0);
            uint8_t* stg = ring + pos;
            if (!bad)
                for (const uint8_t* q = a1 + lane; q < want; q += 32) stg[q - a0] = *q;
            __syncwarp();
            if (lane == 0) {
                DecEntry& e = S.q[slot];
                e.c = c;
                e.pos = pos;
                e.size = size;
                e.delta = delta;
                e.bad = bad;
                e.rend = head;
                if (bulk) {
                    mbar_arrive_tx(smem_u32(&S.full[slot]), bulk);
                    bulk_g2s(smem_u32(stg), a0, bulk, smem_u32(&S.full[slot]));
                }
            }
            __syncwarp();
            if (PFPL_DEC_LANE_ARRIVE ? (lane != 0 || !bulk) : (lane == 0 && !bulk))
                mbar_arrive(smem_u32(&S.full[slot]));
        }
        return;
    }

    // ============================ compute warps ============================
    QF<T> q;
    q.load(p.qc);
    const bool raw = (p.qc.flags & HF_RAWWORDS) != 0;
    const float c23 = u2f((uint32_t)p.c23);
    const bool fastdq = sizeof(T) == 4 && MODE == MODE_ABS && !isinf(c23);
    typename std::conditional<VER, VerAcc<T>, VerNone<T>>::type vacc;
    const T* const orig = (const T*)p.orig;
    for (uint32_t it = 0;; ++it) {
        const int slot = it % NQD;
        mbar_wait_wd(smem_u32(&S.full[slot]), (it / NQD) & 1u, 0x22);
        const DecEntry md = S.q[slot];
        const uint64_t c = md.c;
        if (c >= C) break;
        const uint32_t m = (uint32_t)min((uint64_t)CW, (uint64_t)(p.n - c * (uint64_t)CW));
        const uint8_t* pay = ring + md.pos + md.delta;
        uint8_t* const dstc = (uint8_t*)p.out + c * (uint64_t)kChunkBytes;
        auto release = [&]() {          // after a CTA barrier: every read of the payload is done
            if (tid == 0) mbar_arrive(smem_u32(&S.empty[slot]));
        };
        if (md.bad) {
            named_sync(1, NTC);
            if (tid == 0) set_err(p.err);
            release();
            continue;
        }
        if (md.size == m * S_) {
            // raw chunk: the stored bytes are the original values
            const uint32_t nw = md.size / 4;
            for (uint32_t j = tid; j < nw; j += NTC) {
                const uint32_t a = smem_u32(pay + 4 * j) & 3u;
                const uint32_t* sw = (const uint32_t*)(pay + 4 * j - a);
                ((uint32_t*)dstc)[j] = __funnelshift_r(sw[0], sw[1], 8u * a);
            }
            named_sync(1, NTC);
            release();
            if constexpr (VER) {       // the chunk's words were written by the whole CTA
                for (uint32_t e = tid; e < m; e += NTC)
                    vacc.add(orig[c * (uint64_t)CW + e], ((const T*)dstc)[e], p);
                vacc.flush_chunk(S.vacc);
            }
            continue;
        }
        // ---- levels 4 -> 3 -> 2, derived by every warp (no barrier) ----
        // Corrupt-stream safety: every level's section must fit in
        // the stored size BEFORE it is read, so a bad bitmap can never steer a read past
        // the payload's ring slice.  A level that does not fit is treated as empty (no
        // reads) and the chunk is reported as corrupt; the checks are CTA-uniform (every
        // warp derives the same counts from the same bytes).
        uint32_t M4 = (uint32_t)pay[0] | ((uint32_t)pay[1] << 8) | ((uint32_t)pay[2] << 16) |
                      ((uint32_t)pay[3] << 24);
        bool fits = 4u + (uint32_t)__popc(M4) <= md.size;
        if (!fits) M4 = 0u;
        const uint32_t n4 = __popc(M4);
        const uint8_t* z4 = pay + 4;
        const uint32_t c4 = __popc(M4 & (lane == 31 ? 0xFFFFFFFFu : ((2u << lane) - 1u)));
        uint32_t m3 = c4 ? z4[c4 - 1] : 0u;                     // M3 byte `lane`
        uint32_t cnt3 = __popc(m3);
        uint32_t inc3 = warp_incl_scan(cnt3, lane);
        if (4u + n4 + __shfl_sync(PFPL_FULL, inc3, 31) > md.size) {
            fits = false;
            m3 = cnt3 = inc3 = 0u;
        }
        const uint32_t n3 = __shfl_sync(PFPL_FULL, inc3, 31);
        const uint8_t* z3 = z4 + n4;
        uint32_t m2lo = 0, m2hi = 0;                            // M2 bytes 8*lane .. 8*lane+7
#if PFPL_DEC_LUT
        {
            // two 4-byte groups, each one unaligned read + one repeat-selector PRMT
            const uint32_t e3 = inc3 - cnt3;
            uint32_t carry = e3 ? (uint32_t)z3[e3 - 1] : 0u;
            uint32_t r0 = e3;
#pragma unroll
            for (int g = 0; g < 2; ++g) {
                const uint32_t nib = (m3 >> (4 * g)) & 0xFu;
                const uint8_t* pz = z3 + r0;
                const uint32_t mis = smem_u32(pz) & 3u;
                const uint32_t* wp = (const uint32_t*)(pz - mis);
                const uint32_t w = __byte_perm(__funnelshift_r(wp[0], wp[1], 8u * mis), carry, S.selr[nib]);
                if (g == 0) m2lo = w; else m2hi = w;
                carry = w >> 24;
                r0 += __popc(nib);
            }
        }
#else
#pragma unroll
        for (int j = 0; j < 8; ++j) {
            const uint32_t cj = inc3 - cnt3 + __popc(m3 & ((2u << j) - 1u));
            const uint32_t bv = cj ? z3[cj - 1] : 0u;
            if (j < 4) m2lo |= bv << (8 * j); else m2hi |= bv << (8 * (j - 4));
        }
#endif
        uint32_t pc2 = __popc(m2lo) + __popc(m2hi);
        uint32_t inc2 = warp_incl_scan(pc2, lane);
        if (4u + n4 + n3 + __shfl_sync(PFPL_FULL, inc2, 31) > md.size) {
            fits = false;
            m2lo = m2hi = pc2 = inc2 = 0u;
        }
        const uint32_t n2 = __shfl_sync(PFPL_FULL, inc2, 31);
        const uint8_t* z2 = z3 + n3;
        // ---- level 2 -> M1: thread t owns M1 bytes [NB2*t, NB2*t + NB2) ----
        {
            uint32_t bits, base;
            if (NB2 == 16) {
                const int L = tid >> 2;                          // lane holding M2 bytes 2t, 2t+1
                const uint32_t wlo = __shfl_sync(PFPL_FULL, m2lo, L & 31);
                const uint32_t whi = __shfl_sync(PFPL_FULL, m2hi, L & 31);
                const uint32_t e2 = __shfl_sync(PFPL_FULL, inc2 - pc2, L & 31);
                const int f = tid & 3;                           // 16-bit field within the lane
                const uint32_t wsel = f < 2 ? wlo : whi;
                bits = (wsel >> (16 * (f & 1))) & 0xFFFFu;
                const uint32_t below = (f >= 2 ? __popc(wlo) : 0u) +
                                       __popc(wsel & ((f & 1) ? 0xFFFFu : 0u));
                base = e2 + below;
            } else {
                const int L = tid >> 1;                          // lane holding M2 bytes 4t..4t+3
                const uint32_t wlo = __shfl_sync(PFPL_FULL, m2lo, L & 31);
                const uint32_t whi = __shfl_sync(PFPL_FULL, m2hi, L & 31);
                const uint32_t e2 = __shfl_sync(PFPL_FULL, inc2 - pc2, L & 31);
                bits = (tid & 1) ? whi : wlo;
                base = e2 + ((tid & 1) ? __popc(wlo) : 0u);
            }
            uint32_t wv[NB2 / 4];
            if (bits == 0) {
                const uint32_t b = base ? z2[base - 1] : 0u;
#pragma unroll
                for (int i = 0; i < NB2 / 4; ++i) wv[i] = b * 0x01010101u;
            } else {
#if PFPL_DEC_LUT
                // 4 M1 bytes at a time: the new (non-repeated) bytes of the group are
                // contiguous in Z2; one unaligned read and one PRMT whose selector (selr[])
                // takes byte j from the group's k-th new byte, or repeats the byte before
                // the group (the carry, operand byte 4) -- repeat elimination's inverse
                uint32_t carry = base ? (uint32_t)z2[base - 1] : 0u;
                uint32_t r0 = base;
#pragma unroll
                for (int i = 0; i < NB2 / 4; ++i) {
                    const uint32_t nib = (bits >> (4 * i)) & 0xFu;
                    const uint8_t* pz = z2 + r0;
                    const uint32_t mis = smem_u32(pz) & 3u;
                    const uint32_t* wp = (const uint32_t*)(pz - mis);
                    const uint32_t w = __byte_perm(__funnelshift_r(wp[0], wp[1], 8u * mis), carry, S.selr[nib]);
                    wv[i] = w;
                    carry = w >> 24;
                    r0 += __popc(nib);
                }
#else
#pragma unroll
                for (int i = 0; i < NB2 / 4; ++i) {
                    uint32_t w = 0;
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        const int bit = 4 * i + k;
                        const uint32_t cj = base + __popc(bits & (bit == 31 ? 0xFFFFFFFFu : ((2u << bit) - 1u)));
                        w |= (cj ? (uint32_t)z2[cj - 1] : 0u) << (8 * k);
                    }
                    wv[i] = w;
                }
#endif
            }
#pragma unroll
            for (int i = 0; i < NB2 / 4; i += 4)
                *(uint4*)(S.m1 + NB2 * tid + 4 * i) = make_uint4(wv[i], wv[i + 1], wv[i + 2], wv[i + 3]);
            // 16-byte M1 segment g = (plane g / NWC, warp g % NWC) is non-zero?
#pragma unroll
            for (int sg = 0; sg < NB2 / 16; ++sg)
                S.act[(NB2 / 16) * tid + sg] = (wv[4 * sg] | wv[4 * sg + 1] | wv[4 * sg + 2] | wv[4 * sg + 3]) != 0;
        }
        named_sync(1, NTC);    // M1 and segment flags complete

        // ---- level 1: active planes of this warp, counts, offsets, gather ----
        int P;
        uint64_t all;
        {
            const uint32_t a0 = S.act[lane * NWC + warp];                 // plane p = lane
            const uint32_t a1 = B == 64 ? S.act[(lane + 32) * NWC + warp] : 0u;
            const uint32_t ml = __ballot_sync(PFPL_FULL, a0 != 0);        // bit p: plane p
            const uint32_t mh = __ballot_sync(PFPL_FULL, a1 != 0);        // bit p: plane 32+p
            // bit b of `all` = bit b of the residuals active (plane B-1-b)
            all = B == 32 ? (uint64_t)__brev(ml)
                                         : (((uint64_t)__brev(ml) << 32) | __brev(mh));
            P = all ? 64 - __clzll((long long)all) : 0;
        }
        // X0 (f32 ABS): planes above the rest of this warp's planes in which only byte 0 of
        // the warp's segment is non-zero (M1 segment = 01 00 .. 00): their byte carries bits of
        // the warp's first 8 elements only, so they are counted here and OR-ed into thread 0's
        // values after the inverse transpose, and the tier covers the other planes
        constexpr bool kX0 = X0 && sizeof(T) == 4 && MODE == MODE_ABS;
        uint32_t xh = 0;
        if constexpr (kX0) {
            const uint4 sg = *(const uint4*)(S.m1 + (B - 1 - lane) * (CW / 64) + 16 * warp);   // bit `lane`
            const uint32_t cb = __ballot_sync(PFPL_FULL, sg.x == 1u && (sg.y | sg.z | sg.w) == 0u);
            const uint32_t allw = (uint32_t)all;            // bit b: plane of residual bit b active
            const uint32_t rest = allw & ~cb;
            const int P0 = rest ? 32 - __clz(rest) : 0;
            // the tier's planes (PFPL_DEC_TIER's widths) stay in the gather; only candidates
            // above it are folded (each plane is counted and read exactly once)
            const int K = P0 == 0 ? 0 : P0 <= 4 ? 4 : P0 <= 8 ? 8 : P0 <= 16 ? 16 : 32;
            xh = allw & ~(K >= 32 ? 0xFFFFFFFFu : (1u << K) - 1u);     // all candidates (rest < 2^P0)
            P = P0;
        }
        uint32_t nb[64], ex[16];
        PFPL_DEC_TIER(dec1_count, S.m1, S, tid, lane, warp, nb, ex);
        if (kX0 && xh && lane == 31) {
            // one byte per folded plane in this warp's counts (after the row's own stores)
#pragma unroll
            for (int b0 = 0; b0 < 32; b0 += 4) {
                const uint32_t nb4 = (xh >> b0) & 0xFu;
                if (nb4) *(uint32_t*)&S.wcnt[warp][b0] += (nb4 * 0x00204081u) & 0x01010101u;
            }
        }
        named_sync(1, NTC);    // counts visible
        uint32_t offl, offh, n1;
        {
            uint32_t myl = 0, myh = 0, tl = 0, th = 0;
#pragma unroll
            for (int w = 0; w < NWC; ++w) {
                const uint32_t a = S.wcnt[w][lane];
                const uint32_t b = B == 64 ? S.wcnt[w][32 + lane] : 0u;
                if (w < warp) { myl += a; myh += b; }
                tl += a;
                th += b;
            }
            uint32_t sl = tl, sh = th;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t a = __shfl_down_sync(PFPL_FULL, sl, d);
                const uint32_t b = B == 64 ? __shfl_down_sync(PFPL_FULL, sh, d) : 0u;
                if (lane + d < 32) { sl += a; sh += b; }
            }
            const uint32_t tot_h = B == 64 ? __shfl_sync(PFPL_FULL, sh, 0) : 0u;
            const uint32_t tot_l = __shfl_sync(PFPL_FULL, sl, 0);
            offl = tot_h + sl - tl + myl;
            offh = sh - th + myh;
            n1 = tot_l + tot_h;
        }
        const uint8_t* z1 = z2 + n2;
        const bool consistent = fits && 4 + n4 + n3 + n2 + n1 == md.size;
        if (!consistent) P = 0;           // no Z1 reads: the gather offsets are not trusted
        uint32_t lo[32], hi[32];
        PFPL_DEC_TIER(dec1_gather, lo, hi, z1, lane, nb, ex, offl, offh, S.sel);
        if (kX0 && xh && consistent) {
#pragma unroll 1
            for (uint32_t mm = xh; mm; mm &= mm - 1u) {
                const int b = __ffs(mm) - 1;
                const uint32_t o = __shfl_sync(PFPL_FULL, offl, b);   // this warp's segment start
                if (lane == 0) {
                    const uint32_t v = z1[o];
#pragma unroll
                    for (int e = 0; e < 8; ++e) lo[e] |= ((v >> e) & 1u) << b;
                }
            }
        }

        // ---- residual decode + delta decoder's inclusive scan ----
        W dq[32];
        W tsum = 0;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
            const W r = sizeof(W) == 8 ? (W)(((uint64_t)hi[i] << 32) | lo[i]) : (W)lo[i];
            tsum += rdecode<MSR>(r);
            dq[i] = tsum;
        }
        W incw = tsum;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const W t = __shfl_up_sync(PFPL_FULL, incw, d);
            if (lane >= d) incw += t;
        }
        if (lane == 31) S.wtot[warp] = (unsigned long long)incw;
        if (tid == 0) bulk_wait_read0();     // previous chunk's TMA store has read the staging
        named_sync(1, NTC);    // payload consumed; warp totals visible
        release();
        if (!__all_sync(PFPL_FULL, consistent) && lane == 0) set_err(p.err);
        W carry = incw - tsum;
#pragma unroll
        for (int w = 0; w < NWC; ++w)
            if (w < warp) carry += (W)S.wtot[w];

        // ---- dequantize into swizzled rows ----
        if (m == CW) {
            auto emit = [&](auto dqf) {
#pragma unroll
                for (int i = 0; i < 2 * S_; ++i) {
                    T x[16 / S_];
#pragma unroll
                    for (int k = 0; k < 16 / S_; ++k) x[k] = dqf((W)(carry + dq[i * (16 / S_) + k]));
                    uint4 v;
                    memcpy(&v, x, 16);
                    const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                    *(uint4*)(stage_out + r * 128 + (((i & 7) ^ (r & 7)) << 4)) = v;
                }
            };
            bool done = false;
            if constexpr (sizeof(T) == 4 && MODE == MODE_ABS) {
                if (fastdq) {
                    // all words of this thread are bins (the common case): no raw-word select
                    W wor = PFPL_DEC_WORCHK ? 0u : 0x00800000u;
#if PFPL_DEC_WORCHK
#pragma unroll
                    for (int i = 0; i < 32; ++i) wor |= (W)(carry + dq[i]);
#endif
                    if (wor < 0x00800000u)
                        emit([&](W w) { return (T)q.abs_dq_bins((uint32_t)w, c23); });
                    else
                        emit([&](W w) { return (T)q.abs_dq_fast((uint32_t)w, c23); });
                    done = true;
                }
            }
            if constexpr (MODE == MODE_REL || sizeof(T) == 8) {
                // long dequantizers (REL's pow2p, f64): stage the words, then dequantize
                // them in place in a rolled loop (unrolled over 32 values the code
                // overflows the instruction cache; see the encoder's TWO_PASS)
                emit([&](W w) { T y; memcpy(&y, &w, sizeof(T)); return y; });
#pragma unroll kTpUnrollD
                for (int i = 0; i < 2 * S_; ++i) {
                    const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                    uint4* const a = (uint4*)(stage_out + r * 128 + (((i & 7) ^ (r & 7)) << 4));
                    uint4 v = *a;
                    W w[16 / S_];
                    T y[16 / S_];
                    memcpy(w, &v, 16);
                    if constexpr (sizeof(T) == 4 && MODE == MODE_REL) {
                        const uint64_t y01 = q.rel_dq2((uint32_t)w[0], (uint32_t)w[1], p.nz2);
                        const uint64_t y23 = q.rel_dq2((uint32_t)w[2], (uint32_t)w[3], p.nz2);
                        v = make_uint4((uint32_t)y01, (uint32_t)(y01 >> 32), (uint32_t)y23, (uint32_t)(y23 >> 32));
                        (void)y;
                    } else if constexpr (sizeof(T) == 8 && MODE == MODE_REL && PFPL_DQ64_BF) {
                        y[0] = q.rel_dq_bf((uint64_t)w[0]);
                        y[1] = q.rel_dq_bf((uint64_t)w[1]);
                        memcpy(&v, y, 16);
                    } else {
#pragma unroll
                        for (int k = 0; k < 16 / S_; ++k) y[k] = dequantize<T, MODE>(q, w[k], raw);
                        memcpy(&v, y, 16);
                    }
                    *a = v;
                }
                done = true;
            }
            if (!done) emit([&](W w) { return dequantize<T, MODE>(q, w, raw); });
            fence_proxy_async();
            named_sync(1, NTC);    // staging complete
            if (tid == 0) {
                tma_store_2d(&tmap, 0, (int)(c * 128), smem_u32(stage_out));
                bulk_commit();
            }
            if constexpr (VER) {
                // the staged chunk against the originals: thread t takes the 16-byte pieces
                // t, t + NTC, ... of the chunk, so every load instruction of a warp reads
                // 512 contiguous bytes (the staged piece q sits in row q/8, swizzled)
#pragma unroll 1
                for (int i = 0; i < 2 * S_; ++i) {
                    const int q = i * NTC + tid;                 // 16-byte piece of the chunk
                    const int r = q >> 3;
                    const uint4 v = *(const uint4*)(stage_out + r * 128 + (((q & 7) ^ (r & 7)) << 4));
                    const uint4 o = ldg_nc_v4(orig + c * (uint64_t)CW + (uint64_t)q * (16 / S_));
                    T y[16 / S_], x[16 / S_];
                    memcpy(y, &v, 16);
                    memcpy(x, &o, 16);
#pragma unroll
                    for (int k = 0; k < 16 / S_; ++k) vacc.add(x[k], y[k], p);
                }
                vacc.flush_chunk(S.vacc);
            }
        } else {
            // tail chunk: plain stores of the first m values
#pragma unroll
            for (int i = 0; i < 32; ++i) {
                const uint32_t e = 32 * tid + i;
                if (e < m) {
                    const T yv = dequantize<T, MODE>(q, (W)(carry + dq[i]), raw);
                    ((T*)dstc)[e] = yv;
                    if constexpr (VER) vacc.add(orig[c * (uint64_t)CW + e], yv, p);
                }
            }
            if constexpr (VER) vacc.flush_chunk(S.vacc);
        }
    }
    if constexpr (VER) {
        named_sync(1, NTC);        // every compute warp has flushed its last chunk
        if (tid == 0) decltype(vacc)::flush_cta(S.vacc, p);
    }
    if (tid == 0) bulk_wait0();    // all TMA stores of this CTA complete before exit
}

}  // namespace pfpl
