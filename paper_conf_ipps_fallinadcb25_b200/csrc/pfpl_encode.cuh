// pfpl_encode.cu -- fused PFPL chunk encoder for sm_100a.
//
// Persistent, warp-specialised CTAs.  One 16 KiB chunk is the unit of work
// (P:141); chunks are taken in order from an atomic ticket (P:158
// "dynamically assign the chunks").  Every stage is fused so the input is read
// once and the output written once.
//
//   compute warps (4 for f32, 2 for f64)          IO warp (1 per CTA)
//   ------------------------------------          -------------------
//   wait full[s]; read rows of chunk c from the   pop (chunk, arena slice) from
//   TMA-swizzled stage s; warp 0 refills s with   the queue; decoupled look-back
//   the next ticket's chunk (TMA, 2-stage ring);  for the byte offset;
//   quantize + verify, delta +         size table entry; copy the
//   negabinary, bit-plane transpose in    payload (or the raw chunk,
//   registers, zero-byte           P:158) to HBM with 16-byte
//   elimination with packed warp scans (P:129,    stores; release the arena
//   P:164) into a reserved arena slice, 3 repeat  slice
//   levels, raw decision; publish
//   the aggregate; push (chunk, slice) to the IO
//
// Input refills never wait for output: payloads live in a per-CTA circular
// arena, so a slow look-back only delays the IO warp.
// Thread t of the compute warps owns elements 32t..32t+31, so its 32 bits of
// each bit plane are one aligned word of the shuffled chunk.
// Arena slice of a chunk at pos: Z1 at [pos, pos + n1); the prefix M4 | Z4 | Z3 | Z2
// (section order of R16) ends at pos + a16(n1) + PRE3 + n2, with Z2 at a fixed
// offset PRE3 past Z1 (so all warps can scatter it before n3/n4 are known) and
// M4 | Z4 | Z3 packed immediately before Z2.  A slice is reserved for the worst
// case (a16(n1) + a16(PRE3 + zroom(n1))) but occupies only a16(n1) + a16(PRE3 + n2): on smooth
// data the prefix is a few dozen bytes, so the arena holds many chunks.
#pragma once
#include <cuda.h>
#include "pfpl_device.cuh"

namespace pfpl {

#ifndef PFPL_ENC_NIN
#define PFPL_ENC_NIN 1
#endif
#ifndef PFPL_ENC_MINB
#define PFPL_ENC_MINB 5
#endif
#ifndef PFPL_ENC_ARENA
#define PFPL_ENC_ARENA 24576
#endif
constexpr int NIN = PFPL_ENC_NIN;    // input stages (TMA ring)
constexpr int DATAB = 16384;         // bytes per chunk
constexpr int PRE3 = 4 + 32 + 256;   // M4 + Z4 + Z3 at most
#ifndef PFPL_ENC_NQ
#define PFPL_ENC_NQ 8
#endif
#ifndef PFPL_STATS
#define PFPL_STATS 1
#endif
#ifndef PFPL_TP_UNROLL
#define PFPL_TP_UNROLL 1     // quantize loop of the REL/f64 paths (4 or 2 values per iteration)
#endif
constexpr int kTpUnroll = PFPL_TP_UNROLL;
#ifndef PFPL_MIN_TIER
#define PFPL_MIN_TIER 8
#endif
#ifndef PFPL_TIER4
#define PFPL_TIER4 0        // P <= 4 uses the 8-plane tier: less hot code (+7% NYX)
#endif
#ifndef PFPL_UNIFIED_L1
#define PFPL_UNIFIED_L1 -1    // level-1 code: 1 one windowed path for all tiers, 0 one copy per
                              // tier, -1 per instantiation (see the kernel)
#endif
#ifndef PFPL_STAGED_L1
#define PFPL_STAGED_L1 1      // REL: level 1 from plane words staged in shared memory
#endif
#ifndef PFPL_LANE_ARRIVE
#define PFPL_LANE_ARRIVE 0    // compute lanes arrive on mq_full one by one (else lane 0 after __syncwarp)
#endif
#ifndef PFPL_LANE_ARRIVE_IO
#define PFPL_LANE_ARRIVE_IO 1 // IO lanes arrive on mq_empty one by one
#endif
// arrive on an IO-queue barrier after this lane's own shared-memory accesses (LANES:
// each lane is its own release, as compute-sanitizer racecheck models it; 32 arrivals)
// or after the warp's (lane 0, behind __syncwarp; 1 arrival)
template <bool LANES>
__device__ __forceinline__ void q_arrive(uint32_t bar, int lane) {
    if (LANES) {
        mbar_arrive(bar);
    } else {
        __syncwarp();
        if (lane == 0) mbar_arrive(bar);
    }
}
#ifndef PFPL_PACKED_REL
#define PFPL_PACKED_REL 0     // the f32 REL fast path on FP32x2 pairs (measured 5% slower: off)
#endif
#ifndef PFPL_REL_FASTW
#define PFPL_REL_FASTW 1       // REL fast path: rel_q_fast_w (ftz lg2, one |L| compare, lossless values counted)
#endif
#ifndef PFPL_X0
#define PFPL_X0 1             // f32 ABS: a second encoder form with the first-residual split
#endif
#ifndef PFPL_PACKED_Q
#define PFPL_PACKED_Q 1       // the f32 ABS/NOA fast-path quantizer on FFMA2/FADD2 pairs
#endif
#ifndef PFPL_LB_NS
#define PFPL_LB_NS 1500
#endif
constexpr int NQ = PFPL_ENC_NQ;      // IO queue depth

// hand-off from the compute warps to the IO warp, one per chunk
struct QEntry {
    unsigned long long c;
    uint32_t start, plen, z1, stored, raw, rend;   // prefix at start (plen bytes), Z1 at z1
};

struct EncShared {
    uint8_t m1[2048];
    uint8_t m2[256];
    uint8_t wcnt[128];               // per-warp per-plane Z1 counts, [warp * B + bit]
    uint32_t scan2[4];               // level-2 warp totals
    uint32_t head, rel;                // arena: next free byte / released up to (monotone counters)
    uint32_t xh;                       // X0 form: extra planes of the chunk's first residual
    unsigned long long in_c[NIN];
    QEntry q[NQ];
    unsigned long long full[NIN], mq_full[NQ], mq_empty[NQ];
};
constexpr int ARENA_OFF = NIN * DATAB;
// per element type: arena bytes, shared-memory layout and CTAs per SM (f64 CTAs have 2
// compute warps, so more of them fit; f64 streams are smoother per byte)
#ifndef PFPL_ENC_ARENA64
#define PFPL_ENC_ARENA64 24576
#endif
#ifndef PFPL_ENC_MINB64
#define PFPL_ENC_MINB64 5
#endif
template <typename T> struct EncCfg {
    static constexpr int ARENA = sizeof(T) == 4 ? PFPL_ENC_ARENA : PFPL_ENC_ARENA64;
    static constexpr int SHARED_OFF = ARENA_OFF + ARENA + 64;
    static constexpr int SMEM = SHARED_OFF + (int)sizeof(EncShared);
    static constexpr int MINB = sizeof(T) == 4 ? PFPL_ENC_MINB : PFPL_ENC_MINB64;
    static constexpr int THREADS = Tr<T>::NT + 32;          // compute warps + the IO warp
    static constexpr int TICKETS = NIN + 1;                 // tickets a CTA draws beyond its chunks
    static_assert(SMEM <= 233472 / MINB - 1024, "MINB CTAs per SM must fit in shared memory");
    static_assert(DATAB + 16 + ((PRE3 + 15) & ~15) <= ARENA, "the arena must hold a worst-case slice");
};
constexpr int ENC_SMEM = EncCfg<float>::SMEM;   // f32 layout (host code: enc_smem(dtype))

__device__ __forceinline__ void put_u64(uint8_t* p, uint64_t v) {
#pragma unroll
    for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i));
}

static __device__ void write_header(uint8_t* out, const EncParams& p, const QConst& qc) {
    out[0] = 'P'; out[1] = 'F'; out[2] = 'P'; out[3] = 'L';
    out[4] = 1; out[5] = (uint8_t)p.dtype; out[6] = (uint8_t)p.bound; out[7] = (uint8_t)qc.flags;
    put_u64(out + 8, p.n_total);
    put_u64(out + 16, d2u(p.eps));
    put_u64(out + 24, qc.qconst);
    put_u64(out + 32, d2u(qc.range));
    put_u64(out + 40, (uint64_t)kChunkBytes);
}

// [stage] byte scatter (Z1/Z2/Z3 stores)
// scatter the bytes of w whose marker (0x01 per byte in hh) is set to z[o...]
__device__ __forceinline__ uint32_t scatter_word(uint8_t* z, uint32_t o, uint32_t w, uint32_t hh) {
    const uint32_t incl = hh * 0x01010101u;
    if (hh & 0x1u) z[o] = (uint8_t)w;
    if (hh & 0x100u) z[o + (incl & 0xFFu)] = (uint8_t)(w >> 8);
    if (hh & 0x10000u) z[o + ((incl >> 8) & 0xFFu)] = (uint8_t)(w >> 16);
    if (hh & 0x1000000u) z[o + ((incl >> 16) & 0xFFu)] = (uint8_t)(w >> 24);
    return o + (incl >> 24);
}
// same with the marker at bit 7 (H = nzmark(w)); ranks from one IMAD.WIDE
__device__ __forceinline__ void scatter_marked(uint8_t* z, uint32_t o, uint32_t w, uint32_t H) {
    const uint32_t rk = (uint32_t)rankcount(H);          // byte k = rank of byte k
    if (H & 0x80u) z[o] = (uint8_t)w;
    if (H & 0x8000u) z[o + __byte_perm(rk, 0, 0x4441)] = (uint8_t)(w >> 8);
    if (H & 0x800000u) z[o + __byte_perm(rk, 0, 0x4442)] = (uint8_t)(w >> 16);
    if (H & 0x80000000u) z[o + (rk >> 24)] = (uint8_t)(w >> 24);
}

// [stage] IO warp: copy-out
// copy len bytes from shared memory to global memory, any alignment on either
// side: 16-byte aligned stores for the body (coalesced even for
// unaligned compressed data), byte stores for the head and the tail.  Reads up
// to 20 bytes past src + len (inside the arena's padding).
#ifndef PFPL_COPY_INLINE    // one out-of-line copy: less hot code for the IO warp
static __device__ __noinline__
#else
__device__ __forceinline__
#endif
void warp_copy_s2g(uint8_t* o, const uint8_t* src, uint32_t len, int lane) {
    const uint32_t mis = (uint32_t)((uintptr_t)o & 15u);
    uint32_t head = (16u - mis) & 15u;
    if (head > len) head = len;
    const uint32_t body = (len - head) >> 4;
    const uint32_t tail0 = head + (body << 4);
    if ((uint32_t)lane < head) o[lane] = src[lane];
    if ((uint32_t)lane < len - tail0) o[tail0 + lane] = src[tail0 + lane];
    for (uint32_t j = lane; j < body; j += 32) {
        const uint8_t* sp = src + head + (j << 4);
        const uint32_t a = smem_u32(sp) & 3u;
        const uint32_t* sw = (const uint32_t*)(sp - a);
        const uint32_t w0 = sw[0], w1 = sw[1], w2 = sw[2], w3 = sw[3], w4 = sw[4];
        const uint32_t sh = a * 8u;
        uint4 v;
        v.x = __funnelshift_r(w0, w1, sh);
        v.y = __funnelshift_r(w1, w2, sh);
        v.z = __funnelshift_r(w2, w3, sh);
        v.w = __funnelshift_r(w3, w4, sh);
        *(uint4*)(o + head + (j << 4)) = v;
    }
}

// [stage] arena allocation
// ---------------------------------------------------------------------------
// bit shuffle + level-1 zero-byte elimination for one chunk.
// KL planes from the low 32 bits of the residuals, KH from the high 32 (f64).
// Plane word j holds bit b_j of the thread's 32 residuals; its shuffled
// position is plane p = B-1-b_j, byte p*CW/8 + 4*tid (reading R13).
// Z1 (plane-major, non-zero bytes in order) goes to the chunk's arena slice.
// ---------------------------------------------------------------------------
// Arena slice for a chunk with n1 Z1 bytes: every compute warp derives the same
// position from S.head (advanced by warp 0 only after the Z1 scatter) and waits
// only if the IO warp lags by more than the arena's capacity.
__device__ __forceinline__ uint32_t a16(uint32_t x) { return (x + 15u) & ~15u; }
// room reserved for Z2: at most 2048 bytes, and never more than a non-raw chunk
// can use (4 + n4 + n3 + n2 + n1 < 16384); a chunk whose n2 exceeds it is raw
// (P:158), so its Z2 is not written.  A slice therefore never exceeds
// 16400 + a16(PRE3) bytes, and a raw chunk's slice holds its 16384 staged bytes.
__device__ __forceinline__ uint32_t zroom(uint32_t n1) { return min(2048u, (uint32_t)DATAB + 16u - a16(n1)); }
// bytes a slice occupies once n2 is known
__device__ __forceinline__ uint32_t slice_bytes(uint32_t n1, uint32_t n2) {
    return a16(n1) + a16(PRE3 + min(n2, zroom(n1)));
}
// Arena release protocol: the IO warp arrives on mq_empty[j % NQ] once it has read
// (copied out) chunk j's slice; a compute warp that needs arena bytes still held by
// chunk j waits on that barrier phase itself before writing them, so every reuse of
// arena bytes is ordered by an mbarrier (release/acquire in the PTX memory model, and
// visible to compute-sanitizer racecheck).  S.rel = end (monotone byte counter) of
// chunk it-1-NQ's slice, recorded by the duty warp of iteration it-1 right after its
// own wait on that chunk (published by this iteration's first CTA barrier).  Queue
// entries of chunks it-NQ .. it-1 are intact here: the duty warp overwrites chunk
// it-NQ's only after the third barrier.  The parity wait on chunk j cannot alias: slot
// j % NQ completes again only for chunk j + NQ >= it, which is not yet pushed.
template <int ARENA>
__device__ __forceinline__ uint32_t slice_start(const EncShared& S, uint32_t n1, uint32_t it) {
    const uint32_t R = a16(n1) + a16(PRE3 + zroom(n1));     // worst case
    const uint32_t head0 = S.head;
    uint32_t head = head0;
    const uint32_t p0 = head % ARENA;
    if (p0 + R > (uint32_t)ARENA) head += ARENA - p0;      // a slice never wraps
    // the new slice [head, head+R) is free when every byte before rel is released and
    // the live range [rel, head0) plus the slice spans at most ARENA bytes, or when the
    // arena is empty (rel == head0; the gap skipped to avoid wrapping is never
    // released by itself)
    auto fits = [&](uint32_t rel) { return rel == head0 || head + R - rel <= (uint32_t)ARENA; };
    if (!fits(S.rel)) {
        for (uint32_t j = it - min(it, (uint32_t)NQ); j < it; ++j) {    // oldest first
            mbar_wait_wd(smem_u32(&S.mq_empty[j % NQ]), (j / NQ) & 1u, 0x13);
            if (fits(S.q[j % NQ].rend)) break;
        }
    }
    return head;                                            // monotone byte counter
}

// [stage] level 1: plane counts + scans
// ---- level-1 phase A: transpose in place, per-plane counts, packed warp scans.
// KL planes from the low 32 bits of the residuals, KH from the high 32 (f64).
// Plane word j holds bit b_j of the thread's 32 residuals (b_j = j, or 32+j-KL).
// Writes this warp's full row of per-plane counts (zero above its tier).
template <typename T, int KL, int KH>
__device__ __forceinline__ void rze1_count(uint32_t (&lo)[32], uint32_t (&hi)[32], EncShared& S,
                                           int lane, int warp, uint64_t wor, uint32_t (&ex)[16]) {
    constexpr int B = Tr<T>::B;
    constexpr int NG = (KL + KH) / 4;
    if constexpr (KL > 0) transpose_fwd<KL>(lo);
    if constexpr (KH > 0) transpose_fwd<KH>(hi);
    auto PW = [&](int j) -> uint32_t { return j < KL ? lo[j] : hi[j - KL]; };
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        const int b0 = 4 * g < KL ? 4 * g : 32 + 4 * g - KL;
        uint32_t inc = 0, v = 0;
        if (wor & (0xFull << b0)) {          // skip groups empty in this whole warp
#pragma unroll
            for (int i = 0; i < 4; ++i)
                v = __byte_perm(v, (uint32_t)(rankcount(nzmark(PW(4 * g + i))) >> 32),
                                i == 0 ? 0x3214 : i == 1 ? 0x3240 : i == 2 ? 0x3410 : 0x4210);
            inc = warp_incl_scan(v, lane);
        }
        ex[g] = inc - v;
        if (lane == 31) *(uint32_t*)&S.wcnt[warp * B + b0] = inc;
    }
    if (lane == 31) {
#pragma unroll
        for (int b0 = KL; b0 < 32; b0 += 4) *(uint32_t*)&S.wcnt[warp * B + b0] = 0u;
#pragma unroll
        for (int b0 = 32 + KH; b0 < B; b0 += 4) *(uint32_t*)&S.wcnt[warp * B + b0] = 0u;
    }
}

// [stage] level 1: Z1/M1 scatter
// ---- level-1 phase B: scatter the non-zero bytes of this thread's plane words
// to Z1 (plane-major order, R13) and its M1 nibbles; offl/offh = this warp's
// Z1 offset of the segment of bit `lane` / `32+lane`.
template <typename T, int KL, int KH>
__device__ __forceinline__ void rze1_scatter(const uint32_t (&lo)[32], const uint32_t (&hi)[32],
                                             uint8_t* z1, uint8_t* m1, int tid, int lane,
                                             uint64_t wor, const uint32_t (&ex)[16],
                                             uint32_t offl, uint32_t offh) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW;
    constexpr int NP = KL + KH;
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const uint32_t w = j < KL ? lo[j] : hi[j - KL];
        const int b = j < KL ? j : 32 + j - KL;
        // wor bit b is set iff some lane's plane word b is non-zero (wor is the warp's
        // OR of the residuals)
        if (!((wor >> b) & 1u)) continue;                       // plane empty in this warp
        const int pl = B - 1 - b;
        const uint32_t H = nzmark(w);
        const uint32_t o = __shfl_sync(PFPL_FULL, j < KL ? offl : offh, b & 31) +
                           __byte_perm(ex[j / 4], 0, 0x4440 + (j % 4));
        scatter_marked(z1, o, w, H);
        const uint32_t nb = nib(H >> 7);
        const uint32_t nb2 = __shfl_xor_sync(PFPL_FULL, nb, 1);
        if (!(lane & 1)) m1[pl * (CW / 64) + (tid >> 1)] = (uint8_t)(nb | (nb2 << 4));
    }
}

// [stage] level 1: plane counts + scans
// ---- level 1 with one copy of the count/scatter code for every tier: only the
// transpose is specialised on the tier (P <= 8, 16, 32 planes; f64 adds the high
// half), which leaves plane word b of the thread's residuals in lo[b] / hi[b - 32]
// for every tier.  Counts and scatter then walk windows of 8 planes guarded by the
// active-plane count P (planes >= P are zero in the whole warp), so a CTA whose
// warps run different tiers executes one code path: the tiered copies overflowed
// the 32 KB instruction cache on rough data (ncu: 31% no_instruction stalls).
template <typename T>
__device__ __forceinline__ void rze1_transpose(uint32_t (&lo)[32], uint32_t (&hi)[32], int P) {
    if (P == 0) {
    } else if (Tr<T>::B == 32 || P <= 32) {
        if (P <= 8 && PFPL_MIN_TIER <= 8) transpose_fwd<8>(lo);
        else if (P <= 16 && PFPL_MIN_TIER <= 16) transpose_fwd<16>(lo);
        else transpose_fwd<32>(lo);
    } else {
        transpose_fwd<32>(lo);
        if (P <= 40) transpose_fwd<8>(hi);
        else if (P <= 48) transpose_fwd<16>(hi);
        else transpose_fwd<32>(hi);
    }
}
template <typename T>
__device__ __forceinline__ void rze1_count_w(const uint32_t (&lo)[32], const uint32_t (&hi)[32], EncShared& S,
                                             int lane, int warp, uint64_t wor, int P, uint32_t (&ex)[16]) {
    constexpr int B = Tr<T>::B;
#pragma unroll
    for (int w8 = 0; w8 < B / 8; ++w8) {
        if (P > 8 * w8) {
#pragma unroll
            for (int gg = 0; gg < 2; ++gg) {
                const int b0 = 8 * w8 + 4 * gg;
                uint32_t inc = 0, v = 0;
                if (wor & (0xFull << b0)) {          // skip groups empty in this whole warp
#pragma unroll
                    for (int i = 0; i < 4; ++i) {
                        const uint32_t w = b0 + i < 32 ? lo[(b0 + i) & 31] : hi[(b0 + i) & 31];
                        v = __byte_perm(v, (uint32_t)(rankcount(nzmark(w)) >> 32),
                                        i == 0 ? 0x3214 : i == 1 ? 0x3240 : i == 2 ? 0x3410 : 0x4210);
                    }
                    inc = warp_incl_scan(v, lane);
                }
                ex[b0 / 4] = inc - v;
                if (lane == 31) *(uint32_t*)&S.wcnt[warp * B + b0] = inc;
            }
        } else if (lane == 31) {
            *(uint32_t*)&S.wcnt[warp * B + 8 * w8] = 0u;
            *(uint32_t*)&S.wcnt[warp * B + 8 * w8 + 4] = 0u;
        }
    }
}
// [stage] level 1: Z1/M1 scatter
template <typename T>
__device__ __forceinline__ void rze1_scatter_w(const uint32_t (&lo)[32], const uint32_t (&hi)[32],
                                               uint8_t* z1, uint8_t* m1, int tid, int lane, uint64_t wor,
                                               int P, const uint32_t (&ex)[16], uint32_t offl, uint32_t offh) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW;
#pragma unroll
    for (int w8 = 0; w8 < B / 8; ++w8) {
        if (P <= 8 * w8) break;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
            const int b = 8 * w8 + i;
            const uint32_t w = b < 32 ? lo[b & 31] : hi[b & 31];
            if (!((wor >> b) & 1u)) continue;                       // plane empty in this warp
            const int pl = B - 1 - b;
            const uint32_t H = nzmark(w);
            const uint32_t o = __shfl_sync(PFPL_FULL, b < 32 ? offl : offh, b & 31) +
                               __byte_perm(ex[b / 4], 0, 0x4440 + (b % 4));
            scatter_marked(z1, o, w, H);
            const uint32_t nb = nib(H >> 7);
            const uint32_t nb2 = __shfl_xor_sync(PFPL_FULL, nb, 1);
            if (!(lane & 1)) m1[pl * (CW / 64) + (tid >> 1)] = (uint8_t)(nb | (nb2 << 4));
        }
    }
}

// [stage] level 1: plane counts + scans
// ---- staged level 1 (the two-pass REL / f64 quantizers, whose stage rows are
// already rewritten in place): after the transpose every thread stores its plane
// words to its own stage rows (group g of 4 planes = one swizzled 16-byte slot),
// so counts and scatter are rolled loops over plane groups -- ~2 KB of code for
// every tier and both halves of f64 instead of an unrolled copy per plane -- and
// the planes need no registers across the CTA barrier.  The stage is refilled by
// TMA only after the scatter.
template <typename T>
__device__ __forceinline__ uint8_t* plane_slot(uint8_t* wbuf, int tid, int g) {
    const int r = sizeof(T) == 4 ? tid : 2 * tid + (g >> 3);
    return wbuf + r * 128 + (((g & 7) ^ (r & 7)) << 4);
}
// number of non-zero bytes of each of the 4 words, one per byte (each <= 4)
__device__ __forceinline__ uint32_t nzcount4(const uint4 v) {
    uint32_t c = (uint32_t)(rankcount(nzmark(v.x)) >> 32);
    c = __byte_perm(c, (uint32_t)(rankcount(nzmark(v.y)) >> 32), 0x3240);
    c = __byte_perm(c, (uint32_t)(rankcount(nzmark(v.z)) >> 32), 0x3410);
    c = __byte_perm(c, (uint32_t)(rankcount(nzmark(v.w)) >> 32), 0x4210);
    return c;
}
template <typename T>
__device__ __forceinline__ void rze1_stage_planes(const uint32_t (&lo)[32], const uint32_t (&hi)[32],
                                                  uint8_t* wbuf, int tid, int P) {
#pragma unroll
    for (int g = 0; g < Tr<T>::B / 4; ++g) {
        if (4 * g < P) {
            const uint32_t* src = g < 8 ? lo + 4 * g : hi + 4 * (g - 8);
            *(uint4*)plane_slot<T>(wbuf, tid, g) = make_uint4(src[0], src[1], src[2], src[3]);
        }
    }
}
template <typename T>
__device__ __forceinline__ void rze1_count_s(uint8_t* wbuf, EncShared& S, int tid, int lane, int warp,
                                             uint64_t wor, int P) {
    constexpr int B = Tr<T>::B;
    const int ng = (P + 3) >> 2;
#pragma unroll 1
    for (int g = 0; g < B / 4; ++g) {
        uint32_t tot = 0;
        if (g < ng && (wor & (0xFull << (4 * g)))) {        // warp-uniform
            const uint4 v4 = *(const uint4*)plane_slot<T>(wbuf, tid, g);
            tot = __reduce_add_sync(PFPL_FULL, nzcount4(v4));  // bytes <= 128: no carries
        }
        if (lane == 31) *(uint32_t*)&S.wcnt[warp * B + 4 * g] = tot;
    }
}
// [stage] level 1: Z1/M1 scatter
template <typename T>
__device__ __forceinline__ void rze1_scatter_s(uint8_t* wbuf, uint8_t* z1, uint8_t* m1, int tid, int lane,
                                               uint64_t wor, int P, uint32_t offl, uint32_t offh) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW;
    const int ng = (P + 3) >> 2;
#pragma unroll 1
    for (int g = 0; g < ng; ++g) {
        const uint32_t wg = (uint32_t)(wor >> (4 * g)) & 0xFu;   // warp-uniform
        if (!wg) continue;
        const uint4 v4 = *(const uint4*)plane_slot<T>(wbuf, tid, g);
        const uint32_t cnt = nzcount4(v4);
        const uint32_t ex = warp_incl_scan(cnt, lane) - cnt;
        const uint32_t w4[4] = {v4.x, v4.y, v4.z, v4.w};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
            const int b = 4 * g + i;
            const uint32_t w = w4[i];
            if (!((wg >> i) & 1u)) continue;                    // plane empty in this warp
            const uint32_t H = nzmark(w);
            const uint32_t o = __shfl_sync(PFPL_FULL, b < 32 ? offl : offh, b & 31) +
                               __byte_perm(ex, 0, 0x4440 + i);
            scatter_marked(z1, o, w, H);
            const uint32_t nb = nib(H >> 7);
            const uint32_t nb2 = __shfl_xor_sync(PFPL_FULL, nb, 1);
            if (!(lane & 1)) m1[(B - 1 - b) * (CW / 64) + (tid >> 1)] = (uint8_t)(nb | (nb2 << 4));
        }
    }
}

// [stage] IO warp: look-back
// Decoupled look-back (Merrill-Garland) over descriptors hi, hi-1, ..., lo,
// nearest first, in 32-wide windows (lane l reads descriptor top - l).  rd(idx, &flag)
// returns the value of descriptor idx and its flag (LB_P inclusive prefix, LB_A
// aggregate, 0 not yet published).  Returns the sum of the values from the nearest
// inclusive prefix up to hi and sets *found, or the sum over all of lo..hi if none of
// them is an inclusive prefix.  Chunks handed out in the same "round" are processed
// concurrently by the other CTAs' IO warps, so the nearest inclusive prefix is
// typically one round (~#CTAs chunks) back.  A window is re-read (sleeping between
// polls, so polling costs the compute warps almost no issue slots) until every
// descriptor it needs is published.
template <typename RD>
__device__ __forceinline__ uint64_t lookback(RD rd, int64_t hi, int64_t lo, int lane, bool* found,
                                             uint32_t site) {
    uint64_t acc = 0;
    const uint64_t t0 = globaltimer();
    for (int64_t top = hi; top >= lo;) {
        const int64_t idx = top - lane;
        const bool valid = idx >= lo;
        uint32_t flag = 0;
        const uint64_t v = valid ? rd(idx, flag) : 0ull;
        const uint32_t pm = __ballot_sync(PFPL_FULL, valid && flag == (uint32_t)LB_P);
        const uint32_t nr = __ballot_sync(PFPL_FULL, valid && flag == 0u);
        const uint32_t need = pm ? ((pm & (0u - pm)) << 1) - 1u : PFPL_FULL;
        if (nr & need) {
            if (globaltimer() - t0 > kWatchdogNs) watchdog_fire(site, (uint32_t)top);
            __nanosleep(PFPL_LB_NS);
            continue;
        }
        acc += warp_sum64((valid && ((need >> lane) & 1u)) ? v : 0ull);
        if (pm) {
            *found = true;
            return acc;
        }
        top -= 32;
    }
    *found = false;
    return acc;
}

// [stage] misc (tier dispatch, stats)
#define PFPL_TIER_DISPATCH(FN, ...)                                                     \
    do {                                                                                \
        if (P == 0) FN<T, 0, 0>(__VA_ARGS__);                                           \
        else if (B == 32 || P <= 32) {                                                  \
            if (PFPL_TIER4 && P <= 4) FN<T, 4, 0>(__VA_ARGS__);                         \
            else if (P <= 8 && PFPL_MIN_TIER <= 8) FN<T, 8, 0>(__VA_ARGS__);            \
            else if (P <= 16 && PFPL_MIN_TIER <= 16) FN<T, 16, 0>(__VA_ARGS__);         \
            else FN<T, 32, 0>(__VA_ARGS__);                                             \
        } else {                                                                        \
            if (P <= 36) FN<T, 32, 4>(__VA_ARGS__);                                     \
            else if (P <= 40) FN<T, 32, 8>(__VA_ARGS__);                                \
            else if (P <= 48) FN<T, 32, 16>(__VA_ARGS__);                               \
            else FN<T, 32, 32>(__VA_ARGS__);                                            \
        }                                                                               \
    } while (0)

// A word is a bin (quantized value) iff it lies in the bin range of its mode: ABS/NOA
// zigzag bins below the normal range (R8; f32 words carry the encoder's bias), REL bins
// 1 + payload in the (inverted) negative-NaN pattern (R10, R11).  Everything else, and
// every word in raw-words mode, is an unquantizable value stored losslessly.
template <typename T, int MODE>
__device__ __forceinline__ bool is_bin_word(typename Tr<T>::W w, typename Tr<T>::W qbias, bool raw) {
    typedef typename Tr<T>::W W;
    constexpr W LIM = sizeof(T) == 4 ? (W)0x00800000u : (W)0x0010000000000000ull;
    if (!PFPL_STATS) return true;
    if (MODE == MODE_RAW || (MODE == MODE_NOA && raw)) return false;
    if (MODE == MODE_REL) return (W)(w - 1) < (W)(LIM - 1);
    return (W)(w - qbias) < LIM;
}

// [stage] kernel setup + tickets
// the hint for the next f32 ABS call (IO warp of CTA 0, off the compute warps' code): the
// split form pays when chunks start with a large bin on a smooth field, i.e. first residuals
// reach 2^8 while the others stay below: at >= 4 of 8 chunk starts |bin| = |v| / (2 eps) >= 64
// and the next value is within 4 bins of it (on a rough field the other residuals keep warp 0
// wide anyway, and there the plain form is faster: the rough NYX variant's neighbours are
// 3-70 bins apart)
__device__ __forceinline__ void x0_hint_update(const EncParams& p, float b) {
    int big = 0;
    for (int k = 0; k < 8; ++k) {
        const uint64_t e = (p.C * (uint64_t)k / 8u) * 4096u;
        if (e + 1 >= p.n) continue;
        const float v0 = ((const float*)p.in)[e], v1 = ((const float*)p.in)[e + 1];
        big += (fabsf(v0) * b >= 64.0f && fabsf(v1 - v0) * b < 4.0f) ? 1 : 0;    // NaN: no
    }
    *(volatile unsigned int*)p.x0_hint = big >= 4 ? 1u : 0u;
}

// X0 selects the form with the first-residual split (kX0 below); both forms write the same
// bytes.  The host picks the form from a hint that CTA 0 of every f32 ABS launch leaves in
// mapped host memory (x0_hint_of below), so a hint takes effect from the next call.
template <typename T, int MODE, bool MSR, bool X0>
__global__ void __launch_bounds__(Tr<T>::NT + 32, EncCfg<T>::MINB)
encode_kernel(const EncParams p, const __grid_constant__ CUtensorMap tmap) {
    typedef typename Tr<T>::W W;
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NTC = Tr<T>::NT, NWC = Tr<T>::NW, S_ = Tr<T>::S;
    constexpr int NB2 = 2048 / NTC;     // level-2 bytes per compute thread (16 or 32)
    constexpr int NWD2 = NB2 / 4;

    constexpr int ARENA = EncCfg<T>::ARENA;
    extern __shared__ __align__(1024) uint8_t smem[];
    EncShared& S = *reinterpret_cast<EncShared*>(smem + EncCfg<T>::SHARED_OFF);
    uint8_t* const arena = smem + ARENA_OFF;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint64_t C = p.C;
    const uint64_t full_chunks = p.n / CW;

    QConst qc = p.qc;
    if (MODE == MODE_NOA) qc = *p.qc_dev;

    // ticket -> input stage s (compute warp 0 lane 0 only)
    auto issue = [&](int s, unsigned long long t) {
        S.in_c[s] = t;
        if (t < full_chunks) {
            fence_proxy_async();
            mbar_arrive_tx(smem_u32(&S.full[s]), DATAB);
            tma_load_2d(smem_u32(smem + s * DATAB), &tmap, 0, (int)(t * 128), smem_u32(&S.full[s]));
        } else {
            mbar_arrive(smem_u32(&S.full[s]));     // tail chunk (loaded by the compute warps) or end
        }
    };
    unsigned long long next = 0;
    if (tid == 0) {
        g_pfpl_wd = p.wd;
        if (blockIdx.x == 0 && p.stats_next) { p.stats_next[0] = 0; p.stats_next[1] = 0; }
        if (smem_u32(smem) & 1023u) __trap();       // TMA SWIZZLE_128B needs 1024-byte alignment
        for (int s = 0; s < NIN; ++s) mbar_init(smem_u32(&S.full[s]), 1);
        for (int k = 0; k < NQ; ++k) {
            mbar_init(smem_u32(&S.mq_full[k]), (PFPL_LANE_ARRIVE ? 32 : 1) * NWC);  // compute lanes/warps
            mbar_init(smem_u32(&S.mq_empty[k]), PFPL_LANE_ARRIVE_IO ? 32 : 1);     // IO lanes/warp
        }
        S.head = 0;
        S.rel = 0;
        fence_barrier_init();
        prefetch_tmap(&tmap);
    }
    __syncthreads();
    if (tid == 0) {
        for (int s = 0; s < NIN; ++s) issue(s, atomicAdd(p.ticket, 1ull) - p.ticket_base);
        next = atomicAdd(p.ticket, 1ull);
    }

    if (warp == NWC) {
// [stage] IO warp: queue
        // =========================== IO warp ===========================
        if (sizeof(T) == 4 && (MODE == MODE_ABS || MODE == MODE_NOA) && PFPL_X0 && p.x0_hint &&
            blockIdx.x == 0 && lane == 0)
            x0_hint_update(p, u2f((uint32_t)qc.b));     // NOA: the device-derived constants
        const uint64_t EP = (uint64_t)p.epoch << 48;
        for (uint32_t k = 0;; ++k) {
            const int slot = k % NQ;
            mbar_wait_wd(smem_u32(&S.mq_full[slot]), (k / NQ) & 1u, 0x11);
            const QEntry e = S.q[slot];
            if (e.c >= C) break;
            const uint64_t c = e.c;
            const uint32_t stored = e.stored, start = e.start;
            const bool israw = e.raw != 0;
// [stage] IO warp: look-back
            // ---- decoupled look-back ----
            uint64_t excl = 0;
            if (c > 0) {
                // chunk descriptors: [63:48] epoch | [47:46] flag | [45:0] value
                auto rd_chunk = [&](int64_t i, uint32_t& flag) -> uint64_t {
                    const uint64_t d = ld_relaxed(&p.status[i]);
                    flag = ((uint32_t)(d >> 48) == p.epoch) ? (uint32_t)((d >> 46) & 3u) : 0u;
                    return d & LB_VAL;
                };
                bool found = false;
#if defined(PFPL_LB_FAKE)
                (void)rd_chunk; (void)found;
                excl = c * 1024u;    // timing experiment only: no look-back (invalid stream)
#else
                excl = lookback(rd_chunk, (int64_t)c - 1, 0, lane, &found, 0x12);
#endif
                if (lane == 0) st_relaxed(&p.status[c], EP | (LB_P << 46) | (excl + stored));
            }
// [stage] IO warp: table + copy
            const uint64_t dst = p.payload_off + excl;
            if (lane == 0) {
                p.table[c] = stored;
                if (c == C - 1) {
                    // stream bytes, and the status word of pfpl_compress_async (pfpl.h):
                    // offsets are monotone, so the last chunk's end is the stream's end
                    p.result[0] = dst + stored;
                    if (dst + stored > p.cap) ((int*)p.result)[2] = -3;     // PFPL_ERR_CAPACITY
                }
                if (c == 0 && p.write_header) write_header(p.out, p, qc);
            }
#if defined(PFPL_NO_COPY)
            if (false) {         // timing experiment only: no copy-out (invalid stream)
#else
            if (dst + stored <= p.cap) {
#endif
                if (israw) {
                    // raw chunk (R17): stage the original bytes in this chunk's
                    // arena slice (always large enough: slice >= payload >= raw bytes)
                    uint8_t* stg = arena + start;
                    const uint8_t* g = (const uint8_t*)p.in + c * (uint64_t)kChunkBytes;
                    for (uint32_t i = lane; i < stored / 16; i += 32) ((uint4*)stg)[i] = ldg_nc_v4(g + 16 * i);
                    for (uint32_t i = (stored / 16) * 4 + lane; i < stored / 4; i += 32)
                        ((uint32_t*)stg)[i] = ((const uint32_t*)g)[i];
                    __syncwarp();
                    warp_copy_s2g(p.out + dst, arena + start, stored, lane);
                } else {
                    // payload = prefix (M4 | Z4 | Z3 | Z2) then Z1 (R16)
                    warp_copy_s2g(p.out + dst, arena + start, e.plen, lane);
                    warp_copy_s2g(p.out + dst + e.plen, arena + e.z1, stored - e.plen, lane);
                }
            }
            q_arrive<PFPL_LANE_ARRIVE_IO>(smem_u32(&S.mq_empty[slot]), lane);   // reads of the slice and entry are done
        }
        return;
    }

// [stage] compute: stage wait + M1 zero
    // ============================ compute warps ============================
    QF<T> q;
    q.load(qc);
    const bool raw = (qc.flags & HF_RAWWORDS) != 0;
    // bias of quantize_b(): only the f32 ABS/NOA bin path is biased
    const uint64_t qbias = (sizeof(T) == 4 && (MODE == MODE_ABS || (MODE == MODE_NOA && !raw)))
                               ? 0x4B000000ull : 0ull;
    // kX0 (f32 ABS fast path, the X0 form): the chunk's first residual x0 is taken against
    // q[-1] = 0, so it carries the whole first bin and alone would lift warp 0 out of
    // the 8-plane tier.  When every other residual of warp 0 is below 2^8, its bits >= 8
    // become "extra" planes, in which only element 0 is set: one byte 0x01 at the start of
    // warp 0's segment of the plane (R13) and M1 byte 0x01, added outside the tiered level-1
    // code (counts when the offsets are formed, bytes right after).  The decision is a vote
    // taken before the warp OR is reduced.  Same bytes as the plain shuffle.
    constexpr bool kX0 = X0 && sizeof(T) == 4 && (MODE == MODE_ABS || MODE == MODE_NOA) &&
                         !(PFPL_UNIFIED_L1 == 1) && !PFPL_TIER4 && PFPL_MIN_TIER <= 8;
    uint32_t it = 0;
    for (;; ++it) {
        const int s = it % NIN;
        mbar_wait_wd(smem_u32(&S.full[s]), (it / NIN) & 1u, 0x14);
        const uint64_t c = S.in_c[s];
        if (c >= C) break;
        const uint8_t* buf = smem + s * DATAB;
        uint8_t* const m1 = S.m1;
        const uint32_t m = (uint32_t)min((uint64_t)CW, p.n - c * (uint64_t)CW);
        if constexpr (MODE != MODE_REL) {
            // zero this thread's part of M1
#pragma unroll
            for (int i = 0; i < 2048 / 16 / NTC; ++i)
                ((uint4*)m1)[tid * (2048 / 16 / NTC) + i] = make_uint4(0, 0, 0, 0);
        }


// [stage] quantize + delta (loop)
        // ---- quantize + verify, delta, residual code ----
        uint32_t lo[32], hi[32];
        W orv = 0;
        // unquantizable values (0 on the fast path): counted on the other paths only
        auto add_raw = [&](uint32_t nraw) {
            const uint32_t t = __reduce_add_sync(PFPL_FULL, nraw);
            if (lane == 0 && t && p.stats) atomicAdd(&p.stats[0], (unsigned long long)t);
        };
        // kX0: warp 0's extra planes of this chunk, read by every warp after the counts barrier
        // (0 unless the fast path splits x0)
        if (kX0 && tid == 0) S.xh = 0u;
        {
            // biased words (quantize_b): q + bias; the bias cancels in q[i] - q[i-1]
            W qprev = (W)qbias;
            bool done = false;
            if constexpr (sizeof(T) == 4 && (MODE == MODE_ABS || MODE == MODE_NOA)) {
                if (m == CW && !raw) {
                    // fast path: no per-element select or raw word; the
                    // checks of all 32 values accumulate into one predicate
                    uint32_t zp = (uint32_t)qbias, orw = 0u;
                    // 8 independent predicate chains (a single chain would serialise
                    // 64 dependent FSETPs per thread)
                    bool ok[8] = {true, true, true, true, true, true, true, true};
                    if (tid > 0) {
                        const int r = tid - 1;
                        zp = q.abs_qf(*(const float*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 12), ok[7]);
                    }
#pragma unroll
                    for (int i = 0; i < 8; ++i) {
                        const uint4 v = *(const uint4*)(buf + tid * 128 + (((i & 7) ^ (tid & 7)) << 4));
                        bool* o = ok + 4 * (i & 1);
#if PFPL_PACKED_Q
                        uint32_t z0, z1, z2, z3;
                        q.abs_qf2(((uint64_t)v.y << 32) | v.x, o[0], o[1], z0, z1, p.nz2);
                        q.abs_qf2(((uint64_t)v.w << 32) | v.z, o[2], o[3], z2, z3, p.nz2);
#else
                        const uint32_t z0 = q.abs_qf(u2f(v.x), o[0]), z1 = q.abs_qf(u2f(v.y), o[1]);
                        const uint32_t z2 = q.abs_qf(u2f(v.z), o[2]), z3 = q.abs_qf(u2f(v.w), o[3]);
#endif
                        const uint32_t r0 = rcode<MSR>(z0 - zp), r1 = rcode<MSR>(z1 - z0);
                        const uint32_t r2 = rcode<MSR>(z2 - z1), r3 = rcode<MSR>(z3 - z2);
                        zp = z3;
                        orw |= (kX0 && i == 0 ? 0u : r0) | r1;    // kX0: lo[0] is ORed after the loop
                        orw |= r2 | r3;
                        lo[4 * i] = r0; lo[4 * i + 1] = r1; lo[4 * i + 2] = r2; lo[4 * i + 3] = r3;
                    }
                    done = __all_sync(PFPL_FULL, ok[0] && ok[1] && ok[2] && ok[3] && ok[4] && ok[5] &&
                                                     ok[6] && ok[7]);
                    if constexpr (kX0) {
                        // every residual of the warp below 2^8, x0's bits >= 8 aside?
                        const bool small = __all_sync(PFPL_FULL, (orw | (tid ? lo[0] : lo[0] & 0xFFu)) < 256u);
                        if (tid == 0) {
                            const uint32_t xh = (done && small) ? lo[0] & ~0xFFu : 0u;
                            lo[0] ^= xh;
                            S.xh = xh;
                        }
                        orw |= lo[0];          // x0 whole unless split (a failed fast path redoes lo[])
                    }
                    orv = (W)orw;
                }
            }
            // long quantizers (REL's log2p/pow2p/divisions, f64): quantize the stage in
            // place in a rolled loop, then delta-code the words.  Fully unrolling them
            // over 32 values overflows the instruction cache (ncu: no_instruction stalls
            // were 42% of REL samples).
            constexpr bool TWO_PASS = MODE == MODE_REL || sizeof(T) == 8;
            if constexpr (TWO_PASS) {
                if (m == CW) {
                    uint8_t* const wbuf = smem + s * DATAB;
                    T pv = (T)0;
                    if (tid > 0) {
                        if (lane == 0) {
                            // the previous row belongs to another warp, which may
                            // already have overwritten it: read the input again (L2)
                            pv = ((const T*)p.in)[c * (uint64_t)CW + 32 * tid - 1];
                        } else if (sizeof(T) == 4) {
                            const int r = tid - 1;
                            pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 12);
                        } else {
                            const int r = 2 * tid - 1;
                            pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 8);
                        }
                    }
                    __syncwarp();
                    uint32_t nraw = 0;
                    uint32_t slowm = 0;     // REL: values whose fast-path bin is not certain
                    uint32_t rawm = 0;      // REL: values stored raw by the fast path
#pragma unroll kTpUnroll
                    for (int i = 0; i < 2 * S_; ++i) {
                        const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                        uint4* const a = (uint4*)(wbuf + r * 128 + (((i & 7) ^ (r & 7)) << 4));
                        uint4 v = *a;
                        T x[16 / S_];
                        W w[16 / S_];
                        memcpy(x, &v, 16);
                        if constexpr (MODE == MODE_REL && sizeof(T) == 4 && PFPL_PACKED_REL) {
                            // shift-in masks (value j ends at bit 31 - j), two values at a time
                            uint32_t s01, r01, s23, r23;
                            const uint64_t w01 = q.rel_q_fast2(v.x, v.y, p.nz2, s01, r01);
                            const uint64_t w23 = q.rel_q_fast2(v.z, v.w, p.nz2, s23, r23);
                            slowm = slowm * 16u + (__brev(s01 | (s23 << 2)) >> 28);
                            rawm = rawm * 16u + (r01 | (r23 << 2));
                            v = make_uint4((uint32_t)w01, (uint32_t)(w01 >> 32), (uint32_t)w23, (uint32_t)(w23 >> 32));
                            *a = v;
                            continue;
                        }
#pragma unroll
                        for (int k = 0; k < 16 / S_; ++k) {
                            if constexpr (MODE == MODE_REL && PFPL_REL_FASTW) {
                                bool sl;
                                w[k] = q.rel_q_fast_w(x[k], sl, nraw);
                                slowm = slowm * 2u + (sl ? 1u : 0u);     // shift-in mask (one LEA)
                            } else if constexpr (MODE == MODE_REL) {
                                bool sl, bn;
                                const W fw = q.rel_q_fast(x[k], sl, bn);
                                // an uncertain value keeps its input bits for the exact pass
                                W xb;
                                memcpy(&xb, &x[k], sizeof(W));
                                w[k] = sl ? xb : fw;
                                // shift-in masks (one LEA each; value j ends at bit 31 - j):
                                // uncertain values, and values stored raw (a non-bin word
                                // is never in the bin range, R11)
                                slowm = slowm * 2u + (sl ? 1u : 0u);
                                rawm = rawm * 2u + ((sl || bn) ? 0u : 1u);   // REL never runs in raw-words mode (host: MODE_RAW)
                            } else {
                                w[k] = quantize_b<T, MODE>(q, x[k], raw);
                                nraw += is_bin_word<T, MODE>(w[k], (W)qbias, raw) ? 0u : 1u;
                            }
                        }
                        memcpy(&v, w, 16);
                        *a = v;
                    }
                    if constexpr (MODE == MODE_REL) {
                        static_assert(2 * S_ * (16 / S_) == 32, "32 values per thread");
                        slowm = __brev(slowm);
                        if (!PFPL_REL_FASTW) nraw = __popc(rawm);
                        // the exact quantizer (rel_q, the format's definition) for the few
                        // uncertain values, spread over the warp's lanes: each
                        // lane lists its values (element id = 32 * lane + j) in this warp's
                        // share of M1 (zeroed only afterwards), then lane l takes entries
                        // l, l + 32, ...; above 256 entries every lane does its own
                        const uint32_t cnt = __popc(slowm);
                        const uint32_t inc = warp_incl_scan(cnt, lane);
                        const uint32_t total = __shfl_sync(PFPL_FULL, inc, 31);
                        auto exact_at = [&](int ol, int j) {
                            const int i = j / (16 / S_), k = j % (16 / S_);
                            const int t = 32 * warp + ol;
                            const int r = sizeof(T) == 4 ? t : 2 * t + (i >> 3);
                            W* const e = (W*)(wbuf + r * 128 + (((i & 7) ^ (r & 7)) << 4)) + k;
                            T xv;
                            memcpy(&xv, e, sizeof(T));
                            const W wv = quantize_b<T, MODE>(q, xv, raw);
                            *e = wv;
                            nraw += is_bin_word<T, MODE>(wv, (W)qbias, raw) ? 0u : 1u;
                        };
                        if (total && total <= 256) {
                            // this warp's own share of M1 (the part its threads zero next)
                            uint16_t* const list = (uint16_t*)(S.m1 + (2048 / NWC) * warp);
                            uint32_t o = inc - cnt;
#pragma unroll 1
                            for (uint32_t mm = slowm; mm; mm &= mm - 1u) list[o++] = (uint16_t)((lane << 5) | (__ffs(mm) - 1));
                            __syncwarp();
#pragma unroll 1
                            for (uint32_t g = lane; g < total; g += 32) {
                                const uint32_t id = list[g];
                                exact_at((int)(id >> 5), (int)(id & 31u));
                            }
                            __syncwarp();
                        } else if (total) {
#pragma unroll 1
                            for (uint32_t mm = slowm; mm; mm &= mm - 1u) exact_at(lane, __ffs(mm) - 1);
                            __syncwarp();
                        }
                    }
                    add_raw(nraw);
                    if (tid > 0) {
                        if constexpr (MODE == MODE_REL) {
                            bool sl;
                            qprev = q.rel_q_fast(pv, sl);
                            if (sl) qprev = quantize_b<T, MODE>(q, pv, raw);
                        } else {
                            qprev = quantize_b<T, MODE>(q, pv, raw);
                        }
                    }
                    fence_proxy_async();      // the stage is refilled by TMA after the next barrier
#pragma unroll
                    for (int i = 0; i < 2 * S_; ++i) {
                        const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                        const uint4 v = *(const uint4*)(buf + r * 128 + (((i & 7) ^ (r & 7)) << 4));
                        W x[16 / S_];
                        memcpy(x, &v, 16);
#pragma unroll
                        for (int k = 0; k < 16 / S_; ++k) {
                            const W r2 = rcode<MSR>((W)(x[k] - qprev));
                            qprev = x[k];
                            orv |= r2;
                            lo[i * (16 / S_) + k] = (uint32_t)r2;
                            hi[i * (16 / S_) + k] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r2 >> 32) : 0u;
                        }
                    }
                    done = true;
                }
            }
            if (done) {
            } else if (!TWO_PASS && m == CW) {
                if (tid > 0) {
                    T pv;
                    if (sizeof(T) == 4) {
                        const int r = tid - 1;
                        pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 12);
                    } else {
                        const int r = 2 * tid - 1;
                        pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 8);
                    }
                    qprev = quantize_b<T, MODE>(q, pv, raw);
                }
                uint32_t nraw = 0;
#pragma unroll
                for (int i = 0; i < 2 * S_; ++i) {
                    const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                    const uint4 v = *(const uint4*)(buf + r * 128 + (((i & 7) ^ (r & 7)) << 4));
                    T x[16 / S_];
                    memcpy(x, &v, 16);
#pragma unroll
                    for (int k = 0; k < 16 / S_; ++k) {
                        const W qw = quantize_b<T, MODE>(q, x[k], raw);
                        nraw += is_bin_word<T, MODE>(qw, (W)qbias, raw) ? 0u : 1u;
                        const W r2 = rcode<MSR>((W)(qw - qprev));
                        qprev = qw;
                        orv |= r2;
                        lo[i * (16 / S_) + k] = (uint32_t)r2;
                        hi[i * (16 / S_) + k] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r2 >> 32) : 0u;
                    }
                }
                add_raw(nraw);
            } else {
                // tail chunk: plain loads; R12 pads with the last value -> zero residuals
                const T* src = (const T*)p.in + c * (uint64_t)CW;
                if (tid > 0) qprev = quantize_b<T, MODE>(q, src[min(32 * tid - 1, (int)m - 1)], raw);
                uint32_t nraw = 0;
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                    const W qw = quantize_b<T, MODE>(q, src[min(32 * tid + i, (int)m - 1)], raw);
                    if (32 * tid + i < (int)m) nraw += is_bin_word<T, MODE>(qw, (W)qbias, raw) ? 0u : 1u;
                    const W r2 = rcode<MSR>((W)(qw - qprev));
                    qprev = qw;
                    orv |= r2;
                    lo[i] = (uint32_t)r2;
                    hi[i] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r2 >> 32) : 0u;
                }
                add_raw(nraw);
            }
        }
        // zero this thread's part of M1; REL after its quantizer, which uses this warp's
        // share as scratch (M1 is written only after the next CTA barrier)
        if constexpr (MODE == MODE_REL) {
#pragma unroll
            for (int i = 0; i < 2048 / 16 / NTC; ++i)
                ((uint4*)m1)[tid * (2048 / 16 / NTC) + i] = make_uint4(0, 0, 0, 0);
        }
// [stage] compute: active planes
        // this warp's active planes (warp-uniform tier; other warps may differ)
        const uint32_t ol = __reduce_or_sync(PFPL_FULL, (uint32_t)orv);
        const uint32_t oh = sizeof(W) == 8 ? __reduce_or_sync(PFPL_FULL, (uint32_t)((uint64_t)orv >> 32)) : 0u;
        const uint64_t wor = ((uint64_t)oh << 32) | ol;
        const int P = wor ? 64 - __clzll((long long)wor) : 0;

// [stage] level 1: plane counts + scans
        // ---- bit shuffle + level-1 zero elimination ----
        uint32_t ex[16];
        // level-1 code shape (PFPL_UNIFIED_L1): one copy per tier lets the compiler
        // free the registers of planes above the tier, which the smooth f32 ABS fields
        // (NYX: +13%) need; the shared windowed path keeps the hot code of the REL / NOA
        // quantizers and of f64 inside the instruction cache (Miranda f64 +17-25%,
        // rough f32 +7%; profiles/r02_encoder_budget.md)
        constexpr bool kUni = PFPL_UNIFIED_L1 == 1 ||
                              (PFPL_UNIFIED_L1 < 0 && !(sizeof(T) == 4 && (MODE == MODE_ABS || MODE == MODE_RAW)));
        // staged level 1 for REL (two-pass quantizer): Hurricane +18%, Miranda f64 +5%;
        // f64 ABS/NOA lose 6-8% to the later stage refill and keep the windowed path
        constexpr bool kStg = PFPL_STAGED_L1 && MODE == MODE_REL;
        uint8_t* const sbuf = smem + s * DATAB;
        if constexpr (kStg) {
            rze1_transpose<T>(lo, hi, P);
            rze1_stage_planes<T>(lo, hi, sbuf, tid, P);
            rze1_count_s<T>(sbuf, S, tid, lane, warp, wor, P);
        } else if constexpr (kUni) {
            rze1_transpose<T>(lo, hi, P);
            rze1_count_w<T>(lo, hi, S, lane, warp, wor, P, ex);
        } else {
            PFPL_TIER_DISPATCH(rze1_count, lo, hi, S, lane, warp, wor, ex);
        }
        named_sync(1, NTC);    // counts visible; every row of stage s consumed
        if (!kStg && tid == 0) {
            // refill stage s with the prefetched ticket; prefetch the next one
            // (the raw ticket is kept: subtracting the base here would wait for the
            // atomic's round trip right before the next barrier)
            const unsigned long long t = next - p.ticket_base;
            next = atomicAdd(p.ticket, 1ull);
            issue(s, t);
        }
// [stage] level 1: offsets + arena
        // Z1 offsets of this warp's segments: planes in decreasing bit order,
        // then warps (lane l owns bit l and 32+l)
        uint32_t offl, offh, n1, head;
        const uint32_t xsw = kX0 ? S.xh : 0u;     // kX0: warp 0's extra planes (every warp reads it)
        {
            uint32_t myl = 0, myh = 0, tl = 0, th = 0;
#pragma unroll
            for (int w = 0; w < NWC; ++w) {
                const uint32_t a = S.wcnt[w * B + lane] + ((kX0 && w == 0) ? (xsw >> lane) & 1u : 0u);
                const uint32_t b = B == 64 ? S.wcnt[w * B + 32 + lane] : 0u;
                if (w < warp) { myl += a; myh += b; }
                tl += a;
                th += b;
            }
            uint32_t sl = tl, sh = th;   // inclusive suffix sums over lanes
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
            head = slice_start<ARENA>(S, n1, it);
        }
        uint8_t* const z1 = arena + head % ARENA;
        if (kX0 && warp == 0 && ((xsw >> lane) & 1u)) {
            // extra plane `lane`: byte 0x01 at the start of warp 0's segment (offl of this
            // lane) and M1 byte 0x01
            z1[offl] = 1;
            m1[(B - 1 - lane) * (CW / 64)] = 1;
        }
// [stage] level 1: Z1/M1 scatter
        if constexpr (kStg) {
            rze1_scatter_s<T>(sbuf, z1, m1, tid, lane, wor, P, offl, offh);
            fence_proxy_async();      // the planes' stage is refilled by TMA after the barrier
        } else if constexpr (kUni) {
            rze1_scatter_w<T>(lo, hi, z1, m1, tid, lane, wor, P, ex, offl, offh);
        } else {
            PFPL_TIER_DISPATCH(rze1_scatter, lo, hi, z1, m1, tid, lane, wor, ex, offl, offh);
        }
        named_sync(1, NTC);    // Z1 and M1 complete
        if (kStg && tid == 0) {
            const unsigned long long t = next - p.ticket_base;
            next = atomicAdd(p.ticket, 1ull);
            issue(s, t);
        }
        uint8_t* const z2 = z1 + a16(n1) + PRE3;

// [stage] level 2
        // ---- level 2: repeated-byte elimination of M1 (2048 B -> M2 + Z2), P:131 ----
        const int slot = it % NQ;
        {
            uint32_t w2[NWD2], h2[NWD2];
            const uint32_t* m1w = (const uint32_t*)m1;
#pragma unroll
            for (int i = 0; i < NWD2; i += 4) {
                const uint4 v = *(const uint4*)(m1w + NWD2 * tid + i);
                w2[i] = v.x; w2[i + 1] = v.y; w2[i + 2] = v.z; w2[i + 3] = v.w;
            }
            const uint32_t pred = tid ? m1w[NWD2 * tid - 1] : 0u;
            uint32_t bits2 = 0, any = pred;
#pragma unroll
            for (int i = 0; i < NWD2; ++i) any |= w2[i];
            if (__any_sync(PFPL_FULL, any != 0)) {           // M1 of inactive planes is all zero
#pragma unroll
                for (int i = 0; i < NWD2; ++i) {
                    const uint32_t pw = i ? w2[i - 1] : pred;
                    h2[i] = nzbytes(w2[i] ^ __funnelshift_l(pw, w2[i], 8));
                    bits2 |= nib(h2[i]) << (4 * i);
                }
            }
            if (NB2 == 16) ((uint16_t*)S.m2)[tid] = (uint16_t)bits2;
            else ((uint32_t*)S.m2)[tid] = bits2;
            const uint32_t cnt2 = __popc(bits2);
            uint32_t inc = cnt2;
            if (__any_sync(PFPL_FULL, cnt2 != 0)) inc = warp_incl_scan(cnt2, lane);
            if (lane == 31) S.scan2[warp] = inc;
            named_sync(1, NTC);    // M2 complete, level-2 warp totals visible
            uint32_t base = 0, n2 = 0;
#pragma unroll
            for (int w = 0; w < NWC; ++w) {
                const uint32_t v = S.scan2[w];
                if (w < warp) base += v;
                n2 += v;
            }
            if (tid == 0) S.head = head + slice_bytes(n1, n2);
            if (cnt2 && n2 <= zroom(n1)) {        // else the chunk is raw (see zroom)
                uint32_t o = base + inc - cnt2;
#pragma unroll
                for (int i = 0; i < NWD2; ++i) o = scatter_word(z2, o, w2[i], h2[i]);
            }

// [stage] levels 3-4 + hand-off
            // ---- levels 3 and 4 on the 256-byte M2, size, raw decision,
            // aggregate, hand-off: one duty warp, rotating so no warp is always late ----
            if (warp != (int)(it % NWC)) {
                // this warp's Z2 bytes are written: release them to the IO warp (the
                // entry's phase completes only with the duty warp's arrival)
                q_arrive<PFPL_LANE_ARRIVE>(smem_u32(&S.mq_full[slot]), lane);
                continue;
            }
            const uint2 v = ((const uint2*)S.m2)[lane];
            uint32_t pm2 = __shfl_up_sync(PFPL_FULL, v.y, 1);
            if (lane == 0) pm2 = 0;
            const uint32_t h0 = nzbytes(v.x ^ __funnelshift_l(pm2, v.x, 8));
            const uint32_t h1 = nzbytes(v.y ^ __funnelshift_l(v.x, v.y, 8));
            const uint32_t m3 = nib(h0) | (nib(h1) << 4);
            const uint32_t cnt3 = __popc(m3);
            const uint32_t inc3 = warp_incl_scan(cnt3, lane);
            const uint32_t n3 = __shfl_sync(PFPL_FULL, inc3, 31);
            uint32_t pm3 = __shfl_up_sync(PFPL_FULL, m3, 1);
            if (lane == 0) pm3 = 0;
            const bool dif = m3 != pm3;
            const uint32_t M4 = __ballot_sync(PFPL_FULL, dif);
            const uint32_t n4 = __popc(M4);
            uint8_t* z3 = z2 - n3;
            scatter_word(z3, scatter_word(z3, inc3 - cnt3, v.x, h0), v.y, h1);
            uint8_t* z4 = z3 - n4;
            if (dif) z4[__popc(M4 & ((1u << lane) - 1u))] = (uint8_t)m3;
            if (lane < 4) z4[lane - 4] = (uint8_t)(M4 >> (8 * lane));
            const uint32_t size = 4 + n4 + n3 + n2 + n1;
            const uint32_t rawb = m * S_;
            const bool israw = size >= rawb;
            if (israw && lane == 0 && p.stats) atomicAdd(&p.stats[1], 1ull);
            const uint32_t stored = israw ? rawb : size;
            if (lane == 0) {
                const uint64_t EP = (uint64_t)p.epoch << 48;
                st_relaxed(&p.status[c], EP | ((c == 0 ? LB_P : LB_A) << 46) | stored);
                mbar_wait_wd(smem_u32(&S.mq_empty[slot]), ((it / NQ) & 1u) ^ 1u, 0x15);
                QEntry& e = S.q[slot];
                if (it >= NQ) S.rel = e.rend;       // chunk it-NQ's slice is released
                e.c = c;
                e.stored = stored;
                e.raw = israw ? 1u : 0u;
                e.start = israw ? head % ARENA : (uint32_t)(z4 - 4 - arena);
                e.plen = 4 + n4 + n3 + n2;
                e.z1 = head % ARENA;
                e.rend = head + slice_bytes(n1, n2);
            }
            __syncwarp();
            q_arrive<PFPL_LANE_ARRIVE>(smem_u32(&S.mq_full[slot]), lane);
        }
    }
// [stage] kernel exit
    // end of work: tell the IO warp (queue position `it` gets a terminal entry;
    // all compute warps leave at the same `it` and each arrives once)
    {
        const int slot = it % NQ;
        if (tid == 0) {
            mbar_wait_wd(smem_u32(&S.mq_empty[slot]), ((it / NQ) & 1u) ^ 1u, 0x16);
            S.q[slot].c = ~0ull;
        }
        __syncwarp();
        q_arrive<PFPL_LANE_ARRIVE>(smem_u32(&S.mq_full[slot]), lane);
    }
}

}  // namespace pfpl
