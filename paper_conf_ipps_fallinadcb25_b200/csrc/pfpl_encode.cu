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
// Arena slice of a chunk: [pos, pos + ZPRE + n1) with Z1 at pos + ZPRE and
// M4 | Z4 | Z3 | Z2 packed immediately before it (section order of R16).
#include <cuda.h>
#include "pfpl_device.cuh"

namespace pfpl {

constexpr int NIN = 2;               // input stages (TMA ring)
constexpr int DATAB = 16384;         // bytes per chunk
constexpr int ZPRE = 2352;           // >= 4 + 32 + 256 + 2048, multiple of 16
constexpr int NQ = 8;                // IO queue depth
constexpr int ARENA = 20800;         // circular payload arena (bytes, multiple of 16)

struct QEntry {
    unsigned long long c;
    uint32_t start, stored, raw, rend;
};

struct EncShared {
    uint8_t m1[2048];
    uint8_t m2[256];
    uint8_t wcnt[4][64];
    uint16_t off[4][64];
    unsigned long long wor[4];
    uint32_t scan[4];
    uint32_t n1, apos, head, tail;
    unsigned long long in_c[NIN];
    QEntry q[NQ];
    unsigned long long full[NIN], mq_full[NQ], mq_empty[NQ];
};
constexpr int ARENA_OFF = NIN * DATAB;
constexpr int SHARED_OFF = ARENA_OFF + ARENA + 64;
constexpr int ENC_SMEM = SHARED_OFF + (int)sizeof(EncShared);
static_assert(ENC_SMEM <= 57344, "4 CTAs per SM need <= 56 KiB of shared memory each");
static_assert(ZPRE + DATAB <= ARENA, "the arena must hold a worst-case chunk");

__device__ __forceinline__ void put_u64(uint8_t* p, uint64_t v) {
#pragma unroll
    for (int i = 0; i < 8; ++i) p[i] = (uint8_t)(v >> (8 * i));
}

__device__ void write_header(uint8_t* out, const EncParams& p, const QConst& qc) {
    out[0] = 'P'; out[1] = 'F'; out[2] = 'P'; out[3] = 'L';
    out[4] = 1; out[5] = (uint8_t)p.dtype; out[6] = (uint8_t)p.bound; out[7] = (uint8_t)qc.flags;
    put_u64(out + 8, p.n_total);
    put_u64(out + 16, d2u(p.eps));
    put_u64(out + 24, qc.qconst);
    put_u64(out + 32, d2u(qc.range));
    put_u64(out + 40, (uint64_t)kChunkBytes);
}

// scatter the bytes of w whose marker (0x01 per byte in hh) is set to z[o...]
__device__ __forceinline__ uint32_t scatter_word(uint8_t* z, uint32_t o, uint32_t w, uint32_t hh) {
    const uint32_t incl = hh * 0x01010101u;
    if (hh & 0x1u) z[o] = (uint8_t)w;
    if (hh & 0x100u) z[o + (incl & 0xFFu)] = (uint8_t)(w >> 8);
    if (hh & 0x10000u) z[o + ((incl >> 8) & 0xFFu)] = (uint8_t)(w >> 16);
    if (hh & 0x1000000u) z[o + ((incl >> 16) & 0xFFu)] = (uint8_t)(w >> 24);
    return o + (incl >> 24);
}

// ---------------------------------------------------------------------------
// bit shuffle + level-1 zero-byte elimination for one chunk.
// KL planes from the low 32 bits of the residuals, KH from the high 32 (f64).
// Plane word j holds bit b_j of the thread's 32 residuals; its shuffled
// position is plane p = B-1-b_j, byte p*CW/8 + 4*tid (reading R13).
// Z1 (plane-major, non-zero bytes in order) goes to the chunk's arena slice.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t ld_volatile_u32(const uint32_t* p) {
    return *(const volatile uint32_t*)p;
}

// reserve ZPRE + n1 bytes of the arena (compute warp 0, lane 0); waits only if
// the IO warp lags by more than the arena's capacity
__device__ __forceinline__ void reserve_arena(EncShared& S, uint32_t n1) {
    const uint32_t R = (ZPRE + n1 + 15u) & ~15u;
    uint32_t head = S.head;
    const uint32_t p0 = head % ARENA;
    if (p0 + R > (uint32_t)ARENA) head += ARENA - p0;      // do not wrap a slice
    while (head + R - ld_volatile_u32(&S.tail) > (uint32_t)ARENA) __nanosleep(64);
    S.apos = head % ARENA;
    S.head = head + R;
}

template <typename T, int KL, int KH>
__device__ __forceinline__ void rze1(uint32_t (&lo)[32], uint32_t (&hi)[32], uint8_t* arena,
                                     EncShared& S, int tid, int lane, int warp) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NW = Tr<T>::NW, NTC = Tr<T>::NT;
    constexpr int NP = KL + KH, NG = NP / 4;
    transpose_fwd<KL>(lo);
    if constexpr (KH > 0) transpose_fwd<KH>(hi);
    auto PW = [&](int j) -> uint32_t { return j < KL ? lo[j] : hi[j - KL]; };
    // per-plane non-zero byte counts (0..4), 4 planes per word, 8 bits each
    uint32_t ex[NG];
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        uint32_t v = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) v += ((nzbytes(PW(4 * g + i)) * 0x01010101u) >> 24) << (8 * i);
        uint32_t inc = v;
        if (__any_sync(PFPL_FULL, v != 0)) inc = warp_incl_scan(v, lane);
        ex[g] = inc - v;
        const int b0 = 4 * g < KL ? 4 * g : 32 + 4 * g - KL;
        if (lane == 31) *(uint32_t*)&S.wcnt[warp][b0] = inc;
    }
    named_sync(1, NTC);
    if (warp == 0) {
        // plane order = decreasing bit index; lane l owns bit l (and 32+l)
        uint32_t wl[NW], wh[NW], tl = 0, th = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            wl[w] = lane < KL ? S.wcnt[w][lane] : 0u;
            wh[w] = lane < KH ? S.wcnt[w][32 + lane] : 0u;
            tl += wl[w];
            th += wh[w];
        }
        uint32_t sl = tl, sh = th;   // inclusive suffix sums over lanes
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t a = __shfl_down_sync(PFPL_FULL, sl, d);
            const uint32_t b = KH > 0 ? __shfl_down_sync(PFPL_FULL, sh, d) : 0u;
            if (lane + d < 32) { sl += a; sh += b; }
        }
        const uint32_t tot_h = KH > 0 ? __shfl_sync(PFPL_FULL, sh, 0) : 0u;
        const uint32_t tot_l = __shfl_sync(PFPL_FULL, sl, 0);
        uint32_t run = tot_h + sl - tl;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            if (lane < KL) S.off[w][lane] = (uint16_t)run;
            run += wl[w];
        }
        if (KH > 0) {
            run = sh - th;
#pragma unroll
            for (int w = 0; w < NW; ++w) {
                if (lane < KH) S.off[w][32 + lane] = (uint16_t)run;
                run += wh[w];
            }
        }
        if (lane == 0) {
            S.n1 = tot_l + tot_h;
            reserve_arena(S, tot_l + tot_h);
        }
    }
    named_sync(1, NTC);
    uint8_t* z1 = arena + S.apos + ZPRE;
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const uint32_t w = PW(j);
        if (!__any_sync(PFPL_FULL, w != 0)) continue;          // warp-uniform skip of empty planes
        const int b = j < KL ? j : 32 + j - KL;
        const int pl = B - 1 - b;
        const uint32_t hj = nzbytes(w);
        const uint32_t o = S.off[warp][b] + ((ex[j / 4] >> (8 * (j % 4))) & 0xFFu);
        scatter_word(z1, o, w, hj);
        const uint32_t nb = nib(hj);
        const uint32_t nb2 = __shfl_xor_sync(PFPL_FULL, nb, 1);
        if (!(lane & 1)) S.m1[pl * (CW / 64) + (tid >> 1)] = (uint8_t)(nb | (nb2 << 4));
    }
}

template <typename T, int MODE, bool MSR>
__global__ void __launch_bounds__(Tr<T>::NT + 32, 4)
encode_kernel(const EncParams p, const __grid_constant__ CUtensorMap tmap) {
    typedef typename Tr<T>::W W;
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NTC = Tr<T>::NT, NWC = Tr<T>::NW, S_ = Tr<T>::S;
    constexpr int NB2 = 2048 / NTC;     // level-2 bytes per compute thread (16 or 32)
    constexpr int NWD2 = NB2 / 4;

    extern __shared__ __align__(1024) uint8_t smem[];
    EncShared& S = *reinterpret_cast<EncShared*>(smem + SHARED_OFF);
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
        if (smem_u32(smem) & 1023u) __trap();       // TMA SWIZZLE_128B needs 1024-byte alignment
        for (int s = 0; s < NIN; ++s) mbar_init(smem_u32(&S.full[s]), 1);
        for (int k = 0; k < NQ; ++k) {
            mbar_init(smem_u32(&S.mq_full[k]), 1);
            mbar_init(smem_u32(&S.mq_empty[k]), 1);
        }
        S.head = 0;
        S.tail = 0;
        fence_barrier_init();
        prefetch_tmap(&tmap);
    }
    __syncthreads();
    if (tid == 0) {
        for (int s = 0; s < NIN; ++s) issue(s, atomicAdd(p.ticket, 1ull) - p.ticket_base);
        next = atomicAdd(p.ticket, 1ull) - p.ticket_base;
    }

    if (warp == NWC) {
        // =========================== IO warp ===========================
        const uint64_t EP = (uint64_t)p.epoch << 48;
        for (uint32_t k = 0;; ++k) {
            const int slot = k % NQ;
            mbar_wait(smem_u32(&S.mq_full[slot]), (k / NQ) & 1u);
            const QEntry e = S.q[slot];
            if (e.c >= C) break;
            const uint64_t c = e.c;
            // ---- decoupled look-back; compute published the aggregate ----
            uint64_t excl = 0;
            if (c > 0) {
                int64_t look = (int64_t)c - 1;
                for (;;) {
                    const int64_t idx = look - lane;
                    uint64_t val = 0, flag = LB_P;
                    if (idx >= 0) {
                        for (;;) {
                            const uint64_t d = ld_relaxed(&p.status[idx]);
                            flag = ((uint32_t)(d >> 48) == p.epoch) ? ((d >> 46) & 3u) : 0u;
                            if (flag) { val = d & LB_VAL; break; }
                            __nanosleep(32);
                        }
                    }
                    const uint32_t pm = __ballot_sync(PFPL_FULL, flag == LB_P);
                    if (pm) {
                        const int first = __ffs(pm) - 1;
                        excl += warp_sum64(lane <= first ? val : 0ull);
                        break;
                    }
                    excl += warp_sum64(val);
                    look -= 32;
                }
                if (lane == 0) st_relaxed(&p.status[c], EP | (LB_P << 46) | (excl + e.stored));
            }
            const uint64_t dst = p.payload_off + excl;
            if (lane == 0) {
                p.table[c] = e.stored;
                if (c == C - 1) p.result[0] = dst + e.stored;
                if (c == 0 && p.write_header) write_header(p.out, p, qc);
            }
            if (dst + e.stored <= p.cap) {
                const uint8_t* src = arena + e.start;
                if (e.raw) {
                    // raw chunk (R17): stage the original bytes in this chunk's
                    // arena slice (always large enough: slice >= payload >= raw bytes)
                    uint8_t* stg = arena + e.start;
                    const uint8_t* g = (const uint8_t*)p.in + c * (uint64_t)kChunkBytes;
                    for (uint32_t i = lane; i < e.stored / 16; i += 32) ((uint4*)stg)[i] = ldg_nc_v4(g + 16 * i);
                    for (uint32_t i = (e.stored / 16) * 4 + lane; i < e.stored / 4; i += 32)
                        ((uint32_t*)stg)[i] = ((const uint32_t*)g)[i];
                    __syncwarp();
                }
                // 16-byte aligned stores for the body (coalesced even for
                // unaligned compressed data), bytes for the head and tail
                uint8_t* o = p.out + dst;
                const uint32_t mis = (uint32_t)((uintptr_t)o & 15u);
                uint32_t head = (16u - mis) & 15u;
                if (head > e.stored) head = e.stored;
                const uint32_t body = (e.stored - head) >> 4;
                const uint32_t tail0 = head + (body << 4);
                if ((uint32_t)lane < head) o[lane] = src[lane];
                if ((uint32_t)lane < e.stored - tail0) o[tail0 + lane] = src[tail0 + lane];
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
            __syncwarp();
            if (lane == 0) {
                *(volatile uint32_t*)&S.tail = e.rend;     // release the arena slice
                mbar_arrive(smem_u32(&S.mq_empty[slot]));
            }
        }
        return;
    }

    // ============================ compute warps ============================
    QF<T> q;
    q.load(qc);
    const bool raw = (qc.flags & HF_RAWWORDS) != 0;
    uint32_t it = 0;
    for (;; ++it) {
        const int s = it % NIN;
        mbar_wait(smem_u32(&S.full[s]), (it / NIN) & 1u);
        const uint64_t c = S.in_c[s];
        if (c >= C) break;
        const uint8_t* buf = smem + s * DATAB;
        const uint32_t m = (uint32_t)min((uint64_t)CW, p.n - c * (uint64_t)CW);

        // zero this thread's part of M1
#pragma unroll
        for (int i = 0; i < 2048 / 16 / NTC; ++i)
            ((uint4*)S.m1)[tid * (2048 / 16 / NTC) + i] = make_uint4(0, 0, 0, 0);

        // ---- quantize + verify, delta, residual code ----
        uint32_t lo[32], hi[32];
        W orv = 0;
        {
            W qprev = 0;
            if (m == CW) {
                if (tid > 0) {
                    T pv;
                    if (sizeof(T) == 4) {
                        const int r = tid - 1;
                        pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 12);
                    } else {
                        const int r = 2 * tid - 1;
                        pv = *(const T*)(buf + r * 128 + ((7 ^ (r & 7)) << 4) + 8);
                    }
                    qprev = quantize<T, MODE>(q, pv, raw);
                }
#pragma unroll
                for (int i = 0; i < 2 * S_; ++i) {
                    const int r = sizeof(T) == 4 ? tid : 2 * tid + (i >> 3);
                    const uint4 v = *(const uint4*)(buf + r * 128 + (((i & 7) ^ (r & 7)) << 4));
                    T x[16 / S_];
                    memcpy(x, &v, 16);
#pragma unroll
                    for (int k = 0; k < 16 / S_; ++k) {
                        const W qw = quantize<T, MODE>(q, x[k], raw);
                        const W r2 = rcode<MSR>((W)(qw - qprev));
                        qprev = qw;
                        orv |= r2;
                        lo[i * (16 / S_) + k] = (uint32_t)r2;
                        hi[i * (16 / S_) + k] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r2 >> 32) : 0u;
                    }
                }
            } else {
                // tail chunk: plain loads; R12 pads with the last value -> zero residuals
                const T* src = (const T*)p.in + c * (uint64_t)CW;
                if (tid > 0) qprev = quantize<T, MODE>(q, src[min(32 * tid - 1, (int)m - 1)], raw);
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                    const W qw = quantize<T, MODE>(q, src[min(32 * tid + i, (int)m - 1)], raw);
                    const W r2 = rcode<MSR>((W)(qw - qprev));
                    qprev = qw;
                    orv |= r2;
                    lo[i] = (uint32_t)r2;
                    hi[i] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r2 >> 32) : 0u;
                }
            }
        }
        {
            const uint32_t ol = __reduce_or_sync(PFPL_FULL, (uint32_t)orv);
            const uint32_t oh = sizeof(W) == 8 ? __reduce_or_sync(PFPL_FULL, (uint32_t)((uint64_t)orv >> 32)) : 0u;
            if (lane == 0) S.wor[warp] = ((unsigned long long)oh << 32) | ol;
        }
        named_sync(1, NTC);    // rows of stage s consumed, M1 zeroed, active planes known
        if (tid == 0) {
            // refill stage s with the prefetched ticket; prefetch the next one
            const unsigned long long t = next;
            next = atomicAdd(p.ticket, 1ull) - p.ticket_base;
            issue(s, t);
        }
        unsigned long long bor = 0;
#pragma unroll
        for (int w = 0; w < NWC; ++w) bor |= S.wor[w];
        const int P = bor ? 64 - __clzll((long long)bor) : 0;

        // ---- bit shuffle + level-1 zero elimination (block-uniform tier) ----
        if (P == 0) {
            if (tid == 0) {
                S.n1 = 0;
                reserve_arena(S, 0);
            }
        } else if (B == 32 || P <= 32) {
            if (P <= 4) rze1<T, 4, 0>(lo, hi, arena, S, tid, lane, warp);
            else if (P <= 8) rze1<T, 8, 0>(lo, hi, arena, S, tid, lane, warp);
            else if (P <= 16) rze1<T, 16, 0>(lo, hi, arena, S, tid, lane, warp);
            else rze1<T, 32, 0>(lo, hi, arena, S, tid, lane, warp);
        } else {
            if (P <= 36) rze1<T, 32, 4>(lo, hi, arena, S, tid, lane, warp);
            else if (P <= 40) rze1<T, 32, 8>(lo, hi, arena, S, tid, lane, warp);
            else if (P <= 48) rze1<T, 32, 16>(lo, hi, arena, S, tid, lane, warp);
            else rze1<T, 32, 32>(lo, hi, arena, S, tid, lane, warp);
        }
        named_sync(1, NTC);    // Z1 and M1 complete

        // ---- level 2: repeated-byte elimination of M1 (2048 B -> M2 + Z2) ----
        const uint32_t n1 = S.n1;
        uint8_t* const z1 = arena + S.apos + ZPRE;
        uint32_t n2 = 0;
        {
            uint32_t w2[NWD2], h2[NWD2];
            const uint32_t* m1w = (const uint32_t*)S.m1;
#pragma unroll
            for (int i = 0; i < NWD2; i += 4) {
                const uint4 v = *(const uint4*)(m1w + NWD2 * tid + i);
                w2[i] = v.x; w2[i + 1] = v.y; w2[i + 2] = v.z; w2[i + 3] = v.w;
            }
            const uint32_t pred = tid ? m1w[NWD2 * tid - 1] : 0u;
            uint32_t bits2 = 0;
#pragma unroll
            for (int i = 0; i < NWD2; ++i) {
                const uint32_t pw = i ? w2[i - 1] : pred;
                h2[i] = nzbytes(w2[i] ^ __funnelshift_l(pw, w2[i], 8));
                bits2 |= nib(h2[i]) << (4 * i);
            }
            const uint32_t cnt2 = __popc(bits2);
            uint32_t inc = cnt2;
            if (__any_sync(PFPL_FULL, cnt2 != 0)) inc = warp_incl_scan(cnt2, lane);
            if (lane == 31) S.scan[warp] = inc;
            named_sync(1, NTC);
            uint32_t base = 0;
#pragma unroll
            for (int w = 0; w < NWC; ++w) {
                const uint32_t v = S.scan[w];
                if (w < warp) base += v;
                n2 += v;
            }
            if (cnt2) {
                uint8_t* z2 = z1 - n2;
                uint32_t o = base + inc - cnt2;
#pragma unroll
                for (int i = 0; i < NWD2; ++i) o = scatter_word(z2, o, w2[i], h2[i]);
            }
            if (NB2 == 16) ((uint16_t*)S.m2)[tid] = (uint16_t)bits2;
            else ((uint32_t*)S.m2)[tid] = bits2;
        }
        if (warp != 0) {
            named_arrive(2, NTC);
            continue;
        }
        named_sync(2, NTC);

        // ---- levels 3 and 4, size, raw decision, hand-off to the IO warp (warp 0) ----
        {
            const uint2 v = ((const uint2*)S.m2)[lane];
            const uint32_t pred = lane ? ((const uint32_t*)S.m2)[2 * lane - 1] : 0u;
            const uint32_t h0 = nzbytes(v.x ^ __funnelshift_l(pred, v.x, 8));
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
            uint8_t* z3 = z1 - n2 - n3;
            scatter_word(z3, scatter_word(z3, inc3 - cnt3, v.x, h0), v.y, h1);
            uint8_t* z4 = z3 - n4;
            if (dif) z4[__popc(M4 & ((1u << lane) - 1u))] = (uint8_t)m3;
            if (lane < 4) z4[lane - 4] = (uint8_t)(M4 >> (8 * lane));
            const uint32_t size = 4 + n4 + n3 + n2 + n1;
            const uint32_t rawb = m * S_;
            const bool israw = size >= rawb;
            const uint32_t stored = israw ? rawb : size;
            __syncwarp();
            if (lane == 0) {
                const uint64_t EP = (uint64_t)p.epoch << 48;
                st_relaxed(&p.status[c], EP | ((c == 0 ? LB_P : LB_A) << 46) | stored);
                const int slot = it % NQ;
                mbar_wait(smem_u32(&S.mq_empty[slot]), ((it / NQ) & 1u) ^ 1u);
                QEntry& e = S.q[slot];
                e.c = c;
                e.stored = stored;
                e.raw = israw ? 1u : 0u;
                e.start = israw ? S.apos : (uint32_t)(z4 - 4 - arena);
                e.rend = S.head;
                mbar_arrive(smem_u32(&S.mq_full[slot]));
            }
        }
    }
    // end of work: tell the IO warp (the ring position `it` holds the first c >= C)
    if (tid == 0) {
        const int slot = it % NQ;
        mbar_wait(smem_u32(&S.mq_empty[slot]), ((it / NQ) & 1u) ^ 1u);
        S.q[slot].c = ~0ull;
        mbar_arrive(smem_u32(&S.mq_full[slot]));
    }
}

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
template <typename T, int MODE, bool MSR>
static void* enc_fn() { return (void*)encode_kernel<T, MODE, MSR>; }

static void* pick_enc(int dtype, int mode, bool ms) {
#define PFPL_E(T)                                                                  \
    switch (mode) {                                                                \
        case MODE_ABS: return ms ? enc_fn<T, MODE_ABS, true>() : enc_fn<T, MODE_ABS, false>(); \
        case MODE_REL: return ms ? enc_fn<T, MODE_REL, true>() : enc_fn<T, MODE_REL, false>(); \
        case MODE_RAW: return ms ? enc_fn<T, MODE_RAW, true>() : enc_fn<T, MODE_RAW, false>(); \
        default: return ms ? enc_fn<T, MODE_NOA, true>() : enc_fn<T, MODE_NOA, false>();       \
    }
    if (dtype == 0) { PFPL_E(float) } else { PFPL_E(double) }
#undef PFPL_E
}

static int enc_threads(int dtype) { return (dtype == 0 ? Tr<float>::NT : Tr<double>::NT) + 32; }

static cudaError_t prepare_enc(void* fn) {
    return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, ENC_SMEM);
}

int encode_grid(int dtype, int mode, bool ms, uint64_t C) {
    static int cache[2][4][2] = {};
    int& g = cache[dtype][mode][ms];
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        void* fn = pick_enc(dtype, mode, ms);
        prepare_enc(fn);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, enc_threads(dtype), ENC_SMEM);
        g = sms * (per > 0 ? per : 1);
    }
    return (int)(C < (uint64_t)g ? C : (uint64_t)g);
}

int encode_stages() { return NIN; }

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn get_encode_tiled() {
    static EncodeTiledFn fn = nullptr;
    if (!fn) {
        void* f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (EncodeTiledFn)f;
    }
    return fn;
}

// 2-D view of the input as 128-byte rows of 32 u32 words; a chunk = 128 rows.
cudaError_t make_row_tmap(const void* base, uint64_t bytes, CUtensorMap* map) {
    memset(map, 0, sizeof(*map));
    const uint64_t rows = bytes / 128;
    if (rows < 128) return cudaSuccess;            // no full chunk: map never used
    EncodeTiledFn fn = get_encode_tiled();
    if (!fn) return cudaErrorNotSupported;
    cuuint64_t dims[2] = {32, rows};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {32, 128};
    cuuint32_t es[2] = {1, 1};
    CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<void*>(base), dims, strides,
                    box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

cudaError_t launch_encode(int dtype, int mode, bool ms, const EncParams& p, int grid,
                          cudaStream_t s) {
    alignas(64) CUtensorMap map;
    cudaError_t e = make_row_tmap(p.in, p.n * (dtype == 0 ? 4u : 8u), &map);
    if (e != cudaSuccess) return e;
    void* fn = pick_enc(dtype, mode, ms);
    static bool prepared[2][4][2] = {};
    if (!prepared[dtype][mode][ms]) {
        e = prepare_enc(fn);
        if (e != cudaSuccess) return e;
        prepared[dtype][mode][ms] = true;
    }
    void* args[] = {(void*)&p, (void*)&map};
    return cudaLaunchKernel(fn, dim3(grid), dim3(enc_threads(dtype)), args, ENC_SMEM, s);
}

}  // namespace pfpl
