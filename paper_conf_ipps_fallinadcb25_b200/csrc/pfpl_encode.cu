// pfpl_encode.cu -- fused PFPL chunk encoder for sm_100a.
//
// One CTA per 16 KiB chunk at a time, persistent CTAs that take chunks
// from an atomic ticket ("dynamically assign the chunks"), all stages
// fused so the input is read once and the output written once:
//   load 16 KiB (16-byte coalesced, padded smem rows) -> quantize + verify
//    -> delta + negabinary -> bit-plane transpose in
//   registers -> zero-byte elimination with packed warp scans
//    -> 3 levels of repeated-byte elimination -> raw
//   fallback -> decoupled look-back for the byte offset ->
//   realigned 16-byte stores of the payload.
// Thread t owns elements 32t..32t+31, so its 32 bits of every bit plane form
// one aligned 32-bit word of the shuffled chunk.
#include "pfpl_device.cuh"

namespace pfpl {

constexpr int ZOFF = 2352;   // Z1 starts here in the assembly buffer; M4|Z4|Z3|Z2 precede it

template <typename T> struct EncGeom {
    static constexpr int NT = Tr<T>::NT, S = Tr<T>::S;
    static constexpr int ROWB = 32 * S + 16;                       // padded 32-element row
    static constexpr int STAGE_IN = NT * ROWB;
    static constexpr int STAGE = (STAGE_IN > ZOFF + 16384 ? STAGE_IN : ZOFF + 16384) + 32;
};

// copy len bytes from shared memory (any alignment) to global memory (any
// alignment) with 16-byte aligned vector stores for the body (P:166
// "coalesced memory accesses ... even when writing unaligned compressed data")
__device__ __forceinline__ void copy_smem_to_global(uint8_t* dst, const uint8_t* src, uint32_t len,
                                                    int tid, int nt) {
    const uint32_t mis = (uint32_t)((uintptr_t)dst & 15u);
    uint32_t head = (16u - mis) & 15u;
    if (head > len) head = len;
    const uint32_t body = (len - head) >> 4;
    const uint32_t tail0 = head + (body << 4);
    if ((uint32_t)tid < head) dst[tid] = src[tid];
    if ((uint32_t)tid < len - tail0) dst[tail0 + tid] = src[tail0 + tid];
    for (uint32_t j = tid; j < body; j += nt) {
        const uint8_t* s = src + head + (j << 4);
        const uint32_t a = (uint32_t)__cvta_generic_to_shared(s) & 3u;
        const uint32_t* sw = (const uint32_t*)(s - a);
        uint32_t w0 = sw[0], w1 = sw[1], w2 = sw[2], w3 = sw[3], w4 = sw[4];
        const uint32_t sh = a * 8u;
        uint4 v;
        v.x = __funnelshift_r(w0, w1, sh);
        v.y = __funnelshift_r(w1, w2, sh);
        v.z = __funnelshift_r(w2, w3, sh);
        v.w = __funnelshift_r(w3, w4, sh);
        *(uint4*)(dst + head + (j << 4)) = v;
    }
}

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

// ---------------------------------------------------------------------------
// level-1 zero-byte elimination over the active bit planes.
// KL planes from the low 32 bits of the residuals, KH from the high 32 (f64).
// Plane j of the thread holds bit b_j of its 32 residuals; shuffled position
// of that word: plane p = B-1-b_j, byte offset p*CW/8 + 4*tid (reading R13).
// ---------------------------------------------------------------------------
template <typename T, int KL, int KH>
__device__ __forceinline__ void rze1(const uint32_t (&lo)[32], const uint32_t (&hi)[32],
                                     uint8_t* s_z1, uint8_t* s_m1, uint8_t (*s_wcnt)[64],
                                     uint16_t (*s_off)[64], uint32_t* s_n1, int tid, int lane,
                                     int warp) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NW = Tr<T>::NW;
    constexpr int NP = KL + KH;
    constexpr int NG = NP / 4;
    uint32_t pw[NP];
    {
        uint32_t t[KL];
        transpose_fwd<KL>(lo, t);
#pragma unroll
        for (int j = 0; j < KL; ++j) pw[j] = t[j];
    }
    if constexpr (KH > 0) {
        uint32_t t[KH];
        transpose_fwd<KH>(hi, t);
#pragma unroll
        for (int j = 0; j < KH; ++j) pw[KL + j] = t[j];
    }
    uint32_t h[NP];
#pragma unroll
    for (int j = 0; j < NP; ++j) h[j] = nzbytes(pw[j]);
    // per-plane counts (0..4) packed 4 planes per word, 8 bits each (warp totals <= 128)
    uint32_t ex[NG];
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        uint32_t v = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) v |= ((h[4 * g + i] * 0x01010101u) >> 24) << (8 * i);
        uint32_t inc = warp_incl_scan(v, lane);
        ex[g] = inc - v;
        const int b0 = 4 * g < KL ? 4 * g : 32 + 4 * g - KL;
        if (lane == 31) *(uint32_t*)&s_wcnt[warp][b0] = inc;
    }
    __syncthreads();
    if (warp == 0) {
        // plane order = decreasing bit index; lane l owns bit l (and 32+l)
        uint32_t wl[NW], wh[NW], tl = 0, th = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            wl[w] = lane < KL ? s_wcnt[w][lane] : 0u;
            wh[w] = lane < KH ? s_wcnt[w][32 + lane] : 0u;
            tl += wl[w];
            th += wh[w];
        }
        uint32_t sl = tl, sh = th;   // inclusive suffix sums over lanes
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            uint32_t a = __shfl_down_sync(PFPL_FULL, sl, d);
            uint32_t b = __shfl_down_sync(PFPL_FULL, sh, d);
            if (lane + d < 32) { sl += a; sh += b; }
        }
        const uint32_t tot_h = __shfl_sync(PFPL_FULL, sh, 0);
        const uint32_t tot_l = __shfl_sync(PFPL_FULL, sl, 0);
        uint32_t run = tot_h + sl - tl;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            if (lane < KL) s_off[w][lane] = (uint16_t)run;
            run += wl[w];
        }
        run = sh - th;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            if (lane < KH) s_off[w][32 + lane] = (uint16_t)run;
            run += wh[w];
        }
        if (lane == 0) *s_n1 = tot_l + tot_h;
    }
    __syncthreads();
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const int b = j < KL ? j : 32 + j - KL;
        const int pl = B - 1 - b;
        const uint32_t hj = h[j], w = pw[j];
        const uint32_t o = s_off[warp][b] + ((ex[j / 4] >> (8 * (j % 4))) & 0xFFu);
        const uint32_t incl = hj * 0x01010101u;
        if (hj & 0x1u) s_z1[o] = (uint8_t)w;
        if (hj & 0x100u) s_z1[o + (incl & 0xFFu)] = (uint8_t)(w >> 8);
        if (hj & 0x10000u) s_z1[o + ((incl >> 8) & 0xFFu)] = (uint8_t)(w >> 16);
        if (hj & 0x1000000u) s_z1[o + ((incl >> 16) & 0xFFu)] = (uint8_t)(w >> 24);
        const uint32_t nb = nib(hj);
        const uint32_t nb2 = __shfl_xor_sync(PFPL_FULL, nb, 1);
        if (!(lane & 1)) s_m1[pl * (CW / 64) + (tid >> 1)] = (uint8_t)(nb | (nb2 << 4));
    }
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

template <typename T, int MODE, bool MSR>
__global__ void __launch_bounds__(Tr<T>::NT) encode_kernel(const EncParams p) {
    typedef typename Tr<T>::W W;
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NT = Tr<T>::NT, NW = Tr<T>::NW, S = Tr<T>::S;
    constexpr int ROWB = EncGeom<T>::ROWB;
    constexpr int NB2 = 2048 / NT;     // level-2 bytes per thread (16 or 32)
    constexpr int NWD2 = NB2 / 4;

    __shared__ __align__(16) uint8_t s_stage[EncGeom<T>::STAGE];
    __shared__ __align__(16) uint8_t s_m1[2048];
    __shared__ __align__(16) uint8_t s_m2[256];
    __shared__ __align__(16) uint8_t s_wcnt[NW][64];
    __shared__ __align__(16) uint16_t s_off[NW][64];
    __shared__ uint32_t s_scan[NW];
    __shared__ W s_wor[NW];
    __shared__ unsigned long long s_c;
    __shared__ uint32_t s_n1, s_n2, s_start, s_stored, s_write;
    __shared__ unsigned long long s_dst;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    QConst qc = p.qc;
    if (MODE == MODE_NOA) qc = *p.qc_dev;
    QF<T> q;
    q.load(qc);
    const bool raw = (qc.flags & HF_RAWWORDS) != 0;
    uint8_t* const s_z1 = s_stage + ZOFF;

    for (;;) {
        if (tid == 0) s_c = atomicAdd(p.ticket, 1ull) - p.ticket_base;
        __syncthreads();
        const uint64_t c = s_c;
        if (c >= p.C) break;
        const uint32_t m = (uint32_t)min((uint64_t)CW, p.n - c * (uint64_t)CW);
        if (c == 0 && p.write_header && tid == 0) write_header(p.out, p, qc);

        // ---- zero M1, load the chunk into padded rows ----
        for (int i = tid; i < 2048 / 16; i += NT) ((uint4*)s_m1)[i] = make_uint4(0, 0, 0, 0);
        const uint8_t* src = (const uint8_t*)p.in + c * (uint64_t)kChunkBytes;
        if (m == CW) {
#pragma unroll
            for (int i = 0; i < 1024 / NT; ++i) {
                const int k = i * NT + tid;
                const uint4 v = ldg_nc_v4(src + 16 * k);
                *(uint4*)(s_stage + (k / (2 * S)) * ROWB + (k % (2 * S)) * 16) = v;
            }
        } else {
            // R12: pad a short chunk with its last value -> identical words -> zero residuals
            for (int e = tid; e < CW; e += NT) {
                const int se = e < (int)m ? e : (int)m - 1;
                *(T*)(s_stage + (e / 32) * ROWB + (e % 32) * S) = ((const T*)src)[se];
            }
        }
        __syncthreads();

        // ---- quantize + verify ----
        W qv[32];
        {
            const uint4* row = (const uint4*)(s_stage + tid * ROWB);
#pragma unroll
            for (int j = 0; j < 2 * S; ++j) {
                const uint4 v = row[j];
                T x[16 / S];
                memcpy(x, &v, 16);
#pragma unroll
                for (int i = 0; i < 16 / S; ++i) qv[j * (16 / S) + i] = quantize<T, MODE>(q, x[i], raw);
            }
        }
        // ---- delta (predecessor of the first value is 0) + residual code ----
        W qprev = __shfl_up_sync(PFPL_FULL, qv[31], 1);
        if (lane == 0) {
            qprev = 0;
            if (tid > 0) qprev = quantize<T, MODE>(q, *(const T*)(s_stage + (tid - 1) * ROWB + 31 * S), raw);
        }
        uint32_t lo[32], hi[32];
        W orv = 0;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
            const W r = rcode<MSR>((W)(qv[i] - (i ? qv[i - 1] : qprev)));
            orv |= r;
            lo[i] = (uint32_t)r;
            hi[i] = sizeof(W) == 8 ? (uint32_t)((uint64_t)r >> 32) : 0u;
        }
        {
            const uint32_t ol = __reduce_or_sync(PFPL_FULL, (uint32_t)orv);
            const uint32_t oh = sizeof(W) == 8 ? __reduce_or_sync(PFPL_FULL, (uint32_t)((uint64_t)orv >> 32)) : 0u;
            if (lane == 0) s_wor[warp] = (W)((sizeof(W) == 8 ? ((uint64_t)oh << 32) : 0ull) | ol);
        }
        __syncthreads();   // all rows consumed; active planes known
        uint64_t bor = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) bor |= (uint64_t)s_wor[w];
        const int P = bor ? 64 - __clzll((long long)bor) : 0;   // number of active low bits

        // ---- bit shuffle + level-1 zero elimination (block-uniform tier) ----
        if (P == 0) {
            if (tid == 0) s_n1 = 0;
        } else if (B == 32 || P <= 32) {
            if (P <= 4) rze1<T, 4, 0>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 8) rze1<T, 8, 0>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 16) rze1<T, 16, 0>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else rze1<T, 32, 0>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
        } else {
            if (P <= 36) rze1<T, 32, 4>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 40) rze1<T, 32, 8>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 48) rze1<T, 32, 16>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else rze1<T, 32, 32>(lo, hi, s_z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
        }
        __syncthreads();

        // ---- level 2: repeated-byte elimination of M1 (2048 B -> M2 256 B + Z2) ----
        {
            uint32_t w2[NWD2], h2[NWD2];
            const uint32_t* m1w = (const uint32_t*)s_m1;
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
            const uint32_t inc = warp_incl_scan(cnt2, lane);
            if (lane == 31) s_scan[warp] = inc;
            __syncthreads();
            uint32_t base = 0, n2 = 0;
#pragma unroll
            for (int w = 0; w < NW; ++w) {
                const uint32_t v = s_scan[w];
                if (w < warp) base += v;
                n2 += v;
            }
            if (cnt2) {
                uint8_t* z2 = s_z1 - n2;
                uint32_t o = base + inc - cnt2;
#pragma unroll
                for (int i = 0; i < NWD2; ++i) o = scatter_word(z2, o, w2[i], h2[i]);
            }
            if (NB2 == 16) ((uint16_t*)s_m2)[tid] = (uint16_t)bits2;
            else ((uint32_t*)s_m2)[tid] = bits2;
            if (tid == 0) s_n2 = n2;
        }
        __syncthreads();

        // ---- levels 3 and 4, size, raw decision, look-back (warp 0) ----
        if (warp == 0) {
            const uint32_t n1 = s_n1, n2 = s_n2;
            const uint2 v = ((const uint2*)s_m2)[lane];
            const uint32_t pred = lane ? ((const uint32_t*)s_m2)[2 * lane - 1] : 0u;
            const uint32_t h0 = nzbytes(v.x ^ __funnelshift_l(pred, v.x, 8));
            const uint32_t h1 = nzbytes(v.y ^ __funnelshift_l(v.x, v.y, 8));
            const uint32_t m3 = nib(h0) | (nib(h1) << 4);
            const uint32_t cnt3 = __popc(m3);
            const uint32_t inc3 = warp_incl_scan(cnt3, lane);
            const uint32_t n3 = __shfl_sync(PFPL_FULL, inc3, 31);
            uint8_t* z3 = s_z1 - n2 - n3;
            scatter_word(z3, scatter_word(z3, inc3 - cnt3, v.x, h0), v.y, h1);
            // level 4 on M3 (32 bytes, one per lane)
            uint32_t pm3 = __shfl_up_sync(PFPL_FULL, m3, 1);
            if (lane == 0) pm3 = 0;
            const bool dif = m3 != pm3;
            const uint32_t M4 = __ballot_sync(PFPL_FULL, dif);
            const uint32_t n4 = __popc(M4);
            uint8_t* z4 = s_z1 - n2 - n3 - n4;
            if (dif) z4[__popc(M4 & ((1u << lane) - 1u))] = (uint8_t)m3;
            if (lane < 4) z4[lane - 4] = (uint8_t)(M4 >> (8 * lane));
            const uint32_t size = 4 + n4 + n3 + n2 + n1;
            const uint32_t rawb = m * S;
            const bool israw = size >= rawb;
            const uint32_t stored = israw ? rawb : size;
            // decoupled look-back
            const uint64_t EP = (uint64_t)p.epoch << 48;
            if (lane == 0) st_relaxed(&p.status[c], EP | ((c == 0 ? LB_P : LB_A) << 46) | stored);
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
                if (lane == 0) st_relaxed(&p.status[c], EP | (LB_P << 46) | (excl + stored));
            }
            if (lane == 0) {
                const uint64_t dst = p.payload_off + excl;
                p.table[c] = stored;
                if (c == p.C - 1) p.result[0] = dst + stored;
                s_dst = dst;
                s_stored = stored;
                s_start = israw ? 0u : (uint32_t)(ZOFF - 4 - n4 - n3 - n2);
                s_write = (dst + stored <= p.cap) ? (israw ? 2u : 1u) : 0u;
            }
        }
        __syncthreads();
        const uint32_t wr = s_write;
        if (wr == 2) {
            // raw chunk: original input bytes (R17); stage them aligned
            const uint32_t nb = m * S;
            for (uint32_t i = tid; i < nb / 16; i += NT) ((uint4*)s_stage)[i] = ldg_nc_v4(src + 16 * i);
            for (uint32_t i = (nb / 16) * 4 + tid; i < nb / 4; i += NT)
                ((uint32_t*)s_stage)[i] = ((const uint32_t*)src)[i];
            __syncthreads();
        }
        if (wr) copy_smem_to_global(p.out + s_dst, s_stage + s_start, s_stored, tid, NT);
    }
}

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

int encode_grid(int dtype, int mode, bool ms, uint64_t C) {
    static int cache[2][4][2] = {};
    int& g = cache[dtype][mode][ms];
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const int nt = dtype == 0 ? Tr<float>::NT : Tr<double>::NT;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, pick_enc(dtype, mode, ms), nt, 0);
        g = sms * (per > 0 ? per : 1);
    }
    return (int)(C < (uint64_t)g ? C : (uint64_t)g);
}

cudaError_t launch_encode(int dtype, int mode, bool ms, const EncParams& p, int grid,
                          cudaStream_t s) {
    const int nt = dtype == 0 ? Tr<float>::NT : Tr<double>::NT;
    void* args[] = {(void*)&p};
    return cudaLaunchKernel(pick_enc(dtype, mode, ms), dim3(grid), dim3(nt), args, 0, s);
}

}  // namespace pfpl
