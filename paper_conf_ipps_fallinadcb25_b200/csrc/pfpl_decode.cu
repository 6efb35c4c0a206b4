// pfpl_decode.cu -- fused PFPL chunk decoder for sm_100a.
//
// The exact inverse of pfpl_encode.cu: chunk offsets by a single-pass
// look-back over the stored size table ("the decoder computes a prefix
// sum over the stored chunk sizes"), payload staged once in shared memory,
// repeated-byte levels 4->2 and the zero-byte level rebuilt top-down with
// block-wide prefix sums over bitmap popcounts, inverse bit-plane
// transpose in registers, negabinary -> two's complement and the
// delta decoder's block-wide inclusive scan (the decoder bottleneck
// P:302/P:342), dequantize and 16-byte coalesced stores.
#include <type_traits>
#include "pfpl_device.cuh"

namespace pfpl {

template <typename T> struct DecGeom {
    static constexpr int NT = Tr<T>::NT, S = Tr<T>::S;
    static constexpr int ROWB = 32 * S + 16;
    static constexpr int OUTB = NT * ROWB;
    static constexpr int PAYB = 16 + 2352 + 16384 + 64;
    static constexpr int BUF = OUTB > PAYB ? OUTB : PAYB;
};

__device__ __forceinline__ void set_err(int* err) { atomicExch(err, -4); }

// level-1 inverse: gather this thread's plane words from Z1 (plane-major order)
template <typename T, int KL, int KH>
__device__ __forceinline__ void rze1_dec(uint32_t (&lo)[32], uint32_t (&hi)[32], const uint8_t* z1,
                                         const uint8_t* s_m1, uint8_t (*s_wcnt)[64],
                                         uint16_t (*s_off)[64], uint32_t* s_n1, int tid,
                                         int lane, int warp) {
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NW = Tr<T>::NW;
    constexpr int NP = KL + KH, NG = NP / 4;
    uint32_t nb[NP];
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const int b = j < KL ? j : 32 + j - KL;
        const int pl = B - 1 - b;
        nb[j] = (s_m1[pl * (CW / 64) + (tid >> 1)] >> (4 * (tid & 1))) & 0xFu;
    }
    uint32_t ex[NG];
#pragma unroll
    for (int g = 0; g < NG; ++g) {
        uint32_t v = 0;
#pragma unroll
        for (int i = 0; i < 4; ++i) v |= (uint32_t)__popc(nb[4 * g + i]) << (8 * i);
        const uint32_t inc = warp_incl_scan(v, lane);
        ex[g] = inc - v;
        const int b0 = 4 * g < KL ? 4 * g : 32 + 4 * g - KL;
        if (lane == 31) *(uint32_t*)&s_wcnt[warp][b0] = inc;
    }
    __syncthreads();
    if (warp == 0) {
        uint32_t wl[NW], wh[NW], tl = 0, th = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) {
            wl[w] = lane < KL ? s_wcnt[w][lane] : 0u;
            wh[w] = lane < KH ? s_wcnt[w][32 + lane] : 0u;
            tl += wl[w];
            th += wh[w];
        }
        uint32_t sl = tl, sh = th;
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
    uint32_t pw[NP];
#pragma unroll
    for (int j = 0; j < NP; ++j) {
        const int b = j < KL ? j : 32 + j - KL;
        const uint32_t o = s_off[warp][b] + ((ex[j / 4] >> (8 * (j % 4))) & 0xFFu);
        const uint32_t n = nb[j];
        uint32_t w = 0, r = o;
        if (n & 1u) w |= (uint32_t)z1[r++];
        if (n & 2u) w |= (uint32_t)z1[r++] << 8;
        if (n & 4u) w |= (uint32_t)z1[r++] << 16;
        if (n & 8u) w |= (uint32_t)z1[r] << 24;
        pw[j] = w;
    }
#pragma unroll
    for (int j = 0; j < KL; ++j) lo[j] = pw[j];
    transpose_inv<KL>(lo);
    if constexpr (KH > 0) {
#pragma unroll
        for (int j = 0; j < KH; ++j) hi[j] = pw[KL + j];
        transpose_inv<KH>(hi);
    } else {
#pragma unroll
        for (int i = 0; i < 32; ++i) hi[i] = 0;
    }
}

template <typename T, int MODE, bool MSR>
__global__ void __launch_bounds__(Tr<T>::NT) decode_kernel(const DecParams p) {
    typedef typename Tr<T>::W W;
    constexpr int B = Tr<T>::B, CW = Tr<T>::CW, NT = Tr<T>::NT, NW = Tr<T>::NW, S = Tr<T>::S;
    constexpr int ROWB = DecGeom<T>::ROWB;
    constexpr int NB2 = 2048 / NT;
    constexpr int NWD2 = NB2 / 4;
    typedef typename std::conditional<B == 32, uint32_t, unsigned long long>::type ActT;

    __shared__ __align__(16) uint8_t s_buf[DecGeom<T>::BUF];
    __shared__ __align__(16) uint8_t s_m1[2048];
    __shared__ __align__(16) uint8_t s_m2[256];
    __shared__ __align__(16) uint8_t s_wcnt[NW][64];
    __shared__ __align__(16) uint16_t s_off[NW][64];
    __shared__ W s_scanw[NW];
    __shared__ uint32_t s_scan[NW];
    __shared__ ActT s_act[NW];
    __shared__ unsigned long long s_c, s_poff;
    __shared__ uint32_t s_size, s_delta, s_n1, s_n3, s_n4, s_bad;

    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    QF<T> q;
    q.load(p.qc);
    const bool raw = (p.qc.flags & HF_RAWWORDS) != 0;

    for (;;) {
        if (tid == 0) s_c = atomicAdd(p.ticket, 1ull) - p.ticket_base;
        if (tid < NW) s_act[tid] = 0;
        __syncthreads();
        const uint64_t c = s_c;
        if (c >= p.C) break;
        const uint32_t m = (uint32_t)min((uint64_t)CW, p.n - c * (uint64_t)CW);
        const uint32_t rawb = m * S;

        // ---- d1: chunk offset = prefix of stored sizes (look-back) ----
        if (warp == 0) {
            const uint32_t size = p.table[c];
            const uint64_t EP = (uint64_t)p.epoch << 48;
            uint64_t excl = 0;
            int64_t look = (int64_t)c - 1;
            while (look >= 0) {
                const int64_t idx = look - lane;
                uint64_t val = 0;
                bool isP = false;
                if (idx >= 0) {
                    const uint64_t d = ld_relaxed(&p.status[idx]);
                    if ((uint32_t)(d >> 48) == p.epoch && ((d >> 46) & 3u) == LB_P) { isP = true; val = d & LB_VAL; }
                    else val = p.table[idx];
                }
                const uint32_t pm = __ballot_sync(PFPL_FULL, isP);
                if (pm) {
                    const int first = __ffs(pm) - 1;
                    excl += warp_sum64(lane <= first ? val : 0ull);
                    break;
                }
                excl += warp_sum64(val);
                look -= 32;
            }
            if (lane == 0) {
                st_relaxed(&p.status[c], EP | (LB_P << 46) | ((excl + size) & LB_VAL));
                uint32_t bad = 0;
                if (size > rawb || excl + size > p.in_bytes) bad = 1;
                if (c == p.C - 1 && excl + size != p.in_bytes) bad = 1;
                if (size < 4 && size != rawb) bad = 1;
                s_bad = bad;
                s_size = size;
                s_poff = excl;
                s_delta = (uint32_t)((uintptr_t)(p.in + excl) & 15u);
            }
        }
        __syncthreads();
        if (s_bad) {
            if (tid == 0) set_err(p.err);
            continue;
        }
        const uint32_t size = s_size, delta = s_delta;
        // ---- stage the payload: 16-byte aligned blocks, guarded at the ends ----
        {
            const uint8_t* g0 = p.in + s_poff - delta;          // 16-byte aligned
            const uint8_t* lo_ok = p.in;
            const uint8_t* hi_ok = p.in + p.in_bytes;
            const uint32_t nblk = (delta + size + 15) >> 4;
            for (uint32_t j = tid; j < nblk; j += NT) {
                const uint8_t* a = g0 + 16 * j;
                if (a >= lo_ok && a + 16 <= hi_ok) {
                    ((uint4*)s_buf)[j] = ldg_nc_v4(a);
                } else {
                    for (int k = 0; k < 16; ++k)
                        s_buf[16 * j + k] = (a + k >= lo_ok && a + k < hi_ok) ? a[k] : (uint8_t)0;
                }
            }
        }
        __syncthreads();
        uint8_t* const dstc = (uint8_t*)p.out + c * (uint64_t)kChunkBytes;
        if (size == rawb) {
            // raw chunk: the stored bytes are the original values
            {
                const uint8_t* sp = s_buf + delta;
                for (uint32_t j = tid; j < rawb / 4; j += NT) {
                    const uint32_t a = (uint32_t)__cvta_generic_to_shared(sp + 4 * j) & 3u;
                    const uint32_t* sw = (const uint32_t*)(sp + 4 * j - a);
                    ((uint32_t*)dstc)[j] = __funnelshift_r(sw[0], sw[1], 8u * a);
                }
            }
            continue;
        }
        const uint8_t* const pay = s_buf + delta;

        // ---- levels 4 and 3 (warp 0): M4 -> M3 -> M2 ----
        if (warp == 0) {
            const uint32_t M4 = (uint32_t)pay[0] | ((uint32_t)pay[1] << 8) | ((uint32_t)pay[2] << 16) | ((uint32_t)pay[3] << 24);
            const uint32_t n4 = __popc(M4);
            const uint8_t* z4 = pay + 4;
            const uint32_t c4 = __popc(M4 & (lane == 31 ? 0xFFFFFFFFu : ((2u << lane) - 1u)));
            const uint32_t m3 = c4 ? z4[c4 - 1] : 0u;
            const uint32_t cnt3 = __popc(m3);
            const uint32_t inc3 = warp_incl_scan(cnt3, lane);
            const uint32_t n3 = __shfl_sync(PFPL_FULL, inc3, 31);
            const uint8_t* z3 = z4 + n4;
            const uint32_t e3 = inc3 - cnt3;
            uint32_t w0 = 0, w1 = 0;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const uint32_t cj = e3 + __popc(m3 & ((2u << j) - 1u));
                const uint32_t bv = cj ? z3[cj - 1] : 0u;
                if (j < 4) w0 |= bv << (8 * j); else w1 |= bv << (8 * (j - 4));
            }
            ((uint2*)s_m2)[lane] = make_uint2(w0, w1);
            if (lane == 0) { s_n4 = n4; s_n3 = n3; }
        }
        __syncthreads();

        // ---- level 2 (all threads): M2 -> M1, and active (plane, warp) segments ----
        {
            const uint32_t n4 = s_n4, n3 = s_n3;
            const uint32_t bits2 = NB2 == 16 ? (uint32_t)((const uint16_t*)s_m2)[tid] : ((const uint32_t*)s_m2)[tid];
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
            base += inc - cnt2;
            const uint8_t* z2 = pay + 4 + n4 + n3;
            uint32_t wv[NWD2];
            uint32_t anyseg = 0;
#pragma unroll
            for (int i = 0; i < NWD2; ++i) {
                uint32_t w = 0;
#pragma unroll
                for (int k = 0; k < 4; ++k) {
                    const int bit = 4 * i + k;
                    const uint32_t cj = base + __popc(bits2 & (bit == 31 ? 0xFFFFFFFFu : ((2u << bit) - 1u)));
                    w |= (cj ? (uint32_t)z2[cj - 1] : 0u) << (8 * k);
                }
                wv[i] = w;
                if (w) anyseg |= 1u << (i / 4);
            }
#pragma unroll
            for (int i = 0; i < NWD2; i += 4)
                *(uint4*)(s_m1 + NB2 * tid + 4 * i) = make_uint4(wv[i], wv[i + 1], wv[i + 2], wv[i + 3]);
            // 16-byte segment g of M1 = (plane g / NW, warp g % NW)
#pragma unroll
            for (int sgi = 0; sgi < NB2 / 16; ++sgi) {
                if (anyseg & (1u << sgi)) {
                    const int g = (NB2 / 16) * tid + sgi;
                    atomicOr(&s_act[g % NW], (ActT)1 << (g / NW));
                }
            }
            if (tid == 0 && 4 + n4 + n3 + n2 > size) s_bad = 1;
            if (tid == 0) s_n1 = 4 + n4 + n3 + n2;   // temporarily: offset of Z1 in the payload
        }
        __syncthreads();
        if (s_bad) {
            if (tid == 0) set_err(p.err);
            continue;
        }

        // ---- level 1 + inverse bit shuffle ----
        const uint32_t z1off = s_n1;
        const uint8_t* z1 = pay + z1off;
        ActT act = 0;
#pragma unroll
        for (int w = 0; w < NW; ++w) act |= s_act[w];
        // plane p active <=> bit p of act; active low bits P = B - (lowest active plane)
        const int P = act ? B - (B == 32 ? __ffs((uint32_t)act) - 1 : __ffsll((long long)act) - 1) : 0;
        uint32_t lo[32], hi[32];
        if (P == 0) {
#pragma unroll
            for (int i = 0; i < 32; ++i) { lo[i] = 0; hi[i] = 0; }
            if (tid == 0) s_n1 = 0;
        } else if (B == 32 || P <= 32) {
            if (P <= 4) rze1_dec<T, 4, 0>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 8) rze1_dec<T, 8, 0>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 16) rze1_dec<T, 16, 0>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else rze1_dec<T, 32, 0>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
        } else {
            if (P <= 36) rze1_dec<T, 32, 4>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 40) rze1_dec<T, 32, 8>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else if (P <= 48) rze1_dec<T, 32, 16>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
            else rze1_dec<T, 32, 32>(lo, hi, z1, s_m1, s_wcnt, s_off, &s_n1, tid, lane, warp);
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
        if (lane == 31) s_scanw[warp] = incw;
        __syncthreads();   // all Z1 reads done; totals visible
        W carry = incw - tsum;
#pragma unroll
        for (int w = 0; w < NW; ++w)
            if (w < warp) carry += s_scanw[w];
        if (tid == 0 && z1off + s_n1 != size) s_bad = 1;
        // ---- dequantize into padded rows ----
        {
            uint4* row = (uint4*)(s_buf + tid * ROWB);
#pragma unroll
            for (int j = 0; j < 2 * S; ++j) {
                T x[16 / S];
#pragma unroll
                for (int i = 0; i < 16 / S; ++i) x[i] = dequantize<T, MODE>(q, (W)(carry + dq[j * (16 / S) + i]), raw);
                uint4 v;
                memcpy(&v, x, 16);
                row[j] = v;
            }
        }
        __syncthreads();
        if (s_bad) {
            if (tid == 0) set_err(p.err);
            continue;
        }
        if (m == CW) {
#pragma unroll
            for (int i = 0; i < 1024 / NT; ++i) {
                const int k = i * NT + tid;
                const uint4 v = *(const uint4*)(s_buf + (k / (2 * S)) * ROWB + (k % (2 * S)) * 16);
                *(uint4*)(dstc + 16 * k) = v;
            }
        } else {
            for (uint32_t e = tid; e < m; e += NT)
                ((T*)dstc)[e] = *(const T*)(s_buf + (e / 32) * ROWB + (e % 32) * S);
        }
    }
}

template <typename T, int MODE, bool MSR>
static void* dec_fn() { return (void*)decode_kernel<T, MODE, MSR>; }

static void* pick_dec(int dtype, int mode, bool ms) {
#define PFPL_D(T)                                                                  \
    switch (mode) {                                                                \
        case MODE_ABS: return ms ? dec_fn<T, MODE_ABS, true>() : dec_fn<T, MODE_ABS, false>(); \
        case MODE_REL: return ms ? dec_fn<T, MODE_REL, true>() : dec_fn<T, MODE_REL, false>(); \
        default: return ms ? dec_fn<T, MODE_RAW, true>() : dec_fn<T, MODE_RAW, false>();       \
    }
    if (dtype == 0) { PFPL_D(float) } else { PFPL_D(double) }
#undef PFPL_D
}

int decode_grid(int dtype, int mode, bool ms, uint64_t C) {
    static int cache[2][4][2] = {};
    int& g = cache[dtype][mode][ms];
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        const int nt = dtype == 0 ? Tr<float>::NT : Tr<double>::NT;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, pick_dec(dtype, mode, ms), nt, 0);
        g = sms * (per > 0 ? per : 1);
    }
    return (int)(C < (uint64_t)g ? C : (uint64_t)g);
}

cudaError_t launch_decode(int dtype, int mode, bool ms, const DecParams& p, int grid,
                          cudaStream_t s) {
    const int nt = dtype == 0 ? Tr<float>::NT : Tr<double>::NT;
    void* args[] = {(void*)&p};
    return cudaLaunchKernel(pick_dec(dtype, mode, ms), dim3(grid), dim3(nt), args, 0, s);
}

}  // namespace pfpl
