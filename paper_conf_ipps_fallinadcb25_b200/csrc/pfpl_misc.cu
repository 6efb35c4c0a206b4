// pfpl_misc.cu -- NOA min/max reduction, device-side
// derivation of the NOA quantizer constants (reading R3/R4), header-only streams.
#include <cfloat>
#include "pfpl_device.cuh"

namespace pfpl {

constexpr int MM_THREADS = 256;

__device__ __forceinline__ void block_minmax(double& mn, double& mx, double* out2) {
    __shared__ double smn[MM_THREADS / 32], smx[MM_THREADS / 32];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
        const double a = __shfl_xor_sync(PFPL_FULL, mn, d), b = __shfl_xor_sync(PFPL_FULL, mx, d);
        mn = a < mn ? a : mn;
        mx = b > mx ? b : mx;
    }
    if (lane == 0) { smn[warp] = mn; smx[warp] = mx; }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < MM_THREADS / 32; ++w) {
            mn = smn[w] < mn ? smn[w] : mn;
            mx = smx[w] > mx ? smx[w] : mx;
        }
        out2[0] = mn;
        out2[1] = mx;
    }
}

// Native-precision accumulation (a T value converts to double exactly, and min/max
// commute with that conversion): per element two FMNMX and one FSETP that records
// whether any non-finite value was seen.  Only a thread that saw one re-reads its
// elements with the finite filter (R2).  Zeros are canonicalised at the end (-0 and +0
// compare equal, so which one survives the reduction never matters).
template <typename T, bool CAREFUL>
__device__ __forceinline__ void mm_t(T x, T& mn, T& mx, bool& nf) {
    if (CAREFUL) {
        if (isfinite(x)) { mn = x < mn ? x : mn; mx = x > mx ? x : mx; }
    } else {
        mn = fmin(mn, x);
        mx = fmax(mx, x);
        nf = nf || !(fabs(x) < (T)INFINITY);
    }
}
template <typename T, bool CAREFUL>
__device__ __forceinline__ void mm_pass(const T* in, uint64_t n, T& mn, T& mx, bool& nf) {
    constexpr int V = 16 / sizeof(T);
    const uint64_t nv = n / V;
    const uint64_t stride = (uint64_t)gridDim.x * MM_THREADS;
    uint64_t i = (uint64_t)blockIdx.x * MM_THREADS + threadIdx.x;
    for (; i + 3 * stride < nv; i += 4 * stride) {      // 4 loads in flight per thread
        uint4 v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) v[u] = ldg_nc_v4(in + (i + u * stride) * V);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
            T x[V];
            memcpy(x, &v[u], 16);
#pragma unroll
            for (int k = 0; k < V; ++k) mm_t<T, CAREFUL>(x[k], mn, mx, nf);
        }
    }
    for (; i < nv; i += stride) {
        const uint4 v = ldg_nc_v4(in + i * V);
        T x[V];
        memcpy(x, &v, 16);
#pragma unroll
        for (int k = 0; k < V; ++k) mm_t<T, CAREFUL>(x[k], mn, mx, nf);
    }
    for (uint64_t j = nv * V + (uint64_t)blockIdx.x * MM_THREADS + threadIdx.x; j < n; j += stride)
        mm_t<T, CAREFUL>(in[j], mn, mx, nf);
}
template <typename T>
__global__ void __launch_bounds__(MM_THREADS) minmax_kernel(const T* in, uint64_t n, double* partial) {
    T mn = (T)INFINITY, mx = -(T)INFINITY;
    bool nf = false;
    mm_pass<T, false>(in, n, mn, mx, nf);
    if (nf) {                                   // rare: inf/NaN among this thread's values
        mn = (T)INFINITY;
        mx = -(T)INFINITY;
        mm_pass<T, true>(in, n, mn, mx, nf);
    }
    double dmn = (double)mn, dmx = (double)mx;
    if (dmn == 0.0) dmn = 0.0;                  // canonical +0 (R2)
    if (dmx == 0.0) dmx = 0.0;
    block_minmax(dmn, dmx, partial + 2 * blockIdx.x);
}

__global__ void __launch_bounds__(MM_THREADS) minmax_final_kernel(const double* partial, int blocks,
                                                                  double* mnmx) {
    double mn = u2d(0x7FF0000000000000ull), mx = -mn;
    for (int i = threadIdx.x; i < blocks; i += MM_THREADS) {
        const double a = partial[2 * i], b = partial[2 * i + 1];
        mn = a < mn ? a : mn;
        mx = b > mx ? b : mx;
    }
    block_minmax(mn, mx, mnmx);
}

// NOA constants (abs = eps * (max - min); R3: two round-downs so the
// derived bound never exceeds the exact product; R1: largest T <= it; R4:
// degenerate -> raw-words mode).  One thread.
__global__ void noa_derive_kernel(int dtype, const double* mnmx, double eps, uint32_t ms_flag,
                                  QConst* out) {
    const double mn = mnmx[0], mx = mnmx[1];
    const bool have = mn <= mx;
    const double d = have ? mx - mn : 0.0;
    const double r_lo = d > 0.0 ? u2d(d2u(d) - 1u) : 0.0;
    const double e = eps * r_lo;
    const double eps_abs = e > 0.0 ? u2d(d2u(e) - 1u) : 0.0;
    QConst qc;
    qc.a = qc.b = qc.c = qc.qconst = 0;
    qc.range = d;
    qc.flags = ms_flag;
    qc.pad = 0;
    if (dtype == 0) {
        float ee = 0.0f;
        if (eps_abs > 0.0) {
            ee = __double2float_rn(eps_abs);
            if (isinf(ee)) ee = FLT_MAX;
            if ((double)ee > eps_abs) ee = u2f(f2u(ee) - 1u);
        }
        if (ee > FLT_MAX / 2) ee = FLT_MAX / 2;
        if (!(ee >= FLT_MIN)) {
            qc.flags |= HF_RAWWORDS;
        } else {
            qc.a = f2u(ee);
            qc.b = f2u(0.5f / ee);
            qc.c = f2u(2.0f * ee);
            qc.qconst = f2u(ee);
        }
    } else {
        double ee = eps_abs;
        if (ee > DBL_MAX / 2) ee = DBL_MAX / 2;
        if (!(ee >= DBL_MIN)) {
            qc.flags |= HF_RAWWORDS;
        } else {
            qc.a = d2u(ee);
            qc.b = d2u(0.5 / ee);
            qc.c = d2u(2.0 * ee);
            qc.qconst = d2u(ee);
        }
    }
    *out = qc;
}

__global__ void header_only_kernel(uint8_t* out, uint64_t n, int dtype, int bound, double eps,
                                   QConst qc, const QConst* qc_dev, uint64_t* result) {
    if (qc_dev) qc = *qc_dev;
    uint8_t h[48];
    h[0] = 'P'; h[1] = 'F'; h[2] = 'P'; h[3] = 'L';
    h[4] = 1; h[5] = (uint8_t)dtype; h[6] = (uint8_t)bound; h[7] = (uint8_t)qc.flags;
    const uint64_t f[5] = {n, d2u(eps), qc.qconst, d2u(qc.range), (uint64_t)kChunkBytes};
    for (int i = 0; i < 5; ++i)
        for (int k = 0; k < 8; ++k) h[8 + 8 * i + k] = (uint8_t)(f[i] >> (8 * k));
    for (int i = 0; i < 48; ++i) out[i] = h[i];
    result[0] = 48;
}

// ---------------------------------------------------------------------------
// d1: exclusive prefix sum of the stored chunk sizes ("the decoder
// computes a prefix sum over the stored chunk sizes"), one pass with a
// decoupled look-back over 8192-entry tiles.  offs[c] = byte offset of chunk c
// in the payload area; offs[C] = total.  Sizes are validated against the raw
// chunk size; the total must equal the payload bytes (else *err = CORRUPT).
// ---------------------------------------------------------------------------
// 1024-entry tiles (NYX: 32 CTAs instead of 4), each thread 8 consecutive sizes read
// with two 16-byte loads and written as four 16-byte stores
constexpr int SCAN_T = 128, SCAN_PER = 8, SCAN_TILE = SCAN_T * SCAN_PER;

__global__ void __launch_bounds__(SCAN_T) size_scan_kernel(const uint32_t* table, uint64_t C,
                                                            uint64_t n, uint32_t cw, uint32_t s_bytes,
                                                            uint64_t in_bytes, uint64_t* offs,
                                                            unsigned long long* status, uint32_t epoch,
                                                            unsigned long long* ticket, uint64_t tbase,
                                                            int* err, unsigned int* wd) {
    __shared__ unsigned long long sh_tile;
    __shared__ uint64_t wsum[SCAN_T / 32];
    __shared__ uint64_t sh_excl;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    if (tid == 0) {
        g_pfpl_wd = wd;
        sh_tile = atomicAdd(ticket, 1ull) - tbase;
    }
    __syncthreads();
    const uint64_t t = sh_tile;
    const uint64_t c0 = t * SCAN_TILE + (uint64_t)tid * SCAN_PER;
    uint64_t v[SCAN_PER];
    uint32_t szs[SCAN_PER];
    uint64_t sum = 0;
    bool bad = false;
    if (c0 + SCAN_PER <= C) {
        const uint4 a = *(const uint4*)(table + c0), b = *(const uint4*)(table + c0 + 4);
        szs[0] = a.x; szs[1] = a.y; szs[2] = a.z; szs[3] = a.w;
        szs[4] = b.x; szs[5] = b.y; szs[6] = b.z; szs[7] = b.w;
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_PER; ++i) szs[i] = c0 + i < C ? table[c0 + i] : 0u;
    }
#pragma unroll
    for (int i = 0; i < SCAN_PER; ++i) {
        const uint64_t c = c0 + i;
        const uint64_t sz = szs[i];
        if (c < C) {
            const uint64_t m = c + 1 < C ? cw : n - c * cw;
            if (sz > m * s_bytes || (sz < 4 && sz != m * s_bytes)) bad = true;
        }
        v[i] = sum;
        sum += sz;
    }
    uint64_t inc = warp_incl_scan64(sum, lane);
    if (lane == 31) wsum[warp] = inc;
    __syncthreads();
    uint64_t before = 0, agg = 0;
#pragma unroll
    for (int w = 0; w < SCAN_T / 32; ++w) {
        if (w < warp) before += wsum[w];
        agg += wsum[w];
    }
    if (warp == 0) {
        const uint64_t EP = (uint64_t)epoch << 48;
        if (lane == 0) st_relaxed(&status[t], EP | ((t == 0 ? LB_P : LB_A) << 46) | agg);
        uint64_t excl = 0;
        if (t > 0) {
            int64_t look = (int64_t)t - 1;
            for (;;) {
                const int64_t idx = look - lane;
                uint64_t val = 0, flag = LB_P;
                if (idx >= 0) {
                    const uint64_t t0 = globaltimer();
                    for (;;) {
                        const uint64_t d = ld_relaxed(&status[idx]);
                        flag = ((uint32_t)(d >> 48) == epoch) ? ((d >> 46) & 3u) : 0u;
                        if (flag) { val = d & LB_VAL; break; }
                        // bounded like every spin loop of the library (watchdog -> trap)
                        if (globaltimer() - t0 > kWatchdogNs) watchdog_fire(0x31, (uint32_t)idx);
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
            if (lane == 0) st_relaxed(&status[t], EP | (LB_P << 46) | (excl + agg));
        }
        if (lane == 0) sh_excl = excl;
    }
    __syncthreads();
    const uint64_t base = sh_excl + before + inc - sum;
    if (c0 + SCAN_PER <= C) {
#pragma unroll
        for (int i = 0; i < SCAN_PER; i += 2)
            *(ulonglong2*)(offs + c0 + i) = make_ulonglong2(base + v[i], base + v[i + 1]);
    } else {
#pragma unroll
        for (int i = 0; i < SCAN_PER; ++i)
            if (c0 + i < C) offs[c0 + i] = base + v[i];
    }
#pragma unroll
    for (int i = 0; i < SCAN_PER; ++i) {
        const uint64_t c = c0 + i;
        if (c == C - 1) {
            if (base + v[i] + szs[i] != in_bytes) bad = true;
            offs[C] = base + v[i] + szs[i];
        }
    }
    if (bad) atomicExch(err, -4);
}

int scan_grid(uint64_t C) { return (int)((C + SCAN_TILE - 1) / SCAN_TILE); }

cudaError_t launch_size_scan(const uint32_t* table, uint64_t C, uint64_t n, uint32_t cw,
                             uint32_t s_bytes, uint64_t in_bytes, uint64_t* offs,
                             unsigned long long* status, uint32_t epoch,
                             unsigned long long* ticket, uint64_t tbase, int* err,
                             unsigned int* wd, cudaStream_t s) {
    size_scan_kernel<<<scan_grid(C), SCAN_T, 0, s>>>(table, C, n, cw, s_bytes, in_bytes, offs,
                                                     status, epoch, ticket, tbase, err, wd);
    return cudaGetLastError();
}

cudaError_t launch_minmax(int dtype, const void* in, uint64_t n, double* partial, int blocks,
                          cudaStream_t s) {
    if (dtype == 0) minmax_kernel<float><<<blocks, MM_THREADS, 0, s>>>((const float*)in, n, partial);
    else minmax_kernel<double><<<blocks, MM_THREADS, 0, s>>>((const double*)in, n, partial);
    return cudaGetLastError();
}

cudaError_t launch_minmax_final(const double* partial, int blocks, double* mnmx, cudaStream_t s) {
    minmax_final_kernel<<<1, MM_THREADS, 0, s>>>(partial, blocks, mnmx);
    return cudaGetLastError();
}

cudaError_t launch_noa_derive(int dtype, const double* mnmx, double eps, uint32_t ms_flag,
                              QConst* qc_out, cudaStream_t s) {
    noa_derive_kernel<<<1, 1, 0, s>>>(dtype, mnmx, eps, ms_flag, qc_out);
    return cudaGetLastError();
}

cudaError_t launch_header_only(uint8_t* out, uint64_t n, int dtype, int bound, double eps,
                               const QConst qc, const QConst* qc_dev, uint64_t* result,
                               cudaStream_t s) {
    header_only_kernel<<<1, 1, 0, s>>>(out, n, dtype, bound, eps, qc, qc_dev, result);
    return cudaGetLastError();
}

float log2p_host_f32(float a) { return log2p_f32(a); }
double log2p_host_f64(double a) { return log2p_f64(a); }

}  // namespace pfpl
