// pfpl_api.cu -- host side of the C ABI declared in include/pfpl.h.
//
// Validation, quantizer constants (readings R1, R4, R5 of DESIGN.md 3),
// per-(device, stream) scratch (look-back descriptors, monotone tickets,
// epochs), and kernel launches.  No computation of the codec happens here:
// every step of the path runs in the kernels of pfpl_encode.cu /
// pfpl_decode.cu / pfpl_misc.cu.
#include <atomic>
#include <cfloat>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <utility>

#include "../../include/pfpl.h"
#include "pfpl_internal.h"

using namespace pfpl;

namespace {

std::atomic<int> g_last_cuda{0};
std::atomic<uint64_t> g_launches{0};

struct Scratch {
    unsigned long long* status = nullptr;
    uint64_t status_cap = 0;
    unsigned long long* ticket = nullptr;
    uint64_t ticket_val = 0;
    uint32_t epoch = 0;
    QConst* qc_dev = nullptr;
    double* mnmx = nullptr;
    double* partial = nullptr;
    uint64_t* result = nullptr;      // [0] stream bytes, [1] error word
    uint64_t* host = nullptr;        // pinned mirror of result
    uint8_t* hdr_host = nullptr;     // pinned 64 bytes
    uint32_t* table_dev = nullptr;   // for pfpl_decompress_chunks
    uint64_t table_cap = 0;
    uint64_t* offs = nullptr;        // decoder chunk offsets (C + 1)
    uint64_t offs_cap = 0;
    unsigned long long* stats = nullptr;   // 2 slots x {unquantizable values, raw chunks}
    unsigned long long* vm = nullptr;      // verify-mode metric accumulators (8)
    uint64_t stat_seq = 0;                 // compress calls enqueued (slot = seq & 1)
};

std::mutex g_mu;
std::map<std::pair<int, void*>, Scratch*> g_scratch;
unsigned int* g_wd_host = nullptr;     // mapped pinned watchdog report {site, block, thread, detail}
unsigned int* g_wd_dev = nullptr;

std::once_flag g_wd_once;
// f32 ABS encoder form hint (pfpl_encode.cuh, encode_kernel): one mapped host word per
// process, written by CTA 0 of every f32 ABS launch, read here without a sync (so a hint
// takes effect from the next call; both forms write the same bytes)
std::once_flag g_x0_once;
unsigned int* g_x0_host = nullptr;
unsigned int* g_x0_dev = nullptr;
unsigned int* x0_hint_ptr() {
    std::call_once(g_x0_once, [] {
        if (cudaHostAlloc(&g_x0_host, 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) { g_x0_host = nullptr; return; }
        memset(g_x0_host, 0, 64);
        if (cudaHostGetDevicePointer(&g_x0_dev, g_x0_host, 0) != cudaSuccess) g_x0_dev = nullptr;
    });
    return g_x0_dev;
}

unsigned int* watchdog_ptr() {
    std::call_once(g_wd_once, [] {
        if (cudaHostAlloc(&g_wd_host, 64, cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess) { g_wd_host = nullptr; return; }
        memset(g_wd_host, 0, 64);
        if (cudaHostGetDevicePointer(&g_wd_dev, g_wd_host, 0) != cudaSuccess) g_wd_dev = nullptr;
    });
    return g_wd_dev;
}

constexpr int kMinmaxBlocks = 1184;   // 8 CTAs of 256 threads per SM

int cuda_fail(cudaError_t e) {
    g_last_cuda = (int)e;
    return PFPL_ERR_CUDA;
}
#define CK(x)                                             \
    do {                                                  \
        cudaError_t _e = (x);                             \
        if (_e != cudaSuccess) return cuda_fail(_e);      \
    } while (0)

int get_scratch(cudaStream_t s, uint64_t C, Scratch** out) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    std::lock_guard<std::mutex> lk(g_mu);
    Scratch*& sc = g_scratch[{dev, (void*)s}];
    if (!sc) {
        sc = new Scratch();
        CK(cudaMalloc(&sc->ticket, 64));
        CK(cudaMemsetAsync(sc->ticket, 0, 64, s));
        CK(cudaMalloc(&sc->qc_dev, sizeof(QConst)));
        CK(cudaMalloc(&sc->mnmx, 4 * sizeof(double)));
        CK(cudaMalloc(&sc->partial, 2 * kMinmaxBlocks * sizeof(double)));
        CK(cudaMalloc(&sc->result, 4 * sizeof(uint64_t)));
        CK(cudaMallocHost(&sc->host, 4 * sizeof(uint64_t)));
        CK(cudaMallocHost(&sc->hdr_host, 64));
        CK(cudaMalloc(&sc->stats, 4 * sizeof(unsigned long long)));
        CK(cudaMemsetAsync(sc->stats, 0, 4 * sizeof(unsigned long long), s));
    }
    // look-back descriptors: one per chunk (encoder) / per 1024-chunk tile (size scan)
    auto desc_words = [](uint64_t cap) { return cap; };
    if (C > sc->status_cap) {
        if (sc->status) CK(cudaFreeAsync(sc->status, s));
        uint64_t cap = C < 1024 ? 1024 : C + C / 4;
        CK(cudaMallocAsync(&sc->status, desc_words(cap) * sizeof(unsigned long long), s));
        CK(cudaMemsetAsync(sc->status, 0, desc_words(cap) * sizeof(unsigned long long), s));
        sc->status_cap = cap;
        sc->epoch = 0;
    }
    // epochs tag look-back descriptors so no per-call memset is needed
    if (++sc->epoch >= 0xFFFFu) {
        CK(cudaMemsetAsync(sc->status, 0, desc_words(sc->status_cap) * sizeof(unsigned long long), s));
        sc->epoch = 1;
    }
    *out = sc;
    return PFPL_OK;
}

uint32_t f2u_h(float x) { uint32_t u; memcpy(&u, &x, 4); return u; }
float u2f_h(uint32_t u) { float x; memcpy(&x, &u, 4); return x; }
uint64_t d2u_h(double x) { uint64_t u; memcpy(&u, &x, 8); return u; }
double u2d_h(uint64_t u) { double x; memcpy(&x, &u, 8); return x; }

// R1: largest binary32 <= x (x > 0)
float round_down_f32_h(double x) {
    float f = (float)x;
    if (std::isinf(f)) f = FLT_MAX;
    if ((double)f > x) f = u2f_h(f2u_h(f) - 1u);
    return f;
}

// quantizer constants for ABS / REL on the host (NOA is derived on the device)
int host_qconst(int dtype, int bound, double eps, unsigned opts, QConst* qc, int* mode) {
    memset(qc, 0, sizeof(*qc));
    qc->flags = (opts & PFPL_OPT_MS_RESIDUALS) ? HF_MS : 0u;
    if (!(eps > 0.0) || std::isinf(eps)) return PFPL_ERR_BOUND;
    if (bound == PFPL_NOA) { *mode = MODE_NOA; return PFPL_OK; }
    if (bound == PFPL_ABS) {
        *mode = MODE_ABS;
        if (dtype == PFPL_F32) {
            float ee = round_down_f32_h(eps);
            if (ee > FLT_MAX / 2) ee = FLT_MAX / 2;
            if (!(ee >= FLT_MIN)) return PFPL_ERR_BOUND;
            qc->a = f2u_h(ee); qc->b = f2u_h(0.5f / ee); qc->c = f2u_h(2.0f * ee); qc->qconst = f2u_h(ee);
        } else {
            double ee = eps;
            if (ee > DBL_MAX / 2) ee = DBL_MAX / 2;
            if (!(ee >= DBL_MIN)) return PFPL_ERR_BOUND;
            qc->a = d2u_h(ee); qc->b = d2u_h(0.5 / ee); qc->c = d2u_h(2.0 * ee); qc->qconst = d2u_h(ee);
        }
        return PFPL_OK;
    }
    // REL (P:90 with R5): c_lo = largest T <= 1+eps; w = 2 log2p(c_lo); inv_w = 0.5/log2p(c_lo)
    *mode = MODE_REL;
    if (dtype == PFPL_F32) {
        float c;
        if (eps < 4503599627370496.0) {
            c = (float)(1.0 + eps);
            if (std::isinf(c)) c = FLT_MAX;
            while ((double)c - 1.0 > eps) c = u2f_h(f2u_h(c) - 1u);
        } else {
            c = round_down_f32_h(eps);
        }
        const float lw = log2p_host_f32(c);
        const float w = 2.0f * lw;
        if (!(w > 0.0f) || std::isinf(w)) { qc->flags |= HF_RAWWORDS; *mode = MODE_RAW; return PFPL_OK; }
        qc->a = f2u_h(c); qc->b = f2u_h(w); qc->c = f2u_h(0.5f / lw); qc->qconst = f2u_h(w);
        // fast-path margin in bin units: |log2p - lg2.approx| <= 3.6e-7 +
        // 2.4e-7 |L|, the roundings of s (2.4e-7 |L| c), y, the R7 window and pow2p
        // (<= 2.2e-6 + 7.4e-7 |L| in all, in log2 units), with >= 2.7x headroom
        const double cinv = 0.5 / (double)lw;
        const double m1 = cinv * 2e-6, m2 = cinv * 8e-6;
        qc->m1 = f2u_h(0.0f); qc->m2 = f2u_h(1.0f);          // 1: the fast path never certifies
        if (m2 < 0.2 && m1 * 128.0 + m2 < 0.25) { qc->m1 = f2u_h((float)m1); qc->m2 = f2u_h((float)m2); }
    } else {
        double c;
        if (eps < 4503599627370496.0) {
            c = 1.0 + eps;
            if (c - 1.0 > eps) c = u2d_h(d2u_h(c) - 1u);
        } else {
            c = eps;
            if (std::isinf(c)) c = DBL_MAX;
        }
        const double lw = log2p_host_f64(c);
        const double w = 2.0 * lw;
        if (!(w > 0.0) || std::isinf(w)) { qc->flags |= HF_RAWWORDS; *mode = MODE_RAW; return PFPL_OK; }
        qc->a = d2u_h(c); qc->b = d2u_h(w); qc->c = d2u_h(0.5 / lw); qc->qconst = d2u_h(w);
        // f64 fast path: L from the exact exponent + lg2.approx.f32 of the mantissa (abs
        // error <= ~4e-7), margin with ~4x headroom
        const double cinv = 0.5 / lw;
        const double m1 = cinv * 1e-12, m2 = cinv * 2e-6;
        qc->m1 = d2u_h(0.0); qc->m2 = d2u_h(1.0);
        if (m2 < 0.2 && m1 * 1024.0 + m2 < 0.25) { qc->m1 = d2u_h(m1); qc->m2 = d2u_h(m2); }
    }
    return PFPL_OK;
}

inline uint64_t tsz(int dtype) { return dtype == PFPL_F32 ? 4u : 8u; }
inline uint64_t chunks_of(uint64_t n, int dtype) {
    const uint64_t cw = kChunkBytes / tsz(dtype);
    return (n + cw - 1) / cw;
}
inline bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

// Enqueue one compression (or shard) on s.  Writes stream bytes to sc->result[0].
int enqueue_compress(const void* in, uint64_t n, uint64_t n_total, int dtype, int bound,
                     double eps, unsigned opts, const double* mnmx_given, uint8_t* out,
                     uint64_t cap, uint32_t* table, uint64_t payload_off, int write_header,
                     uint64_t* result, cudaStream_t s, Scratch** sc_out) {
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    if (bound != PFPL_ABS && bound != PFPL_REL && bound != PFPL_NOA) return PFPL_ERR_ARG;
    if (n > (1ull << 40) || n_total > (1ull << 40)) return PFPL_ERR_ARG;
    if ((n && !in) || !out) return PFPL_ERR_ARG;
    if (!aligned16(in) || !aligned16(out)) return PFPL_ERR_ALIGN;
    QConst qc;
    int mode = 0;
    int st = host_qconst(dtype, bound, eps, opts, &qc, &mode);
    if (st != PFPL_OK) return st;
    const uint64_t C = chunks_of(n, dtype);
    if (cap < payload_off) return PFPL_ERR_CAPACITY;
    Scratch* sc = nullptr;
    st = get_scratch(s, C, &sc);
    if (st != PFPL_OK) return st;
    if (sc_out) *sc_out = sc;
    if (!result) result = sc->result;
    const QConst* qdev = nullptr;
    if (mode == MODE_NOA) {
        const double* mm = mnmx_given;
        if (!mm) {
            CK(launch_minmax(dtype, in, n, sc->partial, kMinmaxBlocks, s));
            CK(launch_minmax_final(sc->partial, kMinmaxBlocks, sc->mnmx, s));
            g_launches += 2;
            mm = sc->mnmx;
        }
        CK(launch_noa_derive(dtype, mm, eps, qc.flags, sc->qc_dev, s));
        g_launches += 1;
        qdev = sc->qc_dev;
    }
    // statistics slot of this call; the kernel zeroes the other slot for the next one
    unsigned long long* const st_cur = sc->stats + 2 * (sc->stat_seq & 1);
    unsigned long long* const st_next = sc->stats + 2 * ((sc->stat_seq + 1) & 1);
    sc->stat_seq += 1;
    if (C == 0) {
        // no kernel runs to zero the next slot: clear both
        CK(cudaMemsetAsync(sc->stats, 0, 4 * sizeof(unsigned long long), s));
        if (write_header) {
            CK(launch_header_only(out, n_total, dtype, bound, eps, qc, qdev, result, s));
        } else {
            CK(cudaMemsetAsync(result, 0, 8, s));
            // payload size 0 -> stream bytes = payload_off
            uint64_t v = payload_off;
            CK(cudaMemcpyAsync(result, &v, 8, cudaMemcpyHostToDevice, s));
            CK(cudaStreamSynchronize(s));
        }
        g_launches += 1;
        return PFPL_OK;
    }
    EncParams p;
    memset(&p, 0, sizeof(p));
    p.in = in;
    p.n = n;
    p.C = C;
    p.out = out;
    p.cap = cap;
    p.table = table;
    p.payload_off = payload_off;
    p.status = sc->status;
    p.ticket = sc->ticket;
    p.ticket_base = sc->ticket_val;
    p.epoch = sc->epoch;
    p.write_header = write_header;
    p.qc = qc;
    p.qc_dev = qdev;
    p.result = result;
    p.n_total = n_total;
    p.eps = eps;
    p.dtype = (uint32_t)dtype;
    p.bound = (uint32_t)bound;
    p.wd = watchdog_ptr();
    p.stats = st_cur;
    p.stats_next = st_next;
    p.nz2 = 0x8000000080000000ull;
    bool x0 = false;
    if (dtype == PFPL_F32 && (mode == MODE_ABS || mode == MODE_NOA)) {
        // one hint word per bound (ABS, NOA): their bins differ on the same field
        const int k = mode == MODE_NOA ? 1 : 0;
        unsigned int* const h = x0_hint_ptr();
        p.x0_hint = h ? h + k : nullptr;
        x0 = p.x0_hint && ((volatile unsigned int*)g_x0_host)[k] == 1u;
    }
    const bool ms = (opts & PFPL_OPT_MS_RESIDUALS) != 0;
    const int grid = encode_grid(dtype, mode, ms, C);
    CK(launch_encode(dtype, mode, ms, x0, p, grid, s));
    g_launches += 1;
    // each persistent encoder CTA consumes (stages + 1) tickets per pipeline beyond its chunks
    sc->ticket_val += C + (uint64_t)grid * (uint64_t)encode_tickets_per_cta(dtype);
    return PFPL_OK;
}

int parse_header(const uint8_t* h, uint64_t bytes, uint64_t* n, int* dtype, int* bound,
                 double* eps, unsigned* flags, uint64_t* qconst, double* range) {
    if (bytes < kHeaderBytes) return PFPL_ERR_CORRUPT;
    if (h[0] != 'P' || h[1] != 'F' || h[2] != 'P' || h[3] != 'L' || h[4] != 1) return PFPL_ERR_CORRUPT;
    if (h[5] > 1 || h[6] > 2 || (h[7] & ~3u)) return PFPL_ERR_CORRUPT;
    uint64_t f[5];
    for (int i = 0; i < 5; ++i) {
        f[i] = 0;
        for (int k = 7; k >= 0; --k) f[i] = (f[i] << 8) | h[8 + 8 * i + k];
    }
    if (f[4] != kChunkBytes) return PFPL_ERR_CORRUPT;    // chunk bytes + reserved 0
    if (f[0] > (1ull << 40)) return PFPL_ERR_CORRUPT;
    if (n) *n = f[0];
    if (dtype) *dtype = h[5];
    if (bound) *bound = h[6];
    if (eps) *eps = u2d_h(f[1]);
    if (flags) *flags = h[7];
    if (qconst) *qconst = f[2];
    if (range) *range = u2d_h(f[3]);
    return PFPL_OK;
}

// decoder constants from the header (validated: corrupt constants -> error)
int decode_qconst(int dtype, int bound, unsigned flags, uint64_t qk, QConst* qc, int* mode) {
    memset(qc, 0, sizeof(*qc));
    qc->flags = flags;
    if (flags & HF_RAWWORDS) { *mode = MODE_RAW; return PFPL_OK; }
    if (dtype == PFPL_F32) {
        if (qk >> 32) return PFPL_ERR_CORRUPT;
        const float c = u2f_h((uint32_t)qk);
        if (bound == PFPL_REL) {
            if (!(c > 0.0f) || std::isinf(c)) return PFPL_ERR_CORRUPT;
            qc->b = f2u_h(c);
            *mode = MODE_REL;
        } else {
            if (!(c >= FLT_MIN && c <= FLT_MAX / 2)) return PFPL_ERR_CORRUPT;
            qc->a = f2u_h(c); qc->c = f2u_h(2.0f * c);
            *mode = MODE_ABS;
        }
    } else {
        const double c = u2d_h(qk);
        if (bound == PFPL_REL) {
            if (!(c > 0.0) || std::isinf(c)) return PFPL_ERR_CORRUPT;
            qc->b = d2u_h(c);
            *mode = MODE_REL;
        } else {
            if (!(c >= DBL_MIN && c <= DBL_MAX / 2)) return PFPL_ERR_CORRUPT;
            qc->a = d2u_h(c); qc->c = d2u_h(2.0 * c);
            *mode = MODE_ABS;
        }
    }
    return PFPL_OK;
}

int enqueue_decompress(const uint8_t* hdr, const uint32_t* table_dev, uint64_t first_chunk,
                       uint64_t nchunks, const uint8_t* payload, uint64_t payload_bytes,
                       void* out, uint64_t cap, int* err_dev, cudaStream_t s, uint64_t* n_out,
                       const void* orig = nullptr, unsigned long long* vm = nullptr) {
    uint64_t n = 0, qk = 0;
    int dtype = 0, bound = 0;
    unsigned flags = 0;
    double eps_h = 0.0, range_h = 0.0;
    int st = parse_header(hdr, kHeaderBytes, &n, &dtype, &bound, &eps_h, &flags, &qk, &range_h);
    if (st != PFPL_OK) return st;
    QConst qc;
    int mode = 0;
    st = decode_qconst(dtype, bound, flags, qk, &qc, &mode);
    if (st != PFPL_OK) return st;
    const uint64_t cw = kChunkBytes / tsz(dtype);
    const uint64_t C = chunks_of(n, dtype);
    if (first_chunk > C || nchunks > C - first_chunk) return PFPL_ERR_ARG;
    const uint64_t e0 = first_chunk * cw;
    const uint64_t nloc = nchunks ? ((first_chunk + nchunks) * cw < n ? nchunks * cw : n - e0) : 0;
    if (n_out) *n_out = nloc;
    if (cap < nloc * tsz(dtype)) return PFPL_ERR_CAPACITY;
    if (!aligned16(out)) return PFPL_ERR_ALIGN;
    if (nchunks == 0) return payload_bytes == 0 ? PFPL_OK : PFPL_ERR_CORRUPT;
    Scratch* sc = nullptr;
    st = get_scratch(s, nchunks, &sc);
    if (st != PFPL_OK) return st;
    // d1: a separate prefix-sum launch for large streams; small ones (at most
    // kFusedScanChunks chunks) let the decoder's IO warps sum the size table themselves,
    // which saves the launch (CESM-sized fields: +18% decode) but puts a window sum on
    // the IO warp's path per chunk (large rough fields: -7%)
    const int grid = decode_grid(dtype, mode, (flags & HF_MS) != 0, nchunks);
    const bool fused_scan = nchunks <= kFusedScanChunks;
    if (!fused_scan && nchunks + 1 > sc->offs_cap) {
        if (sc->offs) CK(cudaFreeAsync(sc->offs, s));
        sc->offs_cap = nchunks + 1 < 1024 ? 1024 : (nchunks + 1) + (nchunks + 1) / 4;
        CK(cudaMallocAsync(&sc->offs, sc->offs_cap * sizeof(uint64_t), s));
    }
    if (!fused_scan) {
        // d1: prefix sum of the stored sizes -> chunk offsets
        CK(launch_size_scan(table_dev, nchunks, nloc, (uint32_t)cw, (uint32_t)tsz(dtype), payload_bytes,
                            sc->offs, sc->status, sc->epoch, sc->ticket, sc->ticket_val, err_dev,
                            watchdog_ptr(), s));
        g_launches += 1;
        sc->ticket_val += (uint64_t)scan_grid(nchunks);
    }
    DecParams p;
    memset(&p, 0, sizeof(p));
    p.offs = fused_scan ? nullptr : sc->offs;
    p.in = payload;
    p.in_bytes = payload_bytes;
    p.table = table_dev;
    p.n = nloc;
    p.C = nchunks;
    p.out = out;
    p.status = sc->status;
    p.ticket = sc->ticket;
    p.ticket_base = sc->ticket_val;
    p.epoch = sc->epoch;
    p.qc = qc;
    p.err = err_dev;
    p.wd = watchdog_ptr();
    p.c23 = dtype == PFPL_F32 ? f2u_h(u2f_h((uint32_t)qc.c) * 8388608.0f) : 0u;   // exact or inf
    p.orig = orig;
    p.vm = vm;
    p.vbound = bound;
    p.veps = eps_h;
    p.vrange = range_h;
    p.nz2 = 0x8000000080000000ull;
    const bool ms = (flags & HF_MS) != 0;
    // the decoder form follows the encoder-form hint of the stream's bound (pfpl_encode.cuh:
    // both decoder forms decode every stream; the hint only predicts the chunks' shape)
    bool x0 = false;
    if (dtype == PFPL_F32 && mode == MODE_ABS && (bound == PFPL_ABS || bound == PFPL_NOA) && g_x0_host)
        x0 = ((volatile unsigned int*)g_x0_host)[bound == PFPL_NOA ? 1 : 0] == 1u;
    CK(launch_decode(dtype, mode, ms, x0, p, grid, s));
    g_launches += 1;
    sc->ticket_val += (uint64_t)grid * (uint64_t)decode_tickets_per_cta();   // decoder: no tickets
    return PFPL_OK;
}

}  // namespace

namespace pfpl {
int record_cuda_error(int e) { return cuda_fail((cudaError_t)e); }

int grid_limit() {
    static const int v = [] {
        const char* e = getenv("PFPL_GRID_LIMIT");
        const long x = e ? atol(e) : 0;
        return x > 0 ? (int)(x < (1 << 30) ? x : (1 << 30)) : (1 << 30);
    }();
    return v;
}

// every argument check pfpl_compress_async makes before enqueueing anything
int check_compress_args(const void* in, uint64_t n, int dtype, int bound, double eps,
                        unsigned opts, const void* out, uint64_t cap) {
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    if (bound != PFPL_ABS && bound != PFPL_REL && bound != PFPL_NOA) return PFPL_ERR_ARG;
    if (n > (1ull << 40)) return PFPL_ERR_ARG;
    if ((n && !in) || !out) return PFPL_ERR_ARG;
    if (!aligned16(in) || !aligned16(out)) return PFPL_ERR_ALIGN;
    QConst qc;
    int mode = 0;
    const int st = host_qconst(dtype, bound, eps, opts, &qc, &mode);
    if (st != PFPL_OK) return st;
    if (cap < kHeaderBytes + 4 * chunks_of(n, dtype)) return PFPL_ERR_CAPACITY;
    return PFPL_OK;
}
}  // namespace pfpl

extern "C" {

uint64_t pfpl_max_compressed_bytes(uint64_t n, int dtype) {
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return 0;
    return kHeaderBytes + 4 * chunks_of(n, dtype) + n * tsz(dtype);
}

int pfpl_compress_async(const void* in, uint64_t n, int dtype, int bound, double eps,
                        unsigned opts, void* out, uint64_t cap, uint64_t* result_dev,
                        void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    const uint64_t C = chunks_of(n, dtype);
    if (cap < kHeaderBytes + 4 * C) return PFPL_ERR_CAPACITY;
    if (result_dev) CK(cudaMemsetAsync(result_dev, 0, 16, s));
    return enqueue_compress(in, n, n, dtype, bound, eps, opts, nullptr, (uint8_t*)out, cap,
                            (uint32_t*)((uint8_t*)out + kHeaderBytes), kHeaderBytes + 4 * C, 1,
                            result_dev, s, nullptr);
}

int pfpl_compress_ex(const void* in, uint64_t n, int dtype, int bound, double eps, unsigned opts,
                     void* out, uint64_t* out_bytes, void* stream) {
    if (!out_bytes) return PFPL_ERR_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    const uint64_t C = chunks_of(n, dtype);
    const uint64_t cap = *out_bytes;
    if (cap < kHeaderBytes + 4 * C) return PFPL_ERR_CAPACITY;
    Scratch* sc = nullptr;
    int st = enqueue_compress(in, n, n, dtype, bound, eps, opts, nullptr, (uint8_t*)out, cap,
                              (uint32_t*)((uint8_t*)out + kHeaderBytes), kHeaderBytes + 4 * C, 1,
                              nullptr, s, &sc);
    if (st != PFPL_OK) return st;
    CK(cudaMemcpyAsync(sc->host, sc->result, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const uint64_t total = sc->host[0];
    if (total > cap) return PFPL_ERR_CAPACITY;
    *out_bytes = total;
    return PFPL_OK;
}

int pfpl_compress(const void* in, uint64_t n, int dtype, int bound, double eps, void* out,
                  uint64_t* out_bytes, void* stream) {
    return pfpl_compress_ex(in, n, dtype, bound, eps, 0u, out, out_bytes, stream);
}

int pfpl_peek_header(const void* hdr, uint64_t bytes, uint64_t* n, int* dtype, int* bound,
                     double* eps, unsigned* flags) {
    if (!hdr) return PFPL_ERR_ARG;
    return parse_header((const uint8_t*)hdr, bytes, n, dtype, bound, eps, flags, nullptr, nullptr);
}

int pfpl_decompress_async(const void* in, uint64_t in_bytes, const void* hdr_host, void* out,
                          uint64_t cap, uint64_t* result_dev, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (!in || !hdr_host || !result_dev) return PFPL_ERR_ARG;
    if (!aligned16(in)) return PFPL_ERR_ALIGN;
    uint64_t n = 0;
    int dtype = 0;
    int st = parse_header((const uint8_t*)hdr_host, kHeaderBytes, &n, &dtype, nullptr, nullptr,
                          nullptr, nullptr, nullptr);
    if (st != PFPL_OK) return st;
    if (in_bytes < kHeaderBytes) return PFPL_ERR_CORRUPT;
    const uint64_t C = chunks_of(n, dtype);
    if (in_bytes < kHeaderBytes + 4 * C) return PFPL_ERR_CORRUPT;
    CK(cudaMemsetAsync(result_dev, 0, 16, s));
    const uint8_t* base = (const uint8_t*)in;
    uint64_t nout = 0;
    return enqueue_decompress((const uint8_t*)hdr_host, (const uint32_t*)(base + kHeaderBytes), 0,
                              C, base + kHeaderBytes + 4 * C, in_bytes - kHeaderBytes - 4 * C, out,
                              cap, (int*)(result_dev + 1), s, &nout);
}

int pfpl_decompress(const void* in, uint64_t in_bytes, void* out, uint64_t* out_bytes,
                    void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (!in || !out_bytes) return PFPL_ERR_ARG;
    if (!aligned16(in)) return PFPL_ERR_ALIGN;
    if (in_bytes < kHeaderBytes) return PFPL_ERR_CORRUPT;
    Scratch* sc = nullptr;
    int st = get_scratch(s, 0, &sc);
    if (st != PFPL_OK) return st;
    CK(cudaMemcpyAsync(sc->hdr_host, in, kHeaderBytes, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    uint8_t hdr[kHeaderBytes];
    memcpy(hdr, sc->hdr_host, kHeaderBytes);
    uint64_t n = 0;
    int dtype = 0;
    st = parse_header(hdr, kHeaderBytes, &n, &dtype, nullptr, nullptr, nullptr, nullptr, nullptr);
    if (st != PFPL_OK) return st;
    const uint64_t C = chunks_of(n, dtype);
    if (in_bytes < kHeaderBytes + 4 * C) return PFPL_ERR_CORRUPT;
    CK(cudaMemsetAsync(sc->result + 1, 0, 8, s));
    const uint8_t* base = (const uint8_t*)in;
    uint64_t nout = 0;
    st = enqueue_decompress(hdr, (const uint32_t*)(base + kHeaderBytes), 0, C,
                            base + kHeaderBytes + 4 * C, in_bytes - kHeaderBytes - 4 * C, out,
                            *out_bytes, (int*)(sc->result + 1), s, &nout);
    if (st != PFPL_OK) return st;
    CK(cudaMemcpyAsync(sc->host + 1, sc->result + 1, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int err = (int)(int32_t)(uint32_t)sc->host[1];
    if (err) return err;
    *out_bytes = nout * tsz(dtype);
    return PFPL_OK;
}

int pfpl_decompress_verify(const void* in, uint64_t in_bytes, const void* orig, void* out,
                           uint64_t* out_bytes, pfpl_metrics* m, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (!in || !out_bytes || !orig || !m) return PFPL_ERR_ARG;
    if (!aligned16(in) || !aligned16(orig)) return PFPL_ERR_ALIGN;
    if (in_bytes < kHeaderBytes) return PFPL_ERR_CORRUPT;
    memset(m, 0, sizeof(*m));
    Scratch* sc = nullptr;
    int st = get_scratch(s, 0, &sc);
    if (st != PFPL_OK) return st;
    if (!sc->vm) CK(cudaMalloc(&sc->vm, 8 * sizeof(unsigned long long)));
    CK(cudaMemcpyAsync(sc->hdr_host, in, kHeaderBytes, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    uint8_t hdr[kHeaderBytes];
    memcpy(hdr, sc->hdr_host, kHeaderBytes);
    uint64_t n = 0;
    int dtype = 0, bound = 0;
    double eps = 0.0, range = 0.0;
    st = parse_header(hdr, kHeaderBytes, &n, &dtype, &bound, &eps, nullptr, nullptr, &range);
    if (st != PFPL_OK) return st;
    const uint64_t C = chunks_of(n, dtype);
    if (in_bytes < kHeaderBytes + 4 * C) return PFPL_ERR_CORRUPT;
    // accumulators: zeros, min = order(+inf), max = order(-inf)
    static const unsigned long long init[8] = {0, 0, 0, 0, 0, 0xFFF0000000000000ull /* ord(+inf) */,
                                               ~0xFFF0000000000000ull /* ord(-inf) */, 0};
    CK(cudaMemcpyAsync(sc->vm, init, sizeof(init), cudaMemcpyHostToDevice, s));
    CK(cudaMemsetAsync(sc->result + 1, 0, 8, s));
    const uint8_t* base = (const uint8_t*)in;
    uint64_t nout = 0;
    st = enqueue_decompress(hdr, (const uint32_t*)(base + kHeaderBytes), 0, C,
                            base + kHeaderBytes + 4 * C, in_bytes - kHeaderBytes - 4 * C, out,
                            *out_bytes, (int*)(sc->result + 1), s, &nout, orig, sc->vm);
    if (st != PFPL_OK) return st;
    unsigned long long v[8];
    CK(cudaMemcpyAsync(sc->host + 1, sc->result + 1, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(v, sc->vm, sizeof(v), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int err = (int)(int32_t)(uint32_t)sc->host[1];
    if (err) return err;
    *out_bytes = nout * tsz(dtype);
    auto unord = [](unsigned long long o) { return u2d_h((o >> 63) ? (o & 0x7FFFFFFFFFFFFFFFull) : ~o); };
    m->n = n;
    m->n_finite = v[4];
    m->max_abs_err = u2d_h(v[0]);
    m->max_rel_err = u2d_h(v[1]);
    m->sum_sq_err = u2d_h(v[2]);
    m->violations = v[3];
    m->value_min = v[4] ? unord(v[5]) : 0.0;
    m->value_max = v[4] ? unord(v[6]) : 0.0;
    m->mse = v[4] ? m->sum_sq_err / (double)v[4] : 0.0;
    const double rng = m->value_max - m->value_min;
    m->psnr = (m->mse > 0.0 && rng > 0.0) ? 20.0 * log10(rng) - 10.0 * log10(m->mse) : INFINITY;
    return PFPL_OK;
}

int pfpl_minmax(const void* in, uint64_t n, int dtype, double* mnmx_dev, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    if ((n && !in) || !mnmx_dev) return PFPL_ERR_ARG;
    if (!aligned16(in)) return PFPL_ERR_ALIGN;
    Scratch* sc = nullptr;
    int st = get_scratch(s, 0, &sc);
    if (st != PFPL_OK) return st;
    CK(launch_minmax(dtype, in, n, sc->partial, kMinmaxBlocks, s));
    CK(launch_minmax_final(sc->partial, kMinmaxBlocks, mnmx_dev, s));
    g_launches += 2;
    return PFPL_OK;
}

int pfpl_compress_shard(const void* in, uint64_t n_local, uint64_t first_chunk, uint64_t n_total,
                        int dtype, int bound, double eps, unsigned opts, const double* mnmx_dev,
                        void* out, uint64_t cap, uint64_t* payload_bytes, void* hdr_out_host,
                        void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    if (!payload_bytes) return PFPL_ERR_ARG;
    const uint64_t cw = kChunkBytes / tsz(dtype);
    const uint64_t Ct = chunks_of(n_total, dtype);
    const uint64_t Cl = chunks_of(n_local, dtype);
    if (first_chunk + Cl > Ct) return PFPL_ERR_ARG;
    if (first_chunk * cw + n_local > n_total) return PFPL_ERR_ARG;
    if (n_local % cw && first_chunk * cw + n_local != n_total) return PFPL_ERR_ARG;
    if (bound == PFPL_NOA && !mnmx_dev) return PFPL_ERR_ARG;
    if (cap < 4 * Cl) return PFPL_ERR_CAPACITY;
    Scratch* sc = nullptr;
    int st = enqueue_compress(in, n_local, n_total, dtype, bound, eps, opts, mnmx_dev,
                              (uint8_t*)out, cap, (uint32_t*)out, 4 * Cl, 0, nullptr, s, &sc);
    if (st != PFPL_OK) return st;
    CK(cudaMemcpyAsync(sc->host, sc->result, 8, cudaMemcpyDeviceToHost, s));
    QConst qc;
    int mode = 0;
    host_qconst(dtype, bound, eps, opts, &qc, &mode);
    QConst qch;
    if (bound == PFPL_NOA) CK(cudaMemcpyAsync(&qch, sc->qc_dev, sizeof(QConst), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    if (bound == PFPL_NOA) qc = qch;
    const uint64_t total = sc->host[0];
    if (total > cap) return PFPL_ERR_CAPACITY;
    *payload_bytes = total - 4 * Cl;
    if (hdr_out_host) {
        uint8_t* h = (uint8_t*)hdr_out_host;
        memset(h, 0, kHeaderBytes);
        h[0] = 'P'; h[1] = 'F'; h[2] = 'P'; h[3] = 'L';
        h[4] = 1; h[5] = (uint8_t)dtype; h[6] = (uint8_t)bound; h[7] = (uint8_t)qc.flags;
        const uint64_t f[5] = {n_total, d2u_h(eps), qc.qconst, d2u_h(qc.range), (uint64_t)kChunkBytes};
        for (int i = 0; i < 5; ++i)
            for (int k = 0; k < 8; ++k) h[8 + 8 * i + k] = (uint8_t)(f[i] >> (8 * k));
    }
    return PFPL_OK;
}

int pfpl_decompress_chunks(const void* hdr_host, const uint32_t* table_host, uint64_t first_chunk,
                           uint64_t n_chunks, const void* payload, uint64_t payload_bytes,
                           void* out, uint64_t cap, void* stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (!hdr_host || (n_chunks && (!table_host || !payload))) return PFPL_ERR_ARG;
    if (payload && !aligned16(payload)) return PFPL_ERR_ALIGN;
    Scratch* sc = nullptr;
    int st = get_scratch(s, n_chunks, &sc);
    if (st != PFPL_OK) return st;
    if (n_chunks > sc->table_cap) {
        if (sc->table_dev) CK(cudaFree(sc->table_dev));
        CK(cudaMalloc(&sc->table_dev, n_chunks * 4));
        sc->table_cap = n_chunks;
    }
    if (n_chunks) CK(cudaMemcpyAsync(sc->table_dev, table_host, n_chunks * 4, cudaMemcpyHostToDevice, s));
    CK(cudaMemsetAsync(sc->result + 1, 0, 8, s));
    uint64_t nout = 0;
    st = enqueue_decompress((const uint8_t*)hdr_host, sc->table_dev, first_chunk, n_chunks,
                            (const uint8_t*)payload, payload_bytes, out, cap, (int*)(sc->result + 1),
                            s, &nout);
    if (st != PFPL_OK) return st;
    CK(cudaMemcpyAsync(sc->host + 1, sc->result + 1, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    const int err = (int)(int32_t)(uint32_t)sc->host[1];
    return err ? err : PFPL_OK;
}

const char* pfpl_strerror(int st) {
    switch (st) {
        case PFPL_OK: return "ok";
        case PFPL_ERR_ARG: return "invalid argument";
        case PFPL_ERR_BOUND: return "invalid error bound";
        case PFPL_ERR_CAPACITY: return "output capacity too small";
        case PFPL_ERR_CORRUPT: return "corrupt stream";
        case PFPL_ERR_ALIGN: return "buffer not 16-byte aligned";
        case PFPL_ERR_CUDA: return "CUDA runtime error";
        default: return "unknown status";
    }
}

int pfpl_last_cuda_error(void) { return g_last_cuda.load(); }

int pfpl_watchdog_report(unsigned int* out4) {
    if (!g_wd_host || !out4) return 0;
    for (int i = 0; i < 4; ++i) out4[i] = ((volatile unsigned int*)g_wd_host)[i];
    return out4[0] != 0;
}

int pfpl_release_scratch(void) {
    int dev = 0;
    CK(cudaGetDevice(&dev));
    release_pipes(dev);
    release_lanes(dev);
    std::lock_guard<std::mutex> lk(g_mu);
    for (auto it = g_scratch.begin(); it != g_scratch.end();) {
        if (it->first.first != dev) { ++it; continue; }
        Scratch* sc = it->second;
        cudaDeviceSynchronize();
        cudaFree(sc->status); cudaFree(sc->ticket); cudaFree(sc->qc_dev); cudaFree(sc->mnmx);
        cudaFree(sc->partial); cudaFree(sc->result); cudaFreeHost(sc->host);
        cudaFreeHost(sc->hdr_host); cudaFree(sc->table_dev); cudaFree(sc->offs);
        cudaFree(sc->stats); cudaFree(sc->vm);
        delete sc;
        it = g_scratch.erase(it);
    }
    return PFPL_OK;
}

int pfpl_last_stats(void* stream, uint64_t* unquantizable, uint64_t* raw_chunks) {
    if (!unquantizable || !raw_chunks) return PFPL_ERR_ARG;
    *unquantizable = 0;
    *raw_chunks = 0;
    cudaStream_t s = (cudaStream_t)stream;
    int dev = 0;
    CK(cudaGetDevice(&dev));
    Scratch* sc = nullptr;
    {
        std::lock_guard<std::mutex> lk(g_mu);
        auto it = g_scratch.find({dev, (void*)s});
        if (it != g_scratch.end()) sc = it->second;
    }
    if (!sc || sc->stat_seq == 0) return PFPL_OK;          // no compression on this stream yet
    unsigned long long v[2];
    CK(cudaMemcpyAsync(v, sc->stats + 2 * ((sc->stat_seq - 1) & 1), sizeof(v), cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    *unquantizable = v[0];
    *raw_chunks = v[1];
    return PFPL_OK;
}

uint64_t pfpl_launch_count(void) { return g_launches.load(); }
int pfpl_f32_encoder_form(int bound) {
    if (!g_x0_host || (bound != PFPL_ABS && bound != PFPL_NOA)) return 0;
    return ((volatile unsigned int*)g_x0_host)[bound == PFPL_NOA ? 1 : 0] == 1u ? 1 : 0;
}

const char* pfpl_version(void) { return "pfpl-b200 1.0 sm_100a (stream format v1)"; }

}  // extern "C"
