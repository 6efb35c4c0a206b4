// pfpl_pipeline.cu -- host-resident (out-of-core) compression and decompression
// (SURVEY 8(f) NEXT-4).  The array lives in host memory and may exceed HBM; it
// is streamed through two device segment buffers.  Per segment of S chunks:
//   H2D (copy stream) -> pfpl_compress_shard (compute stream) -> D2H (copy stream)
// with segment k+1's upload and segment k-1's download overlapping segment k's
// kernel.  Chunks are independent, so the shard of chunks
// [k*S, (k+1)*S) produces exactly the size-table slice and payload bytes the
// single-device call would (the payload offsets are a prefix sum of the
// chunk sizes, here carried across segments on the host).  The stream is
// therefore byte-identical to pfpl_compress of the whole array.  The paper
// excludes transfers from its timings; this path is what a user whose
// data sits in host memory (multi-GB fields) pays end to end.
#include <cuda_runtime.h>

#include <cstring>
#include <map>
#include <mutex>
#include <utility>
#include <vector>

#include "../../include/pfpl.h"
#include "pfpl_internal.h"

using namespace pfpl;

namespace {

constexpr uint64_t kDefaultSegChunks = 2048;   // 32 MiB of input per segment

// Per-(device, stream) pipeline state, cached across calls: two non-blocking
// copy streams, the hand-off events and the two pairs of segment buffers.
// Creating streams and mapping 256 MiB of buffers on every call costs more
// than the transfers themselves (measured: 14 GB/s vs 51 GB/s sequential).
struct Pipe {
    std::mutex mu;                  // held for a whole call: one user of the buffers at a time
    cudaStream_t s = nullptr;       // caller's compute stream
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t in_ready[2] = {}, in_free[2] = {}, out_free[2] = {};
    uint8_t* inbuf[2] = {};
    uint8_t* outbuf[2] = {};
    uint64_t in_cap = 0, out_cap = 0;

    cudaError_t ensure(cudaStream_t cs, uint64_t in_bytes, uint64_t out_bytes) {
        s = cs;
        cudaError_t e;
        if (!h2d) {
            if ((e = cudaStreamCreateWithFlags(&h2d, cudaStreamNonBlocking))) return e;
            if ((e = cudaStreamCreateWithFlags(&d2h, cudaStreamNonBlocking))) return e;
            for (int b = 0; b < 2; ++b) {
                if ((e = cudaEventCreateWithFlags(&in_ready[b], cudaEventDisableTiming))) return e;
                if ((e = cudaEventCreateWithFlags(&in_free[b], cudaEventDisableTiming))) return e;
                if ((e = cudaEventCreateWithFlags(&out_free[b], cudaEventDisableTiming))) return e;
            }
        }
        if (in_bytes > in_cap || out_bytes > out_cap) {
            if ((e = cudaDeviceSynchronize())) return e;
            if (in_bytes > in_cap) {
                for (int b = 0; b < 2; ++b) {
                    if (inbuf[b]) cudaFree(inbuf[b]);
                    inbuf[b] = nullptr;
                }
                in_cap = 0;
                for (int b = 0; b < 2; ++b)
                    if ((e = cudaMalloc((void**)&inbuf[b], in_bytes))) return e;
                in_cap = in_bytes;
            }
            if (out_bytes > out_cap) {
                for (int b = 0; b < 2; ++b) {
                    if (outbuf[b]) cudaFree(outbuf[b]);
                    outbuf[b] = nullptr;
                }
                out_cap = 0;
                for (int b = 0; b < 2; ++b)
                    if ((e = cudaMalloc((void**)&outbuf[b], out_bytes))) return e;
                out_cap = out_bytes;
            }
        }
        // buffers are free once the caller's stream reaches this point
        for (int b = 0; b < 2; ++b) {
            if ((e = cudaEventRecord(in_free[b], s))) return e;
            if ((e = cudaEventRecord(out_free[b], s))) return e;
        }
        return cudaSuccess;
    }
    void drain() {
        if (h2d) cudaStreamSynchronize(h2d);
        if (d2h) cudaStreamSynchronize(d2h);
        cudaStreamSynchronize(s);
    }
};

std::mutex g_pipe_mu;
std::map<std::pair<int, void*>, Pipe*> g_pipes;

// owns the pipe for one call (two host threads passing the same stream are
// serialised instead of sharing its buffers and events); drains the pipe's
// streams when the call leaves, on every path, before releasing it
struct PipeUse {
    Pipe* p = nullptr;
    std::unique_lock<std::mutex> lk;
    ~PipeUse() {
        if (p) p->drain();
    }
};

cudaError_t get_pipe(cudaStream_t cs, uint64_t in_bytes, uint64_t out_bytes, PipeUse* use) {
    int dev = 0;
    cudaError_t e = cudaGetDevice(&dev);
    if (e) return e;
    Pipe* p;
    {
        std::lock_guard<std::mutex> lk(g_pipe_mu);
        Pipe*& slot = g_pipes[{dev, (void*)cs}];
        if (!slot) slot = new Pipe();
        p = slot;
    }
    use->lk = std::unique_lock<std::mutex>(p->mu);
    use->p = p;
    return p->ensure(cs, in_bytes, out_bytes);
}

#define PK(x)                                                         \
    do {                                                              \
        cudaError_t _e = (x);                                         \
        if (_e != cudaSuccess) return record_cuda_error((int)_e);   \
    } while (0)

inline uint64_t tsz_of(int dtype) { return dtype == PFPL_F32 ? 4u : 8u; }

}  // namespace

void pfpl::release_pipes(int dev) {
    std::lock_guard<std::mutex> lk(g_pipe_mu);
    for (auto it = g_pipes.begin(); it != g_pipes.end();) {
        if (it->first.first != dev) { ++it; continue; }
        Pipe* p = it->second;
        cudaDeviceSynchronize();
        for (int b = 0; b < 2; ++b) {
            cudaFree(p->inbuf[b]); cudaFree(p->outbuf[b]);
            cudaEventDestroy(p->in_ready[b]); cudaEventDestroy(p->in_free[b]);
            cudaEventDestroy(p->out_free[b]);
        }
        if (p->h2d) cudaStreamDestroy(p->h2d);
        if (p->d2h) cudaStreamDestroy(p->d2h);
        delete p;
        it = g_pipes.erase(it);
    }
}

extern "C" {

int pfpl_compress_host(const void* in_host, uint64_t n, int dtype, int bound, double eps,
                       unsigned opts, void* out_host, uint64_t* out_bytes, uint64_t seg_chunks,
                       void* stream) {
    if (dtype != PFPL_F32 && dtype != PFPL_F64) return PFPL_ERR_ARG;
    if (bound != PFPL_ABS && bound != PFPL_REL && bound != PFPL_NOA) return PFPL_ERR_ARG;
    if (!out_host || !out_bytes || (n && !in_host)) return PFPL_ERR_ARG;
    if (n > (1ull << 40)) return PFPL_ERR_ARG;
    const uint64_t ts = tsz_of(dtype);
    const uint64_t cw = kChunkBytes / ts;
    const uint64_t C = (n + cw - 1) / cw;
    // S in [1, max(C, 1)]: a larger request means one segment (and keeps S*cw,
    // k*S*kChunkBytes and the segment count free of overflow)
    uint64_t S = seg_chunks ? seg_chunks : kDefaultSegChunks;
    if (S > C) S = C ? C : 1;
    const uint64_t cap = *out_bytes;
    const uint64_t pay_base = kHeaderBytes + 4 * C;
    if (cap < pay_base) return PFPL_ERR_CAPACITY;
    const uint8_t* src = (const uint8_t*)in_host;
    uint8_t* dst = (uint8_t*)out_host;
    cudaStream_t cs = (cudaStream_t)stream;
    const uint64_t nseg = C ? (C + S - 1) / S : 1;
    const uint64_t seg_in = (C < S ? C : S) * kChunkBytes;
    const uint64_t seg_out = 4 * (C < S ? C : S) + seg_in;

    PipeUse use;
    PK(get_pipe(cs, seg_in ? seg_in : 16, seg_out ? seg_out : 16, &use));
    Pipe& p = *use.p;
    auto seg_elems = [&](uint64_t k) {
        const uint64_t e0 = k * S * cw;
        const uint64_t rest = n - e0;
        return rest < S * cw ? rest : S * cw;
    };
    auto upload = [&](uint64_t k) -> cudaError_t {
        const int b = (int)(k & 1);
        cudaError_t e = cudaStreamWaitEvent(p.h2d, p.in_free[b], 0);
        if (!e && seg_elems(k))
            e = cudaMemcpyAsync(p.inbuf[b], src + k * S * kChunkBytes, seg_elems(k) * ts,
                                cudaMemcpyHostToDevice, p.h2d);
        if (!e) e = cudaEventRecord(p.in_ready[b], p.h2d);
        return e;
    };

    // NOA needs the global {min, max} before any chunk is quantized:
    // a first streaming pass, one pfpl_minmax per segment, combined on the host
    // (min/max are order-independent, so the result equals the one-pass value).
    double* mm_dev = nullptr;
    if (bound == PFPL_NOA) {
        PK(cudaMallocAsync((void**)&mm_dev, 2 * nseg * sizeof(double), cs));
        std::vector<double> mm_vec(2 * nseg);
        double* mm_host = mm_vec.data();
        int st = PFPL_OK;
        cudaError_t e = upload(0);
        for (uint64_t k = 0; k < nseg && !e && st == PFPL_OK; ++k) {
            const int b = (int)(k & 1);
            if (k + 1 < nseg) e = upload(k + 1);
            if (!e) e = cudaStreamWaitEvent(cs, p.in_ready[b], 0);
            if (e) break;
            st = pfpl_minmax(p.inbuf[b], seg_elems(k), dtype, mm_dev + 2 * k, cs);
            if (st == PFPL_OK) e = cudaEventRecord(p.in_free[b], cs);
        }
        if (!e && st == PFPL_OK)
            e = cudaMemcpyAsync(mm_host, mm_dev, 2 * nseg * sizeof(double),
                                cudaMemcpyDeviceToHost, cs);
        if (!e && st == PFPL_OK) e = cudaStreamSynchronize(cs);
        double mn = __builtin_inf(), mx = -__builtin_inf();
        for (uint64_t k = 0; k < nseg && !e && st == PFPL_OK; ++k) {
            const double a = mm_host[2 * k], b = mm_host[2 * k + 1];
            mn = a < mn ? a : mn;
            mx = b > mx ? b : mx;
        }
        mm_host[0] = mn;
        mm_host[1] = mx;
        if (!e && st == PFPL_OK)
            e = cudaMemcpyAsync(mm_dev, mm_host, 2 * sizeof(double), cudaMemcpyHostToDevice, cs);
        if (!e && st == PFPL_OK) e = cudaStreamSynchronize(cs);
        if (e) {
            cudaFreeAsync(mm_dev, cs);
            return record_cuda_error((int)e);
        }
        if (st != PFPL_OK) {
            cudaFreeAsync(mm_dev, cs);
            return st;
        }
    }

    int st = PFPL_OK;
    cudaError_t e = upload(0);
    uint64_t pay_off = 0;
    for (uint64_t k = 0; k < nseg && !e && st == PFPL_OK; ++k) {
        const int b = (int)(k & 1);
        if (k + 1 < nseg) e = upload(k + 1);
        if (!e) e = cudaStreamWaitEvent(cs, p.in_ready[b], 0);
        if (!e) e = cudaStreamWaitEvent(cs, p.out_free[b], 0);
        if (e) break;
        const uint64_t nk = seg_elems(k);
        const uint64_t Ck = (nk + cw - 1) / cw;
        uint64_t pb = 0;
        uint8_t hdr[kHeaderBytes];
        st = pfpl_compress_shard(p.inbuf[b], nk, k * S, n, dtype, bound, eps, opts, mm_dev,
                                 p.outbuf[b], seg_out ? seg_out : 16, &pb, k == 0 ? hdr : nullptr,
                                 cs);   // synchronises cs
        if (st != PFPL_OK) break;
        if (k == 0) memcpy(dst, hdr, kHeaderBytes);
        e = cudaEventRecord(p.in_free[b], cs);
        if (e) break;
        if (pay_base + pay_off + pb > cap) {
            st = PFPL_ERR_CAPACITY;
            break;
        }
        if (Ck) e = cudaMemcpyAsync(dst + kHeaderBytes + 4 * k * S, p.outbuf[b], 4 * Ck,
                                    cudaMemcpyDeviceToHost, p.d2h);
        if (!e && pb) e = cudaMemcpyAsync(dst + pay_base + pay_off, p.outbuf[b] + 4 * Ck, pb,
                                          cudaMemcpyDeviceToHost, p.d2h);
        if (!e) e = cudaEventRecord(p.out_free[b], p.d2h);
        pay_off += pb;
    }
    if (!e) e = cudaStreamSynchronize(p.d2h);
    if (mm_dev) cudaFreeAsync(mm_dev, cs);
    if (e) return record_cuda_error((int)e);
    if (st != PFPL_OK) return st;
    *out_bytes = pay_base + pay_off;
    return PFPL_OK;
}

int pfpl_decompress_host(const void* in_host, uint64_t in_bytes, void* out_host,
                         uint64_t* out_bytes, uint64_t seg_chunks, void* stream) {
    if (!in_host || !out_host || !out_bytes) return PFPL_ERR_ARG;
    if (in_bytes < kHeaderBytes) return PFPL_ERR_CORRUPT;
    uint64_t n = 0;
    int dtype = 0, bound = 0;
    double eps = 0;
    unsigned flags = 0;
    int st = pfpl_peek_header(in_host, in_bytes, &n, &dtype, &bound, &eps, &flags);
    if (st != PFPL_OK) return st;
    const uint64_t ts = tsz_of(dtype);
    const uint64_t cw = kChunkBytes / ts;
    const uint64_t C = (n + cw - 1) / cw;
    if (in_bytes < kHeaderBytes + 4 * C) return PFPL_ERR_CORRUPT;
    if (*out_bytes < n * ts) return PFPL_ERR_CAPACITY;
    const uint8_t* src = (const uint8_t*)in_host;
    const uint32_t* table = (const uint32_t*)(src + kHeaderBytes);   // may be unaligned
    const uint8_t* payload = src + kHeaderBytes + 4 * C;
    const uint64_t pay_bytes = in_bytes - kHeaderBytes - 4 * C;
    if (C == 0) {                       // header only: nothing may follow it
        if (in_bytes != kHeaderBytes) return PFPL_ERR_CORRUPT;
        *out_bytes = 0;
        return PFPL_OK;
    }
    uint64_t S = seg_chunks ? seg_chunks : kDefaultSegChunks;
    if (S > C) S = C;
    const uint64_t nseg = (C + S - 1) / S;
    // segment payload offsets: host prefix sum of the size table.  Every
    // entry is validated here, with the rules of the device path (a chunk holds at
    // most its raw bytes; a compressed chunk at least the 4-byte M4; the sizes sum
    // to exactly the payload), so a corrupt table is rejected before any device
    // buffer is sized from it.
    uint64_t* seg_off = new uint64_t[nseg + 1];
    uint32_t* tab = new uint32_t[C];
    memcpy(tab, table, 4 * C);
    struct Free {
        uint64_t* a; uint32_t* b;
        ~Free() { delete[] a; delete[] b; }
    } fr{seg_off, tab};
    uint64_t acc = 0, seg_max = 0;
    for (uint64_t k = 0; k < nseg; ++k) {
        seg_off[k] = acc;
        const uint64_t c1 = (k + 1) * S < C ? (k + 1) * S : C;
        for (uint64_t c = k * S; c < c1; ++c) {
            const uint64_t m = c + 1 < C ? cw : n - c * cw;
            const uint64_t rawb = m * ts;
            if (tab[c] > rawb || (tab[c] < 4 && tab[c] != rawb)) return PFPL_ERR_CORRUPT;
            acc += tab[c];
        }
        if (acc - seg_off[k] > seg_max) seg_max = acc - seg_off[k];
    }
    seg_off[nseg] = acc;
    if (acc != pay_bytes) return PFPL_ERR_CORRUPT;
    cudaStream_t cs = (cudaStream_t)stream;
    const uint64_t seg_out = (C < S ? C : S) * kChunkBytes;
    PipeUse use;
    PK(get_pipe(cs, seg_max ? seg_max : 16, seg_out, &use));
    Pipe& p = *use.p;
    const uint8_t* hdr = src;
    uint8_t* dst = (uint8_t*)out_host;
    auto upload = [&](uint64_t k) -> cudaError_t {
        const int b = (int)(k & 1);
        cudaError_t e = cudaStreamWaitEvent(p.h2d, p.in_free[b], 0);
        const uint64_t bytes = seg_off[k + 1] - seg_off[k];
        if (!e && bytes)
            e = cudaMemcpyAsync(p.inbuf[b], payload + seg_off[k], bytes, cudaMemcpyHostToDevice,
                                p.h2d);
        if (!e) e = cudaEventRecord(p.in_ready[b], p.h2d);
        return e;
    };
    cudaError_t e = upload(0);
    for (uint64_t k = 0; k < nseg && !e && st == PFPL_OK; ++k) {
        const int b = (int)(k & 1);
        if (k + 1 < nseg) e = upload(k + 1);
        if (!e) e = cudaStreamWaitEvent(cs, p.in_ready[b], 0);
        if (!e) e = cudaStreamWaitEvent(cs, p.out_free[b], 0);
        if (e) break;
        const uint64_t c0 = k * S;
        const uint64_t Ck = (c0 + S < C ? S : C - c0);
        const uint64_t e0 = c0 * cw;
        const uint64_t nk = (n - e0 < Ck * cw) ? n - e0 : Ck * cw;
        st = pfpl_decompress_chunks(hdr, tab + c0, c0, Ck, p.inbuf[b], seg_off[k + 1] - seg_off[k],
                                    p.outbuf[b], seg_out, cs);   // synchronises cs
        if (st != PFPL_OK) break;
        e = cudaEventRecord(p.in_free[b], cs);
        if (!e) e = cudaMemcpyAsync(dst + e0 * ts, p.outbuf[b], nk * ts, cudaMemcpyDeviceToHost,
                                    p.d2h);
        if (!e) e = cudaEventRecord(p.out_free[b], p.d2h);
    }
    if (!e) e = cudaStreamSynchronize(p.d2h);
    if (e) return record_cuda_error((int)e);
    if (st != PFPL_OK) return st;
    *out_bytes = n * ts;
    return PFPL_OK;
}

}  // extern "C"
