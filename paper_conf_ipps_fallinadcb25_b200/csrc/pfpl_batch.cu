// pfpl_batch.cu -- many independent fields in one call (compress and decompress) (SURVEY 8(f) NEXT-4:
// multi-field batches such as CESM's 33 per-timestep fields).  A small
// field (CESM: 1,583 chunks, 26 MB) keeps the persistent encoder busy for only
// ~2 chunks per CTA, so one field per launch is bound by ramp-up and drain.
// The batch forks the fields over a cached pool of non-blocking streams so
// consecutive fields' launches overlap each other's tails, then joins back
// onto the caller's stream with one D2H of every stream size.  Each field's
// stream is exactly pfpl_compress's (same kernel, same arguments).
#include <cuda_runtime.h>

#include <cstdlib>
#include <map>
#include <mutex>
#include <utility>

#include "../../include/pfpl.h"
#include "pfpl_internal.h"

using namespace pfpl;

namespace {

constexpr int kMaxLanes = 16;

// lanes (internal streams) a batch forks over; PFPL_BATCH_LANES overrides (tuning)
int lanes_cfg() {
    static int v = [] {
        const char* e = getenv("PFPL_BATCH_LANES");
        int x = e ? atoi(e) : 4;
        return x < 1 ? 1 : (x > kMaxLanes ? kMaxLanes : x);
    }();
    return v;
}

struct Lanes {
    std::mutex mu;                  // held for a whole batch call (one user of res/hdr at a time)
    cudaStream_t st[kMaxLanes] = {};
    cudaEvent_t done[kMaxLanes] = {};
    cudaEvent_t fork = nullptr;
    uint64_t* res_dev = nullptr;    // 2 words per field (pfpl_compress_async's result)
    uint64_t* res_host = nullptr;
    int res_cap = 0;
    uint8_t* hdr_host = nullptr;    // kHeaderBytes per field (decompress)
    int hdr_cap = 0;
};

std::mutex g_mu;
std::map<std::pair<int, void*>, Lanes*> g_lanes;

#define BK(x)                                                       \
    do {                                                            \
        cudaError_t _e = (x);                                       \
        if (_e != cudaSuccess) return record_cuda_error((int)_e);   \
    } while (0)

int init_lanes(Lanes* L, cudaStream_t s, int count, Lanes** out) {
    if (!L->fork) {
        for (int i = 0; i < kMaxLanes; ++i) {
            BK(cudaStreamCreateWithFlags(&L->st[i], cudaStreamNonBlocking));
            BK(cudaEventCreateWithFlags(&L->done[i], cudaEventDisableTiming));
        }
        BK(cudaEventCreateWithFlags(&L->fork, cudaEventDisableTiming));
    }
    if (count > L->res_cap) {
        BK(cudaStreamSynchronize(s));
        if (L->res_dev) BK(cudaFree(L->res_dev));
        if (L->res_host) BK(cudaFreeHost(L->res_host));
        L->res_dev = nullptr;
        L->res_host = nullptr;
        L->res_cap = 0;
        BK(cudaMalloc((void**)&L->res_dev, 16ull * count));
        BK(cudaMallocHost((void**)&L->res_host, 16ull * count));
        L->res_cap = count;
    }
    *out = L;
    return PFPL_OK;
}

int get_lanes(cudaStream_t s, int count, Lanes** out, std::unique_lock<std::mutex>* own) {
    int dev = 0;
    BK(cudaGetDevice(&dev));
    std::unique_lock<std::mutex> lk(g_mu);
    Lanes*& L = g_lanes[{dev, (void*)s}];
    if (!L) L = new Lanes();
    Lanes* const Lp = L;
    lk.unlock();
    *own = std::unique_lock<std::mutex>(Lp->mu);     // two threads on one stream are serialised
    return init_lanes(Lp, s, count, out);
}

int ensure_hdr(Lanes* L, cudaStream_t s, int count) {
    if (count <= L->hdr_cap) return PFPL_OK;
    BK(cudaStreamSynchronize(s));
    if (L->hdr_host) BK(cudaFreeHost(L->hdr_host));
    L->hdr_host = nullptr;
    L->hdr_cap = 0;
    BK(cudaMallocHost((void**)&L->hdr_host, (size_t)kHeaderBytes * count));
    L->hdr_cap = count;
    return PFPL_OK;
}

}  // namespace

void pfpl::release_lanes(int dev) {
    std::lock_guard<std::mutex> lk(g_mu);
    for (auto it = g_lanes.begin(); it != g_lanes.end();) {
        if (it->first.first != dev) { ++it; continue; }
        Lanes* L = it->second;
        cudaDeviceSynchronize();
        for (int i = 0; i < kMaxLanes; ++i) {
            if (L->st[i]) cudaStreamDestroy(L->st[i]);
            if (L->done[i]) cudaEventDestroy(L->done[i]);
        }
        if (L->fork) cudaEventDestroy(L->fork);
        cudaFree(L->res_dev); cudaFreeHost(L->res_host); cudaFreeHost(L->hdr_host);
        delete L;
        it = g_lanes.erase(it);
    }
}

extern "C" {

int pfpl_compress_batch(int count, const void* const* in, const uint64_t* n, int dtype, int bound,
                        double eps, unsigned opts, void* const* out, uint64_t* out_bytes,
                        void* stream) {
    if (count < 0 || (count && (!in || !n || !out || !out_bytes))) return PFPL_ERR_ARG;
    if (count == 0) return PFPL_OK;
    // every field's argument errors before anything is enqueued (pfpl.h)
    for (int f = 0; f < count; ++f) {
        const int e = check_compress_args(in[f], n[f], dtype, bound, eps, opts, out[f], out_bytes[f]);
        if (e != PFPL_OK) return e;
    }
    cudaStream_t s = (cudaStream_t)stream;
    Lanes* L = nullptr;
    std::unique_lock<std::mutex> own;
    int st = get_lanes(s, count, &L, &own);
    if (st != PFPL_OK) return st;
    BK(cudaEventRecord(L->fork, s));
    const int lanes = count < lanes_cfg() ? count : lanes_cfg();
    for (int i = 0; i < lanes; ++i) BK(cudaStreamWaitEvent(L->st[i], L->fork, 0));
    int first_err = PFPL_OK;
    for (int f = 0; f < count; ++f) {
        st = pfpl_compress_async(in[f], n[f], dtype, bound, eps, opts, out[f], out_bytes[f],
                                 L->res_dev + 2 * f, L->st[f % lanes]);
        if (st != PFPL_OK) {
            first_err = st;
            break;
        }
    }
    // join every lane (also after an error, so nothing is left in flight)
    for (int i = 0; i < lanes; ++i) {
        BK(cudaEventRecord(L->done[i], L->st[i]));
        BK(cudaStreamWaitEvent(s, L->done[i], 0));
    }
    if (first_err != PFPL_OK) {
        BK(cudaStreamSynchronize(s));
        return first_err;
    }
    BK(cudaMemcpyAsync(L->res_host, L->res_dev, 16ull * count, cudaMemcpyDeviceToHost, s));
    BK(cudaStreamSynchronize(s));
    for (int f = 0; f < count; ++f) {
        const uint64_t total = L->res_host[2 * f];
        const int code = (int)(int32_t)(uint32_t)L->res_host[2 * f + 1];
        if (code != 0 || total > out_bytes[f]) {
            if (first_err == PFPL_OK) first_err = code ? code : PFPL_ERR_CAPACITY;
        } else {
            out_bytes[f] = total;
        }
    }
    return first_err;
}

int pfpl_decompress_batch(int count, const void* const* in, const uint64_t* in_bytes,
                          void* const* out, uint64_t* out_bytes, void* stream) {
    if (count < 0 || (count && (!in || !in_bytes || !out || !out_bytes))) return PFPL_ERR_ARG;
    if (count == 0) return PFPL_OK;
    for (int f = 0; f < count; ++f)
        if (!in[f] || in_bytes[f] < kHeaderBytes) return PFPL_ERR_CORRUPT;
    cudaStream_t s = (cudaStream_t)stream;
    Lanes* L = nullptr;
    std::unique_lock<std::mutex> own;
    int st = get_lanes(s, count, &L, &own);
    if (st == PFPL_OK) st = ensure_hdr(L, s, count);
    if (st != PFPL_OK) return st;
    // every header in one round trip (n and dtype size each output)
    for (int f = 0; f < count; ++f)
        BK(cudaMemcpyAsync(L->hdr_host + (size_t)kHeaderBytes * f, in[f], kHeaderBytes,
                           cudaMemcpyDeviceToHost, s));
    BK(cudaStreamSynchronize(s));
    BK(cudaEventRecord(L->fork, s));
    const int lanes = count < lanes_cfg() ? count : lanes_cfg();
    for (int i = 0; i < lanes; ++i) BK(cudaStreamWaitEvent(L->st[i], L->fork, 0));
    int first_err = PFPL_OK;
    for (int f = 0; f < count; ++f) {
        st = pfpl_decompress_async(in[f], in_bytes[f], L->hdr_host + (size_t)kHeaderBytes * f,
                                   out[f], out_bytes[f], L->res_dev + 2 * f, L->st[f % lanes]);
        if (st != PFPL_OK) {
            first_err = st;
            break;
        }
    }
    for (int i = 0; i < lanes; ++i) {
        BK(cudaEventRecord(L->done[i], L->st[i]));
        BK(cudaStreamWaitEvent(s, L->done[i], 0));
    }
    if (first_err != PFPL_OK) {
        BK(cudaStreamSynchronize(s));
        return first_err;
    }
    BK(cudaMemcpyAsync(L->res_host, L->res_dev, 16ull * count, cudaMemcpyDeviceToHost, s));
    BK(cudaStreamSynchronize(s));
    for (int f = 0; f < count; ++f) {
        const int code = (int)(int32_t)(uint32_t)L->res_host[2 * f + 1];
        if (code != 0) {
            if (first_err == PFPL_OK) first_err = code;
            continue;
        }
        uint64_t n = 0;
        int dtype = 0, bound = 0;
        double eps = 0;
        unsigned flags = 0;
        pfpl_peek_header(L->hdr_host + (size_t)kHeaderBytes * f, kHeaderBytes, &n, &dtype, &bound,
                         &eps, &flags);
        out_bytes[f] = n * (dtype == PFPL_F32 ? 4u : 8u);
    }
    return first_err;
}

}  // extern "C"
