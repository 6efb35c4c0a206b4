// pfpl_encode_host.cu -- launch-side code of the fused encoder (pfpl_encode.cuh):
// kernel selection, grid sizing, the TMA tensor map of the input.
#include <cstring>
#include "pfpl_encode.cuh"

namespace pfpl {

// ---------------------------------------------------------------------------
// host side
// ---------------------------------------------------------------------------
// one instantiation TU per (dtype, mode): pfpl_enc_inst.cu built with -DPFPL_DT/-DPFPL_MODE
#define PFPL_DECL(D, M) void* enc_ptr_##D##_##M(bool ms, bool x0);
PFPL_DECL(0, 0) PFPL_DECL(0, 1) PFPL_DECL(0, 2) PFPL_DECL(0, 3)
PFPL_DECL(1, 0) PFPL_DECL(1, 1) PFPL_DECL(1, 2) PFPL_DECL(1, 3)
#undef PFPL_DECL

static void* pick_enc(int dtype, int mode, bool ms, bool x0 = false) {
    static void* (*const tab[2][4])(bool, bool) = {{enc_ptr_0_0, enc_ptr_0_1, enc_ptr_0_2, enc_ptr_0_3},
                                            {enc_ptr_1_0, enc_ptr_1_1, enc_ptr_1_2, enc_ptr_1_3}};
    return tab[dtype ? 1 : 0][mode & 3](ms, x0);
}

static int enc_threads(int dtype) { return dtype == 0 ? EncCfg<float>::THREADS : EncCfg<double>::THREADS; }

static int enc_smem(int dtype) { return dtype == 0 ? EncCfg<float>::SMEM : EncCfg<double>::SMEM; }

static cudaError_t prepare_enc(void* fn, int dtype) {
    return cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, enc_smem(dtype));
}

int encode_grid(int dtype, int mode, bool ms, uint64_t C) {
    static int cache[2][4][2] = {};
    int& g = cache[dtype][mode][ms];
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        void* fn = pick_enc(dtype, mode, ms);
        prepare_enc(fn, dtype);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, enc_threads(dtype), enc_smem(dtype));
        g = sms * (per > 0 ? per : 1);
        if (g > grid_limit()) g = grid_limit();
    }
    return (int)(C < (uint64_t)g ? C : (uint64_t)g);
}

int encode_tickets_per_cta(int dtype) { return dtype == 0 ? EncCfg<float>::TICKETS : EncCfg<double>::TICKETS; }

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

cudaError_t launch_encode(int dtype, int mode, bool ms, bool x0, const EncParams& p, int grid,
                          cudaStream_t s) {
    alignas(64) CUtensorMap map;
    cudaError_t e = make_row_tmap(p.in, p.n * (dtype == 0 ? 4u : 8u), &map);
    if (e != cudaSuccess) return e;
    void* fn = pick_enc(dtype, mode, ms, x0);
    static bool prepared[2][4][2][2] = {};
    if (!prepared[dtype][mode][ms][x0]) {
        e = prepare_enc(fn, dtype);
        if (e != cudaSuccess) return e;
        prepared[dtype][mode][ms][x0] = true;
    }
    void* args[] = {(void*)&p, (void*)&map};
    return cudaLaunchKernel(fn, dim3(grid), dim3(enc_threads(dtype)), args, enc_smem(dtype), s);
}

}  // namespace pfpl
