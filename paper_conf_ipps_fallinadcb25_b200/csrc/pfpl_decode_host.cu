// pfpl_decode_host.cu -- launch-side code of the fused decoder (pfpl_decode.cuh).
#include "pfpl_decode.cuh"

namespace pfpl {

// one instantiation TU per (dtype, mode): pfpl_dec_inst.cu built with -DPFPL_DT/-DPFPL_MODE
#define PFPL_DECL(D, M) void* dec_ptr_##D##_##M(bool ms, bool ver, bool x0);
PFPL_DECL(0, 0) PFPL_DECL(0, 1) PFPL_DECL(0, 2) PFPL_DECL(1, 0) PFPL_DECL(1, 1) PFPL_DECL(1, 2)
#undef PFPL_DECL

static void* pick_dec(int dtype, int mode, bool ms, bool ver = false, bool x0 = false) {
    static void* (*const tab[2][3])(bool, bool, bool) = {{dec_ptr_0_0, dec_ptr_0_1, dec_ptr_0_2},
                                            {dec_ptr_1_0, dec_ptr_1_1, dec_ptr_1_2}};
    const int m = mode == MODE_ABS ? 0 : mode == MODE_REL ? 1 : 2;
    return tab[dtype ? 1 : 0][m](ms, ver, x0);
}

static int dec_threads(int dtype) { return (dtype == 0 ? Tr<float>::NT : Tr<double>::NT) + 32; }

int decode_grid(int dtype, int mode, bool ms, uint64_t C) {
    static int cache[2][4][2] = {};
    int& g = cache[dtype][mode][ms];
    if (!g) {
        int dev = 0, sms = 148, per = 1;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        void* fn = pick_dec(dtype, mode, ms);
        cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, DEC_SMEM);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, fn, dec_threads(dtype), DEC_SMEM);
        g = sms * (per > 0 ? per : 1);
        if (g > grid_limit()) g = grid_limit();
    }
    return (int)(C < (uint64_t)g ? C : (uint64_t)g);
}

int decode_tickets_per_cta() { return 0; }   // static chunk assignment

cudaError_t make_row_tmap(const void* base, uint64_t bytes, CUtensorMap* map);

cudaError_t launch_decode(int dtype, int mode, bool ms, bool x0, const DecParams& p, int grid,
                          cudaStream_t s) {
    alignas(64) CUtensorMap map;
    cudaError_t e = make_row_tmap(p.out, p.n * (dtype == 0 ? 4u : 8u), &map);
    if (e != cudaSuccess) return e;
    const bool ver = p.orig != nullptr;
    x0 = x0 && !ver;
    void* fn = pick_dec(dtype, mode, ms, ver, x0);
    static bool prepared[2][4][2][2][2] = {};
    if (!prepared[dtype][mode][ms][ver][x0]) {
        e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, DEC_SMEM);
        if (e != cudaSuccess) return e;
        prepared[dtype][mode][ms][ver][x0] = true;
    }
    void* args[] = {(void*)&p, (void*)&map};
    return cudaLaunchKernel(fn, dim3(grid), dim3(dec_threads(dtype)), args, DEC_SMEM, s);
}

}  // namespace pfpl
