// pfpl_inst.cu -- explicit instantiation of one (dtype, mode) pair of the fused
// encoder or decoder, so the 28 kernel variants compile in parallel.  Built by
// _build.py with -DPFPL_KIND=0 (encode) / 1 (decode), -DPFPL_DT, -DPFPL_MODE.
#if PFPL_KIND == 0
#include "pfpl_encode.cuh"
#define PFPL_KERNEL encode_kernel
#define PFPL_PREFIX enc_ptr_
#else
#include "pfpl_decode.cuh"
#define PFPL_KERNEL decode_kernel
#define PFPL_PREFIX dec_ptr_
#endif

#define PFPL_CAT3(a, b, c, d) a##b##_##d
#define PFPL_NAME(p, d, m) PFPL_CAT3(p, d, _, m)

namespace pfpl {
#if PFPL_DT == 0
typedef float InstT;
#else
typedef double InstT;
#endif
#if PFPL_KIND == 0
// encoder: (residual code, first-residual split form; the latter exists for f32 ABS only)
void* PFPL_NAME(PFPL_PREFIX, PFPL_DT, PFPL_MODE)(bool ms, bool x0) {
#if PFPL_DT == 0 && (PFPL_MODE == 0 || PFPL_MODE == 3)
    if (x0) return ms ? (void*)PFPL_KERNEL<InstT, PFPL_MODE, true, true> : (void*)PFPL_KERNEL<InstT, PFPL_MODE, false, true>;
#else
    (void)x0;
#endif
    return ms ? (void*)PFPL_KERNEL<InstT, PFPL_MODE, true, false> : (void*)PFPL_KERNEL<InstT, PFPL_MODE, false, false>;
}
#else
// decoder: (residual code, verify mode); verify is instantiated for the default residuals
// and for zigzag residuals alike
void* PFPL_NAME(PFPL_PREFIX, PFPL_DT, PFPL_MODE)(bool ms, bool ver, bool x0) {
#if PFPL_DT == 0 && PFPL_MODE == 0
    // f32 ABS (and NOA streams): the form that folds a warp's first-byte-only top planes
    if (x0 && !ver) return ms ? (void*)PFPL_KERNEL<InstT, PFPL_MODE, true, false, true>
                              : (void*)PFPL_KERNEL<InstT, PFPL_MODE, false, false, true>;
#else
    (void)x0;
#endif
    if (ver) return ms ? (void*)PFPL_KERNEL<InstT, PFPL_MODE, true, true>
                       : (void*)PFPL_KERNEL<InstT, PFPL_MODE, false, true>;
    return ms ? (void*)PFPL_KERNEL<InstT, PFPL_MODE, true, false> : (void*)PFPL_KERNEL<InstT, PFPL_MODE, false, false>;
}
#endif
}  // namespace pfpl
