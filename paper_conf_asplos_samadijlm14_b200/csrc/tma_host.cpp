// tma_host.cpp -- cuTensorMapEncodeTiled through the runtime's driver entry
// point (the library does not link libcuda directly).
#include <cudaTypedefs.h>

#include <cstdlib>
#include <mutex>

#include "tma.cuh"

namespace ppx {

static PFN_cuTensorMapEncodeTiled_v12000 get_encoder() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

// L2 promotion of the TMA loads: 256 B (r01 A/B of none / 64 / 128 / 256 B:
// within +-1 %)
static CUtensorMapL2promotion l2_promotion(int bytes) {
    return bytes >= 256 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
                        : bytes >= 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
                                       : bytes >= 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                                                     : CU_TENSOR_MAP_L2_PROMOTION_NONE;
}

bool encode_tmap_3d(CUtensorMap* map, const float* base, int w, int rows, int n, long long pitch,
                    long long fstride, int box_w, int box_h, int l2_promo) {
    auto enc = get_encoder();
    if (!enc) return false;
    if ((reinterpret_cast<uintptr_t>(base) & 15) != 0) return false;
    if ((pitch * 4) % 16 != 0 || (fstride * 4) % 16 != 0) return false;
    if (box_w > 256 || box_h > 256 || (box_w * 4) % 16 != 0) return false;
    if (pitch * 4 >= (1LL << 40) || fstride * 4 >= (1LL << 40)) return false;
    cuuint64_t dims[3] = {(cuuint64_t)w, (cuuint64_t)rows, (cuuint64_t)n};
    cuuint64_t strides[2] = {(cuuint64_t)(pitch * 4), (cuuint64_t)(fstride * 4)};
    cuuint32_t box[3] = {(cuuint32_t)box_w, (cuuint32_t)box_h, 1};
    cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, const_cast<float*>(base), dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, l2_promotion(l2_promo),
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
}

}  // namespace ppx
