// k_svg_launch.cuh -- per-MODE launcher template of the staged SV kernel (instantiated in
// k_svg_tma.cu and k_svg_async.cu so the instances compile in parallel).
#pragma once
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "k_split.cuh"
#include "k_svg.cuh"

namespace ug {

PFN_cuTensorMapEncodeTiled_v12000 svg_encode_fn();

template <int MODE, int KE, int GOP, int VEC, int BM>
static cudaError_t svg_launch_one(const CUtensorMap &tm, const GraphArgs &g, const OpArgs &op, const SplitPlan &plan,
                                  int n_tiles, float *scratch, int64_t sld, cudaStream_t s) {
    constexpr size_t smem = svg_smem_bytes<MODE, VEC>();
    auto kern = k_svg<MODE, KE, GOP, VEC, BM>;
    static int per_sm = 0;
    static int n_sm = 0;
    static std::once_flag once;
    std::call_once(once, [&] {
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        int dev = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&n_sm, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, UG_SVG_WARPS * 32, smem);
        if (per_sm < 1) per_sm = 1;
    });
    const int64_t units = plan.n_chunks * n_tiles;
    const int64_t want = cdiv(units, UG_SVG_WARPS);
    const int64_t grid = std::max<int64_t>(1, std::min<int64_t>(want, (int64_t)per_sm * n_sm));
    kern<<<(unsigned)grid, UG_SVG_WARPS * 32, smem, s>>>(tm, g, op, reinterpret_cast<const int4 *>(plan.d_chunk),
                                                       (int)plan.n_chunks, n_tiles, scratch, sld);
    return cudaGetLastError();
}

template <int MODE>
cudaError_t launch_svg_mode(int kedge, int gather, const GraphArgs &g, const OpArgs &op, int vec, int bm,
                            const SplitPlan &plan, float *scratch, cudaStream_t s) {
    const int TW = 32 * vec;
    const int n_tiles = (int)cdiv(op.W, TW);
    if (plan.n_chunks * n_tiles >= (int64_t)1 << 30) return cudaErrorInvalidValue;   // 32-bit unit cursor
    const int64_t sld = cdiv(op.W, 4) * 4;
    CUtensorMap tm;
    std::memset(&tm, 0, sizeof(tm));
    if constexpr (MODE == 0) {
        const cuuint64_t dims[2] = {(cuuint64_t)op.F, (cuuint64_t)g.V_src};
        const cuuint64_t strides[1] = {(cuuint64_t)op.A.ld * 4};
        const cuuint32_t box[2] = {(cuuint32_t)TW, 1};
        const cuuint32_t estr[2] = {1, 1};
        CUresult r = svg_encode_fn()(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float *>(op.A.p), dims,
                                     strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                                     CU_TENSOR_MAP_L2_PROMOTION_L2_128B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) return cudaErrorInvalidValue;
    }
    cudaError_t err = cudaSuccess;
#define UG_SVG_BM(KEV, GOPV, VECV)                                                                             \
    switch (bm) {                                                                                              \
    case 1: err = svg_launch_one<MODE, KEV, GOPV, VECV, 1>(tm, g, op, plan, n_tiles, scratch, sld, s); break; \
    case 2: err = svg_launch_one<MODE, KEV, GOPV, VECV, 2>(tm, g, op, plan, n_tiles, scratch, sld, s); break; \
    default: err = cudaErrorInvalidValue; break;                                                               \
    }
    UG_DISPATCH_VEC(vec, VEC,
        UG_DISPATCH_RED(gather, GOP, {
            switch (kedge) {
            case K_COPY: err = svg_launch_one<MODE, K_COPY, GOP, VEC, 0>(tm, g, op, plan, n_tiles, scratch, sld, s); break;
            case K_ADD: UG_SVG_BM(K_ADD, GOP, VEC); break;
            case K_SUB: UG_SVG_BM(K_SUB, GOP, VEC); break;
            case K_MUL: UG_SVG_BM(K_MUL, GOP, VEC); break;
            default: UG_SVG_BM(K_DIV, GOP, VEC); break;
            }
        }));
#undef UG_SVG_BM
    return err;
}

}  // namespace ug
