// k_svg.cu -- launcher of the staged SV kernel (k_svg.cuh): tensor map of the A operand (TMA
// mode), persistent grid sized to the resident warps, then the split-row fix-up of k_split.cuh.
// The instances of each MODE live in their own translation unit (k_svg_tma.cu / k_svg_async.cu).
#include <cstring>

#include "k_svg_launch.cuh"

namespace ug {

PFN_cuTensorMapEncodeTiled_v12000 svg_encode_fn() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    });
    return fn;
}

bool svg_supported(const OpArgs &op, int vec, int mode) {
    if (vec != 1 && vec != 2 && vec != 4) return false;
    const uintptr_t a = reinterpret_cast<uintptr_t>(op.A.p);
    if (op.A.div != 1 || op.A.type != UG_T_SRC_V) return false;
    if (mode == 0) return svg_encode_fn() != nullptr && a % 16 == 0 && (op.A.ld * 4) % 16 == 0;
    // cp.async of 4 * vec bytes per lane: every chunk start aligned to its size
    return a % (4 * vec) == 0 && op.A.ld % vec == 0;
}

extern template cudaError_t launch_svg_mode<0>(int, int, const GraphArgs &, const OpArgs &, int, int,
                                               const SplitPlan &, float *, cudaStream_t);
extern template cudaError_t launch_svg_mode<1>(int, int, const GraphArgs &, const OpArgs &, int, int,
                                               const SplitPlan &, float *, cudaStream_t);

cudaError_t launch_split_staged(int mode, int kedge, int gather, const GraphArgs &g, const OpArgs &op, int vec,
                                int bm, const SplitPlan &plan, float *scratch, cudaStream_t s, cudaEvent_t ev_begin,
                                cudaEvent_t ev_end) {
    if (plan.n_chunks == 0) return cudaSuccess;
    if (ev_begin) cudaEventRecord(ev_begin, s);
    cudaError_t err = mode == 0 ? launch_svg_mode<0>(kedge, gather, g, op, vec, bm, plan, scratch, s)
                                : launch_svg_mode<1>(kedge, gather, g, op, vec, bm, plan, scratch, s);
    if (ev_end) cudaEventRecord(ev_end, s);
    if (err != cudaSuccess || plan.n_split_rows == 0) return err;
    const int64_t sld = cdiv(op.W, 4) * 4;
    const int64_t per_row = cdiv(op.W, vec);
    const int64_t fgrid = cdiv(plan.n_split_rows * per_row, 256);
    const int4 *split = reinterpret_cast<const int4 *>(plan.d_split);
    UG_DISPATCH_VEC(vec, VEC,
        UG_DISPATCH_RED(gather, GOP,
            k_split_fix<GOP, VEC><<<(unsigned)fgrid, 256, 0, s>>>(g, op, split, plan.n_split_rows, scratch, sld)));
    return cudaGetLastError();
}

}  // namespace ug
