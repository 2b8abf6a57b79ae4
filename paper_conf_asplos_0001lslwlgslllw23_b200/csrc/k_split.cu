// k_split.cu -- SV launcher: dispatch on edge_op to the per-KE instantiations (k_split*.cu
// split the instances over translation units so they compile in parallel).
#include "k_split.cuh"

namespace ug {

UG_SV_INSTANTIATE(K_COPY)
// instantiated in k_split_addsub.cu / k_split_mul.cu / k_split_div.cu
extern template cudaError_t launch_split_ke<K_ADD>(int, const GraphArgs &, const OpArgs &, const LaunchCfg &,
                                                   const SplitPlan &, float *, cudaStream_t, cudaEvent_t, cudaEvent_t,
                                                   int32_t *);
extern template cudaError_t launch_split_ke<K_SUB>(int, const GraphArgs &, const OpArgs &, const LaunchCfg &,
                                                   const SplitPlan &, float *, cudaStream_t, cudaEvent_t, cudaEvent_t,
                                                   int32_t *);
extern template cudaError_t launch_split_ke<K_MUL>(int, const GraphArgs &, const OpArgs &, const LaunchCfg &,
                                                   const SplitPlan &, float *, cudaStream_t, cudaEvent_t, cudaEvent_t,
                                                   int32_t *);
extern template cudaError_t launch_split_ke<K_DIV>(int, const GraphArgs &, const OpArgs &, const LaunchCfg &,
                                                   const SplitPlan &, float *, cudaStream_t, cudaEvent_t, cudaEvent_t,
                                                   int32_t *);

cudaError_t launch_split_vertex(int kedge, int gather, const GraphArgs &g, const OpArgs &op,
                                const LaunchCfg &c, const SplitPlan &plan, float *scratch,
                                cudaStream_t s, cudaEvent_t ev_begin, cudaEvent_t ev_end, int32_t *counters) {
    switch (kedge) {
    case K_COPY: return launch_split_ke<K_COPY>(gather, g, op, c, plan, scratch, s, ev_begin, ev_end, counters);
    case K_ADD: return launch_split_ke<K_ADD>(gather, g, op, c, plan, scratch, s, ev_begin, ev_end, counters);
    case K_SUB: return launch_split_ke<K_SUB>(gather, g, op, c, plan, scratch, s, ev_begin, ev_end, counters);
    case K_MUL: return launch_split_ke<K_MUL>(gather, g, op, c, plan, scratch, s, ev_begin, ev_end, counters);
    default: return launch_split_ke<K_DIV>(gather, g, op, c, plan, scratch, s, ev_begin, ev_end, counters);
    }
}

}  // namespace ug
