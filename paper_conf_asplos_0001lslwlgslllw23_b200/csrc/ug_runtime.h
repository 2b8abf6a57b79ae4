// ug_runtime.h -- host-side helpers shared by the runtime translation units.
#pragma once
#include <string>

#include "ug.h"
#include "ug_internal.h"

namespace ug {

ug_status set_error(ug_status s, const std::string &msg);

// Operator after lowering (validation + pass 1 of PAPER.md:405: copy ops fused, copy_rhs
// rewritten as copy_lhs on B, operand broadcast factors resolved).
struct Lowered {
    int kedge;          // K_COPY .. K_DIV, or -1 for dot
    bool dot;
    int gather;         // UG_GATHER_*
    bool to_edges;      // C is an Edge tensor (message creation)
    OpArgs args;
    int max_vec;        // widest legal feature vector for every tensor (1, 2, 4)
    int a_vec, b_vec, c_vec;   // per tensor
    bool pack_ok;       // A is a full-width Src_V operand whose rows are not 128-byte aligned
    // selector key
    int op_class;       // 0 msg, 1 agg (copy, sum/mean), 2 dot msg, 3 dot agg, 4 agg_bin, 5 agg_ext
};

ug_status lower(const ug_graph *g, const ug_op_info *op, Lowered *out);

// Concrete launch configuration for a (graph, lowered op, schedule).
ug_status resolve(const ug_graph *g, const Lowered &lw, const ug_schedule &s, LaunchCfg *cfg);

// Selector (ug_selector.cpp).
ug_status select_schedule(const ug_graph *g, const Lowered &lw, ug_schedule *out);

}  // namespace ug
