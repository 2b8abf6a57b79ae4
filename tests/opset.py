"""The 160-operator test matrix, derived from Table 2's counts
 and Table 4, readings R3-R5 in DESIGN.md.

An op is (edge_op, lhs, rhs, gather_op, c_type); lhs/rhs are tensor types "u" (Src_V),
"v" (Dst_V), "e" (Edge) or None (NULL).  Test-side enumeration only.
"""
import itertools

BINARY = ("add", "sub", "mul", "div", "dot")
REDUCERS = ("sum", "max", "min", "mean")


def message_functions():
    """32 DGL message functions: copy_u, copy_e, and 5 binary ops x 6 ordered distinct pairs."""
    out = [("copy_lhs", "u", None), ("copy_lhs", "e", None)]
    for op in BINARY:
        for lhs, rhs in itertools.permutations(("u", "v", "e"), 2):
            out.append((op, lhs, rhs))
    return out


def all_ops():
    """160 ops: 32 message creation (gather assign, C=e) + 32 x 4 aggregations (C=v)."""
    ops = []
    for (eo, l, r) in message_functions():
        ops.append((eo, l, r, "assign", "e"))
    for (eo, l, r) in message_functions():
        for g in REDUCERS:
            ops.append((eo, l, r, g, "v"))
    return ops


def name(op):
    eo, l, r, g, c = op
    if eo == "copy_lhs":
        base = f"copy_{l}"
    else:
        base = f"{l}_{eo}_{r}"
    return base if g == "assign" else f"{base}_{g}"


def table2_class(op):
    """(input class, output type) as in Table 2: input 'V', 'E' or 'V&E'."""
    eo, l, r, g, c = op
    kinds = {t for t in (l, r) if t is not None}
    has_v = bool(kinds & {"u", "v"})
    has_e = "e" in kinds
    inp = "V&E" if (has_v and has_e) else ("V" if has_v else "E")
    return inp, ("E" if c == "e" else "V")
