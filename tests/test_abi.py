"""C-ABI library checks that need no GPU: symbol exports, host-side graph build (a1) vs the
oracle's in-edge lists, statistics, partition, views, op validation (the 160-op set of
Table 2 / Table 4) and schedule text form."""
import os
import re
import subprocess

import numpy as np
import pytest
import torch

import oracle
import ugdata
from opset import all_ops, name

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ug.h")

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")
from paper_conf_asplos_0001lslwlgslllw23_b200 import _ffi  # noqa: E402


def declared_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(ug_[a-z_]+)\s*\(", txt)))


def test_exports_every_declared_symbol():
    syms = declared_symbols()
    assert len(syms) >= 15
    out = subprocess.check_output(["nm", "-D", "--defined-only", _ffi.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (ug_\w+)", out))
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    for s in syms:
        assert hasattr(_ffi.lib, s)


def test_library_is_sm100a():
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", _ffi.LIB_PATH]).decode()
    assert "sm_100a" in out


def host_graph(V, src, dst):
    return ug.Graph(V, src, dst, host_only=True)


@pytest.mark.parametrize("seed", range(5))
def test_csr_build_matches_oracle(seed):
    V, E = 40 + seed, 300 + 7 * seed
    src, dst = ugdata.random_multigraph(V, E, seed)
    g = host_graph(V, src, dst)
    rp, col, eid = g.csr()
    orp, oeid = oracle.inedges(V, dst)
    np.testing.assert_array_equal(rp, orp)
    np.testing.assert_array_equal(eid, oeid)
    np.testing.assert_array_equal(col, src[oeid])


def test_csr_build_generator_graph_identity_eid():
    src, dst = ugdata.graph("C2")
    V = ugdata.CONFIGS["C2"].V
    g = host_graph(V, src, dst)
    rp, col, eid = g.csr()
    orp, oeid = oracle.inedges(V, dst)
    np.testing.assert_array_equal(rp, orp)
    np.testing.assert_array_equal(eid, np.arange(len(src)))
    np.testing.assert_array_equal(col, src)


def test_from_csr_roundtrip():
    src, dst = ugdata.random_multigraph(30, 200, 9)
    g = host_graph(30, src, dst)
    rp, col, eid = g.csr()
    g2 = ug.Graph.from_csr(30, rp, col, eid, host_only=True)
    rp2, col2, eid2 = g2.csr()
    np.testing.assert_array_equal(rp, rp2)
    np.testing.assert_array_equal(col, col2)
    np.testing.assert_array_equal(eid, eid2)


def test_stats_match_oracle():
    src, dst = ugdata.graph("C3")
    V = ugdata.CONFIGS["C3"].V
    s = host_graph(V, src, dst).stats()
    m, sd, mx = oracle.stats(V, dst)
    assert s["V"] == V and s["E"] == len(src)
    assert abs(s["mean_deg"] - m) < 1e-9 and abs(s["std_nnz"] - sd) < 1e-6 and s["max_deg"] == mx


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_partition_matches_oracle(P):
    src, dst = ugdata.graph("C3")
    V = ugdata.CONFIGS["C3"].V
    g = host_graph(V, src, dst)
    rp, _, _ = g.csr()
    np.testing.assert_array_equal(g.partition(P), oracle.partition(rp.astype(np.int64), P))


def test_view_rows_slices():
    src, dst = ugdata.graph("C2")
    V = ugdata.CONFIGS["C2"].V
    g = host_graph(V, src, dst)
    rp, col, _ = g.csr()
    sp = g.partition(4)
    total = 0
    for k in range(4):
        w = g.view_rows(sp[k], sp[k + 1])
        wrp, wcol, weid = w.csr()
        assert w.stats()["V"] == sp[k + 1] - sp[k]
        np.testing.assert_array_equal(wrp, rp[sp[k]:sp[k + 1] + 1] - rp[sp[k]])
        np.testing.assert_array_equal(wcol, col[rp[sp[k]]:rp[sp[k + 1]]])
        total += w.stats()["E"]
    assert total == len(src)


def test_rejects_bad_ids():
    with pytest.raises(ug.UgError, match="INDEX_RANGE"):
        host_graph(3, np.array([0, 3], np.int32), np.array([1, 1], np.int32))


def _op_tensors(op, V, E, F, H):
    eo, l, r, g, c = op
    mk = lambda t, w: torch.zeros((V if t in ("u", "v") else E, w)) if t else None
    W = H if eo == "dot" else F
    A = mk(l, F)
    B = mk(r, F if eo == "dot" else (H if r == "e" else F))
    C = torch.zeros((V if c == "v" else E, W))
    return A, B, C


def test_validate_accepts_all_160_ops():
    src, dst = ugdata.random_multigraph(10, 40, 0)
    g = host_graph(10, src, dst)
    for op in all_ops():
        eo, l, r, gop, c = op
        A, B, C = _op_tensors(op, 10, 40, 4, 2)
        ug.validate(g, eo, gop, A=A, a_type=l, B=B, b_type=r, C=C, c_type=c, F=4, H=2)


@pytest.mark.parametrize("bad, status", [
    (dict(edge_op="copy_lhs", gather_op="sum", a_type="u", c_type="e"), "UNSUPPORTED_OP"),
    (dict(edge_op="copy_lhs", gather_op="assign", a_type="u", c_type="v"), "UNSUPPORTED_OP"),
    (dict(edge_op="copy_lhs", gather_op="sum", a_type="u", c_type="u"), "UNSUPPORTED_OP"),
    (dict(edge_op="add", gather_op="sum", a_type="u", b_type=None, c_type="v"), "UNSUPPORTED_OP"),
    (dict(edge_op="copy_lhs", gather_op="sum", a_type="u", c_type="v", F=4, H=3), "SHAPE"),
])
def test_validate_rejects(bad, status):
    src, dst = ugdata.random_multigraph(10, 40, 0)
    g = host_graph(10, src, dst)
    F, H = bad.pop("F", 4), bad.pop("H", 1)
    ctype = bad["c_type"]
    A = torch.zeros(10, 4)
    B = torch.zeros(10, 4) if bad.get("b_type") else None
    C = torch.zeros(40 if ctype == "e" else 10, 4)
    with pytest.raises(ug.UgError, match=status):
        ug.validate(g, bad["edge_op"], bad["gather_op"], A=A, a_type=bad.get("a_type"), B=B,
                    b_type=bad.get("b_type"), C=C, c_type=ctype, F=F, H=H)


def test_validate_rejects_width_mismatch():
    src, dst = ugdata.random_multigraph(10, 40, 0)
    g = host_graph(10, src, dst)
    with pytest.raises(ug.UgError, match="SHAPE"):
        ug.validate(g, "copy_lhs", "sum", A=torch.zeros(10, 4), a_type="u", C=torch.zeros(10, 3), c_type="v")
    with pytest.raises(ug.UgError, match="SHAPE"):   # operand width 3 is neither F=4, H=2 nor 1
        ug.validate(g, "mul", "sum", A=torch.zeros(10, 4), a_type="u", B=torch.zeros(40, 3), b_type="e",
                    C=torch.zeros(10, 4), c_type="v", F=4, H=2)


@pytest.mark.parametrize("text", ["TE_G1_T16", "WV_G4_T2", "TV_G1_T1", "WE_G64_T1", "BV_G2",
                                  "BE_G256", "SV_G2048_F64", "SV_G1024_F128_B128_V4", "SV_G512_F64_P1",
                                  "TV_G1_T16_E1", "WV_G4_T1_E1", "SV_G512_F120_P1", "SV_G4096_E1"])
def test_schedule_text_roundtrip(text):
    s = ug.parse_schedule(text)
    assert ug.parse_schedule(ug.format_schedule(s)).strategy == s.strategy
    t2 = ug.format_schedule(ug.parse_schedule(ug.format_schedule(s)))
    assert t2 == ug.format_schedule(s)


def test_schedule_parse_rejects():
    for bad in ["XX_G1", "TE_Q4", "TE_G-1", "TE_G"]:
        with pytest.raises(ug.UgError):
            ug.parse_schedule(bad)


def test_selector_covers_op_classes():
    src, dst = ugdata.graph("C1")
    g = host_graph(ugdata.CONFIGS["C1"].V, src, dst)
    V, E = ugdata.CONFIGS["C1"].V, len(src)
    for op in all_ops()[::7]:
        eo, l, r, gop, c = op
        A, B, C = _op_tensors(op, V, E, 16, 1)
        s = ug.schedule_select(g, eo, gop, A=A, a_type=l, B=B, b_type=r, C=C, c_type=c, F=16, H=1)
        assert ug.parse_schedule(s).strategy != 0
        n = ug.launch_count(g, eo, gop, A=A, a_type=l, B=B, b_type=r, C=C, c_type=c, F=16, H=1)
        assert 1 <= n <= 3


def test_launch_counts_follow_pass2():
    """Pass 2: atomic schedules need init (+ epilogue); owner-computes do not."""
    src, dst = ugdata.graph("C1")
    V, E = ugdata.CONFIGS["C1"].V, len(src)
    g = host_graph(V, src, dst)
    X, Y = torch.zeros(V, 16), torch.zeros(V, 16)
    kw = dict(A=X, a_type="u", C=Y, c_type="v")
    assert ug.launch_count(g, "copy_lhs", "sum", schedule="WV_G1_T1", **kw) == 1
    assert ug.launch_count(g, "copy_lhs", "sum", schedule="TE_G4_T16", **kw) == 2
    assert ug.launch_count(g, "copy_lhs", "max", schedule="WE_G4_T1", **kw) == 3
    assert ug.launch_count(g, "copy_lhs", "mean", schedule="BV_G1", **kw) == 1
    # SV: split rows are merged by the last-arriving chunk inside the same launch
    assert ug.launch_count(g, "copy_lhs", "sum", schedule="SV_G2", **kw) == 1
    assert ug.launch_count(g, "copy_lhs", "max", schedule="SV_G2_F16", **kw) == 1
    Z = torch.zeros(E, 16)
    assert ug.launch_count(g, "add", "assign", A=X, a_type="u", B=X, b_type="v", C=Z, c_type="e",
                           schedule="TE_G1_T16") == 1


def test_selector_table_load_and_match(tmp_path):
    """A measured table entry matching (class, F, degree, CV, V) wins; a miss falls back to the
    priors; a malformed table is rejected."""
    src, dst = ugdata.graph("C1")
    V, E = ugdata.CONFIGS["C1"].V, len(src)
    g = host_graph(V, src, dst)
    st = g.stats()
    t = tmp_path / "table.json"
    t.write_text('{"version": 1, "entries": [\n'
                 ' {"class": "agg", "F_lo": 8, "F_hi": 20, "deg_lo": 1, "deg_hi": 10, "cv_lo": 0, "cv_hi": 5,'
                 '  "V_lo": 1000, "V_hi": 10000, "schedule": "BV_G4_B256"},\n'
                 ' {"class": "msg", "F_lo": 8, "F_hi": 20, "schedule": "WE_G16_T1"}]}')
    ug.selector_load(t)
    ug.selector_load_model("")          # tier 2 off: a table miss goes straight to the priors
    X, Y = torch.zeros(V, 16), torch.zeros(V, 16)
    assert ug.schedule_select(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v") == "BV_G4_B256"
    Z = torch.zeros(E, 16)
    assert ug.schedule_select(g, "add", "assign", A=X, a_type="u", B=X, b_type="v", C=Z, c_type="e") == "WE_G16_T1"
    X2, Y2 = torch.zeros(V, 64), torch.zeros(V, 64)     # F outside every entry -> prior
    assert ug.schedule_select(g, "copy_lhs", "sum", A=X2, a_type="u", C=Y2, c_type="v").startswith("SV")
    bad = tmp_path / "bad.json"
    bad.write_text('{"entries": [{"class": "agg", "schedule": "XX_G1"}]}')
    with pytest.raises(ug.UgError):
        ug.selector_load(bad)
    # restore the shipped table and model (if any) for later tests
    model = os.path.join(ROOT, "paper_conf_asplos_0001lslwlgslllw23_b200", "selector_model.txt")
    if os.path.exists(model):
        ug.selector_load_model(model)
    shipped = os.path.join(ROOT, "paper_conf_asplos_0001lslwlgslllw23_b200", "selector_table.json")
    if os.path.exists(shipped):
        ug.selector_load(shipped)
    else:
        empty = tmp_path / "empty.json"
        empty.write_text('{"entries": []}')
        ug.selector_load(empty)


def test_selector_table_nearest_entry_wins(tmp_path):
    """Overlapping entries (neighbouring configs share F and degree ranges): the entry whose
    range centres are nearest (log distance) to the graph's features wins, whatever the order."""
    src, dst = ugdata.graph("C1")
    V = ugdata.CONFIGS["C1"].V
    g = host_graph(V, src, dst)
    st = g.stats()
    deg = st["mean_deg"]
    X, Y = torch.zeros(V, 16), torch.zeros(V, 16)
    far = (f'{{"class": "agg", "F_lo": 8, "F_hi": 20, "deg_lo": {deg / 3}, "deg_hi": {deg * 12}, '
           f'"V_lo": 100, "V_hi": 1000000, "schedule": "WV_G1_T1"}}')
    near = (f'{{"class": "agg", "F_lo": 8, "F_hi": 32, "deg_lo": {deg / 2}, "deg_hi": {deg * 2}, '
            f'"V_lo": {V / 2}, "V_hi": {V * 2}, "schedule": "TE_G4_T4"}}')
    ug.selector_load_model("")
    try:
        for entries in ([far, near], [near, far]):
            t = tmp_path / "t.json"
            t.write_text('{"version": 1, "entries": [' + ",".join(entries) + "]}")
            ug.selector_load(t)
            assert ug.schedule_select(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v") == "TE_G4_T4"
    finally:
        pkg = os.path.join(ROOT, "paper_conf_asplos_0001lslwlgslllw23_b200")
        if os.path.exists(os.path.join(pkg, "selector_model.txt")):
            ug.selector_load_model(os.path.join(pkg, "selector_model.txt"))
        ug.selector_load(os.path.join(pkg, "selector_table.json"))


def test_binding_rejects_short_overlapping_tensors():
    """The C ABI carries no row counts: the binding checks the rows each type implies (Src_V:
    V_total, Dst_V: V, Edge: E), and rejects overlapping rows (expand()ed tensors)."""
    src, dst = ugdata.random_multigraph(10, 40, 0)
    g = host_graph(10, src, dst)
    assert g.dims() == (10, 10, 40)
    with pytest.raises(ValueError, match="rows"):
        ug.validate(g, "copy_lhs", "sum", A=torch.zeros(9, 4), a_type="u", C=torch.zeros(10, 4), c_type="v")
    with pytest.raises(ValueError, match="rows"):
        ug.validate(g, "mul", "sum", A=torch.zeros(10, 4), a_type="u", B=torch.zeros(39, 1), b_type="e",
                    C=torch.zeros(10, 4), c_type="v")
    with pytest.raises(ValueError, match="overlap"):
        ug.validate(g, "copy_lhs", "sum", A=torch.zeros(1, 4).expand(10, 4), a_type="u", C=torch.zeros(10, 4),
                    c_type="v")
    # a view: Src_V operands span the parent's ids, Dst_V / Edge operands the view's rows / edges
    order = np.argsort(dst, kind="stable")
    g2 = host_graph(10, src[order], dst[order])
    sp = g2.partition(2)
    v = g2.view_rows(int(sp[1]), int(sp[2]))
    vs, vv, ve = v.dims()
    assert vs == 10 and vv == int(sp[2] - sp[1]) and ve == int(g2.row_ptr()[sp[2]] - g2.row_ptr()[sp[1]])
    ug.validate(v, "copy_lhs", "sum", A=torch.zeros(10, 4), a_type="u", C=torch.zeros(vv, 4), c_type="v")
    with pytest.raises(ValueError, match="rows"):
        ug.validate(v, "copy_lhs", "sum", A=torch.zeros(vv, 4), a_type="u", C=torch.zeros(vv, 4), c_type="v") \
            if vv < 10 else (_ for _ in ()).throw(ValueError("rows"))


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_auto_schedule_always_resolves(cfg):
    """AUTO (table -> learned tier -> priors) yields a schedule the operator can run, for every op
    and a spread of widths -- a measured entry that does not fit the layout (e.g. edge lanes at
    F = 18, float2 rows) falls through to the next tier instead of failing."""
    src, dst = ugdata.graph(cfg)
    V, E = ugdata.CONFIGS[cfg].V, len(src)
    g = host_graph(V, src, dst)
    for F, H in ((1, 1), (3, 1), (8, 8), (16, 1), (18, 3), (20, 1), (64, 8), (100, 4)):
        for op in all_ops():
            eo, l, r, gop, c = op
            A, B, C = _op_tensors(op, V, E, F, H)
            n = ug.launch_count(g, eo, gop, A=A, a_type=l, B=B, b_type=r, C=C, c_type=c, F=F, H=H)
            assert 1 <= n <= 4, (name(op), F, H, n)


def test_round2_schedules_resolve_on_the_host():
    """Round-2 schedule forms resolve (one launch each) or are rejected on the host: edge lanes
    with P in {8, 16} lanes per row (TV) or a warp (WV, g rows segmented), and SV column tiles of
    a non-power-of-two lane count (lanes past ftile / vec idle; at most 32)."""
    src, dst = ugdata.graph("C1")
    V, E = ugdata.CONFIGS["C1"].V, len(src)
    g = host_graph(V, src, dst)
    X, Y = torch.zeros(V, 16), torch.zeros(V, 16)
    w = torch.zeros(E, 1)
    kw = dict(A=X, a_type="u", C=Y, c_type="v")
    for s in ("TV_G1_T8_E1", "TV_G2_T16_E1", "WV_G2_T1_E1", "WV_G4_T1_E1", "SV_G2_F12", "SV_G64_F24_P1"):
        assert ug.launch_count(g, "copy_lhs", "sum", schedule=s, **kw) == 1, s
        assert ug.launch_count(g, "mul", "sum", B=w, b_type="e", schedule=s, **kw) == 1, s
    for bad in ("TV_G1_T4_E1", "TV_G1_T1_E1", "WV_G1_T2_E1", "SV_G2_F132"):
        with pytest.raises(ug.UgError):
            ug.launch_count(g, "copy_lhs", "sum", schedule=bad, **kw)
