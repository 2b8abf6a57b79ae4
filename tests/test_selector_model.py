"""The learned selector tier: the C++ tree walk in ug_schedule_select picks
exactly the leaf the exporter's reference walk (scripts/train_selector.predict_text) picks,
for host-only graphs of varied shape.  CPU only (host-only graphs; no kernels)."""
import math
import os
import sys

import numpy as np
import pytest
import torch

import ugdata

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import train_selector  # noqa: E402

PKG = os.path.dirname(ug.__file__)

TREE = """# hand-made model: root splits on log2 F at 5 (F <= 32), then on CV at 1.0
class agg 5
0 5 5 1 2 -
1 3 1.0 3 4 -
2 -1 0 -1 -1 SV_G32_F128
3 -1 0 -1 -1 TE_G8_T4
4 -1 0 -1 -1 WE_G4_T1
"""


@pytest.fixture()
def empty_table(tmp_path):
    t = tmp_path / "empty.json"
    t.write_text('{"entries": []}')
    ug.selector_load(str(t))
    yield tmp_path
    ug.selector_load(os.path.join(PKG, "selector_table.json"))
    default_model = os.path.join(PKG, "selector_model.txt")
    ug.selector_load_model(default_model if os.path.exists(default_model) else "")


def _features(st, F):
    mean = st["mean_deg"]
    return [math.log2(st["V"]), math.log2(st["E"]), math.log2(mean), st["std_nnz"] / mean,
            math.log2(max(st["max_deg"], 1) / mean), math.log2(F)]


def _select(g, V, F):
    X = torch.empty(V, F)
    Y = torch.empty(V, F)
    return ug.schedule_select(g, "copy_lhs", "sum", A=X, a_type="u", C=Y, c_type="v", F=F)


@pytest.mark.parametrize("sigma", [0.3, 1.4])
@pytest.mark.parametrize("F", [16, 128])
def test_tree_walk_matches_reference(empty_table, sigma, F):
    p = empty_table / "model.txt"
    p.write_text(TREE)
    ug.selector_load_model(str(p))
    V = 3000
    src, dst = ugdata.chung_lu(V, 30000, True, sigma, 0.5, 5)
    g = ug.Graph(V, src, dst, host_only=True)
    lines = [ln for ln in TREE.splitlines() if ln and not ln.startswith("#")]
    want = train_selector.predict_text(lines, _features(g.stats(), F))
    got = _select(g, V, F)
    assert got.startswith(want.split("_F")[0]), (got, want)


def test_model_unloaded_falls_back_to_priors(empty_table):
    ug.selector_load_model("")
    V = 3000
    src, dst = ugdata.chung_lu(V, 30000, True, 1.0, 0.5, 5)
    g = ug.Graph(V, src, dst, host_only=True)
    assert _select(g, V, 8).startswith("WV")         # prior: narrow aggregation -> warp-vertex


def test_bad_model_file_is_rejected(empty_table):
    p = empty_table / "bad.txt"
    p.write_text("class agg 2\n0 5 5 1 7 -\n")
    with pytest.raises(ug.UgError):
        ug.selector_load_model(str(p))


def test_shipped_model_parses():
    path = os.path.join(PKG, "selector_model.txt")
    if not os.path.exists(path):
        pytest.skip("no trained model shipped")
    ug.selector_load_model(path)
    in_knn = 0
    for ln in open(path):
        if ln.startswith("#") or ln.startswith("class"):
            continue
        parts = ln.split()
        if parts[0] == "knn":
            in_knn = 1
            continue
        if parts[0] in ("w", "mu", "sd", "p"):
            continue
        if parts[0] == "s":
            for sc in parts[1:]:
                ug.parse_schedule(sc)
            continue
        if parts[1] == "-1":
            ug.parse_schedule(parts[5])


@pytest.mark.parametrize("sigma", [0.3, 1.4])
@pytest.mark.parametrize("F", [16, 128])
def test_knn_matches_reference(empty_table, sigma, F):
    """The C++ nearest-neighbour rule picks the schedule train_selector.knn_scores ranks first."""
    rng = np.random.default_rng(3)
    X = np.column_stack([rng.uniform(11, 18, 40), rng.uniform(14, 23, 40), rng.uniform(1, 6, 40),
                         rng.uniform(0.3, 2.0, 40), rng.uniform(1, 8, 40), rng.choice([3, 4, 5, 6, 7], 40)])
    scheds = ["TE_G8_T4", "WE_G4_T1", "SV_G32_F32", "WV_G1_T1"]
    Y = rng.uniform(0, 1.5, (40, len(scheds)))
    w = np.array([1, 1, 1, 1, 1, 2.0])
    p = empty_table / "knn.txt"
    p.write_text("\n".join(train_selector.export_knn(X, Y, scheds, "agg", 5, w)) + "\n")
    ug.selector_load_model(str(p))
    V = 3000
    src, dst = ugdata.chung_lu(V, 30000, True, sigma, 0.5, 5)
    g = ug.Graph(V, src, dst, host_only=True)
    x = np.array([_features(g.stats(), F)])
    want = scheds[int(train_selector.knn_scores(X, Y, x, 5, w)[0].argmin())]
    got = _select(g, V, F)
    assert got.split("_")[0] == want.split("_")[0] and got.split("_")[1] == want.split("_")[1], (got, want)
