"""GPU parity of the fused GAT attention chain (ug_gat_attention) against the
fp64 definition in oracle.gat, through the C ABI.

Tolerance (fused chains): out within 1e-5 * sum_e a(e,h) |z[u][f]| (the R11 scale
of the final weighted aggregation-sum), attention within 1e-5 relative.  Graphs: C1 / C2 /
C3-shaped (ugdata), random multigraphs with self-loops, duplicate edges and zero-in-degree
rows, and a star whose hub exceeds the CTA-per-row threshold for every lane layout."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def _run(V, src, dst, H, F, seed, slope=0.2, attn=True, g=None, ld=None):
    el = ugdata.values(V, H, seed, 1)
    er = ugdata.values(V, H, seed, 2)
    z = ugdata.values(V, F, seed, 3)
    g = g or ug.Graph(V, src, dst)
    E = len(src)
    zd = torch.from_numpy(z).cuda()
    if ld is not None:                       # padded row stride for z and out
        buf = torch.zeros(V, ld, device="cuda")
        buf[:, :F] = zd
        zd = buf[:, :F]
    out = torch.full((V, ld or F), float("nan"), device="cuda")[:, :F]
    a = torch.full((E, H), float("nan"), device="cuda") if attn else None
    ug.gat_attention(g, torch.from_numpy(el).cuda(), torch.from_numpy(er).cuda(), zd, H, slope, out=out, attn=a)
    torch.cuda.synchronize()
    ref, aref, bnd = oracle.gat(V, src, dst, el, er, z, H, slope, bound=True)
    got = out.cpu().numpy().astype(np.float64)
    err = np.abs(got - ref)
    bad = ~(err <= 1e-5 * bnd)
    assert not bad.any(), (f"{bad.sum()} outputs out of tolerance; max err/bound "
                           f"{(err / np.maximum(bnd, 1e-30)).max()}")
    if attn:
        ga = a.cpu().numpy().astype(np.float64)
        np.testing.assert_allclose(ga, aref, rtol=1e-5, atol=1e-30)
    return got


@pytest.mark.parametrize("H,F", [(1, 16), (8, 64), (8, 8), (4, 256), (3, 12), (2, 6), (1, 602)])
def test_gat_random_multigraphs(H, F):
    for seed in range(3):
        V = 50 + 40 * seed
        src, dst = ugdata.random_multigraph(V, 6 * V, seed)
        _run(V, src, dst, H, F, 20 + seed)


@pytest.mark.parametrize("H,F", [(1, 16), (8, 64), (2, 6), (4, 256)])
def test_gat_hub_rows_use_cta_path(H, F):
    """A star (hub in-degree 3000) plus a ring: the hub exceeds every long-row threshold."""
    V = 3001
    hub_src = np.arange(1, V, dtype=np.int32)
    ring_src = np.arange(V, dtype=np.int32)
    src = np.concatenate([hub_src, ring_src])
    dst = np.concatenate([np.zeros(V - 1, np.int32), (ring_src + 1) % V]).astype(np.int32)
    _run(V, src, dst, H, F, 5)


@pytest.mark.parametrize("cfg,H,F", [("C1", 1, 16), ("C2", 8, 64), ("C2", 1, 16), ("C3", 4, 64)])
def test_gat_configs(cfg, H, F):
    c = ugdata.CONFIGS[cfg]
    src, dst = ugdata.graph(cfg)
    _run(c.V, src, dst, H, F, c.seed + 1)


def test_gat_padded_ld_and_no_attention():
    V = 300
    src, dst = ugdata.random_multigraph(V, 2000, 4)
    _run(V, src, dst, 4, 64, 8, attn=False, ld=70)      # ld 70: not a multiple of 4 -> float2 path
    _run(V, src, dst, 4, 64, 8, attn=False, ld=72)


def test_gat_unsorted_coo_and_slopes():
    """Edge ids not in dst order (eid != identity): attention lands at edge-id rows."""
    V = 200
    rng = np.random.default_rng(3)
    src = rng.integers(0, V, 1500).astype(np.int32)
    dst = rng.integers(0, V, 1500).astype(np.int32)
    for slope in (0.2, 0.0, 1.0):
        _run(V, src, dst, 2, 8, 11, slope=slope)


def test_gat_empty_graph_and_shape_errors():
    V = 10
    g = ug.Graph(V, np.zeros(0, np.int32), np.zeros(0, np.int32))
    el = torch.randn(V, 2, device="cuda")
    z = torch.randn(V, 8, device="cuda")
    out = ug.gat_attention(g, el, el, z, 2)
    torch.cuda.synchronize()
    assert (out == 0).all()
    with pytest.raises(ug.UgError, match="UG_ERR_SHAPE"):
        ug.gat_attention(g, el, el, torch.randn(V, 7, device="cuda"), 2)


def test_gat_sharded_views_equal_unsharded():
    """Row views (global src ids, local dst rows): the concatenated shards equal one call."""
    c = ugdata.CONFIGS["C2"]
    src, dst = ugdata.graph("C2")
    g = ug.Graph(c.V, src, dst)
    H, F = 8, 64
    el = torch.randn(c.V, H, device="cuda")
    er = torch.randn(c.V, H, device="cuda")
    z = torch.randn(c.V, F, device="cuda")
    full = ug.gat_attention(g, el, er, z, H)
    splits = g.partition(3)
    parts = []
    for k in range(3):
        r0, r1 = int(splits[k]), int(splits[k + 1])
        v = g.view_rows(r0, r1)
        parts.append(ug.gat_attention(v, el, er[r0:r1], z, H))
    torch.cuda.synchronize()
    assert torch.equal(torch.cat(parts), full)


def test_gat_layer_fused_equals_chain():
    """GATConv through the fused call vs the six-operator chain of the shim (both GPU)."""
    from paper_conf_asplos_0001lslwlgslllw23_b200 import gnn
    c = ugdata.CONFIGS["C2"]
    src, dst = ugdata.graph("C2")
    gd = gnn.GraphData(c.V, src, dst)
    torch.manual_seed(0)
    layer = gnn.GATConv(32, 8, heads=4).cuda()
    h = torch.randn(c.V, 32, device="cuda")
    with torch.no_grad():
        a = layer(gd, h, fused=True)
        b = layer(gd, h, fused=False)
    torch.cuda.synchronize()
    torch.testing.assert_close(a, b, rtol=1e-4, atol=1e-5)
