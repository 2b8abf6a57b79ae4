"""GPU parity of the fused dot-product attention chain (ug_dot_attention) against
the fp64 definition oracle.dot_attention, through the C ABI.

Tolerance (R25): out within 1e-5 * sum_e a_e |val[u]| (the R11 scale of the final
weighted aggregation-sum, as for GAT, R23); attention within 1e-5 relative.  Graphs: random
multigraphs with self-loops, duplicate edges and zero-in-degree rows (unsorted COO: edge-id
indirection), a star whose hub is split into many chunks (the chunk merge), and the C2 / C4
shapes of BASELINE.json (Pubmed-shaped H = 8; ogbn-arxiv-shaped F = 128)."""
import numpy as np
import pytest
import torch

import oracle
import ugdata

pytestmark = pytest.mark.gpu

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def _check(V, src, dst, H, Dk, Dv, seed, g=None, attn=True, scale=None):
    q = ugdata.values(V, H * Dk, seed, 1)
    k = ugdata.values(V, H * Dk, seed, 2)
    val = ugdata.values(V, H * Dv, seed, 3)
    g = g or ug.Graph(V, src, dst)
    E = len(src)
    out = torch.full((V, H * Dv), float("nan"), device="cuda")
    a = torch.full((E, H), float("nan"), device="cuda") if attn else None
    ug.dot_attention(g, torch.from_numpy(q).cuda(), torch.from_numpy(k).cuda(), torch.from_numpy(val).cuda(), H,
                     scale=scale, out=out, attn=a)
    torch.cuda.synchronize()
    ref, aref, bnd = oracle.dot_attention(V, src, dst, q, k, val, H, scale=scale, bound=True)
    got = out.cpu().numpy().astype(np.float64)
    err = np.abs(got - ref)
    bad = ~(err <= 1e-5 * bnd)
    assert not bad.any(), f"{bad.sum()} outputs out of tolerance; max err/bound {(err / np.maximum(bnd, 1e-30)).max()}"
    if attn:
        np.testing.assert_allclose(a.cpu().numpy().astype(np.float64), aref, rtol=1e-5, atol=1e-30)


@pytest.mark.parametrize("H,Dk,Dv", [(1, 16, 16), (8, 8, 8), (2, 64, 32), (4, 3, 5), (1, 128, 128), (1, 256, 64),
                                     (3, 30, 50), (1, 512, 512),
                                     (4, 64, 64), (1, 96, 96), (1, 64, 128), (5, 32, 32), (3, 64, 64)])
def test_dotattn_random_multigraphs(H, Dk, Dv):
    for seed in range(3):
        V = 60 + 50 * seed
        src, dst = ugdata.random_multigraph(V, 7 * V, 40 + seed, zero_in_frac=0.15)
        _check(V, src, dst, H, Dk, Dv, 50 + seed)


@pytest.mark.parametrize("H,Dk,Dv", [(1, 16, 16), (8, 8, 8), (2, 128, 64), (4, 64, 64), (5, 32, 32)])
def test_dotattn_hub_split_rows(H, Dk, Dv):
    V = 3001
    s = np.concatenate([np.arange(1, V), np.arange(V)]).astype(np.int32)
    d = np.concatenate([np.zeros(V - 1, np.int32), (np.arange(V) + 1) % V]).astype(np.int32)
    _check(V, s, d, H, Dk, Dv, 7)


@pytest.mark.parametrize("cfg,H,F", [("C2", 8, 64), ("C2", 1, 16), ("C4", 8, 128), ("C4", 1, 128),
                                         ("C4", 4, 256), ("C4", 1, 64)])
def test_dotattn_configs(cfg, H, F):
    c = ugdata.CONFIGS[cfg]
    src, dst = ugdata.graph(cfg)
    _check(c.V, src, dst, H, F // H, F // H, 9, attn=(cfg == "C2"))


def test_dotattn_scale_zero_is_mean():
    """scale 0: uniform attention, out = copy_u_mean(val) (closed form, through the unified op)."""
    V = 500
    src, dst = ugdata.random_multigraph(V, 4000, 3)
    g = ug.Graph(V, src, dst)
    H, D = 2, 16
    q = torch.randn(V, H * D, device="cuda")
    val = torch.randn(V, H * D, device="cuda")
    out = ug.dot_attention(g, q, q, val, H, scale=0.0)
    mean = torch.empty(V, H * D, device="cuda")
    ug.op_run(g, "copy_lhs", "mean", A=val, a_type="u", C=mean, c_type="v")
    torch.cuda.synchronize()
    torch.testing.assert_close(out, mean, rtol=1e-5, atol=1e-6)
