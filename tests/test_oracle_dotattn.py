"""Pins for the dot-product attention oracle (oracle.dot_attention: the FusedMM-style
SDDMM + edge softmax + SpMM chain, PAPER.md:588 / :224) -- no GPU needed.

oracle.dot_attention is the plain fp64 per-destination loop.  It is pinned here to things other
than itself:
  * the textbook masked-attention formulation on a dense matrix: scores S = scale * Q K^T (a
    library matmul over all vertex pairs), entries without an edge masked to -inf, multi-edges
    counted by multiplicity, row softmax, out = P @ Val (a second matmul) -- no edge loop;
  * the same chain composed from the per-op oracle (u_dot_v message creation, then the softmax,
    then u_mul_e_sum aggregation; Fig. 5 / Table 4) -- the paper's own operators;
  * closed forms: k = 0 or scale = 0 -> uniform attention and out = copy_u_mean(val); one
    in-edge -> out = val[src]; attention rows sum to 1; relabelling equivariance;
  * a hand-worked 3-vertex example with literal values (tests/golden/dot_attention.json).
"""
import json
import os

import numpy as np
import pytest

import oracle
import ugdata

HERE = os.path.dirname(os.path.abspath(__file__))


def _dense(V, src, dst, q, k, val, H, scale):
    """Masked dense attention: out[v] = softmax_u(mask(scale q_v . k_u)) @ val (per head)."""
    M = np.zeros((V, V))
    np.add.at(M, (dst, src), 1.0)                      # multiplicity of u -> v
    Dk, Dv = q.shape[1] // H, val.shape[1] // H
    out = np.zeros((V, H * Dv))
    for h in range(H):
        Qh = q[:, h * Dk:(h + 1) * Dk].astype(np.float64)
        Kh = k[:, h * Dk:(h + 1) * Dk].astype(np.float64)
        S = scale * (Qh @ Kh.T)                        # [V(dst), V(src)]
        S = np.where(M > 0, S, -np.inf)
        mx = S.max(axis=1, keepdims=True)
        mx = np.where(np.isfinite(mx), mx, 0.0)
        P = M * np.exp(S - mx)                          # exp(-inf) = 0 off the edges
        den = P.sum(axis=1, keepdims=True)
        P = P / np.where(den > 0, den, 1.0)
        out[:, h * Dv:(h + 1) * Dv] = P @ val[:, h * Dv:(h + 1) * Dv].astype(np.float64)
    return out


def _inputs(V, H, Dk, Dv, seed):
    return (ugdata.values(V, H * Dk, seed, 1), ugdata.values(V, H * Dk, seed, 2),
            ugdata.values(V, H * Dv, seed, 3))


@pytest.mark.parametrize("H,Dk,Dv", [(1, 4, 4), (2, 3, 5), (4, 8, 2), (1, 16, 1)])
def test_dotattn_oracle_equals_dense(H, Dk, Dv):
    for seed in range(5):
        V = 7 + 6 * seed
        src, dst = ugdata.random_multigraph(V, 4 * V + seed, 300 + seed, zero_in_frac=0.2)
        q, k, val = _inputs(V, H, Dk, Dv, seed)
        scale = 1.0 / np.sqrt(Dk)
        out, attn = oracle.dot_attention(V, src, dst, q, k, val, H)
        ref = _dense(V, src, dst, q, k, val, H, scale)
        np.testing.assert_allclose(out, ref, rtol=1e-12, atol=1e-12)


def test_dotattn_oracle_equals_per_op_chain():
    """u_dot_v (message creation, fp32 messages) -> softmax -> u_mul_e_sum: within the fp32
    rounding of the scores and of the per-op aggregation."""
    V, H, Dk, Dv = 40, 2, 6, 3
    src, dst = ugdata.random_multigraph(V, 200, 7, zero_in_frac=0.2)
    q, k, val = _inputs(V, H, Dk, Dv, 9)
    out, attn = oracle.dot_attention(V, src, dst, q, k, val, H, scale=1.0)
    s = oracle.op(V, src, dst, "dot", "assign", A=k, a_type="u", B=q, b_type="v", c_type="e",
                  F=H * Dk, H=H).astype(np.float64)                      # [E, H] scores
    E = len(src)
    a = np.zeros((E, H))
    for v in range(V):
        es = np.nonzero(dst == v)[0]
        if es.size:
            x = np.exp(s[es] - s[es].max(axis=0))
            a[es] = x / x.sum(axis=0)
    np.testing.assert_allclose(attn, a, rtol=1e-5, atol=1e-7)
    y = oracle.op(V, src, dst, "mul", "sum", A=val, a_type="u", B=a.astype(np.float32), b_type="e", c_type="v",
                  F=H * Dv, H=H)
    np.testing.assert_allclose(out, y, rtol=1e-5, atol=1e-6)


def test_dotattn_closed_forms():
    V, H, Dk, Dv = 30, 3, 4, 2
    src, dst = ugdata.random_multigraph(V, 150, 11, zero_in_frac=0.2)
    q, k, val = _inputs(V, H, Dk, Dv, 12)
    mean = oracle.op(V, src, dst, "copy_lhs", "mean", A=val, a_type="u", c_type="v", F=H * Dv).astype(np.float64)
    for kk, sc in ((np.zeros_like(k), 1.0), (k, 0.0)):
        out, attn = oracle.dot_attention(V, src, dst, q, kk, val, H, scale=sc)
        np.testing.assert_allclose(out, mean, rtol=1e-6, atol=1e-7)     # uniform attention = mean
        deg = np.bincount(dst, minlength=V)
        np.testing.assert_allclose(attn, 1.0 / deg[dst][:, None] * np.ones((1, H)), rtol=1e-14)
    # attention rows sum to one; zero in-degree rows are 0
    out, attn = oracle.dot_attention(V, src, dst, q, k, val, H)
    sums = np.zeros((V, H))
    np.add.at(sums, dst, attn)
    deg = np.bincount(dst, minlength=V)
    np.testing.assert_allclose(sums[deg > 0], 1.0, rtol=1e-14)
    assert np.all(out[deg == 0] == 0.0)
    # a single in-edge: out = val[src] exactly
    s1 = np.arange(V, dtype=np.int32)
    d1 = np.roll(s1, 1)
    out1, _ = oracle.dot_attention(V, s1, d1, q, k, val, H)
    np.testing.assert_array_equal(out1[d1], val[s1].astype(np.float64))


def test_dotattn_relabel_equivariance():
    V, H, Dk, Dv = 25, 2, 3, 3
    src, dst = ugdata.random_multigraph(V, 120, 5)
    q, k, val = _inputs(V, H, Dk, Dv, 6)
    out, attn = oracle.dot_attention(V, src, dst, q, k, val, H)
    perm = np.random.default_rng(1).permutation(V)
    inv = np.argsort(perm)
    out2, attn2 = oracle.dot_attention(V, inv[src].astype(np.int32), inv[dst].astype(np.int32), q[perm], k[perm],
                                       val[perm], H)
    np.testing.assert_allclose(out2, out[perm], rtol=1e-13, atol=1e-15)
    np.testing.assert_allclose(attn2, attn, rtol=1e-13)


def test_dotattn_hand_worked():
    g = json.load(open(os.path.join(HERE, "golden", "dot_attention.json")))
    q = np.array(g["q"], np.float32)
    k = np.array(g["k"], np.float32)
    val = np.array(g["val"], np.float32)
    out, attn = oracle.dot_attention(g["V"], np.array(g["src"], np.int32), np.array(g["dst"], np.int32), q, k, val,
                                     g["H"], scale=g["scale"])
    np.testing.assert_allclose(out, np.array(g["expect_out"]), rtol=1e-12)
    np.testing.assert_allclose(attn[:, 0], np.array(g["expect_attn"]), rtol=1e-12)
