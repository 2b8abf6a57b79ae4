"""Pins for the GAT attention-chain oracle (oracle.gat) -- no GPU needed.

oracle.gat is the plain fp64 definition of the chain PAPER.md:224 describes (scores from a
message creation el_u + er_v, GAT's edge softmax, then the weighted aggregation-sum).  It is
pinned here to things other than itself:
  * a dense brute-force formulation (one-hot incidence products, masked dense max) on random
    multigraphs with self-loops, duplicate edges and zero-in-degree vertices;
  * the same chain composed from the per-op oracle (u_add_v, copy_e_max, e_sub_v, copy_e_sum,
    e_div_v, u_mul_e_sum; Fig. 5 / Table 4) -- the paper's own operator sequence;
  * closed forms: equal scores -> attention 1/deg and out = copy_u_mean; slope 1 -> er
    cancels in the softmax; attention rows sum to 1;
  * a hand-worked 3-vertex example with literal values.
"""
import math

import numpy as np
import pytest

import oracle
import ugdata
import dense_ref


def _dense_gat(V, src, dst, el, er, z, H, slope):
    """Dense fp64 formulation: no in-edge lists, no edge loop."""
    S, T = dense_ref.incidence(V, src, dst)                  # [E, V] one-hot
    E = len(src)
    F = z.shape[1]
    D = F // H
    s = S @ el.astype(np.float64) + T @ er.astype(np.float64)   # [E, H]
    s = np.where(s >= 0, s, slope * s)
    mask = T.T > 0                                            # [V, E]
    out = np.zeros((V, F))
    attn = np.zeros((E, H))
    for h in range(H):
        big = np.where(mask, s[:, h][None, :], -np.inf)
        mx = big.max(axis=1)                                  # [V] (-inf for empty rows)
        mx = np.where(np.isfinite(mx), mx, 0.0)
        p = np.exp(s[:, h] - T @ mx)                          # [E]
        den = T.T @ p                                         # [V]
        a = p / (T @ np.where(den > 0, den, 1.0))
        attn[:, h] = a
        zu = S @ z[:, h * D:(h + 1) * D].astype(np.float64)   # [E, D]
        out[:, h * D:(h + 1) * D] = T.T @ (a[:, None] * zu)
    return out, attn


def _inputs(V, H, F, seed):
    el = ugdata.values(V, H, seed, 1)
    er = ugdata.values(V, H, seed, 2)
    z = ugdata.values(V, F, seed, 3)
    return el, er, z


@pytest.mark.parametrize("H,F", [(1, 4), (2, 6), (4, 16)])
@pytest.mark.parametrize("slope", [0.2, 0.0, 1.0])
def test_gat_oracle_equals_dense(H, F, slope):
    for seed in range(5):
        V = 6 + 5 * seed
        E = 4 * V + seed
        src, dst = ugdata.random_multigraph(V, E, seed)
        el, er, z = _inputs(V, H, F, 100 + seed)
        out, attn = oracle.gat(V, src, dst, el, er, z, H, slope)
        dout, dattn = _dense_gat(V, src, dst, el, er, z, H, slope)
        np.testing.assert_allclose(attn, dattn, rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(out, dout, rtol=1e-12, atol=1e-14)


@pytest.mark.parametrize("H,F", [(1, 8), (4, 16)])
def test_gat_oracle_equals_operator_chain(H, F):
    """The definition agrees with the paper's operator chain run through the per-op oracle
    (fp32 messages): u_add_v -> LeakyReLU -> copy_e_max -> e_sub_v -> exp -> copy_e_sum ->
    e_div_v -> u_mul_e_sum, within the R11 scale sum_e a |z|."""
    V, E = 40, 200
    src, dst = ugdata.random_multigraph(V, E, 7)
    el, er, z = _inputs(V, H, F, 9)
    kw = dict(F=H, H=H)
    s = oracle.op(V, src, dst, "add", "assign", A=el, a_type="u", B=er, b_type="v", c_type="e", **kw)
    s = np.where(s >= 0, s, np.float32(0.2) * s).astype(np.float32)
    m = oracle.op(V, src, dst, "copy_lhs", "max", A=s, a_type="e", c_type="v", **kw)
    sh = oracle.op(V, src, dst, "sub", "assign", A=s, a_type="e", B=m, b_type="v", c_type="e", **kw)
    ex = np.exp(sh.astype(np.float64)).astype(np.float32)
    den = oracle.op(V, src, dst, "copy_lhs", "sum", A=ex, a_type="e", c_type="v", **kw)
    a = oracle.op(V, src, dst, "div", "assign", A=ex, a_type="e", B=den, b_type="v", c_type="e", **kw)
    chain = oracle.op(V, src, dst, "mul", "sum", A=z, a_type="u", B=a, b_type="e", c_type="v", F=F, H=H)
    out, attn, bnd = oracle.gat(V, src, dst, el, er, z, H, 0.2, bound=True)
    np.testing.assert_allclose(a, attn, rtol=1e-6, atol=1e-7)
    assert (np.abs(chain - out) <= 1e-5 * bnd + 1e-7).all()


def test_gat_uniform_scores_is_mean():
    """el = er = 0: every score is 0, attention = 1/deg, out = copy_u_mean (R8)."""
    V, E, H, F = 30, 150, 2, 8
    src, dst = ugdata.random_multigraph(V, E, 3)
    z = ugdata.values(V, F, 4, 1)
    zero = np.zeros((V, H), np.float32)
    out, attn = oracle.gat(V, src, dst, zero, zero, z, H)
    deg = np.bincount(dst, minlength=V)
    np.testing.assert_allclose(attn, np.repeat((1.0 / deg[dst])[:, None], H, axis=1), rtol=1e-15)
    mean = oracle.op(V, src, dst, "copy_lhs", "mean", A=z, a_type="u", F=F)
    np.testing.assert_allclose(out, mean, rtol=1e-6, atol=1e-7)


def test_gat_slope_one_er_cancels_and_rows_sum_to_one():
    """With slope 1 LeakyReLU is the identity, so er[v] shifts every score of row v equally and
    the softmax cancels it; attention of every non-empty (row, head) sums to 1."""
    V, E, H, F = 25, 120, 3, 6
    src, dst = ugdata.random_multigraph(V, E, 11)
    el, er, z = _inputs(V, H, F, 12)
    out1, a1 = oracle.gat(V, src, dst, el, er, z, H, 1.0)
    out2, a2 = oracle.gat(V, src, dst, el, np.zeros_like(er), z, H, 1.0)
    np.testing.assert_allclose(a1, a2, rtol=1e-13)
    np.testing.assert_allclose(out1, out2, rtol=1e-12, atol=1e-14)
    _, a3 = oracle.gat(V, src, dst, el, er, z, H, 0.2)
    sums = np.zeros((V, H))
    np.add.at(sums, dst, a3)
    deg = np.bincount(dst, minlength=V)
    np.testing.assert_allclose(sums[deg > 0], 1.0, rtol=1e-14)
    assert (a3 > 0).all()
    zero_rows = deg == 0
    assert zero_rows.any()
    assert (out1[zero_rows] == 0).all()


def test_gat_hand_worked():
    """3 vertices, in-edges of vertex 2: 0->2, 1->2, 2->2 (self-loop); H = 1, slope 0.2.
    el = [-5 ln2, ln2, 0], er[2] = 0 -> scores [0.2*(-5 ln2), ln2, 0] = [-ln2, ln2, 0];
    max = ln2 -> exp = [1/4, 1, 1/2], den = 7/4 -> a = [1/7, 4/7, 2/7];
    z = [7, 14, 21] -> out[2] = 1 + 8 + 6 = 15; vertices 0 and 1 have no in-edges -> 0."""
    ln2 = math.log(2.0)
    src = np.array([0, 1, 2], np.int32)
    dst = np.array([2, 2, 2], np.int32)
    el = np.array([[-5 * ln2], [ln2], [0.0]], np.float32)
    er = np.array([[0.0], [0.0], [0.0]], np.float32)
    z = np.array([[7.0], [14.0], [21.0]], np.float32)
    out, attn = oracle.gat(3, src, dst, el, er, z, 1, 0.2)
    np.testing.assert_allclose(attn[:, 0], [1 / 7, 4 / 7, 2 / 7], rtol=1e-6)
    np.testing.assert_allclose(out[:, 0], [0.0, 0.0, 15.0], rtol=1e-6)
