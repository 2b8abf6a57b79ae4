"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no message, reduction or CSR logic): it only
draws graphs and feature values.  Both sides of every parity check consume the same arrays.

Recipe:
  * Chung-Lu graphs with i.i.d. lognormal expected degrees (sigma per config), exact E,
    multi-edges and self-loops allowed (Table 3 std-of-nnz as skew target).
    Weights are i.i.d. per vertex, so vertex ids carry no degree order.
  * COO is emitted dst-sorted (edge id = position; rows grouped by destination) so that
    edge tensors need no permutation (reading R9).
  * undirected configs store both directions of every sampled pair (reading R20).
  * graph seed = 1000 + k for config Ck; value streams seeded (seed + 1, tag).
"""
from __future__ import annotations

import dataclasses

import numpy as np


@dataclasses.dataclass(frozen=True)
class GraphConfig:
    name: str
    V: int
    E: int
    directed: bool
    sigma_in: float
    sigma_out: float
    seed: int
    widths: tuple      # feature widths F exercised by this config
    note: str
    label: str = ""


# BASELINE.json configs; shapes and skew per SURVEY.md 8(d) (Table 3).
CONFIGS = {
    "C1": GraphConfig("C1", 2708, 10556, False, 1.015, 1.015, 1001, (16,),
                      "Cora-shaped (PAPER.md:148): u_mul_e_sum F=16", "Cora-shaped"),
    "C2": GraphConfig("C2", 19717, 88648, False, 1.108, 1.108, 1002, (16, 64),
                      "Pubmed-shaped (PAPER.md:150, E per BASELINE.json): GAT op set", "Pubmed-shaped"),
    "C3": GraphConfig("C3", 403394, 3387388, True, 1.209, 0.5, 1003, (32, 64, 128),
                      "amazon0601-shaped (PAPER.md:157): GCN/GIN aggregation, schedule sweep", "amazon0601-shaped"),
    "C4": GraphConfig("C4", 169343, 1166243, True, 1.2, 0.5, 1004, (128, 256),
                      "ogbn-arxiv-shaped: u_dot_v SDDMM", "ogbn-arxiv-shaped"),
    "C5": GraphConfig("C5", 232965, 114615892, False, 1.0, 1.0, 1005, (602,),
                      "Reddit-shaped: copy_u_sum / copy_u_mean F=602", "Reddit-shaped"),
}


def _weights(rng, V, sigma):
    w = rng.lognormal(0.0, sigma, V)
    return w / w.sum()


def _sorted_sample(rng, V, n, p):
    """n i.i.d. draws from p, returned sorted ascending, with per-vertex counts."""
    cnt = rng.multinomial(n, p).astype(np.int64)
    return np.repeat(np.arange(V, dtype=np.int32), cnt), cnt


def chung_lu(V, E, directed, sigma_in, sigma_out, seed):
    """Return (src, dst) int32 arrays of length E, dst-sorted (non-decreasing dst)."""
    rng = np.random.default_rng(seed)
    if directed:
        p_in = _weights(rng, V, sigma_in)
        p_out = _weights(rng, V, sigma_out)
        dst, _ = _sorted_sample(rng, V, E, p_in)
        s, _ = _sorted_sample(rng, V, E, p_out)
        src = s[rng.permutation(E)]
        return src, dst
    if E % 2:
        raise ValueError("undirected graph needs an even edge count")
    M = E // 2
    p = _weights(rng, V, sigma_in)
    a, cnt_a = _sorted_sample(rng, V, M, p)           # pair endpoint a_k (sorted)
    bs, cnt_b = _sorted_sample(rng, V, M, p)
    pi = rng.permutation(M)                           # b_k = bs[pi[k]]: i.i.d. endpoint
    # set1: edges b_k -> a_k, already grouped by dst = a_k.
    src1 = bs[pi]
    # set2: edges a_k -> b_k; grouped by dst = bs, position of pair k is pi[k].
    src2 = np.empty(M, dtype=np.int32)
    src2[pi] = a
    # interleave per destination row: row v = [cnt_a[v] set1 edges, cnt_b[v] set2 edges].
    deg = cnt_a + cnt_b
    row0 = np.zeros(V + 1, dtype=np.int64)
    np.cumsum(deg, out=row0[1:])
    start_a = np.zeros(V, dtype=np.int64)
    np.cumsum(cnt_a[:-1], out=start_a[1:])
    start_b = np.zeros(V, dtype=np.int64)
    np.cumsum(cnt_b[:-1], out=start_b[1:])
    k = np.arange(M, dtype=np.int64)
    pos1 = row0[a] + (k - start_a[a])
    pos2 = row0[bs] + cnt_a[bs] + (k - start_b[bs])
    src = np.empty(E, dtype=np.int32)
    dst = np.empty(E, dtype=np.int32)
    src[pos1] = src1
    dst[pos1] = a
    src[pos2] = src2
    dst[pos2] = bs
    return src, dst


def graph(cfg: str | GraphConfig):
    c = CONFIGS[cfg] if isinstance(cfg, str) else cfg
    return chung_lu(c.V, c.E, c.directed, c.sigma_in, c.sigma_out, c.seed)


def random_multigraph(V, E, seed, zero_in_frac=0.2):
    """Tiny unsorted COO multigraph for brute-force pins: self-loops, duplicate edges and
    zero-in-degree vertices are all likely.  NOT dst-sorted (exercises edge-id order)."""
    rng = np.random.default_rng(seed)
    n_live = max(1, int(round(V * (1.0 - zero_in_frac))))
    live = rng.choice(V, n_live, replace=False).astype(np.int32)
    dst = live[rng.integers(0, n_live, E)].astype(np.int32)
    src = rng.integers(0, V, E).astype(np.int32)
    if E >= 4:   # force a duplicate edge and a self-loop
        src[1], dst[1] = src[0], dst[0]
        src[2] = dst[2]
    return src, dst


# ---------------------------------------------------------------- feature values

def values(rows, width, seed, tag, mode="float", role="num", k=8):
    """Feature tensor [rows, width] float32.

    mode "float": U(-1,1) with exact zeros resampled (R12); role "den" draws |x| in
                  [0.5, 1.5] with a random sign (R13).
    mode "int":   integers in [-k, k] \\ {0}; role "den" or "edge" draws from
                  {+-0.5, +-1, +-2, +-4} (integer mode of SURVEY 8(c)).
    mode "pos":   U(0.5, 1.5) (positive-stress: partial sums grow linearly).
    mode "ones":  all 1.0.
    """
    rng = np.random.default_rng([int(seed), int(tag)])
    shape = (int(rows), int(width))
    if mode == "ones":
        return np.ones(shape, dtype=np.float32)
    if mode == "pos":
        return rng.uniform(0.5, 1.5, shape).astype(np.float32)
    if mode == "int":
        if role in ("den", "edge"):
            mags = np.array([0.5, 1.0, 2.0, 4.0], dtype=np.float32)
            x = mags[rng.integers(0, 4, shape)]
            return (x * rng.choice(np.array([-1.0, 1.0], np.float32), shape)).astype(np.float32)
        x = rng.integers(1, k + 1, shape).astype(np.float32)
        return (x * rng.choice(np.array([-1.0, 1.0], np.float32), shape)).astype(np.float32)
    if role == "den":
        x = rng.uniform(0.5, 1.5, shape).astype(np.float32)
        return x * rng.choice(np.array([-1.0, 1.0], np.float32), shape)
    x = rng.uniform(-1.0, 1.0, shape).astype(np.float32)
    z = x == 0.0
    while z.any():
        x[z] = rng.uniform(-1.0, 1.0, int(z.sum())).astype(np.float32)
        z = x == 0.0
    return x


def community_graph(V, E, blocks, p_in, seed, shuffle=True):
    """Stochastic-block-style COO (no method arithmetic): vertex v belongs to block
    v * blocks // V; each edge picks a destination uniformly and, with probability p_in, a
    source in the same block (else anywhere).  Ids are then randomly relabelled (shuffle),
    hiding the locality a renumbering (ug_graph_reorder) can recover.  Returned dst-sorted."""
    rng = np.random.default_rng(seed)
    dst = rng.integers(0, V, E).astype(np.int64)
    blk = dst * blocks // V
    lo = (blk * V + blocks - 1) // blocks
    hi = ((blk + 1) * V + blocks - 1) // blocks
    local = lo + (rng.random(E) * (hi - lo)).astype(np.int64)
    anywhere = rng.integers(0, V, E)
    src = np.where(rng.random(E) < p_in, local, anywhere)
    if shuffle:
        relabel = rng.permutation(V)
        src, dst = relabel[src], relabel[dst]
    order = np.argsort(dst, kind="stable")
    return src[order].astype(np.int32), dst[order].astype(np.int32)
