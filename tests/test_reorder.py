"""Vertex renumbering (ug_graph_reorder): permutation validity and the RCM
bandwidth property on graphs whose optimum is known (CPU, host-only graphs)."""
import numpy as np
import pytest

import ugdata

ug = pytest.importorskip("paper_conf_asplos_0001lslwlgslllw23_b200")


def _bandwidth(perm, src, dst):
    inv = np.empty_like(perm)
    inv[perm] = np.arange(len(perm))
    return int(np.abs(inv[src].astype(np.int64) - inv[dst]).max())


def _shuffled(V, src, dst, seed):
    r = np.random.default_rng(seed).permutation(V).astype(np.int32)
    return r[src], r[dst]


@pytest.mark.parametrize("method", ["degree", "rcm", "community"])
def test_reorder_is_a_permutation(method):
    V = 500
    src, dst = ugdata.random_multigraph(V, 3000, 3)
    g = ug.Graph(V, src, dst, host_only=True)
    p = ug.reorder(g, method)
    assert sorted(p.tolist()) == list(range(V))


def test_rcm_recovers_a_shuffled_path():
    """A path 0-1-...-(V-1) (both directions) under random labels: RCM starts at an endpoint
    (degree 1) and walks the path, so the renumbered bandwidth is 1."""
    V = 1000
    a = np.arange(V - 1, dtype=np.int32)
    src, dst = np.concatenate([a, a + 1]), np.concatenate([a + 1, a])
    src, dst = _shuffled(V, src, dst, 1)
    g = ug.Graph(V, src, dst, host_only=True)
    assert _bandwidth(np.arange(V, dtype=np.int32), src, dst) > 100
    assert _bandwidth(ug.reorder(g, "rcm"), src, dst) == 1


def test_rcm_grid_bandwidth():
    """k x k grid, shuffled: RCM's bandwidth is O(k) (a BFS level holds <= k+1 vertices)."""
    k = 30
    idx = np.arange(k * k).reshape(k, k)
    e = [(idx[:, :-1].ravel(), idx[:, 1:].ravel()), (idx[:-1, :].ravel(), idx[1:, :].ravel())]
    src = np.concatenate([np.concatenate([a, b]) for a, b in e]).astype(np.int32)
    dst = np.concatenate([np.concatenate([b, a]) for a, b in e]).astype(np.int32)
    src, dst = _shuffled(k * k, src, dst, 2)
    g = ug.Graph(k * k, src, dst, host_only=True)
    assert _bandwidth(ug.reorder(g, "rcm"), src, dst) <= 2 * k + 2


def test_degree_order_is_non_increasing():
    V = 800
    src, dst = ugdata.chung_lu(V, 8000, True, 1.2, 0.5, 9)
    g = ug.Graph(V, src, dst, host_only=True)
    p = ug.reorder(g, "degree")
    deg = np.bincount(src, minlength=V) + np.bincount(dst, minlength=V)
    d = deg[p]
    assert (d[:-1] >= d[1:]).all()


def test_reorder_rejects_views():
    V = 50
    src, dst = ugdata.chung_lu(V, 400, True, 1.0, 0.5, 1)
    g = ug.Graph(V, src, dst, host_only=True)
    with pytest.raises(ug.UgError):
        ug.reorder(g.view_rows(0, 10), "rcm")


def test_community_order_recovers_blocks():
    """Block graph (200 blocks of 100 vertices, 90 % of edges inside a block) under random ids:
    after the community order at least 85 % of the edges join vertices < 100 ids apart (all
    intra-block edges, when each block becomes one id range); the shuffled ids have ~0.5 %."""
    V, blocks = 20000, 200
    src, dst = ugdata.community_graph(V, 300000, blocks, 0.9, 3)
    g = ug.Graph(V, src, dst, host_only=True)
    near = lambda p: _near(p, src, dst, V // blocks)
    assert near(np.arange(V, dtype=np.int32)) < 0.02
    assert near(ug.reorder(g, "community")) > 0.85


def _near(perm, src, dst, width):
    inv = np.empty_like(perm)
    inv[perm] = np.arange(len(perm))
    return float((np.abs(inv[src].astype(np.int64) - inv[dst]) < width).mean())
