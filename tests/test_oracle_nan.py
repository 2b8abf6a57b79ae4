"""Pins for the oracle's NaN rule (R12): a max / min over messages any of which is NaN
is NaN -- IEEE 754-2019 maximum / minimum, numpy's np.maximum / np.minimum reductions -- written as
the canonical quiet NaN 0x7FFFFFFF; arg capture returns the FIRST NaN in-edge; sums propagate NaN
by IEEE arithmetic; rows without a NaN message are unaffected (bit-exact vs the NaN-free loop)."""
import numpy as np
import pytest

import oracle
import ugdata

CANON = 0x7FFFFFFF


def _inputs(V, E, F, seed, frac=0.03):
    rng = np.random.default_rng(seed)
    X = ugdata.values(V, F, seed, 1)
    w = ugdata.values(E, 1, seed, 2, role="edge")
    X[rng.random((V, F)) < frac] = np.nan
    w[rng.random((E, 1)) < frac] = np.nan
    return X, w


@pytest.mark.parametrize("gop", ["max", "min"])
def test_nan_max_min_matches_numpy_reduction(gop):
    V, F = 60, 5
    src, dst = ugdata.random_multigraph(V, 400, 17, zero_in_frac=0.2)
    X, w = _inputs(V, len(src), F, 3)
    for eo, B, bt in (("copy_lhs", None, None), ("mul", w, "e")):
        C = oracle.op(V, src, dst, eo, gop, A=X, a_type="u", B=B, b_type=bt, c_type="v", F=F)
        red = np.maximum.reduce if gop == "max" else np.minimum.reduce
        for v in range(V):
            es = np.nonzero(dst == v)[0]
            if es.size == 0:
                assert np.all(C[v] == 0)
                continue
            msgs = X[src[es]].astype(np.float32)
            if B is not None:
                msgs = (msgs * w[es]).astype(np.float32)
            ref = red(msgs, axis=0)                     # numpy propagates NaN
            assert np.array_equal(np.isnan(C[v]), np.isnan(ref)), (eo, v)
            ok = ~np.isnan(ref)
            np.testing.assert_array_equal(C[v][ok], ref[ok])
            assert np.all(C[v][~ok].view(np.uint32) == CANON)


def test_nan_free_rows_unchanged_and_sum_propagates():
    V, F = 50, 4
    src, dst = ugdata.random_multigraph(V, 300, 5, zero_in_frac=0.2)
    X, _ = _inputs(V, len(src), F, 8, frac=0.02)
    clean = np.nan_to_num(X, nan=0.25)
    for gop in ("max", "min", "sum", "mean"):
        a = oracle.op(V, src, dst, "copy_lhs", gop, A=X, a_type="u", c_type="v", F=F)
        b = oracle.op(V, src, dst, "copy_lhs", gop, A=clean, a_type="u", c_type="v", F=F)
        has = np.zeros((V, F), bool)
        np.logical_or.at(has, dst, np.isnan(X[src]))
        assert np.array_equal(np.isnan(a), has), gop
        np.testing.assert_array_equal(a[~has], b[~has])


@pytest.mark.parametrize("gop", ["max", "min"])
def test_nan_arg_is_first_nan_edge(gop):
    V, F = 40, 3
    src, dst = ugdata.random_multigraph(V, 250, 9)
    X, _ = _inputs(V, len(src), F, 11, frac=0.05)
    C, arg = oracle.op_arg(V, src, dst, "copy_lhs", gop, A=X, a_type="u", F=F)
    C2 = oracle.op(V, src, dst, "copy_lhs", gop, A=X, a_type="u", c_type="v", F=F)
    np.testing.assert_array_equal(C.view(np.uint32), C2.view(np.uint32))
    for v in range(V):
        es = np.nonzero(dst == v)[0]
        for f in range(F):
            nan_es = [e for e in es if np.isnan(X[src[e], f])]
            if nan_es:
                assert arg[v, f] == min(nan_es)
                assert C[v, f].view(np.uint32) == CANON
