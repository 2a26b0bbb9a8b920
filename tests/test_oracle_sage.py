"""Pins for the oracle's GraphSAGE mean aggregation (Eq. 1) and its adjoint: a hand-worked block,
constant and one-hot features (closed forms), the adjoint identity <A x, y> = <x, A^T y> for the backward, and
blocks straight out of the oracle sampler."""
from collections import Counter

import numpy as np
import pytest


def test_sage_mean_hand_worked(orc):
    # 3 dst rows: row 0 <- {0, 2}, row 1 <- {} (isolated), row 2 <- {1, 1, 3}
    x = np.array([[1.0, 10.0], [2.0, 20.0], [3.0, 30.0], [4.0, 40.0]])
    off = [0, 2, 2, 5]
    src = [0, 2, 1, 1, 3]
    out = orc.sage_mean(x, off, src)
    assert np.array_equal(out, [[2.0, 20.0], [0.0, 0.0], [8 / 3, 80 / 3]])
    g = np.array([[1.0, 2.0], [5.0, 5.0], [3.0, 6.0]])
    gx = orc.sage_mean_backward(g, off, src, 4)
    # row 0 sends g/2 to 0 and 2; row 2 sends g/3 to 1 (twice) and 3; row 1 sends nothing
    assert np.allclose(gx, [[0.5, 1.0], [2.0, 4.0], [0.5, 1.0], [1.0, 2.0]], rtol=0, atol=1e-15)


def _random_block(rng, n_dst, n_src, max_deg):
    deg = rng.integers(0, max_deg + 1, n_dst)
    off = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    src = rng.integers(0, n_src, int(off[-1])).astype(np.int32)
    return off, src


@pytest.mark.parametrize("seed", range(4))
def test_sage_mean_closed_forms(orc, seed):
    rng = np.random.default_rng(seed)
    n_dst, n_src = 50, 30
    off, src = _random_block(rng, n_dst, n_src, 9)
    deg = np.diff(off)
    # constant features: the mean is the constant wherever there are neighbours
    out = orc.sage_mean(np.full((n_src, 3), 7.25), off, src)
    assert np.array_equal(out[deg > 0], np.full(((deg > 0).sum(), 3), 7.25))
    assert not out[deg == 0].any()
    # one-hot features: row i = histogram of its sources / deg_i (counted independently)
    out = orc.sage_mean(np.eye(n_src), off, src)
    for i in range(n_dst):
        want = np.zeros(n_src)
        for j, c in Counter(src[off[i]:off[i + 1]].tolist()).items():
            want[j] = c / deg[i]
        assert np.allclose(out[i], want, rtol=0, atol=1e-15)
    # adjoint identity of the backward
    x = rng.standard_normal((n_src, 5))
    y = rng.standard_normal((n_dst, 5))
    lhs = float((orc.sage_mean(x, off, src) * y).sum())
    rhs = float((x * orc.sage_mean_backward(y, off, src, n_src)).sum())
    assert abs(lhs - rhs) <= 1e-12 * max(1.0, abs(lhs))


def test_sage_mean_on_sampled_blocks(orc):
    # blocks of the oracle sampler: every row's mean uses exactly min(deg, fanout) sources from F_{h+1}
    rng = np.random.default_rng(3)
    n = 300
    deg = rng.integers(0, 12, n)
    indptr = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    indices = rng.integers(0, n, int(indptr[-1])).astype(np.int32)
    seeds = rng.choice(n, 40, replace=False).astype(np.int64)
    r = orc.sample(indptr, indices, seeds, [5, 3], 99)
    x = rng.standard_normal((len(r["nodes"]), 4))
    for h in range(2):
        off, src = r["offsets"][h], r["src"][h]
        out = orc.sage_mean(x, off, src)
        for i in range(len(off) - 1):
            s = src[off[i]:off[i + 1]]
            want = x[s].mean(axis=0) if len(s) else np.zeros(4)
            assert np.allclose(out[i], want, rtol=1e-14, atol=1e-14)
