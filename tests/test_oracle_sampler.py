"""Pins for the oracle sampler (R3-R6).

* Floyd F2, exhaustively: for every d <= 7 and k <= d, enumerating all prod(j_i + 1) choice tuples
  yields every k-subset of [0, d) exactly k! times (Floyd's theorem: exact uniformity).
* Statistical uniformity of the Philox-driven sampler (chi-square over 20 000 batch seeds).
* Hand-worked cases: path graph (take all), isolated seed, d == k, d == k + 1, a star.
* Invariants on random R-MAT-like graphs: every emitted id is a true CSR neighbour at distinct
  positions, count = min(d, k), F_h is a prefix of F_{h+1}, new ids ascending and not in F_h,
  src consistent with F_{h+1}, |F_{h+1}| <= |F_h| (1 + f_h).
"""
import itertools
import math
from collections import Counter

import numpy as np
import pytest


def test_floyd_exhaustive_uniform(orc):
    for d in range(1, 8):
        for k in range(1, d + 1):
            ranges = [range(d - k + i + 1) for i in range(k)]
            counts = Counter()
            for t in itertools.product(*ranges):
                P = orc.floyd(d, k, list(t))
                assert len(P) == k and len(set(P)) == k and all(0 <= p < d for p in P)
                assert P == sorted(P)
                counts[tuple(P)] += 1
            assert len(counts) == math.comb(d, k)
            assert set(counts.values()) == {math.factorial(k)}


def _csr(n, edges):
    edges = sorted(edges)
    indptr = np.zeros(n + 1, np.int64)
    for u, _ in edges:
        indptr[u + 1] += 1
    indptr = np.cumsum(indptr)
    indices = np.array([v for _, v in edges], np.int32)
    return indptr, indices


def test_sample_node_statistical_uniformity(orc):
    d, k = 5, 2
    trials = 20000
    counts = Counter()
    for s in range(trials):
        counts[tuple(orc.sample_node(s * 7919 + 1, 3, 0, d, k))] += 1
    assert len(counts) == math.comb(d, k)
    exp = trials / math.comb(d, k)
    chi2 = sum((c - exp) ** 2 / exp for c in counts.values())
    assert chi2 < 30.0  # 9 dof; p ~ 4e-4


def test_sample_node_replace_uniform(orc):
    d, k = 7, 4
    counts = Counter()
    for s in range(5000):
        P = orc.sample_node(s + 11, 9, 1, d, k, replace=True)
        assert len(P) == k
        counts.update(P)
    exp = 5000 * k / d
    chi2 = sum((counts[p] - exp) ** 2 / exp for p in range(d))
    assert chi2 < 25.0  # 6 dof


def test_hand_worked_cases(orc):
    # path 0 -> 1 -> 2 -> 3 (deg 1: take all, no draws); isolated vertex 4.
    indptr, indices = _csr(5, [(0, 1), (1, 2), (2, 3)])
    r = orc.sample(indptr, indices, [0, 4], [3, 3], rng_seed=99)
    assert list(r["nodes"]) == [0, 4, 1, 2]
    assert list(r["counts"]) == [2, 3, 4, 1, 2]
    assert list(r["offsets"][0]) == [0, 1, 1]
    assert list(r["src"][0]) == [2]
    assert list(r["offsets"][1]) == [0, 1, 1, 2]
    assert list(r["src"][1]) == [2, 3]
    # d == k and d == k + 1: star centre 0 with 4 leaves
    indptr, indices = _csr(5, [(0, i) for i in range(1, 5)])
    r = orc.sample(indptr, indices, [0], [4], rng_seed=1)
    assert list(r["nodes"]) == [0, 1, 2, 3, 4]
    r = orc.sample(indptr, indices, [0], [3], rng_seed=1)
    assert len(r["nodes"]) == 4 and r["counts"][2] == 3
    # hand-worked star: centre d = 8, k = 3; the three draws come from the KAT-pinned Philox.
    indptr, indices = _csr(9, [(0, i) for i in range(1, 9)])
    seed = 2024
    t = [orc.uniform(orc.draw(seed, 0, 0, i), 8 - 3 + i + 1) for i in range(3)]
    S = []
    for i, ti in enumerate(t):
        j = 8 - 3 + i
        S.append(j if ti in S else ti)
    want = sorted(indices[p] for p in S)
    r = orc.sample(indptr, indices, [0], [3], rng_seed=seed)
    got = list(r["nodes"][1:])
    assert got == want


def test_errors(orc):
    indptr, indices = _csr(3, [(0, 1)])
    with pytest.raises(orc.OracleError):
        orc.sample(indptr, indices, [0, 0], [2], 1)  # repeated seed
    with pytest.raises(orc.OracleError):
        orc.sample(indptr, indices, [3], [2], 1)  # out of range


def random_graph(n, m, seed, skew=True):
    rng = np.random.default_rng(seed)
    if skew:
        w = 1.0 / np.arange(1, n + 1) ** 0.8
        w /= w.sum()
        src = rng.choice(n, size=m, p=w)
        dst = rng.choice(n, size=m, p=w[::-1])
    else:
        src = rng.integers(0, n, m)
        dst = rng.integers(0, n, m)
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    indptr = np.zeros(n + 1, np.int64)
    np.add.at(indptr, src + 1, 1)
    return np.cumsum(indptr), dst.astype(np.int32)


def check_sample_invariants(indptr, indices, seeds, fanout, r, replace=False):
    nodes = r["nodes"]
    counts = r["counts"]
    H = len(fanout)
    F = [int(c) for c in counts[: H + 1]]
    assert list(nodes[: len(seeds)]) == list(seeds)
    assert len(set(nodes.tolist())) == len(nodes)
    for h in range(H):
        prev = set(nodes[: F[h]].tolist())
        new = nodes[F[h]: F[h + 1]]
        assert all(new[i] < new[i + 1] for i in range(len(new) - 1))
        assert not (set(new.tolist()) & prev)
        assert F[h + 1] <= F[h] * (1 + fanout[h])
        off = r["offsets"][h]
        src = r["src"][h]
        assert off[0] == 0 and off[-1] == len(src) == counts[H + 1 + h]
        emitted = set()
        for idx in range(F[h]):
            v = nodes[idx]
            d = int(indptr[v + 1] - indptr[v])
            c = int(off[idx + 1] - off[idx])
            assert c == (fanout[h] if (replace and d > 0) else min(d, fanout[h]))
            got = nodes[src[off[idx]: off[idx + 1]]]
            adj = Counter(indices[indptr[v]: indptr[v + 1]].tolist())
            gc = Counter(got.tolist())
            for u, cu in gc.items():
                assert u in adj
                if not replace:
                    assert cu <= adj[u]
            emitted |= set(got.tolist())
            assert (src[off[idx]: off[idx + 1]] < F[h + 1]).all()
        assert set(new.tolist()) == emitted - prev


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_sampler_invariants_random_graph(orc, seed):
    n, m = 3000, 30000
    indptr, indices = random_graph(n, m, seed)
    rng = np.random.default_rng(seed + 100)
    seeds = rng.choice(n, 200, replace=False)
    fanout = [10, 5, 3]
    r = orc.sample(indptr, indices, seeds, fanout, rng_seed=seed * 31 + 7)
    check_sample_invariants(indptr, indices, seeds, fanout, r)
    r2 = orc.sample(indptr, indices, seeds, fanout, rng_seed=seed * 31 + 7, replace=True)
    check_sample_invariants(indptr, indices, seeds, fanout, r2, replace=True)


def test_sampler_deterministic_and_seed_sensitive(orc):
    indptr, indices = random_graph(2000, 40000, 9)
    seeds = np.arange(0, 2000, 10)
    a = orc.sample(indptr, indices, seeds, [10, 5], 5)
    b = orc.sample(indptr, indices, seeds, [10, 5], 5)
    c = orc.sample(indptr, indices, seeds, [10, 5], 6)
    assert np.array_equal(a["nodes"], b["nodes"])
    assert not np.array_equal(a["nodes"], c["nodes"])


def test_gather_definition(orc):
    rng = np.random.default_rng(0)
    table = rng.integers(0, 255, size=(100, 48), dtype=np.uint8)
    ids = rng.integers(0, 100, 500)
    out = orc.gather(table, ids)
    assert np.array_equal(out, table[ids])
