"""Pins for the oracle planner: max-flow, time bisection, closed-form plan
times (R11), request routing (R12) and DDAK (Eq. 2).

Max-flow: brute-force minimum s-t cut over all 2^(n-2) cuts (max-flow = min-cut theorem), SciPy's
maximum_flow and networkx on random graphs with parallel, antiparallel, zero and INF links; closed
forms (series = min, parallel = sum); flow certificate (capacity, conservation, value).
Time bisection: single path ceil(D/c), parallel paths ceil(D/sum c), a two-socket closed form, and a
linear scan over T for tiny demands. DDAK: exhaustive enumeration of tiny instances, the closed-form
2:1 fill ratio, hierarchy, pool semantics.
"""
import itertools

import networkx as nx
import numpy as np
import pytest
from scipy.sparse import csr_matrix
from scipy.sparse.csgraph import maximum_flow

INF = np.iinfo(np.int64).max


def random_links(n, m, rng, inf_prob=0.05, zero_prob=0.05, maxcap=50):
    links = []
    for _ in range(m):
        u, v = rng.integers(0, n, 2)
        if u == v:
            continue
        r = rng.random()
        cap = INF if r < inf_prob else (0 if r < inf_prob + zero_prob else int(rng.integers(1, maxcap)))
        links.append((int(u), int(v), cap))
        if rng.random() < 0.2:  # antiparallel partner
            links.append((int(v), int(u), int(rng.integers(1, maxcap))))
        if rng.random() < 0.1:  # parallel partner
            links.append((int(u), int(v), int(rng.integers(0, maxcap))))
    return links


def brute_min_cut(n, links, s, t):
    others = [x for x in range(n) if x not in (s, t)]
    best = None
    for mask in range(1 << len(others)):
        S = {s} | {others[i] for i in range(len(others)) if mask >> i & 1}
        c = 0
        for u, v, cap in links:
            if u in S and v not in S:
                c = INF if cap == INF or c == INF else c + cap
        best = c if best is None else min(best, c)
    return best


def check_certificate(n, links, s, t, value, flow):
    bal = [0] * n
    for (u, v, cap), f in zip(links, flow):
        assert 0 <= f and (cap == INF or f <= cap)
        bal[u] -= int(f)
        bal[v] += int(f)
    for x in range(n):
        if x not in (s, t):
            assert bal[x] == 0
    assert bal[t] == value and -bal[s] == value


@pytest.mark.parametrize("seed", range(40))
def test_maxflow_vs_brute_min_cut(orc, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 11))
    links = random_links(n, int(rng.integers(1, 3 * n)), rng)
    s, t = 0, n - 1
    cut = brute_min_cut(n, links, s, t)
    if cut == INF:
        with pytest.raises(orc.OracleError) as e:
            orc.maxflow(n, links, s, t)
        assert e.value.status == orc.EINVAL
        return
    val, flow = orc.maxflow(n, links, s, t)
    assert val == cut
    check_certificate(n, links, s, t, val, flow)


@pytest.mark.parametrize("seed", range(10))
def test_maxflow_vs_scipy_networkx(orc, seed):
    rng = np.random.default_rng(1000 + seed)
    n = 40
    links = random_links(n, 200, rng, inf_prob=0.0, zero_prob=0.1, maxcap=10**6)
    val, flow = orc.maxflow(n, links, 0, n - 1)
    check_certificate(n, links, 0, n - 1, val, flow)
    # scipy wants one entry per (u, v): merge parallel links
    agg = {}
    for u, v, c in links:
        agg[(u, v)] = agg.get((u, v), 0) + c
    rows = [k[0] for k in agg]
    cols = [k[1] for k in agg]
    data = np.array([agg[k] for k in agg], np.int32)
    M = csr_matrix((data, (rows, cols)), shape=(n, n))
    assert maximum_flow(M, 0, n - 1).flow_value == val
    G = nx.DiGraph()
    G.add_nodes_from(range(n))
    for (u, v), c in agg.items():
        G.add_edge(u, v, capacity=c)
    assert nx.maximum_flow_value(G, 0, n - 1) == val


def test_maxflow_closed_forms(orc):
    # series: min; parallel: sum; INF links are transparent when a finite link bounds the path
    assert orc.maxflow(4, [(0, 1, 7), (1, 2, 3), (2, 3, 9)], 0, 3)[0] == 3
    assert orc.maxflow(2, [(0, 1, 7), (0, 1, 3), (0, 1, 0)], 0, 1)[0] == 10
    assert orc.maxflow(3, [(0, 1, INF), (1, 2, 5)], 0, 2)[0] == 5
    assert orc.maxflow(3, [(0, 1, 5)], 0, 2)[0] == 0  # t unreachable
    with pytest.raises(orc.OracleError):
        orc.maxflow(3, [(0, 1, INF), (1, 2, INF)], 0, 2)  # unbounded


def _server(rng, k, with_nvlink):
    """s, host bins (2), PCIe switches (2), GPU ports (k), NVSwitch, compute nodes (k), t; links in MB/s."""
    s, t = 0, 1
    host = [2, 3]
    sw = [4, 5]
    port = [6 + g for g in range(k)]
    nvsw = 6 + k
    comp = [7 + k + g for g in range(k)]
    n = 7 + 2 * k
    links = [(s, h, INF) for h in host]
    links += [(host[j], sw[j], int(rng.integers(10, 60))) for j in range(2)]
    links += [(host[0], host[1], int(rng.integers(1, 20))), (host[1], host[0], int(rng.integers(1, 20)))]  # UPI
    links += [(sw[g * 2 // k], port[g], int(rng.integers(5, 30))) for g in range(k)]
    links += [(port[g], comp[g], INF) for g in range(k)]
    if with_nvlink:
        for g in range(k):
            c = int(rng.integers(50, 200))
            links += [(port[g], nvsw, c), (nvsw, comp[g], c)]
    links += [(comp[g], t, INF) for g in range(k)]
    return n, links, s, t


@pytest.mark.parametrize("seed", range(20))
def test_maxflow_nvlink_never_hurts(orc, seed):
    """Planner sanity: removing the NVLink edges can never increase the max-flow. With every
    compute node an infinite sink (c(v_c, t) = inf) the rate max-flow is the host ingest capacity,
    so here NVLink leaves it unchanged: its value shows up in the per-GPU time plan (R11), not in F."""
    k = 4
    rng = np.random.default_rng(seed)
    n, with_nv, s, t = _server(rng, k, True)
    rng = np.random.default_rng(seed)
    _, without, _, _ = _server(rng, k, False)
    f_with = orc.maxflow(n, with_nv, s, t)[0]
    f_without = orc.maxflow(n, without, s, t)[0]
    assert f_without <= f_with
    assert f_without == f_with
    assert f_with == brute_min_cut(n, with_nv, s, t) if n <= 16 else True
    # the NVLink fabric cannot carry more than the host side supplies: F <= sum of host egress + UPI
    host_out = sum(c for (u, v, c) in with_nv if u in (2, 3) and v in (4, 5))
    assert f_with <= host_out


def _tb(orc, n, links, supply_idx, s, t):
    sup = [1 if i in supply_idx else 0 for i in range(len(links))]
    return orc.time_bisect(n, links, sup, s, t)


def test_time_bisect_closed_forms(orc):
    # single path: s -(D)-> bin -> x -> gpu -> t(INF); T* = ceil(D / c)
    for D, c in [(1, 1), (100, 7), (10**9, 13), (5, 10)]:
        links = [(0, 1, D), (1, 2, c), (2, 3, INF)]
        T, _ = _tb(orc, 4, links, {0}, 0, 3)
        assert T == -(-D // c)
    # parallel paths: T* = ceil(D / sum c)
    links = [(0, 1, 1000), (1, 2, 3), (1, 2, 4), (1, 2, 6), (2, 3, INF)]
    assert _tb(orc, 4, links, {0}, 0, 3)[0] == -(-1000 // 13)
    # zero demand
    assert _tb(orc, 4, [(0, 1, 0), (1, 2, 5), (2, 3, INF)], {0}, 0, 3)[0] == 0
    # infeasible: demanded bin unreachable
    with pytest.raises(orc.OracleError) as e:
        _tb(orc, 4, [(0, 1, 5), (2, 3, INF)], {0}, 0, 3)
    assert e.value.status == orc.EINFEASIBLE


@pytest.mark.parametrize("S0,S1,p,u", [(800, 200, 10, 5), (1000, 1000, 3, 50), (5000, 0, 7, 1), (300, 250, 2, 0)])
def test_time_bisect_two_socket(orc, S0, S1, p, u):
    # two host bins (one per socket), 4 GPU ports per socket of capacity p, UPI u each way.
    # T* = max(ceil((S0+S1)/(8p)), ceil(S0/(4p+u)), ceil(S1/(4p+u)))
    s, h0, h1, c0, c1, t = 0, 1, 2, 3, 4, 5
    gpus = list(range(6, 14))
    links = [(s, h0, S0), (s, h1, S1), (h0, c0, INF), (h1, c1, INF), (c0, c1, u), (c1, c0, u)]
    for i, g in enumerate(gpus):
        links.append((c0 if i < 4 else c1, g, p))
        links.append((g, t, INF))
    T, flow = _tb(orc, 14, links, {0, 1}, s, t)
    want = max(-(-(S0 + S1) // (8 * p)), -(-S0 // (4 * p + u)), -(-S1 // (4 * p + u)))
    assert T == want


def test_time_bisect_linear_scan(orc):
    rng = np.random.default_rng(3)
    for trial in range(15):
        n = 7
        links = [(0, 1, int(rng.integers(1, 40))), (0, 2, int(rng.integers(0, 40)))]
        for _ in range(10):
            u = int(rng.integers(1, 5))
            v = int(rng.integers(3, 6))
            if u != v:
                links.append((u, v, int(rng.integers(1, 6))))
        links += [(5, 6, INF), (3, 6, INF), (4, 6, INF)]
        D = links[0][2] + links[1][2]
        try:
            T, _ = _tb(orc, n, links, {0, 1}, 0, 6)
        except orc.OracleError as e:
            assert e.status == orc.EINFEASIBLE
            continue
        # brute force: smallest T with maxflow(T) == D
        for Tb in range(0, T + 1):
            sc = [(u, v, c if i < 2 else (c if c == INF else c * Tb)) for i, (u, v, c) in enumerate(links)]
            if orc.maxflow(n, sc, 0, 6)[0] == D:
                break
        assert Tb == T


def test_plan_closed_forms_hand_worked(orc):
    # k = 2, HBM bins 0 (GPU0), 1 (GPU1), host bin 2; per GPU per batch d = [100, 60, 40];
    # x for host bin: 30 bytes enter via GPU0, 10 via GPU1 (W = 40).
    own = [0, 1, -1]
    d = [100, 60, 40]
    x = [[0, 0], [0, 0], [30, 10]]
    # GPU0: in = 60 (peer HBM1) + ceil(40*10/40)=10 -> 70; out = 100 (HBM0 to GPU1) + ceil(1*40*30/40)=30 -> 130
    # GPU1: in = 100 + ceil(40*30/40)=30 -> 130; out = 60 + ceil(40*10/40)=10 -> 70
    # max = 130; nvlink cap 7 -> ceil(130/7) = 19
    # HBM: GPU0 = 2*100 + 200 = 400, GPU1 = 2*60 + 200 = 320 -> ceil(400/9) = 45
    tn, th = orc.plan_closed_forms(2, own, d, x, 7, 9)
    assert (tn, th) == (19, 45)
    # single GPU, all local: no NVLink bytes
    tn, th = orc.plan_closed_forms(1, [0], [500], [[0]], 0, 100)
    assert (tn, th) == (0, 10)


def test_bucket_hand_worked_and_properties(orc):
    # one host bin, k = 2, x = [3, 1] (W = 4), 10 requests of rank g = 0:
    # slot = floor(r*4/10) = 0,0,0,1,1,2,2,2,3,3 -> via GPU0 while slot < 3 (r = 0..7), GPU1 for r = 8, 9
    route, qoff, qpos = orc.bucket(0, 2, [-1], [[3, 1]], [0] * 10)
    assert list(route) == [0] * 8 + [1] * 2
    assert list(qoff) == [0, 8, 10]
    rng = np.random.default_rng(0)
    own = [0, 1, 2, -1, -1]
    x = [[0, 0, 0], [0, 0, 0], [0, 0, 0], [5, 3, 2], [0, 0, 0]]
    bins = rng.integers(0, 5, 1000)
    for g in range(3):
        route, qoff, qpos = orc.bucket(g, 3, own, x, bins)
        assert sorted(qpos.tolist()) == list(range(1000))  # every request in exactly one queue
        for q in range(15):
            seg = qpos[qoff[q]: qoff[q + 1]]
            assert (np.diff(seg) > 0).all()  # stable
            assert (route[seg] == q).all()
        for i, b in enumerate(bins):
            if own[b] >= 0:
                assert route[i] == b * 3 + own[b]
            if b == 4:  # W = 0: direct
                assert route[i] == 4 * 3 + g
        nj = int((bins == 3).sum())
        for h in range(3):
            cnt = int((route == 3 * 3 + h).sum())
            assert abs(cnt - nj * x[3][h] / 10) <= 1


def brute_ddak_feasible(hot, caps):
    nb = len(caps)
    sols = []
    for assign in itertools.product(range(nb), repeat=len(hot)):
        used = [assign.count(b) for b in range(nb)]
        if all(used[b] <= caps[b] for b in range(nb)):
            sols.append(assign)
    return sols


@pytest.mark.parametrize("seed", range(12))
def test_ddak_exhaustive_small(orc, seed):
    rng = np.random.default_rng(seed)
    nv = int(rng.integers(1, 8))
    nb = int(rng.integers(1, 4))
    hot = rng.integers(0, 20, nv)
    tier = sorted(rng.integers(0, 2, nb).tolist())
    caps = rng.integers(0, nv + 1, nb)
    if caps.sum() < nv:
        caps[-1] += nv - caps.sum()
    traffic = rng.integers(0, 10, nb)
    sols = brute_ddak_feasible(hot.tolist(), caps.tolist())
    assert sols  # instance is feasible
    for pool in (1, 2, 100):
        bin_of, slot_of, A, U = orc.ddak(hot, tier, caps, traffic, pool)
        assert tuple(bin_of.tolist()) in set(sols)  # a feasible assignment
        for b in range(nb):
            mine = np.where(bin_of == b)[0]
            assert U[b] == len(mine) <= caps[b]
            assert sorted(slot_of[mine].tolist()) == list(range(len(mine)))
            assert A[b] == hot[mine].sum()
        if pool == 1:
            # hierarchy: every vertex placed in the best tier having traffic is at least
            # as hot as every vertex placed in a worse tier.
            best = min((tier[b] for b in range(nb) if traffic[b] > 0), default=None)
            if best is not None:
                hb = [hot[v] for v in range(nv) if tier[bin_of[v]] == best and traffic[bin_of[v]] > 0]
                hw = [hot[v] for v in range(nv) if tier[bin_of[v]] > best]
                if hb and hw:
                    assert min(hb) >= max(hw)


def test_ddak_closed_form_ratio(orc):
    # uniform hotness, T = (4, 1), equal capacity: priority ~ U^2 / T equalises at U0 = 2 U1.
    n = 3000
    _, _, _, U = orc.ddak(np.ones(n, np.uint64), [0, 0], [10**6, 10**6], [4, 1], 1)
    assert U.sum() == n
    assert abs(U[0] - 2 * U[1]) <= 2
    # with pooling the ratio holds to within a pool
    _, _, _, U = orc.ddak(np.ones(n, np.uint64), [0, 0], [10**6, 10**6], [4, 1], 100)
    assert abs(U[0] - 2 * U[1]) <= 200


def test_ddak_single_bin_and_pool_semantics(orc):
    hot = np.array([5, 9, 1, 9, 0, 3], np.uint64)
    bin_of, slot_of, A, U = orc.ddak(hot, [0], [6], [1], 1)
    # single bin fills in hotness order (desc, id asc): 1, 3, 0, 5, 2, 4
    order = [1, 3, 0, 5, 2, 4]
    assert [int(slot_of[v]) for v in order] == list(range(6))
    # pool >= capacity: the first chosen bin fills completely before the next takes anything
    bin_of, slot_of, A, U = orc.ddak(hot, [0, 0], [4, 4], [1, 1], 100)
    assert list(U) == [4, 2]
    assert set(np.where(bin_of == 0)[0].tolist()) == {1, 3, 0, 5}
    # infeasible: total capacity below n
    with pytest.raises(orc.OracleError) as e:
        orc.ddak(hot, [0], [5], [1], 1)
    assert e.value.status == orc.EINFEASIBLE
    # host tier only used once the GPU tier is full
    bin_of, _, _, U = orc.ddak(hot, [0, 1], [2, 10], [1, 100], 1)
    assert list(U) == [2, 4]
    assert set(np.where(bin_of == 0)[0].tolist()) == {1, 3}


# ------------------------------------------------------------------------------------------------
# Replication-aware DDAK (R25) and the replica term of the closed forms
# ------------------------------------------------------------------------------------------------
def hot_order(hot):
    """(hotness desc, id asc) — written out independently of the oracle's qsort comparator."""
    return sorted(range(len(hot)), key=lambda v: (-int(hot[v]), v))


@pytest.mark.parametrize("seed", range(10))
def test_ddak_replicate_exhaustive_small(orc, seed):
    rng = np.random.default_rng(100 + seed)
    nv = int(rng.integers(1, 8))
    nb = int(rng.integers(1, 4))
    hot = rng.integers(0, 20, nv)
    tier = sorted(rng.integers(0, 2, nb).tolist())
    caps = rng.integers(0, nv + 1, nb)
    traffic = rng.integers(0, 10, nb)
    gpu = [b for b in range(nb) if tier[b] == 0]
    for r in range(0, nv + 1):
        if any(caps[b] < r for b in gpu):
            with pytest.raises(orc.OracleError) as e:
                orc.ddak_replicate(hot, tier, caps, traffic, r, 1)
            assert e.value.status == orc.EINFEASIBLE
            continue
        red = [int(caps[b]) - (r if tier[b] == 0 else 0) for b in range(nb)]
        if sum(red) < nv - r:
            continue
        for pool in (1, 3):
            bin_of, slot_of, A, U, rep = orc.ddak_replicate(hot, tier, caps, traffic, r, pool)
            top = hot_order(hot)[:r]
            # replicas: exactly the r first vertices of the order, slot = position in the order
            assert sorted(np.where(bin_of == -2)[0].tolist()) == sorted(top)
            assert [int(slot_of[v]) for v in top] == list(range(r))
            assert rep == int(sum(int(hot[v]) for v in top))
            # the rest: a feasible assignment under the reduced capacities (brute force), slots after the
            # replica region in GPU bins, dense from 0 in the others
            rest = [v for v in range(nv) if v not in top]
            sols = set(brute_ddak_feasible([hot[v] for v in rest], red))
            assert tuple(int(bin_of[v]) for v in rest) in sols
            for b in range(nb):
                mine = [v for v in rest if bin_of[v] == b]
                base = r if tier[b] == 0 else 0
                assert U[b] == len(mine) <= red[b]
                assert sorted(int(slot_of[v]) for v in mine) == list(range(base, base + len(mine)))
                assert A[b] == sum(int(hot[v]) for v in mine)
            # r = 0 is plain DDAK
            if r == 0:
                b0, s0, A0, U0 = orc.ddak(hot, tier, caps, traffic, pool)
                assert np.array_equal(b0, bin_of) and np.array_equal(s0, slot_of)


def test_ddak_replicate_closed_form_split(orc):
    # uniform hotness, GPU bins with traffic (4, 1) and ample capacity: after the r replicas the
    # partition still splits 2:1 (the closed form of test_ddak_closed_form_ratio on n - r vertices)
    n, r = 3300, 300
    bin_of, slot_of, A, U, rep = orc.ddak_replicate(np.ones(n, np.uint64), [0, 0], [10**6, 10**6], [4, 1], r, 1)
    assert rep == r and U.sum() == n - r
    assert abs(U[0] - 2 * U[1]) <= 2
    # replicas are the r lowest ids (all hotness equal: id order)
    assert np.array_equal(np.where(bin_of == -2)[0], np.arange(r))


def test_plan_closed_forms_replica_hand_worked(orc):
    # the k = 2 example of test_plan_closed_forms_hand_worked plus d_rep = 50 bytes per GPU from replicas:
    # NVLink unchanged (19); HBM GPU0 = 2*100 + (200 + 2*50) = 500 -> ceil(500/9) = 56
    own = [0, 1, -1]
    d = [100, 60, 40]
    x = [[0, 0], [0, 0], [30, 10]]
    assert orc.plan_closed_forms(2, own, d, x, 7, 9, 50) == (19, 56)
    # everything replicated (d_b = 0, k = 8): no NVLink bytes, T_hbm = ceil(2 d_rep / hbm)
    assert orc.plan_closed_forms(8, list(range(8)), [0] * 8, [[0] * 8] * 8, 900, 6500, 1000) == (0, 1)
    assert orc.plan_closed_forms(8, list(range(8)), [0] * 8, [[0] * 8] * 8, 0, 6500, 6500) == (0, 2)


def test_ddak_zero_hotness_spreads_by_fill(orc):
    # R16 tie-break: vertices pre-sampling never saw (hotness 0) keep every bin's priority at 0; they go to
    # the less-filled bin, so equal bins split them evenly and unequal ones in proportion to capacity
    hot = np.zeros(1000, np.uint64)
    _, _, _, U = orc.ddak(hot, [1, 1], [600, 600], [5, 5], 1)
    assert list(U) == [500, 500]
    _, _, _, U = orc.ddak(hot, [1, 1], [300, 900], [5, 7], 1)
    assert abs(3 * U[0] - U[1]) <= 3 and U.sum() == 1000
    # hot vertices first by Eq. 2, the cold tail then balances the fill
    hot = np.zeros(1000, np.uint64)
    hot[:10] = 100
    bin_of, _, A, U = orc.ddak(hot, [1, 1], [600, 600], [5, 5], 1)
    assert abs(int(U[0]) - int(U[1])) <= 1 and A[0] > 0 and A[1] > 0


# ---------------------------------------------------------------------------------------------- quotas (R11)
def test_quota_hand_worked_cycle(orc):
    # s=0 -> host bin j=1 -> a=2 <-> b=3 (a cycle a->b->a carrying 3), b -> GPU 5, a -> GPU 6, GPUs -> t=7.
    # Worked by hand in the documented order (DESIGN R11): the walk j->a->b meets a again, cancels the
    # cycle (3 units off a->b and b->a), resumes at a: a->b->g5 (4 units), then a->g6 (6 units).
    links = [(0, 1, 0), (1, 2, 0), (2, 3, 0), (3, 2, 0), (3, 5, 0), (2, 6, 0), (5, 7, 0), (6, 7, 0)]
    flow = [10, 10, 7, 3, 4, 6, 4, 6]
    x = orc.quota(8, links, flow, 0, 7, [5, 6])
    assert x[1].tolist() == [4, 6]
    assert x.sum() == 10 and x[[0, 2, 3, 4, 5, 6, 7]].sum() == 0


def test_quota_hand_worked_shared_switch(orc):
    # two host bins j1=1, j2=2 into one switch x=3, switch -> GPU 4 (6 units) and GPU 5 (4 units).
    # Supply links in order: j1 takes the switch's first out-link (to GPU 4) for all 5 units; j2 then
    # finds 1 unit left on it and the other 4 on the link to GPU 5.
    links = [(0, 1, 0), (0, 2, 0), (1, 3, 0), (2, 3, 0), (3, 4, 0), (3, 5, 0), (4, 6, 0), (5, 6, 0)]
    flow = [5, 5, 5, 5, 6, 4, 6, 4]
    x = orc.quota(7, links, flow, 0, 6, [4, 5])
    assert x[1].tolist() == [5, 0] and x[2].tolist() == [1, 4]
    # GPU ranks follow the order of the gpu list, not node ids
    x = orc.quota(7, links, flow, 0, 6, [5, 4])
    assert x[1].tolist() == [0, 5] and x[2].tolist() == [4, 1]


def test_quota_rejects_unconserved_flow(orc):
    links = [(0, 1, 0), (1, 2, 0), (2, 3, 0)]
    with pytest.raises(orc.OracleError):
        orc.quota(4, links, [5, 5, 4], 0, 3, [2])  # GPU 2 can pass on only 4 of the 5 units


@pytest.mark.parametrize("S0,S1,p", [(800, 200, 10), (1000, 1000, 3), (5000, 0, 7), (300, 250, 2)])
def test_quota_two_socket_without_upi_closed_form(orc, S0, S1, p):
    # no UPI: every GPU is reachable from one socket's bin only, so x[j][h] is unique = the flow on h's sink
    # link for h on j's socket, 0 elsewhere; and T* = max(ceil(S0/4p), ceil(S1/4p)) (the two-socket closed form
    # with u = 0).
    s, h0, h1, c0, c1, t = 0, 1, 2, 3, 4, 5
    gpus = list(range(6, 14))
    links = [(s, h0, S0), (s, h1, S1), (h0, c0, INF), (h1, c1, INF)]
    sink_link = {}
    for i, g in enumerate(gpus):
        links.append((c0 if i < 4 else c1, g, p))
        sink_link[g] = len(links)
        links.append((g, t, INF))
    T, flow = _tb(orc, 14, links, {0, 1}, s, t)
    assert T == max(-(-S0 // (4 * p)), -(-S1 // (4 * p)))
    x = orc.quota(14, links, flow, s, t, gpus)
    for r, g in enumerate(gpus):
        j = h0 if r < 4 else h1
        assert x[j][r] == flow[sink_link[g]]
        assert x[h1 if j == h0 else h0][r] == 0
        assert x[j][r] <= p * T  # the port's capacity at T*
    assert x[h0].sum() == S0 and x[h1].sum() == S1


@pytest.mark.parametrize("seed", range(12))
def test_quota_invariants_random_flows(orc, seed):
    # flows built as sums of random s-j-...-g-t paths plus random cycles (so a decomposition exists), on
    # random graphs; the decomposition must return every supply unit to exactly one GPU reachable from j in
    # the flow's support, with row sums = supply flows and column sums = sink-link flows
    rng = np.random.default_rng(seed)
    n_host, n_mid, k = int(rng.integers(1, 4)), int(rng.integers(2, 6)), int(rng.integers(1, 5))
    s = 0
    host = list(range(1, 1 + n_host))
    mid = list(range(1 + n_host, 1 + n_host + n_mid))
    gpus = list(range(1 + n_host + n_mid, 1 + n_host + n_mid + k))
    t = 1 + n_host + n_mid + k
    N = t + 1
    links, idx = [], {}

    def link(u, v):
        if (u, v) not in idx or rng.random() < 0.2:  # sometimes a parallel link
            idx[(u, v)] = len(links)
            links.append((u, v, INF))
        return idx[(u, v)]

    for j in host:
        link(s, j)
    for g in gpus:
        link(g, t)
    flow = np.zeros(200, np.int64)
    for _ in range(int(rng.integers(1, 12))):  # paths
        j = host[int(rng.integers(0, n_host))]
        g = gpus[int(rng.integers(0, k))]
        hops = [j] + [mid[int(i)] for i in rng.choice(n_mid, int(rng.integers(0, n_mid + 1)), replace=False)] + [g]
        a = int(rng.integers(1, 20))
        flow[link(s, j)] += a
        for u, v in zip(hops, hops[1:]):
            flow[link(u, v)] += a
        flow[link(g, t)] += a
    for _ in range(int(rng.integers(0, 4))):  # cycles among interconnect nodes and GPUs
        cyc = [int(v) for v in rng.choice(mid + gpus, min(3, n_mid + k), replace=False)]
        a = int(rng.integers(1, 10))
        for u, v in zip(cyc, cyc[1:] + cyc[:1]):
            flow[link(u, v)] += a
    flow = flow[: len(links)]
    x = orc.quota(N, links, flow, s, t, gpus)
    assert (x >= 0).all()
    for v in range(N):
        sup = sum(int(f) for (u, w, _), f in zip(links, flow) if u == s and w == v)
        assert x[v].sum() == sup
    for r, g in enumerate(gpus):
        assert x[:, r].sum() == sum(int(f) for (u, w, _), f in zip(links, flow) if u == g and w == t)
    for j in host:
        reach, st = {j}, [j]
        while st:
            u = st.pop()
            for (a_, b_, _), f in zip(links, flow):
                if a_ == u and f > 0 and b_ != t and b_ not in reach:
                    reach.add(b_)
                    st.append(b_)
        for r, g in enumerate(gpus):
            if x[j][r] > 0:
                assert g in reach


# ---------------------------------------------------------------------------------------------- hash baseline (R24)
def _splitmix64_out(state):
    z = (state + 0x9E3779B97F4A7C15) & ((1 << 64) - 1)
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & ((1 << 64) - 1)
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & ((1 << 64) - 1)
    return z ^ (z >> 31)


def test_hash_place_known_answer(orc):
    # SplitMix64 (Steele, Lea, Flood 2014) seeded with 0 first outputs 0xE220A8397B1DCDAF, and with state
    # 0x9E3779B97F4A7C15 (its second step) 0x6E789E6AA1B965F4: the oracle's vertex-0 bin must be the first
    # value mod n_bins when no bin fills
    for nb in (3, 7, 64):
        b, sl, used = orc.hash_place(1, [10] * nb)
        assert b[0] == 0xE220A8397B1DCDAF % nb and sl[0] == 0
    assert _splitmix64_out(0) == 0xE220A8397B1DCDAF and _splitmix64_out(0x9E3779B97F4A7C15) == 0x6E789E6AA1B965F4


@pytest.mark.parametrize("seed", range(10))
def test_hash_place_properties(orc, seed):
    rng = np.random.default_rng(seed)
    nb = int(rng.integers(1, 6))
    n = int(rng.integers(0, 40))
    caps = [int(c) for c in rng.integers(0, 15, nb)]
    if sum(caps) < n:
        with pytest.raises(orc.OracleError) as e:
            orc.hash_place(n, caps)
        assert e.value.status == orc.EINFEASIBLE
        caps[0] += n - sum(caps)
    b, sl, used = orc.hash_place(n, caps)
    for q in range(nb):
        mine = [v for v in range(n) if b[v] == q]
        assert len(mine) == used[q] <= caps[q]
        assert [int(sl[v]) for v in mine] == list(range(len(mine)))  # slots in id order, contiguous
    # a vertex leaves its hash bin only if that bin was already full when its turn came, and then lands in
    # the first bin after it (cyclically) that still had room
    fill = [0] * nb
    for v in range(n):
        h = _splitmix64_out(v) % nb
        if fill[h] < caps[h]:
            assert b[v] == h
        else:
            q = h
            while fill[q] >= caps[q]:
                q = (q + 1) % nb
            assert b[v] == q
        fill[b[v]] += 1


def test_hash_place_uniform_when_roomy(orc):
    # ample capacity: the bin counts of 2^16 ids follow the hash's uniformity (chi-square, 7 dof, p ~ 1e-4)
    n, nb = 1 << 16, 8
    b, _, used = orc.hash_place(n, [n] * nb)
    exp = n / nb
    chi2 = sum((u - exp) ** 2 / exp for u in used)
    assert chi2 < 30
