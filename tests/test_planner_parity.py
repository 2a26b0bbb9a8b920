"""Product host planner (libmoment.so, C++) vs the oracle (CPU, no GPU needed).

P1 topology validation/augmentation, P3 Dinic vs Edmonds-Karp (value + optimality certificate of the
product's own flow), P4 DDAK bit-exact vs the oracle, P5 time bisection (T_ingest vs the oracle's
bisection on the same ingest graph), quota validity and the closed-form NVLink/HBM times recomputed by
the oracle from the product's quotas. Also: every symbol include/moment.h declares is exported.
"""
import os
import re

import numpy as np
import pytest

import paper_conf_sc_shi0s0x0w25_b200 as M

from test_oracle_planner import INF, brute_min_cut, random_links

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "moment.h")).read()
    declared = set(re.findall(r"\b(moment_[a-z_]+)\s*\(", hdr))
    declared -= {"moment_"}
    L = M.lib()
    missing = [s for s in sorted(declared) if not hasattr(L, s)]
    assert not missing, missing
    assert set(M.EXPORTED) == declared
    assert L.moment_version() >= 1


def test_step_batch_argument_checks_on_host():
    """moment_step_batch validates its arrays on the host before touching CUDA: n = 0 is a no-op, null arrays
    with n > 0 are EINVAL (runs without a GPU)."""
    L = M.lib()
    assert L.moment_step_batch(0, None, None, None, 0, None, None, None, None, None, None) == M.OK
    st = L.moment_step_batch(2, None, None, None, 1024, None, None, None, None, None, None)
    assert st == M.EINVAL and b"null" in L.moment_last_error()


def flow_certificate(n, links, s, t, value, flow):
    bal = [0] * n
    for (u, v, c), f in zip(links, flow):
        assert 0 <= f and (c == INF or f <= c)
        bal[u] -= int(f)
        bal[v] += int(f)
    for x in range(n):
        if x not in (s, t):
            assert bal[x] == 0
    assert bal[t] == value
    # min-cut certificate: S = residual-reachable from s; cut capacity == value
    adj = {}
    for (u, v, c), f in zip(links, flow):
        if c == INF or f < c:
            adj.setdefault(u, []).append(v)
        if f > 0:
            adj.setdefault(v, []).append(u)
    S = {s}
    st = [s]
    while st:
        u = st.pop()
        for w in adj.get(u, []):
            if w not in S:
                S.add(w)
                st.append(w)
    assert t not in S
    cut = sum(c for (u, v, c) in links if u in S and v not in S)
    assert cut == value


def layered_topology(rng, n_storage, n_inter, n_compute, n_links):
    """Random valid topology: storage -> interconnect -> ... -> compute."""
    nodes = []
    for i in range(n_storage):
        nodes.append((M.NODE_STORAGE, int(rng.choice([M.TIER_GPU_HBM, M.TIER_HOST_DRAM])), i % max(1, n_compute)))
    for i in range(n_inter):
        nodes.append((M.NODE_INTERCONNECT, M.TIER_NONE, -1))
    for i in range(n_compute):
        nodes.append((M.NODE_COMPUTE, M.TIER_NONE, i))
    S = list(range(n_storage))
    I = list(range(n_storage, n_storage + n_inter))
    Cp = list(range(n_storage + n_inter, n_storage + n_inter + n_compute))
    links = []
    for _ in range(n_links):
        kind = rng.integers(0, 4)
        if kind == 0 and I:
            u, v = int(rng.choice(S)), int(rng.choice(I))
        elif kind == 1 and len(I) > 1:
            u, v = [int(x) for x in rng.choice(I, 2, replace=False)]
        elif kind == 2 and I:
            u, v = int(rng.choice(I)), int(rng.choice(Cp))
        else:
            u, v = int(rng.choice(S)), int(rng.choice(Cp))
        r = rng.random()
        cap = 0 if r < 0.05 else int(rng.integers(1, 100))
        links.append((u, v, cap))
    return nodes, links


@pytest.mark.parametrize("seed", range(30))
def test_maxflow_dinic_vs_oracle(orc, seed):
    rng = np.random.default_rng(seed)
    nodes, links = layered_topology(rng, int(rng.integers(1, 5)), int(rng.integers(0, 6)), int(rng.integers(1, 4)),
                                    int(rng.integers(1, 25)))
    topo = M.topology(nodes, links)
    allnodes, alllinks, s, t = topo.export()
    val, flow = topo.maxflow()
    oval, _ = orc.maxflow(len(allnodes), alllinks, s, t)
    assert val == oval
    flow_certificate(len(allnodes), alllinks, s, t, val, flow)
    if len(allnodes) <= 14:
        assert val == brute_min_cut(len(allnodes), alllinks, s, t)


def test_topology_augmentation_and_errors():
    nodes = [(M.NODE_STORAGE, M.TIER_HOST_DRAM, 0), (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0),
             (M.NODE_COMPUTE, 0, 1)]
    links = [(0, 1, 30), (0, 1, 20), (1, 2, 25), (1, 3, 25)]
    topo = M.topology(nodes, links)
    n, m, s, t = topo.info()
    assert (n, m, s, t) == (6, 7, 4, 5)
    _, L, _, _ = topo.export()
    assert L[4] == (4, 0, 50)  # c(s, v_s) = sum of the storage node's out-capacities (R8)
    assert L[5] == (2, 5, INF) and L[6] == (3, 5, INF)
    assert topo.maxflow()[0] == 50
    bad = [
        ([(M.NODE_COMPUTE, 0, 0), (M.NODE_STORAGE, M.TIER_GPU_HBM, 0)], [(0, 1, 5)]),  # wrong direction
        ([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0)], [(0, 0, 5)]),  # self loop
        ([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_COMPUTE, 0, 0)], [(0, 1, -1)]),  # negative
        ([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_COMPUTE, 0, 0)], [(0, 7, 1)]),  # out of range
        ([(M.NODE_STORAGE, 0, 0)], []),  # storage without tier
        ([(M.NODE_SOURCE, 0, -1), (M.NODE_SOURCE, 0, -1)], []),  # two sources
    ]
    for nd, lk in bad:
        with pytest.raises(M.MomentError) as e:
            M.topology(nd, lk)
        assert e.value.status == M.EINVAL
    # unbounded: INF path from s to t
    with pytest.raises(M.MomentError):
        M.topology([(M.NODE_STORAGE, M.TIER_HOST_DRAM, 0), (M.NODE_COMPUTE, 0, 0)], [(0, 1, INF)]).maxflow()


@pytest.mark.parametrize("seed", range(25))
def test_ddak_bit_exact_vs_oracle(orc, seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 3000))
    nb = int(rng.integers(1, 7))
    hot = (rng.pareto(1.2, n) * 10).astype(np.uint64)
    if seed % 3 == 0:
        hot[:] = rng.integers(0, 3, n)  # many ties
    tier = np.array(sorted(rng.choice([1, 2, 3], nb)), np.int32)
    caps = rng.integers(0, n, nb).astype(np.int64)
    if caps.sum() < n:
        caps[-1] += n - caps.sum()
    traffic = rng.integers(0, 1000, nb).astype(np.int64)
    if seed % 4 == 1:
        traffic[rng.integers(0, nb)] = 0
    for pool in (1, 7, 100):
        b, s, A, U, T = M.place(None, hot, caps, bin_tier=tier, bin_traffic=traffic, pool=pool)
        ob, os_, oA, oU = orc.ddak(hot, tier - 1, caps, traffic, pool)
        assert np.array_equal(b, ob) and np.array_equal(s, os_)
        assert np.array_equal(A, oA) and np.array_equal(U, oU) and np.array_equal(T, traffic)


def test_ddak_large_values_exact(orc):
    # priorities whose cross products need more than 128 bits
    n = 500
    hot = np.full(n, 2**40, np.uint64)
    hot[::3] = 2**40 + 1
    caps = np.array([2**35, 2**35 + 3, 2**34], np.int64)
    traffic = np.array([2**50, 2**50 - 1, 2**49 + 7], np.int64)
    tier = np.array([1, 1, 1], np.int32)
    b, s, *_ = M.place(None, hot, caps, bin_tier=tier, bin_traffic=traffic, pool=3)
    ob, os_, *_ = orc.ddak(hot, tier - 1, caps, traffic, 3)
    assert np.array_equal(b, ob) and np.array_equal(s, os_)


def test_ddak_traffic_from_rate_maxflow(orc):
    # bins = storage nodes; traffic = f(s, b) of the product's rate max-flow
    nodes = [(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 0),
             (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0)]
    links = [(0, 3, 600), (1, 2, 50), (2, 3, 40)]
    topo = M.topology(nodes, links)
    hot = np.arange(100, dtype=np.uint64)
    b, s, A, U, T = M.place(topo, hot, [30, 100])
    assert list(T) == [600, 40]
    assert U[0] == 30 and set(np.where(b == 0)[0]) == set(range(70, 100))  # hottest 30 in HBM
    ob, os_, _, _ = orc.ddak(hot, [0, 1], [30, 100], T, 100)
    assert np.array_equal(b, ob) and np.array_equal(s, os_)


def test_place_pack_and_errors():
    packed = M.place_pack([0, 3, 63], [0, 5, 2**40 - 1])
    assert list(packed) == [0, (3 << 40) | 5, (63 << 40) | (2**40 - 1)]
    with pytest.raises(M.MomentError):
        M.place_pack([64], [0])
    with pytest.raises(M.MomentError) as e:
        M.place(None, [1, 2, 3], [1], bin_tier=[1], bin_traffic=[1])
    assert e.value.status == M.EINFEASIBLE


def two_socket_box(k=8, port=55, upi=40, hbm=6000, nv=770, host_per_socket=True):
    """A B200-like box: 2 NUMA host bins, k GPUs (PCIe port cap each), HBM bin per GPU."""
    nodes, links = [], []
    host = [len(nodes), len(nodes) + 1]
    nodes += [(M.NODE_STORAGE, M.TIER_HOST_DRAM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 1)]
    cpu = [len(nodes), len(nodes) + 1]
    nodes += [(M.NODE_INTERCONNECT, 0, -1)] * 2
    hbm_nodes, gpu_nodes = [], []
    for g in range(k):
        hbm_nodes.append(len(nodes))
        nodes.append((M.NODE_STORAGE, M.TIER_GPU_HBM, g))
    for g in range(k):
        gpu_nodes.append(len(nodes))
        nodes.append((M.NODE_COMPUTE, 0, g))
    links += [(host[0], cpu[0], 400), (host[1], cpu[1], 400), (cpu[0], cpu[1], upi), (cpu[1], cpu[0], upi)]
    for g in range(k):
        links.append((cpu[0] if g < k // 2 else cpu[1], gpu_nodes[g], port))
        links.append((hbm_nodes[g], gpu_nodes[g], hbm))
    return nodes, links, host, hbm_nodes, gpu_nodes


@pytest.mark.parametrize("k,d_host0,d_host1,d_hbm", [(8, 4000, 1000, 500), (4, 100, 9000, 0), (2, 0, 0, 300),
                                                     (8, 12345, 777, 4096), (1, 500, 500, 500)])
def test_plan_vs_oracle(orc, k, d_host0, d_host1, d_hbm):
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=8)
    topo = M.topology(nodes, links)
    N, Lc, s, t = topo.info()
    allnodes, alllinks, _, _ = topo.export()
    demand = np.zeros(N, np.int64)
    demand[host[0]], demand[host[1]] = d_host0, d_host1
    for g in range(k):
        demand[hbm_nodes[g]] = d_hbm
    active = gpu_nodes[:k]
    p = M.plan(topo, active, demand, 770, 6000).info()
    # oracle: T_ingest on the same ingest graph (supplies k*d on host bins, none on HBM, active sinks only)
    il, sup = [], []
    for (u, v, c) in alllinks:
        if u == s:
            tier = allnodes[v][1]
            il.append((u, v, 0 if tier == M.TIER_GPU_HBM else k * demand[v]))
            sup.append(1)
        elif v == t:
            il.append((u, v, INF if u in active else 0))
            sup.append(0)
        else:
            il.append((u, v, c))
            sup.append(0)
    tin, _ = orc.time_bisect(N, il, sup, s, t)
    assert p["t_ingest"] == tin
    # the product's ingest flow is a max flow of the graph at T_ingest (certificate)
    scaled = [(u, v, c if (sp or c == INF) else c * tin) for (u, v, c), sp in zip(il, sup)]
    flow_certificate(N, scaled, s, t, k * (d_host0 + d_host1), p["link_flow"])
    # quotas: row sums = supplies, only host rows, only active GPU columns
    x = p["quota"]
    for v in range(N):
        if v in host:
            assert x[v].sum() == k * demand[v]
        else:
            assert x[v].sum() == 0
    # closed forms recomputed by the oracle from the product's quotas
    bins = [v for v in range(N) if allnodes[v][0] == M.NODE_STORAGE]
    owner = [allnodes[v][2] if allnodes[v][1] == M.TIER_GPU_HBM else -1 for v in bins]
    owner = [o if o < k else -1 for o in owner]
    d = [demand[v] if not (allnodes[v][1] == M.TIER_GPU_HBM and allnodes[v][2] >= k) else 0 for v in bins]
    xb = [x[v] for v in bins]
    tn, th = orc.plan_closed_forms(k, owner, d, xb, 770, 6000)
    assert (p["t_nvlink"], p["t_hbm"]) == (tn, th)
    assert p["t_star"] == max(tin, tn, th)


def test_plan_needs_nvlink_for_peer_traffic(orc):
    # peer HBM reads and relays need the NVLink edges; without them the plan is infeasible
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=4)
    topo = M.topology(nodes, links)
    N = topo.info()[0]
    demand = np.zeros(N, np.int64)
    demand[host[0]] = 10000
    for g in range(4):
        demand[hbm_nodes[g]] = 1000
    with_nv = M.plan(topo, gpu_nodes[:4], demand, 770, 6000).info()["t_star"]
    with pytest.raises(M.MomentError) as e:
        M.plan(topo, gpu_nodes[:4], demand, 0, 6000)  # peer traffic exists but no NVLink
    assert e.value.status == M.EINFEASIBLE
    demand2 = demand.copy()
    for g in range(4):
        demand2[hbm_nodes[g]] = 0
    # less demand never needs more time (monotone plan)
    assert M.plan(topo, gpu_nodes[:4], demand2, 770, 6000).info()["t_star"] <= with_nv


def test_plan_infeasible_and_zero():
    nodes = [(M.NODE_STORAGE, M.TIER_HOST_DRAM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 1),
             (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0)]
    links = [(0, 2, 10), (2, 3, 10)]  # node 1 is unreachable
    topo = M.topology(nodes, links)
    N = topo.info()[0]
    d = np.zeros(N, np.int64)
    d[1] = 5
    with pytest.raises(M.MomentError) as e:
        M.plan(topo, [3], d, 0, 100)
    assert e.value.status == M.EINFEASIBLE
    d[:] = 0
    info = M.plan(topo, [3], d, 0, 100).info()
    assert info["t_ingest"] == 0 and info["t_star"] == 0


# ------------------------------------------------------------------------------------------------
# Replication-aware placement and search (R25)
# ------------------------------------------------------------------------------------------------
@pytest.mark.parametrize("seed", range(16))
def test_ddak_replicate_bit_exact_vs_oracle(orc, seed):
    rng = np.random.default_rng(1000 + seed)
    n = int(rng.integers(1, 4000))
    n_gpu = int(rng.integers(1, 5))
    n_host = int(rng.integers(0, 3))
    nb = n_gpu + n_host
    hot = (rng.pareto(1.1, n) * 10).astype(np.uint64)
    if seed % 3 == 0:
        hot[:] = rng.integers(0, 3, n)  # many ties
    tier = np.array([1] * n_gpu + [2] * n_host, np.int32)
    caps = rng.integers(n // 8, n // 2 + 2, nb).astype(np.int64)
    r_max = int(caps[:n_gpu].min())
    for r in sorted({0, 1, r_max // 2, r_max}):
        need = n - r - int((caps - np.where(tier == 1, r, 0)).sum())
        caps_r = caps.copy()
        if need > 0:
            caps_r[-1] += need
        traffic = rng.integers(1, 1000, nb).astype(np.int64)
        for pool in (1, 100):
            b, s, A, U, T, rep = M.place(None, hot, caps_r, bin_tier=tier, bin_traffic=traffic, pool=pool,
                                         replicate_rows=r, return_replica_access=True)
            ob, os_, oA, oU, orep = orc.ddak_replicate(hot, tier - 1, caps_r, traffic, r, pool)
            assert np.array_equal(b, ob) and np.array_equal(s, os_), (r, pool)
            assert np.array_equal(A, oA) and np.array_equal(U, oU) and rep == orep
            # one rank's device map: replicas point at that rank's own bin
            g = int(rng.integers(0, n_gpu))
            packed = M.place_pack_rank(b, s, g)
            want = np.where(b == M.BIN_REPLICA, g, b).astype(np.uint64) << np.uint64(40) | s.astype(np.uint64)
            assert np.array_equal(packed, want)
            if r > 0:
                with pytest.raises(M.MomentError):
                    M.place_pack(b, s)  # a replica has no single bin


def test_ddak_replicate_errors():
    hot = np.arange(10, dtype=np.uint64)
    with pytest.raises(M.MomentError) as e:  # r above a GPU bin's capacity
        M.place(None, hot, [4, 8, 20], bin_tier=[1, 1, 2], bin_traffic=[1, 1, 1], replicate_rows=5)
    assert e.value.status == M.EINFEASIBLE
    with pytest.raises(M.MomentError) as e:  # hash placement has no replicas
        M.place(None, hot, [10, 10], bin_tier=[1, 2], bin_traffic=[1, 1], replicate_rows=1, mode=M.PLACE_HASH)
    assert e.value.status == M.EINVAL
    with pytest.raises(M.MomentError):
        M.place_pack_rank([M.BIN_REPLICA], [0], 64)
    # r = n with room: everything replicated, nothing partitioned
    b, s, A, U, T = M.place(None, hot, [10, 10, 0], bin_tier=[1, 1, 2], bin_traffic=[1, 1, 1], replicate_rows=10)
    assert (b == M.BIN_REPLICA).all() and list(U) == [0, 0, 0]
    assert list(s[np.argsort(-hot.astype(np.int64), kind="stable")]) == list(range(10))


@pytest.mark.parametrize("k,d_host0,d_hbm,d_rep", [(8, 4000, 500, 700), (2, 0, 300, 10**6), (1, 500, 500, 1)])
def test_plan_replica_demand_vs_oracle(orc, k, d_host0, d_hbm, d_rep):
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=8)
    topo = M.topology(nodes, links)
    N, _, s, t = topo.info()
    allnodes, _, _, _ = topo.export()
    demand = np.zeros(N, np.int64)
    demand[host[0]] = d_host0
    for g in range(k):
        demand[hbm_nodes[g]] = d_hbm
    p0 = M.plan(topo, gpu_nodes[:k], demand, 770, 6000).info()
    p = M.plan(topo, gpu_nodes[:k], demand, 770, 6000, replica_demand=d_rep).info()
    assert p["t_ingest"] == p0["t_ingest"] and p["t_nvlink"] == p0["t_nvlink"]  # replicas: HBM only
    bins = [v for v in range(N) if allnodes[v][0] == M.NODE_STORAGE]
    owner = [allnodes[v][2] if allnodes[v][1] == M.TIER_GPU_HBM and allnodes[v][2] < k else -1 for v in bins]
    d = [demand[v] for v in bins]
    tn, th = orc.plan_closed_forms(k, owner, d, [p["quota"][v] for v in bins], 770, 6000, d_rep)
    assert (p["t_nvlink"], p["t_hbm"]) == (tn, th)
    assert p["t_star"] == max(p["t_ingest"], tn, th)
    with pytest.raises(M.MomentError):
        M.plan(topo, gpu_nodes[:k], demand, 770, 6000, replica_demand=-1)


def _search_setup(k, n, cap_gpu, host_cap, hot, port=55, nv=900, hbm=6500):
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=k, port=port, nv=nv, hbm=hbm)
    topo = M.topology(nodes, links)
    bin_node = hbm_nodes + host
    tier = [M.TIER_GPU_HBM] * k + [M.TIER_HOST_DRAM] * 2
    caps = [cap_gpu] * k + [host_cap, host_cap]
    traffic = [hbm] * k + [10, 10]
    return topo, bin_node, tier, caps, traffic, gpu_nodes, host, hbm_nodes


@pytest.mark.parametrize("seed", range(4))
def test_replicate_search_vs_oracle_composition(orc, seed):
    """Every candidate's T* = the plan (checked against the oracle above) of the demands that the ORACLE's
    replicated placement implies: d_b = floor(R A_b / batches), d_rep = floor(R A_rep / batches)."""
    rng = np.random.default_rng(seed)
    k, n, R, batches = [2, 4, 8, 8][seed], 5000, 512, 64
    hot = (rng.pareto(0.8, n) * 5).astype(np.uint64)
    cap_gpu = [n // k, n // (2 * k), n, n // 3][seed]
    topo, bin_node, tier, caps, traffic, gpu_nodes, host, hbm_nodes = _search_setup(k, n, cap_gpu, n, hot)
    cand = [0, cap_gpu // 4, cap_gpu // 2, cap_gpu, cap_gpu + 1]
    held = (rng.pareto(0.8, n) * 3).astype(np.uint64)  # held-out batches' counts (demand estimate)
    for dem, dem_batches in ((None, 0), (held, 32)):
        ts, best = M.replicate_search(topo, hot, caps, cand, gpu_node=gpu_nodes, nvlink_cap=900, hbm_cap=6500,
                                      row_bytes=R, hot_batches=batches, bin_node=bin_node, bin_tier=tier,
                                      bin_traffic=traffic, demand_counts=dem, demand_batches=dem_batches)
        cnt, nb_ = (hot, batches) if dem is None else (dem, dem_batches)
        N = topo.info()[0]
        for r, t_got in zip(cand, ts):
            if r > cap_gpu:
                assert t_got == -1
                continue
            b, s, A, U, rep = orc.ddak_replicate(hot, np.array(tier) - 1, caps, traffic, r, 100)
            demand = np.zeros(N, np.int64)
            for i, v in enumerate(bin_node):
                demand[v] += int(cnt[b == i].sum()) * R // nb_
            rep_d = int(cnt[b == -2].sum()) * R // nb_
            want = M.plan(topo, gpu_nodes, demand, 900, 6500, replica_demand=rep_d).info()["t_star"]
            assert t_got == want, r
        feas = [i for i, x in enumerate(ts) if x >= 0]
        assert best == min(feas, key=lambda i: (ts[i], i))


def test_replicate_search_closed_forms():
    """Uniform hotness, all rows fit in every GPU (no host rows): replicating everything removes the
    NVLink term; with k = 1 replication changes nothing; with tight GPU capacity, replication pushes rows
    to the host tier and T* grows."""
    n, R, batches, k = 8000, 512, 1, 8
    hot = np.ones(n, np.uint64)
    topo, bin_node, tier, caps, traffic, gpu_nodes, host, hbm_nodes = _search_setup(k, n, n, n, hot, nv=900,
                                                                                      hbm=6500)
    cand = [0, n // 4, n // 2, n]
    ts, best = M.replicate_search(topo, hot, caps, cand, gpu_node=gpu_nodes, nvlink_cap=900, hbm_cap=6500,
                                  row_bytes=R, hot_batches=batches, bin_node=bin_node, bin_tier=tier,
                                  bin_traffic=traffic)
    # per GPU per batch: D = n R bytes. r = 0: DDAK splits evenly (equal traffic), each GPU reads
    # (k-1)/k D over NVLink in and serves the same out: T_nvlink = ceil(7/8 D / 900); r = n: T = ceil(2D/6500)
    D = n * R
    assert ts[0] == max(-(-(D * 7 // 8) // 900), -(-(D + k * D // 8) // 6500))
    assert ts[-1] == -(-(2 * D) // 6500)
    assert list(ts) == sorted(ts, reverse=True) and best == 3
    # tight GPU capacity (n/8 per GPU = the whole table exactly once): every replica forces n/8 rows
    # (spread over 8 bins) to host DRAM over 55 bytes/us ports
    topo, bin_node, tier, caps, traffic, gpu_nodes, host, hbm_nodes = _search_setup(k, n, n // k, n, hot)
    ts, best = M.replicate_search(topo, hot, caps, [0, 100, 500], gpu_node=gpu_nodes, nvlink_cap=900,
                                  hbm_cap=6500, row_bytes=R, hot_batches=batches, bin_node=bin_node, bin_tier=tier,
                                  bin_traffic=traffic)
    assert best == 0 and ts[0] < ts[1] < ts[2]


def test_standalone_traffic_vs_oracle(orc):
    """R7 canonical Bin_traffic: each bin's own max-flow to t (every other supply cut) = the oracle's
    Edmonds-Karp on the same graph; on the symmetric box both host bins get equal traffic, where the rate
    max-flow may give one of them none."""
    for act in ([0], [0, 4], [0, 1, 4, 5], list(range(8))):
        box = M.boxes.hgx_b200(8, active=act)
        topo = box.topology()
        N, L, s, t = topo.info()
        nodes, links, _, _ = topo.export()
        bins = [box.hbm_bin[g] for g in act] + box.host_bin
        hot = np.arange(1000, dtype=np.uint64)
        *_, T = M.place(topo, hot, [10] * len(act) + [1000, 1000], bin_node=bins,
                        traffic_mode=M.TRAFFIC_STANDALONE)
        for i, b in enumerate(bins):
            cut = [(u, v, 0 if (u == s and v != b) else c) for (u, v, c) in links]
            assert T[i] == orc.maxflow(N, cut, s, t)[0]
        if len(act) > 1:
            assert T[-1] == T[-2]
    with pytest.raises(M.MomentError):
        M.place(topo, hot, [10] * 8 + [1000, 1000], bin_node=bins, traffic_mode=7)


def test_signal_barrier_argument_errors():
    # host-side validation happens before anything is enqueued (no GPU needed)
    import ctypes as C
    L = M.lib()
    flags = np.zeros(2, np.uint64)
    peers = (C.c_void_p * 2)(None, flags.ctypes.data)
    for world, rank, epoch, timeout in [(0, 0, 1, 10), (2, 2, 1, 10), (65, 0, 1, 10), (2, 0, 0, 10), (2, 0, 1, 0)]:
        st = L.moment_signal_barrier(world, rank, peers, flags.ctypes.data, epoch, timeout, None, None)
        assert st == M.EINVAL, (world, rank, epoch, timeout)
    # a null peer pointer for another rank
    st = L.moment_signal_barrier(2, 0, (C.c_void_p * 2)(None, None), flags.ctypes.data, 1, 10, None, None)
    assert st == M.EINVAL


# ---------------------------------------------------------------------------------------------- P5 quotas
def _quota_vs_oracle(orc, topo, active, demand, nvlink=770, hbm=6000):
    """moment_plan's x[j][h] == the oracle's decomposition (R11) of the product's own ingest flow, bit-exact;
    column sums == the active GPUs' sink-link flows; row sums == the host bins' supplies."""
    N, _, s, t = topo.info()
    allnodes, alllinks, _, _ = topo.export()
    p = M.plan(topo, active, demand, nvlink, hbm).info()
    x = orc.quota(N, alllinks, p["link_flow"], s, t, active)
    assert np.array_equal(p["quota"], x)
    for r, g in enumerate(active):
        sink = sum(int(f) for (u, v, _), f in zip(alllinks, p["link_flow"]) if u == g and v == t)
        assert p["quota"][:, r].sum() == sink
    k = len(active)
    for v in range(N):
        want = k * demand[v] if allnodes[v][0] == M.NODE_STORAGE and allnodes[v][1] != M.TIER_GPU_HBM else 0
        assert p["quota"][v].sum() == want
    return p


@pytest.mark.parametrize("k,d_host0,d_host1,d_hbm", [(8, 4000, 1000, 500), (4, 100, 9000, 0), (2, 0, 0, 300),
                                                     (8, 12345, 777, 4096), (1, 500, 500, 500), (3, 7, 11, 0)])
def test_plan_quota_bit_exact_two_socket(orc, k, d_host0, d_host1, d_hbm):
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=8)
    topo = M.topology(nodes, links)
    N = topo.info()[0]
    demand = np.zeros(N, np.int64)
    demand[host[0]], demand[host[1]] = d_host0, d_host1
    for g in range(k):
        demand[hbm_nodes[g]] = d_hbm
    _quota_vs_oracle(orc, topo, gpu_nodes[:k], demand)


@pytest.mark.parametrize("k,gps,uplink", [(8, 1, None), (8, 2, None), (4, 2, 30.0), (6, 1, None), (8, 4, 80.0)])
def test_plan_quota_bit_exact_hgx(orc, k, gps, uplink):
    from paper_conf_sc_shi0s0x0w25_b200 import boxes

    act = boxes.spread_gpus(k, gpus_per_switch=gps)
    box = boxes.hgx_b200(8, gpus_per_switch=gps, uplink_gbs=uplink, active=act)
    topo = M.topology(box.nodes, box.links)
    N = topo.info()[0]
    rng = np.random.default_rng(k * 10 + gps)
    demand = np.zeros(N, np.int64)
    for j in box.host_bin:
        demand[j] = int(rng.integers(10**5, 10**8))
    for g in act:
        demand[box.hbm_bin[g]] = int(rng.integers(0, 10**7))
    _quota_vs_oracle(orc, topo, [box.gpu[g] for g in act], demand)


@pytest.mark.parametrize("seed", range(15))
def test_plan_quota_bit_exact_random_topologies(orc, seed):
    # random interconnect between 1-3 host bins and 1-4 GPUs (antiparallel interconnect links make cycles
    # in the flow possible), random capacities and demands
    rng = np.random.default_rng(100 + seed)
    n_host, n_mid, k = int(rng.integers(1, 4)), int(rng.integers(1, 5)), int(rng.integers(1, 5))
    nodes = [(M.NODE_STORAGE, M.TIER_HOST_DRAM, j) for j in range(n_host)]
    mid = list(range(len(nodes), len(nodes) + n_mid))
    nodes += [(M.NODE_INTERCONNECT, M.TIER_NONE, -1)] * n_mid
    gpus = list(range(len(nodes), len(nodes) + k))
    nodes += [(M.NODE_COMPUTE, M.TIER_NONE, g) for g in range(k)]
    links = []
    for j in range(n_host):
        for v in rng.choice(mid, int(rng.integers(1, n_mid + 1)), replace=False):
            links.append((j, int(v), int(rng.integers(1, 100))))
    for a in mid:  # interconnect <-> interconnect (antiparallel pairs) and interconnect -> GPU
        for b in mid + gpus:
            if a != b and rng.random() < 0.5:
                links.append((a, b, int(rng.integers(1, 60))))
    for m_ in mid:  # every interconnect node reaches some GPU
        links.append((m_, gpus[int(rng.integers(0, k))], int(rng.integers(1, 60))))
    topo = M.topology(nodes, links)
    N = topo.info()[0]
    demand = np.zeros(N, np.int64)
    for j in range(n_host):
        demand[j] = int(rng.integers(0, 5000))
    act = sorted(int(g) for g in rng.choice(gpus, int(rng.integers(1, k + 1)), replace=False))
    try:
        _quota_vs_oracle(orc, topo, act, demand, nvlink=100, hbm=1000)
    except M.MomentError as e:
        # a demanded host bin that reaches no active GPU: the oracle's bisection must agree it is infeasible
        assert e.status == M.EINFEASIBLE and "unreachable" in str(e)
        _, alllinks, s, t = topo.export()
        il = [(u, v, k * 0 + (len(act) * demand[v] if u == s else (INF if u in act else 0) if v == t else c))
              for (u, v, c) in alllinks]
        with pytest.raises(orc.OracleError) as oe:
            orc.time_bisect(N, il, [1 if u == s else 0 for (u, _, _) in alllinks], s, t)
        assert oe.value.status == orc.EINFEASIBLE


# ---------------------------------------------------------------------------------------------- hash baseline
@pytest.mark.parametrize("seed", range(12))
def test_hash_place_bit_exact_vs_oracle(orc, seed):
    rng = np.random.default_rng(500 + seed)
    nb = int(rng.integers(1, 9))
    n = int(rng.integers(0, 3000))
    caps = rng.integers(0, max(2, 2 * n // nb + 2), nb)
    if caps.sum() < n:
        caps[int(rng.integers(0, nb))] += n - caps.sum()
    hot = rng.integers(0, 50, n).astype(np.uint64)
    b, sl, acc, used, _ = M.place(None, hot, caps, bin_tier=[1] * nb, bin_traffic=[1] * nb, mode=M.PLACE_HASH)
    ob, osl, oused = orc.hash_place(n, caps)
    assert np.array_equal(b, ob) and np.array_equal(sl, osl) and np.array_equal(used, oused)
    for q in range(nb):
        assert acc[q] == hot[b == q].sum()


def test_hash_place_infeasible():
    with pytest.raises(M.MomentError) as e:
        M.place(None, np.zeros(10, np.uint64), [3, 3], bin_tier=[1, 1], bin_traffic=[1, 1], mode=M.PLACE_HASH)
    assert e.value.status == M.EINFEASIBLE
