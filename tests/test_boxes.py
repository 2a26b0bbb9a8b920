"""The HGX B200 topology builder (P1, boxes.py) and the replication search on it (R25): rate max-flow closed
forms of the two-socket box, and the planner's k-scaling predictions in the cases that have closed forms."""
import numpy as np

import paper_conf_sc_shi0s0x0w25_b200 as M


def test_hgx_rate_maxflow_closed_forms():
    hbm = 6543.4
    # GPU ports straight off the root complexes: host ingest = min(DRAM of both sockets, 8 ports)
    b = M.boxes.hgx_b200(8, port_gbs=55.6, hbm_gbs=hbm, dram_gbs=250, upi_gbs=62)
    F, _ = b.topology().maxflow()
    assert F == 8 * 6543400 + min(2 * 250000, 8 * 55600)
    # 2 GPUs per PCIe switch with a one-port uplink: the 4 uplinks bound the host ingest
    b = M.boxes.hgx_b200(8, port_gbs=55.6, hbm_gbs=hbm, dram_gbs=250, upi_gbs=62, gpus_per_switch=2)
    F, _ = b.topology().maxflow()
    assert F == 8 * 6543400 + 4 * 55600
    # DRAM-bound sockets: a slow socket's rows cross UPI only up to its DRAM rate
    b = M.boxes.hgx_b200(8, port_gbs=55.6, hbm_gbs=hbm, dram_gbs=100, upi_gbs=62)
    assert b.topology().maxflow()[0] == 8 * 6543400 + 2 * 100000
    # two active GPUs on one socket: host ingest = 2 ports; the other socket's rows must cross UPI
    act = [0, 1]
    b = M.boxes.hgx_b200(8, active=act)
    assert [g for g in range(8) if b.gpu[g] is not None] == act
    F, _ = b.topology().maxflow()
    assert F == 2 * 6543400 + 2 * 55600


def test_spread_gpus_balanced():
    assert M.boxes.spread_gpus(2) == [0, 4]
    assert M.boxes.spread_gpus(4, gpus_per_switch=2) == [0, 2, 4, 6]  # one GPU per switch first
    assert M.boxes.spread_gpus(8) == list(range(8))
    for k in (1, 2, 4, 6, 8):
        assert len(set(M.boxes.spread_gpus(k))) == k


def _predict(k, n, hot, cap, R=512, batches=1, candidates=None):
    act = M.boxes.spread_gpus(k)
    box = M.boxes.hgx_b200(8, active=act)
    topo = box.topology()
    cand = candidates or [0, n // 2, n]
    ts, best = M.replicate_search(topo, hot, [cap] * k + [n, n], cand, gpu_node=[box.gpu[g] for g in act],
                                  nvlink_cap=900000, hbm_cap=6543400, row_bytes=R, hot_batches=batches,
                                  bin_node=[box.hbm_bin[g] for g in act] + box.host_bin)
    return ts, best


def test_replication_predicted_scaling():
    """Uniform hotness, table fits one GPU (the C3 case): without replicas each GPU reads (k-1)/k of its batch
    over NVLink, so T* grows with k; with every row replicated T* stays the k = 1 HBM time, i.e. predicted
    seeds/s = k x the single-GPU rate."""
    n, R = 4096, 65536
    hot = np.ones(n, np.uint64)
    D = n * R
    t1 = -(-(2 * D) // 6543400)
    for k in (1, 2, 4, 8):
        ts, best = _predict(k, n, hot, n, R)
        assert ts[-1] == t1  # r = n
        if k > 1:
            assert ts[0] >= -(-(D * (k - 1) // k) // 900000) > t1 and ts[best] == t1
        else:
            assert ts[0] == t1


def test_gpu_subset_classes_counts():
    from itertools import combinations
    # direct ports: a subset is determined up to symmetry by how many GPUs each socket gets
    assert M.boxes.gpu_subset_classes(2) == [[0, 1], [0, 4]]
    assert len(M.boxes.gpu_subset_classes(4)) == 3  # (4,0), (3,1), (2,2)
    # 2 GPUs per switch, k = 2: same switch / same socket other switch / other socket
    assert M.boxes.gpu_subset_classes(2, gpus_per_switch=2) == [[0, 1], [0, 2], [0, 4]]
    # brute force: every subset is equivalent to exactly one representative under the generated group
    def orbit_key(sub, gps):
        per = 4
        cnt = [[0] * (per // gps) for _ in range(2)]
        for g in sub:
            cnt[g // per][(g % per) // gps] += 1
        return tuple(sorted(tuple(sorted(c, reverse=True)) for c in cnt))
    for gps in (1, 2):
        for k in range(1, 9):
            reps = M.boxes.gpu_subset_classes(k, gpus_per_switch=gps)
            keys = {orbit_key(s, gps) for s in combinations(range(8), k)}
            assert len(reps) == len(keys) and {orbit_key(r, gps) for r in reps} == keys


def test_subset_choice_matters_with_shared_switches():
    """Host-bound placement, 2 GPUs per switch: two GPUs on one switch share one uplink, two on different
    switches have two — the plan's T_ingest halves (the PLX contention of P:L157-168)."""
    n, R = 4096, 4096
    hot = np.ones(n, np.uint64)
    out = {}
    for act in ([0, 1], [0, 2]):
        box = M.boxes.hgx_b200(8, gpus_per_switch=2, active=act)
        topo = box.topology()
        b, s, A, U, T = M.place(topo, hot, [0, 0, n, n], bin_node=[box.hbm_bin[g] for g in act] + box.host_bin)
        N = topo.info()[0]
        d = np.zeros(N, np.int64)
        for i, v in enumerate([box.hbm_bin[g] for g in act] + box.host_bin):
            d[v] += int(A[i]) * R
        out[tuple(act)] = M.plan(topo, [box.gpu[g] for g in act], d, 900000, 6543400).info()["t_ingest"]
    assert out[(0, 1)] >= 2 * out[(0, 2)] - 1


def test_upi_bytes_closed_form():
    # all host demand on socket 0's bin, 8 GPUs: the 4 socket-1 ports can only be fed across UPI, so at T*
    # = ceil(8 d / (4 p + u)) (ports p, UPI u, ample DRAM) the plan moves u T* (rounded to the flow) over UPI
    p, u, d = 50_000, 20_000, 3_000_000
    box = M.boxes.hgx_b200(8, port_gbs=p / 1000, upi_gbs=u / 1000, dram_gbs=10_000)
    topo = box.topology()
    N, _, s, t = topo.info()
    _, links, _, _ = topo.export()
    assert all(links[i][0] in box.rc and links[i][1] in box.rc for i in box.upi_links) and len(box.upi_links) == 2
    dem = np.zeros(N, np.int64)
    dem[box.host_bin[0]] = d
    plan = M.plan(topo, box.gpu, dem, 770_000, 6_500_000).info()
    T = plan["t_ingest"]
    assert T == -(-8 * d // (4 * p + u))
    upi = box.upi_bytes(plan["link_flow"])
    assert 8 * d - 4 * p * T <= upi <= u * T  # what the socket-0 ports cannot take crosses, within capacity
    # symmetric demand: no reason to cross sockets at all at T* = ceil(8 d / 8 p)
    dem[box.host_bin[1]] = d
    plan = M.plan(topo, box.gpu, dem, 770_000, 6_500_000).info()
    assert plan["t_ingest"] == -(-8 * d // (4 * p))
    assert box.upi_bytes(plan["link_flow"]) <= u * plan["t_ingest"]


def test_from_probe_provenance():
    one_gpu = {"gpus": 1, "port_gbs": 55.6, "port_remote_gbs": None, "port_concurrent_gbs": None,
               "hbm_gbs": 6500.0, "nvlink_gbs": None}
    kw, src = M.boxes.from_probe(one_gpu)
    assert kw["port_gbs"] == 55.6 and kw["hbm_gbs"] == 6500.0
    assert src["upi_gbs"] == "assumed" and src["dram_gbs"] == "assumed" and src["nvlink_value"] == 770.0
    eight = dict(one_gpu, gpus=8, port_remote_gbs=40.0, port_concurrent_gbs=[50.0] * 7 + [45.0], nvlink_gbs=760.0)
    kw, src = M.boxes.from_probe(eight)
    assert kw["port_gbs"] == 45.0 and kw["upi_gbs"] == 40.0 and src["nvlink_value"] == 760.0
    assert src["port_gbs"].startswith("measured")
    M.boxes.hgx_b200(8, **kw)  # builds
