"""N > 1 host-side paths with world_size 2-3 gloo process groups on CPU (no GPU needed).

* seed sharding: ranks' batches are disjoint slices of the training set;
* the planner is deterministic across ranks: topology, rate max-flow, DDAK placement and the
  time-bisection plan computed independently on every rank agree bit for bit;
* the relay exchange transport (exchange.alltoallv / exchange_counts): requests routed by the oracle's
  routing (R12) travel to their relay rank, are served from its copy of the host rows and come back to
  the right output positions — the same counts / words / rows protocol the GPU path runs.
"""
import numpy as np
import pytest
import torch
import torch.distributed as dist

from mp_util import run_world


def _shard_and_plan(rank, world):
    import paper_conf_sc_shi0s0x0w25_b200 as M
    import workloads as W
    from test_planner_parity import two_socket_box

    g = W.rmat_csr(1 << 12, 1 << 15, device="cpu")
    train = W.training_set(g, min_count=64 * world)
    batches = W.epoch_batches(train, 64, epoch=3, rank=rank, world=world)
    seeds = torch.cat(batches).tolist() if batches else []
    nodes, links, host, hbm_nodes, gpu_nodes = two_socket_box(k=4)
    topo = M.topology(nodes, links)
    N = topo.info()[0]
    demand = np.zeros(N, np.int64)
    demand[host[0]], demand[host[1]] = 7000, 3000
    for h in hbm_nodes[:4]:
        demand[h] = 1000
    info = M.plan(topo, gpu_nodes[:4], demand, 770, 6000).info()
    hot = np.random.default_rng(0).pareto(1.0, 5000).astype(np.uint64)
    bin_of, slot_of, *_ = M.place(topo, hot, [2000, 2000] + [500] * 4)  # storage nodes: 2 host, 4 HBM
    out = {"seeds": seeds, "train": train.tolist(), "t_star": info["t_star"], "quota": info["quota"].tolist(),
           "flow": topo.maxflow()[0], "bin_of": bin_of.tolist(), "slot_of": slot_of.tolist()}
    gathered = [None] * world
    dist.all_gather_object(gathered, {k: out[k] for k in ("t_star", "quota", "flow", "bin_of", "slot_of")})
    out["all"] = gathered
    return out


@pytest.mark.parametrize("world", [2, 3])
def test_seed_sharding_and_planner_agreement(world):
    res = run_world(_shard_and_plan, world)
    train = set(res[0]["train"])
    seen = set()
    for r in res:
        s = set(r["seeds"])
        assert len(s) == len(r["seeds"]) and s <= train
        assert not (s & seen)
        seen |= s
    assert len({len(r["seeds"]) for r in res}) == 1
    for r in res:
        for other in r["all"]:
            assert other == r["all"][0]


def _exchange(rank, world, seed):
    import oracle
    from paper_conf_sc_shi0s0x0w25_b200.exchange import alltoallv, exchange_counts

    oracle.build()
    rng = np.random.default_rng(seed)  # same on every rank: shared placement, quota and host rows
    n_rows, R = 4000, 48
    table = rng.integers(0, 255, size=(n_rows, R), dtype=np.uint8)
    n_bins = world + 2  # one HBM bin per rank + two host bins
    owner = list(range(world)) + [-1, -1]
    bin_of_v = rng.integers(0, n_bins, n_rows).astype(np.int32)
    quota = np.zeros((n_bins, world), np.int64)
    quota[world] = rng.integers(1, 5, world)
    quota[world + 1] = rng.integers(0, 5, world)
    quota[world + 1][0] = 3
    my_ids = np.random.default_rng(seed * 10 + rank).integers(0, n_rows, 700)
    route, qoff, qpos = oracle.bucket(rank, world, owner, quota, bin_of_v[my_ids])
    out = np.zeros((len(my_ids), R), np.uint8)
    # rows this rank reads itself
    direct = np.array([(route[i] % world == rank) or owner[route[i] // world] >= 0 for i in range(len(my_ids))])
    out[direct] = table[my_ids[direct]]
    # pack: destination rank ascending, then host bin ascending (the relay_pack order)
    words, send = [], [0] * world
    for h in range(world):
        if h == rank:
            continue
        for b in range(n_bins):
            if owner[b] >= 0:
                continue
            q = b * world + h
            for i in qpos[qoff[q]:qoff[q + 1]]:
                words.append((int(my_ids[i]), int(i)))
                send[h] += 1
    recv = exchange_counts(torch.tensor(send), None)
    w = torch.tensor(words, dtype=torch.int64).reshape(-1, 2) if words else torch.zeros((0, 2), dtype=torch.int64)
    w_in = alltoallv(w, send, recv)
    served = torch.from_numpy(oracle.gather(table, w_in[:, 0].numpy())) if len(w_in) else torch.zeros((0, R),
                                                                                                       dtype=torch.uint8)
    back = alltoallv(served, recv, send)
    for e, (_, i) in enumerate(words):
        out[i] = back[e].numpy()
    return {"ok": bool(np.array_equal(out, table[my_ids])), "sent": send, "served": recv}


@pytest.mark.parametrize("world,seed", [(2, 1), (3, 2)])
def test_relay_exchange_protocol(world, seed):
    res = run_world(_exchange, world, seed)
    assert all(r["ok"] for r in res)
    # what rank g sent to h is what h served for g
    for g in range(world):
        for h in range(world):
            assert res[g]["sent"][h] == res[h]["served"][g]
    assert sum(sum(r["sent"]) for r in res) > 0
