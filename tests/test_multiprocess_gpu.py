"""One process per rank on the GPU path (H4-H7 with the all-to-all transport), 2 processes sharing cuda:0.

Each rank owns one HBM bin (its feature rows by the DDAK placement); the other rank's bin is mapped
through CUDA IPC (moment_ipc_export / import — the peer-load pointer of the NVLink path); both host bins
are pinned host memory; the quota relays part of every rank's host rows through the other rank. Each rank
samples its own seeds and runs exchange.gather_exchange (bucket -> routed gather -> relay pack ->
all-to-all -> relay serve -> all-to-all -> scatter) over a gloo group; the rows must equal the oracle's
table[ids] byte for byte.
"""
import numpy as np
import pytest
import torch

from mp_util import run_world

pytestmark = pytest.mark.gpu


def _rank_main(rank, world, transport="alltoall"):
    import torch.distributed as dist

    import oracle
    import paper_conf_sc_shi0s0x0w25_b200 as M
    import workloads as W
    from paper_conf_sc_shi0s0x0w25_b200.exchange import ExchangeBuffers, PeerExchange, gather_exchange

    oracle.build()
    torch.cuda.set_device(0)
    dev = "cuda:0"
    cfg = W.CONFIGS["C1"]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=dev)
    n = g.n
    table = W.feature_table(n, 32, torch.float32, device="cpu")  # 128-byte rows
    R = table.shape[1]
    rng = np.random.default_rng(7)  # identical on every rank: one global placement
    hot = rng.pareto(1.0, n).astype(np.uint64)
    owners = list(range(world)) + [-1, -1]
    tiers = [M.TIER_GPU_HBM] * world + [M.TIER_HOST_DRAM] * 2
    caps = [n // (4 * world)] * world + [n // 2, n]
    bin_of, slot_of, *_ = M.place(None, hot, caps, bin_tier=tiers, bin_traffic=[100] * world + [10, 10])
    bins = []
    for b in range(world + 2):
        sel = np.nonzero(bin_of == b)[0]
        buf = torch.zeros((max(1, int(slot_of[sel].max()) + 1 if len(sel) else 1), R), dtype=torch.uint8)
        buf[torch.as_tensor(slot_of[sel])] = table[torch.as_tensor(sel)]
        bins.append(buf)
    mine = bins[rank].to(dev)  # this rank's HBM bin
    handle, off = M.ipc_export(mine)
    shared = [None] * world
    dist.all_gather_object(shared, (handle, off))
    imported = {}
    ptrs = []
    for b in range(world):
        if b == rank:
            ptrs.append(mine.data_ptr())
        else:
            base = M.ipc_import(shared[b][0])
            imported[b] = base
            ptrs.append(base + shared[b][1])
    host = [bins[world].pin_memory(), bins[world + 1].pin_memory()]
    ptrs += [h.data_ptr() for h in host]
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=dev)
    quota = np.zeros((world + 2, world), np.int64)
    quota[world] = [3, 2] if world == 2 else np.arange(1, world + 1)
    quota[world + 1] = [1, 4] if world == 2 else np.arange(world, 0, -1)
    ctx = M.Ctx(n_vertices=n, max_seeds=512, max_fanout=[10, 5], rank=rank, world=world, device=0, row_bytes=R,
                bin_owner=owners, bin_ptr=ptrs, placement=placement, quota=quota)
    train = W.training_set(g, min_count=512 * world)
    seeds = W.epoch_batches(train, 512, 0, rank=rank, world=world)[0]
    bufs = M.SampleBuffers.allocate(512, [10, 5], n, dev)
    ctx.sample(g.indptr, g.indices, seeds, [10, 5], 900 + rank, bufs)
    torch.cuda.synchronize()
    nF = int(bufs.counts[2])
    ids = bufs.nodes[:nF].contiguous()
    want = oracle.gather(table.numpy(), ids.cpu().numpy())
    if transport == "one_call":
        # moment_ctx_set_exchange: each batch is ONE library call (moment_gather, then moment_step = sample +
        # exchange from the ctx's CUDA graph), device barriers inside, nothing host-synchronised between calls
        nmax = [None] * world
        dist.all_gather_object(nmax, int(bufs.nodes.numel()))
        px = PeerExchange(ctx, max(nmax), R, dev, timeout_s=30.0)
        outs = [px.gather(ids, nF).clone() for _ in range(3)]
        torch.cuda.synchronize()
        ok = all(bool(np.array_equal(o.cpu().numpy(), want)) for o in outs)
        steps = []
        for rep in range(4):  # rep 0 captures the graph, the others replay it
            px.step(g.indptr, g.indices, seeds, [10, 5], 900 + rank, bufs)
            steps.append(px.out[:nF].clone())
        torch.cuda.synchronize()
        ok &= int(bufs.counts[2]) == nF
        ok &= all(bool(np.array_equal(o.cpu().numpy(), want)) for o in steps)
        # an empty batch on this rank still serves the other's requests
        out = px.gather(ids, 0 if rank == 0 else nF)
        torch.cuda.synchronize()
        if rank == 1:
            ok &= bool(np.array_equal(out.cpu().numpy(), want))
        px.check()
        # the registered output is required: another buffer is refused
        try:
            ctx.gather(ids, torch.empty_like(px.out), max_n=nF)
            ok = False
        except M.MomentError as e:
            ok &= e.status == M.EINVAL
        px.close()
        info = {"sent": [0] * world, "served": [0] * world}
    elif transport in ("peer", "peer_dev"):
        # the exchange buffers are sized for the largest batch of any rank; two batches check reuse
        nmax = [None] * world
        dist.all_gather_object(nmax, int(bufs.nodes.numel()))
        px = PeerExchange(ctx, max(nmax), R, dev, device_barrier=transport == "peer_dev", timeout_s=30.0,
                          one_call=False)
        ok = True
        for rep in range(2):
            out = px.gather(ids, nF)
            torch.cuda.synchronize()
            ok &= bool(np.array_equal(out.cpu().numpy(), want))
        if transport == "peer_dev":
            # several batches enqueued back to back with no host synchronisation between them
            outs = []
            for rep in range(3):
                outs.append(px.gather(ids, nF).clone())
            torch.cuda.synchronize()
            ok &= all(bool(np.array_equal(o.cpu().numpy(), want)) for o in outs)
            px.check()
        # an empty batch on this rank still serves the other's requests
        out = px.gather(ids, 0 if rank == 0 else nF)
        torch.cuda.synchronize()
        if rank == 1:
            ok &= bool(np.array_equal(out.cpu().numpy(), want))
        if transport == "peer_dev":
            px.check()
        px.close()
        info = {"sent": [0] * world, "served": [0] * world}
    else:
        out = torch.zeros((nF, R), dtype=torch.uint8, device=dev)
        xb = ExchangeBuffers(max_n=nF, row_bytes=R, n_queues=(world + 2) * world, device=torch.device(dev))
        info = gather_exchange(ctx, ids, out, xb, n=nF)
        torch.cuda.synchronize()
        ok = bool(np.array_equal(out.cpu().numpy(), want))
    dist.barrier()  # every rank done with the others' bins before any mapping goes away
    for base in imported.values():
        M.ipc_close(base)
    dist.barrier()
    return {"ok": ok, "sent": info["sent"], "served": info["served"], "nF": nF}


def test_gather_exchange_two_processes_one_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    res = run_world(_rank_main, 2)
    assert all(r["ok"] for r in res), res
    assert res[0]["sent"][1] == res[1]["served"][0] and res[1]["sent"][0] == res[0]["served"][1]
    assert res[0]["sent"][1] > 0 and res[1]["sent"][0] > 0


def test_peer_exchange_two_processes_one_gpu():
    """The same exchange with no all-to-all: requests and relayed rows move by peer stores into CUDA-IPC
    mapped inboxes / outputs (moment_relay_push, moment_relay_serve_push), byte-exact with the oracle."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    res = run_world(_rank_main, 2, "peer")
    assert all(r["ok"] for r in res), res


def test_peer_exchange_device_barrier_two_processes_one_gpu():
    """The peer-memory exchange with device-side signal barriers (moment_signal_barrier) instead of host
    synchronisation: batches enqueued back to back, byte-exact with the oracle, no watchdog expiry."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    res = run_world(_rank_main, 2, "peer_dev")
    assert all(r["ok"] for r in res), res


@pytest.mark.parametrize("world", [2, 3])
def test_one_call_exchange_processes_one_gpu(world):
    """moment_ctx_set_exchange: the whole relay exchange inside ONE moment_gather / moment_step call per batch
    (bucket, own reads, peer-store requests, device barrier, peer-store rows, device barrier), replayed from
    the ctx's CUDA graph with no host barrier between batches; byte-exact with the oracle (2 and 3 processes
    sharing cuda:0, every rank relaying for the others)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    res = run_world(_rank_main, world, "one_call")
    assert all(r["ok"] for r in res), res
