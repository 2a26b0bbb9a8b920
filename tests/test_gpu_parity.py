"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element.

Sampling (H1-H3) is compared bit-exactly: nodes (F_H), per-hop offsets, src and counts. Gathers
(H4-H7) are compared byte-exactly with the oracle's out[i] = table[ids[i]]. Bucketing (H4) is compared
with the oracle's routing given the same quota. Sizes span several tiles and ragged tails; C1 runs at its
full BASELINE size, C2 at full size with the launch configuration bench.py times.
"""
import numpy as np
import pytest
import torch

import paper_conf_sc_shi0s0x0w25_b200 as M
import workloads as W

pytestmark = pytest.mark.gpu

DEV = "cuda:0"


def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


@pytest.fixture(scope="module")
def c1():
    _need_gpu()
    cfg = W.CONFIGS["C1"]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    return cfg, g


def sample_both(orc, g, seeds, fanout, rng_seed, flags=0, ctx=None):
    ctx = ctx or M.Ctx(n_vertices=g.n, max_seeds=max(len(seeds), 1), max_fanout=fanout, device=0)
    bufs = M.SampleBuffers.allocate(len(seeds), fanout, g.n, DEV)
    seeds_d = torch.as_tensor(np.asarray(seeds, np.int64), device=DEV)
    ctx.sample(g.indptr, g.indices, seeds_d, fanout, rng_seed, bufs, flags=flags)
    got = bufs.result()
    want = orc.sample(g.indptr.cpu().numpy(), g.indices.cpu().numpy(), np.asarray(seeds, np.int64), fanout, rng_seed,
                      replace=bool(flags & M.SAMPLE_REPLACE))
    return got, want


def assert_same_sample(got, want):
    assert np.array_equal(got["counts"], want["counts"]), (got["counts"], want["counts"])
    assert np.array_equal(got["nodes"], want["nodes"])
    for h in range(len(want["offsets"])):
        assert np.array_equal(got["offsets"][h], want["offsets"][h]), h
        assert np.array_equal(got["src"][h], want["src"][h]), h


def assert_all_rows(rows, ids, dim, dtype, mod=None):
    """Every gathered row (all |F_H| of them, not a sample) equals the table row of its id (the oracle's
    gather, out[i] = table[ids[i]], with table[v] = featgen(v)); compared on the device in
    chunks so that full-size batches stay cheap."""
    n = len(ids)
    ids_d = torch.as_tensor(np.asarray(ids, np.int64), device=rows.device)
    if mod is not None:
        ids_d = ids_d % mod
    R = rows.shape[1]
    chunk = max(1024, (1 << 28) // (2 * R))
    for c0 in range(0, n, chunk):
        want = W.feature_rows(ids_d[c0:c0 + chunk], dim, dtype)
        got = rows[c0:c0 + len(want), :want.shape[1]]
        if not torch.equal(got, want):
            bad = (got != want).any(1).nonzero().flatten()
            raise AssertionError(f"{len(bad)} of {len(want)} rows differ in chunk at {c0}; first row {c0 + int(bad[0])}")


def test_sample_c1_full_size(orc, c1):
    cfg, g = c1
    train = W.training_set(g, min_count=cfg["batch"])
    for b, seeds in enumerate(W.epoch_batches(train, cfg["batch"], 0)[:2]):
        got, want = sample_both(orc, g, seeds.cpu().numpy(), list(cfg["fanout"]), W.batch_rng_seed(1, 0, 0, b))
        assert_same_sample(got, want)


@pytest.mark.parametrize("fanout", [[15, 10, 5], [3], [1, 1, 1, 1], [25, 10], [33, 2], [64], [200], [7, 11, 13],
                                    [32, 2], [16, 31]])
@pytest.mark.parametrize("n_seeds", [1, 257, 1000])
def test_sample_fanouts_and_ragged(orc, c1, fanout, n_seeds):
    _, g = c1
    rng = np.random.default_rng(n_seeds * 7 + len(fanout))
    seeds = rng.choice(g.n, n_seeds, replace=False)
    got, want = sample_both(orc, g, seeds, fanout, 12345 + n_seeds)
    assert_same_sample(got, want)


@pytest.mark.parametrize("knob", [(("MOMENT_HOP_WARP", "0"),), (("MOMENT_INIT_KERNEL", "1"),),
                                  (("MOMENT_SPARSE_SCAN", "1"),),
                                  (("MOMENT_SPARSE_SCAN", "1"), ("MOMENT_SPARSE_NT", "1024")),
                                  (("MOMENT_RANK_RELABEL", "0"),),
                                  (("MOMENT_RANK_RELABEL", "0"), ("MOMENT_SPARSE_SCAN", "1"))])
@pytest.mark.parametrize("fanout", [[15, 10, 5], [7, 3], [20], [40, 2]])
def test_sample_kernel_variants(orc, c1, fanout, knob, monkeypatch):
    """The other sampler kernels give the same result as the default: MOMENT_HOP_WARP=0 selects the
    power-of-two lane tiles (always used for k > 32), MOMENT_INIT_KERNEL=1 a separate init kernel instead of
    the first hop's sampler initialising the call, MOMENT_SPARSE_SCAN=1 the summary-bitmap bitscan that
    graphs above 8.4 M vertices use (C3-C5), MOMENT_RANK_RELABEL=0 local indices through lidx for every
    node instead of the rank tables (dense and sparse)."""
    _, g = c1
    for k, v in knob:
        monkeypatch.setenv(k, v)
    seeds = np.random.default_rng(5).choice(g.n, 1000, replace=False)
    got, want = sample_both(orc, g, seeds, fanout, 4242)
    assert_same_sample(got, want)
    got, want = sample_both(orc, g, seeds, fanout, 4243, flags=M.SAMPLE_REPLACE)
    assert_same_sample(got, want)


@pytest.mark.parametrize("fanout", [[10, 5], [40], [7, 13]])
def test_sample_replace(orc, c1, fanout):
    _, g = c1
    seeds = np.random.default_rng(3).choice(g.n, 700, replace=False)
    got, want = sample_both(orc, g, seeds, fanout, 99, flags=M.SAMPLE_REPLACE)
    assert_same_sample(got, want)


def test_sample_handmade_graphs(orc):
    _need_gpu()
    # path + isolated vertex + star + self loop + duplicate edges
    edges = [(0, 1), (1, 2), (2, 3), (5, 6), (5, 7), (5, 8), (5, 9), (5, 10), (5, 11), (5, 12), (9, 9), (10, 11),
             (10, 11), (10, 11)]
    n = 13
    edges.sort()
    indptr = np.zeros(n + 1, np.int64)
    for u, _ in edges:
        indptr[u + 1] += 1
    indptr = np.cumsum(indptr)
    indices = np.array([v for _, v in edges], np.int32)
    g = W.Graph(torch.as_tensor(indptr, device=DEV), torch.as_tensor(indices, device=DEV), n, len(edges))
    for seeds, fanout in [([0, 4], [3, 3]), ([5], [3, 2, 1]), ([10, 9], [2, 2]), ([4], [5]), (list(range(13)), [2])]:
        for seed in range(5):
            got, want = sample_both(orc, g, seeds, fanout, seed)
            assert_same_sample(got, want)


def test_sample_empty_batch(orc, c1):
    _, g = c1
    ctx = M.Ctx(n_vertices=g.n, max_seeds=16, max_fanout=[4, 4], device=0)
    bufs = M.SampleBuffers.allocate(0, [4, 4], g.n, DEV)
    ctx.sample(g.indptr, g.indices, torch.zeros(0, dtype=torch.int64, device=DEV), [4, 4], 1, bufs)
    assert list(bufs.counts.cpu().numpy()) == [0, 0, 0, 0, 0]


def test_sample_check_flags_bad_seeds(c1):
    _, g = c1
    ctx = M.Ctx(n_vertices=g.n, max_seeds=16, max_fanout=[4], device=0)
    bufs = M.SampleBuffers.allocate(3, [4], g.n, DEV)
    ctx.sample(g.indptr, g.indices, torch.tensor([1, 2, 1], device=DEV), [4], 1, bufs, flags=M.SAMPLE_CHECK)
    with pytest.raises(M.MomentError):
        ctx.sample_check()
    ctx.sample(g.indptr, g.indices, torch.tensor([1, 2, g.n + 5], device=DEV), [4], 1, bufs, flags=M.SAMPLE_CHECK)
    with pytest.raises(M.MomentError):
        ctx.sample_check()
    ctx.sample(g.indptr, g.indices, torch.tensor([1, 2, 3], device=DEV), [4], 1, bufs, flags=M.SAMPLE_CHECK)
    ctx.sample_check()
    with pytest.raises(M.MomentError) as e:  # host-side argument errors
        ctx.sample(g.indptr, g.indices, torch.tensor([1, 2, 3], device=DEV), [5], 1, bufs)
    assert e.value.status == M.EINVAL


@pytest.mark.parametrize("sparse,relabel", [("0", "1"), ("1", "1"), ("0", "0"), ("1", "0")])
def test_sample_reused_ctx_many_batches(orc, c1, sparse, relabel, monkeypatch):
    """The workspace (lidx, rank tables, bitmaps, summary bitmap, tile descriptors) is reset or rewritten
    correctly between calls, for the dense and the sparse (summary-bitmap) bitscan, with and without rank
    relabelling."""
    cfg, g = c1
    monkeypatch.setenv("MOMENT_SPARSE_SCAN", sparse)
    monkeypatch.setenv("MOMENT_RANK_RELABEL", relabel)
    ctx = M.Ctx(n_vertices=g.n, max_seeds=1024, max_fanout=[10, 5], device=0)
    rng = np.random.default_rng(0)
    for b in range(4):
        seeds = rng.choice(g.n, int(rng.integers(1, 1024)), replace=False)
        got, want = sample_both(orc, g, seeds, [10, 5], b, ctx=ctx)
        assert_same_sample(got, want)


def _gather_path_env(monkeypatch, path):
    """MOMENT_GATHER_PATH; "tma4-rN": tile::gather4 with N-row tiles (MOMENT_TMA4_ROWS; default 16)."""
    if path.startswith("tma4-r"):
        monkeypatch.setenv("MOMENT_TMA4_ROWS", path[len("tma4-r"):])
        path = "tma4"
    monkeypatch.setenv("MOMENT_GATHER_PATH", path)
    return path


@pytest.mark.parametrize("path", ["auto", "ldg", "bulk", "tma4", "tma4-r8", "tma4-r32"])
@pytest.mark.parametrize("dim,dtype", [(4, torch.float32), (12, torch.float32), (100, torch.float32),
                                       (128, torch.float32), (768, torch.float16), (1024, torch.float32)])
def test_gather_replicated(orc, dim, dtype, path, monkeypatch):
    _need_gpu()
    path = _gather_path_env(monkeypatch, path)
    n = 5000
    table = W.feature_table(n, dim, dtype, device=DEV)
    R = table.shape[1]
    rng = np.random.default_rng(dim)
    # counts past one round of tiles (148 SMs x 3 blocks x 16 rows) exercise the ragged last round
    for count in [1, 31, 1000, 4099] + ([15000, 50001] if path == "tma4" else []):
        ids = torch.as_tensor(rng.integers(0, n, count), device=DEV)
        ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], device=0, row_bytes=R, bin_owner=[0],
                    bin_ptr=[table.data_ptr()])
        out = torch.empty((count, R), dtype=torch.uint8, device=DEV)
        ctx.gather(ids, out)
        want = orc.gather(table.cpu().numpy(), ids.cpu().numpy())
        assert np.array_equal(out.cpu().numpy(), want)
        # device count smaller than max_n: only the first n_dev rows are written
        out2 = torch.zeros((count, R), dtype=torch.uint8, device=DEV)
        nd = torch.tensor([count // 2], dtype=torch.int64, device=DEV)
        ctx.gather(ids, out2, n_dev=nd)
        o2 = out2.cpu().numpy()
        assert np.array_equal(o2[: count // 2], want[: count // 2]) and not o2[count // 2:].any()


@pytest.mark.parametrize("path", ["auto", "ldg", "bulk", "tma4", "tma4-r8", "tma4-r32"])
@pytest.mark.parametrize("dim,dtype", [(100, torch.float32), (128, torch.float32), (768, torch.float16)])
def test_gather_one_local_bin_with_placement(orc, dim, dtype, path, monkeypatch):
    """One local bin addressed through a placement map (a DDAK layout on one GPU: row v at a permuted
    slot): tile::gather4 takes the slot as its row coordinate, the bulk gather resolves the placement one
    tile ahead; every path byte-exact with the oracle's table[ids]."""
    _need_gpu()
    path = _gather_path_env(monkeypatch, path)
    n = 7000
    table = W.feature_table(n, dim, dtype, device="cpu")
    R = table.shape[1]
    rng = np.random.default_rng(dim + 1)
    slot_of = rng.permutation(n).astype(np.int64)
    bin_tab = torch.zeros((n, R), dtype=torch.uint8)
    bin_tab[torch.as_tensor(slot_of)] = table
    bin_tab = bin_tab.to(DEV)
    placement = torch.as_tensor(M.place_pack(np.zeros(n, np.int32), slot_of).view(np.int64), device=DEV)
    ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], device=0, row_bytes=R, bin_owner=[0],
                bin_ptr=[bin_tab.data_ptr()], placement=placement)
    for count in [1, 33, 4099, 50001]:
        ids = torch.as_tensor(rng.integers(0, n, count), device=DEV)
        out = torch.empty((count, R), dtype=torch.uint8, device=DEV)
        ctx.gather(ids, out)
        want = orc.gather(table.numpy(), ids.cpu().numpy())
        assert np.array_equal(out.cpu().numpy(), want)
        # a device count below the buffer size, the buffer's tail holding stale, out-of-range ids (as F_H's
        # buffer does past |F_H|): only the first n_dev rows are read and written
        stale = ids.clone()
        stale[count // 2:] = (1 << 40) + 12345
        out2 = torch.zeros_like(out)
        ctx.gather(stale, out2, n_dev=torch.tensor([count // 2], dtype=torch.int64, device=DEV))
        o2 = out2.cpu().numpy()
        assert np.array_equal(o2[: count // 2], want[: count // 2]) and not o2[count // 2:].any()


def build_tiered(table, bin_of, slot_of, owners, host_bins, device=DEV):
    """Materialise bins from a placement: HBM bins as device buffers, host bins as pinned host memory."""
    R = table.shape[1]
    nb = len(owners)
    bins = []
    t_cpu = table.cpu()
    b_t = torch.as_tensor(bin_of)
    s_t = torch.as_tensor(slot_of)
    for b in range(nb):
        sel = torch.nonzero(b_t == b).flatten()
        rows = max(1, int(s_t[sel].max()) + 1) if len(sel) else 1
        buf = torch.zeros((rows, R), dtype=torch.uint8)
        buf[s_t[sel]] = t_cpu[sel]
        if b in host_bins:
            buf = buf.pin_memory()
        else:
            buf = buf.to(device)
        bins.append(buf)
    return bins


def test_gather_tiered_and_bucket_vs_oracle(orc, c1):
    """DDAK placement over 2 HBM bins (local + 'peer') and 2 pinned host bins; routed gather for rank 0."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 32, torch.float32, device=DEV)  # 128-byte rows
    R = table.shape[1]
    train = W.training_set(g, min_count=1024)
    seeds = W.epoch_batches(train, 1024, 0)[0]
    # hotness from product pre-sampling (P2), compared with the oracle sampler's counts
    ctx_s = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], device=0)
    hot = torch.zeros(n, dtype=torch.int64, device=DEV)
    hot_np = np.zeros(n, np.uint64)
    for b in range(3):
        bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
        ctx_s.sample(g.indptr, g.indices, seeds, [10, 5], 1000 + b, bufs)
        ctx_s.hotness(bufs.nodes, hot, n_dev=bufs.counts[2:3], max_n=bufs.nodes.numel())
        ref = orc.sample(g.indptr.cpu().numpy(), g.indices.cpu().numpy(), seeds.cpu().numpy(), [10, 5], 1000 + b)
        np.add.at(hot_np, ref["nodes"], 1)
    assert np.array_equal(hot.cpu().numpy().astype(np.uint64), hot_np)
    owners = [0, 1, -1, -1]
    tiers = [M.TIER_GPU_HBM, M.TIER_GPU_HBM, M.TIER_HOST_DRAM, M.TIER_HOST_DRAM]
    caps = [n // 8, n // 8, n // 2, n]
    bin_of, slot_of, *_ = M.place(None, hot_np, caps, bin_tier=tiers, bin_traffic=[500, 300, 50, 40], pool=100)
    bins = build_tiered(table, bin_of, slot_of, owners, host_bins={2, 3})
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=DEV)
    world = 2
    quota = np.zeros((4, world), np.int64)
    quota[2] = [3, 1]  # host bin 2: 3/4 of rank 0's requests direct, 1/4 via rank 1
    quota[3] = [1, 1]
    ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], rank=0, world=world, device=0, row_bytes=R,
                bin_owner=owners, bin_ptr=[b.data_ptr() for b in bins], placement=placement, quota=quota)
    bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
    ctx.sample(g.indptr, g.indices, seeds, [10, 5], 7, bufs)
    nF = int(bufs.counts[2])
    ids = bufs.nodes[:nF].clone()
    route = torch.empty(nF, dtype=torch.int32, device=DEV)
    qoff = torch.empty(4 * world + 1, dtype=torch.int64, device=DEV)
    qpos = torch.empty(nF, dtype=torch.int64, device=DEV)
    ctx.bucket(ids, route, qoff, qpos)
    o_route, o_qoff, o_qpos = orc.bucket(0, world, owners, quota, bin_of[ids.cpu().numpy()])
    assert np.array_equal(route.cpu().numpy(), o_route)
    assert np.array_equal(qoff.cpu().numpy(), o_qoff)
    assert np.array_equal(qpos.cpu().numpy(), o_qpos)
    # an empty request list right after a full one: empty queues, not the previous call's tile counts
    ctx.bucket(ids, route, qoff, qpos, max_n=0)
    assert not qoff.cpu().numpy().any()
    assert np.array_equal(orc.bucket(0, world, owners, quota, bin_of[ids.cpu().numpy()[:0]])[1], qoff.cpu().numpy())
    # single-rank gather refuses quotas that relay through another rank
    out = torch.empty((nF, R), dtype=torch.uint8, device=DEV)
    with pytest.raises(M.MomentError) as e:
        ctx.gather(ids, out)
    assert e.value.status == M.EUNSUPPORTED


@pytest.mark.parametrize("world", [2, 4])
def test_gather_group_relay_logical_ranks(orc, c1, world):
    """k logical ranks on one GPU: per-rank HBM bins (peer loads), 2 host bins with quota relays."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 100, torch.float32, device=DEV)  # 400-byte rows
    R = table.shape[1]
    rng = np.random.default_rng(world)
    hot = rng.pareto(1.0, n).astype(np.uint64)
    owners = list(range(world)) + [-1, -1]
    tiers = [M.TIER_GPU_HBM] * world + [M.TIER_HOST_DRAM] * 2
    caps = [n // (4 * world)] * world + [n // 2, n]
    bin_of, slot_of, *_ = M.place(None, hot, caps, bin_tier=tiers, bin_traffic=[100] * world + [10, 10])
    bins = build_tiered(table, bin_of, slot_of, owners, host_bins={world, world + 1})
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=DEV)
    quota = np.zeros((world + 2, world), np.int64)
    quota[world] = rng.integers(0, 5, world) + 1
    quota[world + 1] = np.arange(world)  # rank 0 gets nothing directly
    ctxs, ids, outs, nds = [], [], [], []
    train = W.training_set(g, min_count=1024 * world)
    for r in range(world):
        ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], rank=r, world=world, device=0, row_bytes=R,
                    bin_owner=owners, bin_ptr=[b.data_ptr() for b in bins], placement=placement, quota=quota)
        seeds = W.epoch_batches(train, 1024, 0, rank=r, world=world)[0]
        bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
        ctx.sample(g.indptr, g.indices, seeds, [10, 5], 50 + r, bufs)
        ctxs.append(ctx)
        ids.append(bufs.nodes)
        nds.append(bufs.counts[2:3])
        outs.append(torch.zeros((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV))
    max_n = max(t.numel() for t in ids)
    ids = [torch.nn.functional.pad(t, (0, max_n - t.numel())) for t in ids]
    outs = [torch.zeros((max_n, R), dtype=torch.uint8, device=DEV) for _ in range(world)]
    M.gather_group(ctxs, ids, outs, n_dev=nds, max_n=max_n)
    tab = table.cpu().numpy()
    for r in range(world):
        nF = int(nds[r])
        want = orc.gather(tab, ids[r][:nF].cpu().numpy())
        assert np.array_equal(outs[r][:nF].cpu().numpy(), want), r


def test_step_host_matches_device_path(orc, c1):
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 128, torch.float32, device=DEV)
    R = table.shape[1]
    ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], device=0, row_bytes=R, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    train = W.training_set(g, min_count=1024)
    seeds = W.epoch_batches(train, 1024, 0)[0]
    bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
    want = orc.sample(g.indptr.cpu().numpy(), g.indices.cpu().numpy(), seeds.cpu().numpy(), [10, 5], 77)
    nF = int(want["counts"][2])
    # pinned buffers: the kernels read the seeds and write the counts over PCIe themselves; pageable ones go
    # through cudaMemcpyAsync; several steps back to back reuse the graph with new host pointers
    for pinned in (True, False, True):
        counts_h = torch.full((5,), -1, dtype=torch.int64)
        seeds_h = seeds.cpu().clone()
        if pinned:
            counts_h, seeds_h = counts_h.pin_memory(), seeds_h.pin_memory()
        rows.zero_()
        ctx.step_host(g.indptr, g.indices, seeds_h, [10, 5], 77, bufs, rows, counts_h)
        torch.cuda.synchronize()
        assert np.array_equal(counts_h.numpy(), want["counts"]), pinned
        assert np.array_equal(rows[:nF].cpu().numpy(), orc.gather(table.cpu().numpy(), want["nodes"]))
        # the device path after a host step: the call block's host-counts slot is cleared
        bufs.counts.zero_()
        ctx.step(g.indptr, g.indices, seeds, [10, 5], 77, bufs, rows)
        torch.cuda.synchronize()
        assert np.array_equal(bufs.counts.cpu().numpy(), want["counts"])


def test_bind_step_matches_oracle(orc, c1):
    """Ctx.bind_step (the prepared moment_step / moment_step_host the bench issues): per-call seeds, rng seed and
    host counts reach the kernels; interleaved with the unprepared calls on the same ctx."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 128, torch.float32, device=DEV)
    R = table.shape[1]
    ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], device=0, row_bytes=R, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
    s = torch.cuda.Stream()
    run = ctx.bind_step(g.indptr, g.indices, [10, 5], bufs, rows, stream=s)
    run_h = ctx.bind_step(g.indptr, g.indices, [10, 5], bufs, rows, stream=s, host=True)
    batches = W.epoch_batches(W.training_set(g, min_count=4096), 1024, 0)
    ip, ix, tab = g.indptr.cpu().numpy(), g.indices.cpu().numpy(), table.cpu().numpy()
    for b in range(4):
        seeds = batches[b]
        rng = W.batch_rng_seed(9, 0, 0, b)
        want = orc.sample(ip, ix, seeds.cpu().numpy(), [10, 5], rng)
        nF = int(want["counts"][2])
        if b % 2 == 0:
            run(seeds, rng)
            s.synchronize()
            assert np.array_equal(bufs.counts.cpu().numpy(), want["counts"])
        else:
            counts_h = torch.full((5,), -1, dtype=torch.int64).pin_memory()
            seeds_h = seeds.cpu().pin_memory()  # read by the first hop's kernel over PCIe: kept alive until the sync
            run_h(seeds_h, rng, counts_h)
            s.synchronize()
            assert np.array_equal(counts_h.numpy(), want["counts"])
        assert_same_sample(bufs.result(), want)
        assert np.array_equal(rows[:nF].cpu().numpy(), orc.gather(tab, want["nodes"]))
        ctx.step(g.indptr, g.indices, batches[(b + 1) % len(batches)], [10, 5], rng + 1, bufs, rows, stream=s)


def test_step_batch_matches_oracle(orc, c1):
    """moment_step_batch (StepBatch): one call enqueues one step per ctx, device and host variants, fewer
    batches than ctxs, and a repeated ctx is refused."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 128, torch.float32, device=DEV)
    R = table.shape[1]
    P = 3
    ctxs = [M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], device=0, row_bytes=R, bin_owner=[0],
                  bin_ptr=[table.data_ptr()]) for _ in range(P)]
    bufs = [M.SampleBuffers.allocate(1024, [10, 5], n, DEV) for _ in range(P)]
    rows = [torch.empty((b.nodes.numel(), R), dtype=torch.uint8, device=DEV) for b in bufs]
    streams = [torch.cuda.Stream() for _ in range(P)]
    sb = M.StepBatch(ctxs, g.indptr, g.indices, [10, 5], bufs, rows, streams)
    sbh = M.StepBatch(ctxs, g.indptr, g.indices, [10, 5], bufs, rows, streams, host=True)
    batches = W.epoch_batches(W.training_set(g, min_count=4096), 1024, 0)
    ip, ix, tab = g.indptr.cpu().numpy(), g.indices.cpu().numpy(), table.cpu().numpy()
    for k, host in [(3, False), (2, True), (3, True), (1, False)]:
        seeds = [batches[(i + k) % len(batches)] for i in range(k)]
        rngs = [W.batch_rng_seed(11, k, int(host), i) for i in range(k)]
        if host:
            seeds_h = [x.cpu().pin_memory() for x in seeds]
            counts_h = [torch.full((5,), -1, dtype=torch.int64).pin_memory() for _ in range(k)]
            sbh.run(seeds_h, rngs, counts_h)
        else:
            sb.run(seeds, rngs)
        torch.cuda.synchronize()
        for i in range(k):
            want = orc.sample(ip, ix, seeds[i].cpu().numpy(), [10, 5], rngs[i])
            assert_same_sample(bufs[i].result(), want)
            if host:
                assert np.array_equal(counts_h[i].numpy(), want["counts"])
            nF = int(want["counts"][2])
            assert np.array_equal(rows[i][:nF].cpu().numpy(), orc.gather(tab, want["nodes"]))
    bad = M.StepBatch([ctxs[0], ctxs[0]], g.indptr, g.indices, [10, 5], bufs[:2], rows[:2], streams[:2])
    with pytest.raises(M.MomentError) as e:
        bad.run(batches[:2], [1, 2])
    assert e.value.status == M.EINVAL


def test_c2_full_size_bench_configuration(orc):
    """C2 at BASELINE size, in bench.py's launch configuration: whole-batch sample parity + every gathered row."""
    _need_gpu()
    import bench

    st = bench.build_state("C2", device=DEV, rank=0, world=1)
    for b in range(2):
        seeds, rng_seed = st.batch(b)
        st.step(seeds, rng_seed)
        torch.cuda.synchronize()
        got = st.bufs.result()
        want = orc.sample(st.graph.indptr.cpu().numpy(), st.graph.indices.cpu().numpy(), seeds.cpu().numpy(),
                          list(st.fanout), rng_seed)
        assert_same_sample(got, want)
        nF = int(got["counts"][len(st.fanout)])
        assert_all_rows(st.rows[:nF], want["nodes"], st.dim, st.dtype)


def test_moment_step_graph_matches_oracle_across_batches_and_shapes(orc, c1):
    """moment_step replays a cached CUDA graph: per-call seeds / rng_seed must reach the kernels, and a
    new shape (batch size, fanout, buffers) must re-capture."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 32, torch.float32, device=DEV)
    R = table.shape[1]
    ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], device=0, row_bytes=R, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    train = W.training_set(g, min_count=4096)
    batches = W.epoch_batches(train, 1024, 0)
    tab = table.cpu().numpy()
    ip, ix = g.indptr.cpu().numpy(), g.indices.cpu().numpy()
    for fanout, bsz in [([10, 5], 1024), ([10, 5], 1024), ([4, 3], 500), ([10, 5], 1024)]:
        bufs = M.SampleBuffers.allocate(bsz, fanout, n, DEV)
        rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
        for b in range(3):
            seeds = batches[b][:bsz]
            rng = W.batch_rng_seed(5, 0, 0, b * 7 + bsz)
            ctx.step(g.indptr, g.indices, seeds, fanout, rng, bufs, rows)
            torch.cuda.synchronize()
            got = bufs.result()
            want = orc.sample(ip, ix, seeds.cpu().numpy(), fanout, rng)
            assert_same_sample(got, want)
            nF = int(want["counts"][len(fanout)])
            assert np.array_equal(rows[:nF].cpu().numpy(), orc.gather(tab, want["nodes"]))


def test_moment_step_many_in_flight(orc, c1):
    """Several steps enqueued back to back on one ctx/stream (call-block ring in use) stay exact."""
    cfg, g = c1
    n = g.n
    ctx = M.Ctx(n_vertices=n, max_seeds=256, max_fanout=[6, 3], device=0)
    train = W.training_set(g, min_count=256 * 80)
    batches = W.epoch_batches(train, 256, 0)[:80]
    bufs = [M.SampleBuffers.allocate(256, [6, 3], n, DEV) for _ in batches]
    for b, seeds in enumerate(batches):  # 80 > ring size: exercises slot reuse
        ctx.step(g.indptr, g.indices, seeds, [6, 3], 1000 + b, bufs[b], None)
    torch.cuda.synchronize()
    ip, ix = g.indptr.cpu().numpy(), g.indices.cpu().numpy()
    for b in [0, 1, 40, 63, 64, 65, 79]:
        want = orc.sample(ip, ix, batches[b].cpu().numpy(), [6, 3], 1000 + b)
        assert_same_sample(bufs[b].result(), want)


@pytest.mark.parametrize("name", ["C3"])
def test_full_size_config_sample_and_gather(orc, name):
    """BASELINE config at full size (C3: 111 M vertices, 1.6 B edges, 57 GB of 128-d fp32 features in
    HBM): one batch of the bench's shape, whole-sample parity with the oracle and every gathered row of the
    gather checked against the feature generator."""
    _need_gpu()
    cfg = W.CONFIGS[name]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    torch.cuda.empty_cache()
    fan = list(cfg["fanout"])
    train = W.training_set(g, min_count=cfg["batch"])
    seeds = W.epoch_batches(train, cfg["batch"], 0)[0]
    table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device=DEV)
    R = table.shape[1]
    ctx = M.Ctx(n_vertices=g.n, max_seeds=cfg["batch"], max_fanout=fan, device=0, row_bytes=R, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    bufs = M.SampleBuffers.allocate(cfg["batch"], fan, g.n, DEV)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
    rng = W.batch_rng_seed(11, 0, 0, 0)
    ctx.step(g.indptr, g.indices, seeds, fan, rng, bufs, rows)
    torch.cuda.synchronize()
    got = bufs.result()
    want = orc.sample(g.indptr.cpu().numpy(), g.indices.cpu().numpy(), seeds.cpu().numpy(), fan, rng)
    assert_same_sample(got, want)
    nF = int(want["counts"][len(fan)])
    assert_all_rows(rows[:nF], want["nodes"], cfg["dim"], cfg["dtype"])
    del table, g, rows
    torch.cuda.empty_cache()


@pytest.mark.parametrize("name,cache_gib", [("C4", 32), ("C5", 64)])
def test_full_size_tiered_gather(orc, name, cache_gib):
    """C4 / C5 at full graph size (244 M vertices / 1.73 B edges, 768-d fp16; 269 M / 4.0 B edges, 1024-d
    fp32): whole-sample parity, then the tiered gather: the hottest vertices (pre-sampling hotness,
    moment_place DDAK) in a C4: 32 GiB / C5: 64 GiB HBM cache, every other row read zero-copy from pinned
    host DRAM. The features (375 GB / 1.1 TB) exceed the host, so the host tier is a ring of R_phys
    physical rows and row(v) := feature(v mod R_phys) for every tier (SURVEY §8(d) fallback); the checked
    bytes still cross PCIe."""
    _need_gpu()
    cfg = W.CONFIGS[name]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    torch.cuda.empty_cache()
    n, fan, B = g.n, list(cfg["fanout"]), cfg["batch"]
    R = cfg["dim"] * torch.empty(0, dtype=cfg["dtype"]).element_size()
    R_phys = 1 << 22
    chunk = max(1, (1 << 31) // (R // 4 * 8))  # rows per feature_rows call (bounded temporaries)
    train = W.training_set(g, min_count=B * 8)
    batches = W.epoch_batches(train, B, 0)
    ctx0 = M.Ctx(n_vertices=n, max_seeds=B, max_fanout=fan, device=0)
    bufs = M.SampleBuffers.allocate(B, fan, n, DEV)
    hot = torch.zeros(n, dtype=torch.int64, device=DEV)
    for b in range(4):  # P2: pre-sampling hotness
        ctx0.step(g.indptr, g.indices, batches[b], fan, W.batch_rng_seed(3, 99, 0, b), bufs, None)
        ctx0.hotness(bufs.nodes, hot, n_dev=bufs.counts[3:4], max_n=bufs.nodes.numel())
    cap_hbm = (cache_gib << 30) // R
    bin_of, slot_of, *_ = M.place(None, hot.cpu().numpy().astype(np.uint64), [cap_hbm, n], bin_tier=[1, 2],
                                  bin_traffic=[6_469_000, 55_000])
    del hot
    host = bin_of == 1
    slot_of[host] = np.nonzero(host)[0] % R_phys  # ring host tier
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=DEV)
    in_hbm = np.nonzero(~host)[0]
    hbm_v = torch.as_tensor(in_hbm[np.argsort(slot_of[in_hbm])], device=DEV)
    del in_hbm
    hbm = torch.empty((max(1, len(hbm_v)), R), dtype=torch.uint8, device=DEV)
    for c0 in range(0, len(hbm_v), chunk):
        hbm[c0:c0 + chunk] = W.feature_rows(hbm_v[c0:c0 + chunk] % R_phys, cfg["dim"], cfg["dtype"])
    del hbm_v
    ring = torch.empty((R_phys, R), dtype=torch.uint8).pin_memory()
    for c0 in range(0, R_phys, chunk):
        ids = torch.arange(c0, min(R_phys, c0 + chunk), device=DEV)
        ring[c0:c0 + len(ids)] = W.feature_rows(ids, cfg["dim"], cfg["dtype"]).cpu()
    ctx = M.Ctx(n_vertices=n, max_seeds=B, max_fanout=fan, device=0, row_bytes=R, bin_owner=[0, -1],
                bin_ptr=[hbm.data_ptr(), ring.data_ptr()], placement=placement)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
    ip, ix = g.indptr.cpu().numpy(), g.indices.cpu().numpy()
    for b in (5, 6):
        rng = W.batch_rng_seed(3, 0, 0, b)
        ctx.sample(g.indptr, g.indices, batches[b], fan, rng, bufs)
        ctx.gather(bufs.nodes, rows, n_dev=bufs.counts[3:4], max_n=bufs.nodes.numel())
        torch.cuda.synchronize()
        got = bufs.result()
        want = orc.sample(ip, ix, batches[b].cpu().numpy(), fan, rng)
        assert_same_sample(got, want)
        nF = int(want["counts"][len(fan)])
        assert_all_rows(rows[:nF], want["nodes"], cfg["dim"], cfg["dtype"], mod=R_phys)
        frac_hbm = (bin_of[want["nodes"]] == 0).mean()
        assert 0.0 < frac_hbm < 1.0  # both tiers exercised
    del hbm, ring, g, rows
    torch.cuda.empty_cache()


@pytest.mark.parametrize("world", [2, 4])
def test_gather_replicated_hot_rows_per_rank_maps(orc, c1, world):
    """R25: the hottest rows replicated in every rank's HBM bin, the rest DDAK-partitioned over the HBM bins
    and a pinned host bin. Each rank's device map (moment_place_pack_rank) points replicas at its OWN bin:
    byte-exact rows, replicas routed to the local queue, and the replica regions of every other bin
    poisoned while a rank gathers (a replica read from a peer bin would show)."""
    cfg, g = c1
    n = g.n
    table = W.feature_table(n, 32, torch.float32, device=DEV)  # 128-byte rows
    R = table.shape[1]
    rng = np.random.default_rng(7 + world)
    hot = (rng.pareto(0.9, n) * 4).astype(np.uint64)
    r = n // 16
    owners = list(range(world)) + [-1]
    tiers = [M.TIER_GPU_HBM] * world + [M.TIER_HOST_DRAM]
    caps = [r + n // (4 * world)] * world + [n]
    bin_of, slot_of, A, U, T = M.place(None, hot, caps, bin_tier=tiers, bin_traffic=[100] * world + [10],
                                       replicate_rows=r)
    ob, os_, *_ = orc.ddak_replicate(hot, np.array(tiers) - 1, caps, [100] * world + [10], r, 100)
    assert np.array_equal(bin_of, ob) and np.array_equal(slot_of, os_)
    t_cpu = table.cpu()
    rep = np.where(bin_of == M.BIN_REPLICA)[0]
    bins = []
    for b in range(world + 1):
        sel = np.where(bin_of == b)[0]
        rows = r + int(U[b]) if b < world else max(1, int(U[b]))
        buf = torch.zeros((rows, R), dtype=torch.uint8)
        buf[torch.as_tensor(slot_of[sel])] = t_cpu[torch.as_tensor(sel)]
        if b < world:
            buf[torch.as_tensor(slot_of[rep])] = t_cpu[torch.as_tensor(rep)]
            bins.append(buf.to(DEV))
        else:
            bins.append(buf.pin_memory())
    train = W.training_set(g, min_count=1024 * world)
    tab = table.cpu().numpy()
    n_rep_seen = 0
    for rank in range(world):
        placement = torch.as_tensor(M.place_pack_rank(bin_of, slot_of, rank).view(np.int64), device=DEV)
        ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=[10, 5], rank=rank, world=world, device=0,
                    row_bytes=R, bin_owner=owners, bin_ptr=[b.data_ptr() for b in bins], placement=placement)
        seeds = W.epoch_batches(train, 1024, 0, rank=rank, world=world)[0]
        bufs = M.SampleBuffers.allocate(1024, [10, 5], n, DEV)
        ctx.sample(g.indptr, g.indices, seeds, [10, 5], 90 + rank, bufs)
        nF = int(bufs.counts[2])
        ids = bufs.nodes[:nF].clone()
        ids_np = ids.cpu().numpy()
        # routing: replicas to this rank's own bin queue, everything else as the oracle routes it
        route = torch.empty(nF, dtype=torch.int32, device=DEV)
        qoff = torch.empty((world + 1) * world + 1, dtype=torch.int64, device=DEV)
        qpos = torch.empty(nF, dtype=torch.int64, device=DEV)
        ctx.bucket(ids, route, qoff, qpos)
        eff_bin = np.where(bin_of[ids_np] == M.BIN_REPLICA, rank, bin_of[ids_np])
        o_route, o_qoff, o_qpos = orc.bucket(rank, world, owners, np.zeros((world + 1, world), np.int64), eff_bin)
        assert np.array_equal(route.cpu().numpy(), o_route)
        is_rep = bin_of[ids_np] == M.BIN_REPLICA
        n_rep_seen += int(is_rep.sum())
        assert (route.cpu().numpy()[is_rep] == rank * world + rank).all()
        # poison the replica region of every other rank's bin
        for b in range(world):
            if b != rank:
                bins[b][:r].fill_(0xAB)
        out = torch.zeros((nF, R), dtype=torch.uint8, device=DEV)
        ctx.gather(ids, out)
        torch.cuda.synchronize()
        assert np.array_equal(out.cpu().numpy(), orc.gather(tab, ids_np)), rank
        for b in range(world):
            if b != rank:
                bins[b][:r] = t_cpu[torch.as_tensor(rep)].to(DEV)[torch.as_tensor(np.argsort(slot_of[rep]))]
        del ctx
    assert n_rep_seen > 0


def test_near_maximum_frontier_uniform_graph(orc):
    """Workspace bounds at (nearly) their maximum: a uniform random graph with 2^24 vertices and 16 distinct-ish
    out-neighbours each has almost no overlap between frontiers, so one batch of the bench's shape (1024 seeds,
    [15, 10, 5]) comes close to the no-dedup bound 1 081 344 (R-MAT batches stay near 121 k): whole-sample
    parity with the oracle, the padded sampler buffers and the compaction tiles at their largest, the gather of
    ~0.94 M rows (375 MB) checked on a sample of rows, in both bitscan modes."""
    _need_gpu()
    n, deg = 1 << 24, 16
    gen = torch.Generator(device=DEV)
    gen.manual_seed(2024)
    indices = torch.randint(0, n, (n * deg,), device=DEV, generator=gen, dtype=torch.int64)
    indices = indices.view(n, deg).sort(dim=1).values.reshape(-1).to(torch.int32)
    indptr = torch.arange(0, n * deg + 1, deg, device=DEV, dtype=torch.int64)
    fan = [15, 10, 5]
    seeds = torch.randperm(n, device=DEV, generator=gen)[:1024]
    dim = 100
    rows_needed = 1024 * 16 * 11 * 6
    table = W.feature_table(n, dim, torch.float32, device=DEV)
    R = table.shape[1]
    ip, ix = indptr.cpu().numpy(), indices.cpu().numpy()
    want = orc.sample(ip, ix, seeds.cpu().numpy(), fan, 4242)
    nF = int(want["counts"][3])
    # every node of F_h is resampled at hop h (R4), so earlier nodes mostly re-pick neighbours already in the
    # batch: ~0.94 M here, 7.8x an R-MAT batch, 87 % of the no-dedup bound
    assert nF > 900_000 and nF <= rows_needed
    for sparse in ("0", "1"):
        import os
        os.environ["MOMENT_SPARSE_SCAN"] = sparse
        try:
            ctx = M.Ctx(n_vertices=n, max_seeds=1024, max_fanout=fan, device=0, row_bytes=R, bin_owner=[0],
                        bin_ptr=[table.data_ptr()])
        finally:
            del os.environ["MOMENT_SPARSE_SCAN"]
        bufs = M.SampleBuffers.allocate(1024, fan, n, DEV)
        rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
        ctx.step(indptr, indices, seeds, fan, 4242, bufs, rows)
        torch.cuda.synchronize()
        assert_same_sample(bufs.result(), want)
        assert_all_rows(rows[:nF], want["nodes"], dim, torch.float32)
        del ctx, bufs, rows
    del table, indices
    torch.cuda.empty_cache()
