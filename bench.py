"""Benchmark of the Moment hot path on B200: per-batch multi-hop sampling + feature gather.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--impl moment|reference]

One step = one pass of the whole hot path (sample H hops with dedup/relabel, then gather F_H's rows) over
one batch of 1024 seeds per GPU, inputs resident in HBM. N > 1: launched by torch.distributed.run, one
rank per GPU; seeds are sharded (weak scaling), every rank holds the replicated graph and features
(C2 "all features in HBM"), so the data path has no collective. Rank 0 prints ONE JSON line.

The `cpu_baseline` leg and `--impl reference` time the CPU oracle (oracle/, single-threaded C) on a
bounded sample of the same workload — the only places this file touches oracle/.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads as W  # noqa: E402

METRIC = "sampled+gathered seeds/sec and gather GB/s vs per-tier roofline, 1/2/4/8 B200"
RUN_SEED = 20251116


def _peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


LANE_STEPS = None  # steps per timed region (set by main before the lanes are built): see lane_streams
LANE_PRIO = None   # the lane priority mode lane_streams applied (reported in the JSON line's config)


def lane_streams(device, inflight):
    """One stream per lane. MOMENT_LANE_PRIO (default "auto"): "half" = the first half of the lanes on
    high-priority streams (their early, latency-bound hops get the SMs first, so their gathers start sooner and
    overlap the other half's sampling; +0.6 % at K = 200); "hi:N" = the first N lanes high; "auto" = "hi:K mod P"
    for a short region (K < 2P steps on P lanes: the K mod P lanes that run one batch more than the others, whose
    second batch ends the region, go first; K = 20, P = 16: 38.3 -> 38.9 M seeds/s), else "half"; "ramp" = a
    priority gradient (-0.7 %); "none": lane 0 on the current stream, no priorities."""
    mode = os.environ.get("MOMENT_LANE_PRIO", "auto")
    if mode == "auto":
        K = LANE_STEPS
        mode = f"hi:{K % inflight}" if (K is not None and K < 2 * inflight and K % inflight) else "half"
    global LANE_PRIO
    LANE_PRIO = mode
    if mode == "none":
        return [torch.cuda.current_stream(device)] + [torch.cuda.Stream(device) for _ in range(inflight - 1)]
    lo, hi = torch.cuda.Stream.priority_range() if hasattr(torch.cuda.Stream, "priority_range") else (0, -1)
    out = []
    levels = abs(hi - lo) + 1
    for i in range(inflight):
        if mode == "ramp":  # lane i gets the (i * levels / inflight)-th highest priority
            pr = hi + (1 if hi < lo else -1) * min(levels - 1, i * levels // inflight)
        else:
            n_high = int(mode[3:]) if mode.startswith("hi:") else None  # "hi:N": the first N lanes high
            high = ((mode == "half" and i < (inflight + 1) // 2) or (mode == "first" and i == 0)
                    or (n_high is not None and i < n_high))
            pr = hi if high else lo
        out.append(torch.cuda.Stream(device, priority=pr))
    return out


class Lane:
    """One batch in flight: its own device context (workspace), sample buffers, row buffer and stream."""

    def __init__(self, M, cfg, fanout, B, R, rank, world, device, table, stream):
        self.ctx = M.Ctx(n_vertices=cfg["n"], max_seeds=B, max_fanout=fanout, rank=rank, world=world,
                         device=torch.device(device).index or 0, row_bytes=R, row_stride=table.shape[1],
                         bin_owner=[rank],
                         bin_ptr=[table.data_ptr()])
        self.bufs = M.SampleBuffers.allocate(B, fanout, cfg["n"], device)
        self.rows = torch.empty((self.bufs.nodes.numel(), R), dtype=torch.uint8, device=device)
        self.stream = stream


class State:
    """Resident inputs of one rank for one config and `inflight` lanes (the bench and the full-size parity
    test). Every lane shares the replicated graph and feature table (C2: all features in HBM)."""

    def __init__(self, name, device, rank, world, inflight=1):
        import paper_conf_sc_shi0s0x0w25_b200 as M

        self.M = M
        cfg = W.CONFIGS[name]
        self.name, self.cfg = name, cfg
        self.device, self.rank, self.world = device, rank, world
        self.fanout = tuple(cfg["fanout"])
        self.B = cfg["batch"]
        self.dim, self.dtype = cfg["dim"], cfg["dtype"]
        self.graph = W.rmat_csr(cfg["n"], cfg["m"], device=device)
        # replicated, all in HBM; rows start on 64-byte boundaries (HBM burst) so a row costs ceil(R/64) bursts
        self.R = self.dim * torch.empty(0, dtype=self.dtype).element_size()
        self.stride = (self.R + 63) // 64 * 64
        self.table = W.feature_table(cfg["n"], self.dim, self.dtype, device=device, row_stride_bytes=self.stride)
        self.train = W.training_set(self.graph, min_count=self.B * world)
        streams = lane_streams(device, inflight)
        self.lanes = [Lane(M, cfg, self.fanout, self.B, self.R, rank, world, device, self.table, s) for s in streams]
        self.ctx, self.bufs, self.rows = self.lanes[0].ctx, self.lanes[0].bufs, self.lanes[0].rows
        self._batches = []
        self._epoch = 0

    def batch(self, i):
        """(seeds on device, per-batch rng seed) of this rank's i-th batch (cycling epochs)."""
        while i >= len(self._batches):
            self._batches += [(b, self._epoch, j) for j, b in
                              enumerate(W.epoch_batches(self.train, self.B, self._epoch, self.rank, self.world))]
            self._epoch += 1
        seeds, ep, j = self._batches[i]
        return seeds, W.batch_rng_seed(RUN_SEED, ep, self.rank, j)

    def step(self, seeds, rng_seed, stream=None, ev=None, lane=0):
        """Sample + gather one batch on `lane` (its stream unless `stream` is given): one moment_step call,
        replayed from the lane ctx's cached CUDA graph. With `ev` (a pair of timing events) the step runs as
        moment_sample + moment_gather with the events around the gather kernel instead."""
        H = len(self.fanout)
        L = self.lanes[lane]
        s = stream if stream is not None else L.stream
        if ev is None and stream is None:  # the lane's prepared moment_step (one ctypes call per step)
            self.bound(lane)(seeds, rng_seed)
            return
        if ev is None:
            L.ctx.step(self.graph.indptr, self.graph.indices, seeds, self.fanout, rng_seed, L.bufs, L.rows, stream=s)
            return
        L.ctx.sample(self.graph.indptr, self.graph.indices, seeds, self.fanout, rng_seed, L.bufs, stream=s)
        ev[0].record(s)
        L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(), stream=s)
        ev[1].record(s)

    def bound(self, lane, host=False):
        """The lane's moment_step (host: moment_step_host) prepared once on its stream (Ctx.bind_step)."""
        L = self.lanes[lane]
        key = "run_host" if host else "run"
        run = L.__dict__.get(key)
        if run is None:
            run = L.ctx.bind_step(self.graph.indptr, self.graph.indices, self.fanout, L.bufs, L.rows, stream=L.stream,
                                  host=host)
            setattr(L, key, run)
        return run

    def step_host(self, seeds_host, rng_seed, counts_host, lane=0):
        """The same step through moment_step_host: host seeds in, host counts out (asynchronous)."""
        self.bound(lane, host=True)(seeds_host, rng_seed, counts_host)

    def launches_per_step(self):
        # set_call, (sample, bitscan) per hop (the first hop's sampler also initialises the call), compact, gather
        return 1 + 2 * len(self.fanout) + 1 + 1


NVLINK_GBS = 770.0  # measured B200 peer copy per direction (B200_PROFILING.md; 900 GB/s nominal)
PORT_GBS = 55.6     # measured pinned H2D copy of a pool B200 (profiles/r02_probe.json; Gen5 x16 raw 63.0)
PRESAMPLE_EPOCH = 2**32 - 1  # R18: the pre-sample batches use their own rng stream


class PartState(State):
    """Resident inputs of one rank with the feature table PARTITIONED over the ranks' HBM (C3: "knapsack
    placement across 8 GPU caches, max-flow routed"): pre-sampled hotness (P2) summed over the
    ranks, DDAK placement (P4) over the k HBM bins of an HGX B200 topology graph with the rate max-flow's
    per-bin traffic (P3), optionally the hottest rows replicated in every bin (R25), and the plan's predicted
    per-batch time (P5). Each rank holds its own bin; the other ranks' bins are CUDA-IPC mapped, so a batch's
    peer rows are NVLink loads inside the gather kernel (no exchange: there is no host tier to relay)."""

    def __init__(self, name, device, rank, world, inflight, *, dist, shared, placement="ddak", presample=64,
                 replicate_frac=1 / 16, layout=None, cache_gib=32.0):
        import paper_conf_sc_shi0s0x0w25_b200 as M

        self.M = M
        cfg = W.CONFIGS[name]
        self.name, self.cfg = name, cfg
        self.device, self.rank, self.world = device, rank, world
        self.fanout = tuple(cfg["fanout"])
        self.B = cfg["batch"]
        H = len(self.fanout)
        self.dim, self.dtype = cfg["dim"], cfg["dtype"]
        for turn in range(world if shared else 1):  # ranks sharing one GPU (test mode) build one at a time
            if not shared or turn == rank:
                self.graph = W.rmat_csr(cfg["n"], cfg["m"], device=device)
                torch.cuda.empty_cache()
            if shared and dist is not None:
                dist.barrier()
        n = self.graph.n
        self.R = self.dim * torch.empty(0, dtype=self.dtype).element_size()
        self.stride = (self.R + 63) // 64 * 64
        self.train = W.training_set(self.graph, min_count=self.B * world)
        dev_idx = torch.device(device).index or 0
        t0 = time.perf_counter()
        # P2: pre-sampling hotness, every rank its own seeds, counts summed over the ranks
        ctx0 = M.Ctx(n_vertices=n, max_seeds=self.B, max_fanout=self.fanout, rank=rank, world=world, device=dev_idx)
        bufs0 = M.SampleBuffers.allocate(self.B, self.fanout, n, device)
        hot = torch.zeros(n, dtype=torch.int64, device=device)
        pre = W.epoch_batches(self.train, self.B, PRESAMPLE_EPOCH, rank, world)
        for b in range(presample):
            ctx0.step(self.graph.indptr, self.graph.indices, pre[b % len(pre)], self.fanout,
                      W.batch_rng_seed(RUN_SEED, PRESAMPLE_EPOCH, rank, b), bufs0, None)
            ctx0.hotness(bufs0.nodes, hot, n_dev=bufs0.counts[H:H + 1], max_n=bufs0.nodes.numel())
        if dist is not None:
            if shared:
                h_cpu = hot.cpu()
                dist.all_reduce(h_cpu)
                hot.copy_(h_cpu)
            else:
                dist.all_reduce(hot)
        hot_np = hot.cpu().numpy().astype(np.uint64)
        del hot, ctx0, bufs0
        self.t_hotness = time.perf_counter() - t0
        # P1/P3/P4: topology graph of the box, DDAK over the k HBM bins (rate max-flow traffic, R17a)
        if world > 8:
            raise SystemExit("partitioned placement: at most 8 GPUs (one HGX node)")
        active = M.boxes.spread_gpus(world) if world in (1, 2, 4, 8) else list(range(world))
        hbm_gbs = _peaks()[0]
        box = M.boxes.hgx_b200(8, hbm_gbs=hbm_gbs, active=active)
        topo = box.topology()
        tiered = placement == "ddak-tiered"
        bin_node = [box.hbm_bin[g] for g in active] + (box.host_bin if tiered else [])
        r = int(n * replicate_frac) if placement == "ddak-rep" and world > 1 else 0
        if tiered:  # a cache_gib HBM cache per GPU, the rest in one host-DRAM bin per socket (C4 / C5)
            cap = min(n, int(cache_gib * (1 << 30)) // self.stride)
            caps = [cap] * world + [n] * len(box.host_bin)
        else:
            cap = r + -(-(n - r) // world)
            caps = [cap] * world
        t1 = time.perf_counter()
        bin_of, slot_of, A, U, T, rep_acc = M.place(topo, hot_np, caps, bin_node=bin_node,
                                                   replicate_rows=r, traffic_mode=M.TRAFFIC_STANDALONE,
                                                   return_replica_access=True)
        self.t_place = time.perf_counter() - t1
        # host bins hold a ring of r_phys rows (SURVEY 8(d) fallback: the C4 / C5 tables exceed the host), so every
        # tier stores row(v) := feature(v mod r_phys) and a host row of v sits at slot v mod r_phys
        self.r_phys = min(n, 1 << 22) if tiered else n
        if tiered:
            host = bin_of >= world
            slot_of[host] = np.nonzero(host)[0] % self.r_phys
        if layout:  # plan reuse: rank 0 saves the layout; a saved one must match what DDAK recomputed
            if os.path.exists(layout):
                saved = M.layout.load(layout, topo)
                if not (np.array_equal(saved["bin_of"], bin_of) and np.array_equal(saved["slot_of"], slot_of)):
                    raise SystemExit(f"{layout}: saved layout differs from this run's placement")
            elif rank == 0:
                M.layout.save(layout, topo, bin_of=bin_of, slot_of=slot_of, bin_node=bin_node,
                              capacity_rows=caps, replicate_rows=r, note=f"{name} {placement} k={world}")
        # P5: the plan's predicted per-batch time for this layout (in-sample demand per GPU per batch)
        N = topo.info()[0]
        d = np.zeros(N, np.int64)
        for i, v in enumerate(bin_node):
            d[v] = int(A[i]) * self.R // (presample * world)
        self.plan = M.plan(topo, [box.gpu[g] for g in active], d, int(NVLINK_GBS * 1000), int(hbm_gbs * 1000),
                           replica_demand=int(rep_acc) * self.R // (presample * world)).info()
        self.placement_mode, self.replicated_rows = placement, r
        self.bin_rows = [int(x) for x in U]
        self.n_bins = len(bin_node)
        # quota x[j][h] of every host bin (the plan's path decomposition, rank order = active order): the share
        # of this rank's bin-j rows read over GPU h's PCIe port and relayed to it (R11, R12)
        quota = np.zeros((self.n_bins, world), np.int64)
        for i, v in enumerate(bin_node):
            if i >= world:
                quota[i] = self.plan["quota"][v]
        self.quota = quota
        # this rank's HBM bin: replicas at slots 0..r-1, then its partition
        mine = np.nonzero((bin_of == rank) | (bin_of == M.BIN_REPLICA))[0]
        rows_mine = r + int(U[rank])
        self.table = torch.zeros((max(1, rows_mine), self.stride), dtype=torch.uint8, device=device)
        ch = 1 << 20
        for c0 in range(0, len(mine), ch):
            ids = torch.as_tensor(mine[c0:c0 + ch], device=device)
            sl = torch.as_tensor(slot_of[mine[c0:c0 + ch]], device=device)
            self.table[sl, :self.R] = W.feature_rows(ids % self.r_phys, self.dim, self.dtype)
        del mine
        self.host_bins = []
        if tiered:  # every rank pins its own copy of the host rings (each rank reads them over its own port)
            for _ in box.host_bin:
                h = torch.empty((self.r_phys, self.stride), dtype=torch.uint8).pin_memory()
                for c0 in range(0, self.r_phys, ch):
                    c1 = min(self.r_phys, c0 + ch)
                    blk = torch.zeros((c1 - c0, self.stride), dtype=torch.uint8, device=device)
                    blk[:, :self.R] = W.feature_rows(torch.arange(c0, c1, device=device), self.dim, self.dtype)
                    h[c0:c1].copy_(blk)
                self.host_bins.append(h)
        packed = M.place_pack_rank(bin_of, slot_of, rank) if r else M.place_pack(bin_of, slot_of)
        self.placement = torch.as_tensor(packed.view(np.int64), device=device)
        del packed, bin_of, slot_of
        # peer bins: CUDA IPC (NVLink peer pointers between the GPUs of one node)
        self._imported = []
        ptrs = [0] * world
        ptrs[rank] = self.table.data_ptr()
        if world > 1:
            mine_h = M.ipc_export(self.table)
            allh = [None] * world
            dist.all_gather_object(allh, mine_h)
            for h in range(world):
                if h != rank:
                    base = M.ipc_import(allh[h][0])
                    self._imported.append(base)
                    ptrs[h] = base + allh[h][1]
        streams = lane_streams(device, inflight)
        self.lanes = []
        self.exchanges = []
        owners = list(range(world)) + [-1] * len(self.host_bins)
        ptrs = ptrs + [h.data_ptr() for h in self.host_bins]
        for s_ in streams:
            L = Lane.__new__(Lane)
            L.ctx = M.Ctx(n_vertices=n, max_seeds=self.B, max_fanout=self.fanout, rank=rank, world=world,
                          device=dev_idx, row_bytes=self.R, row_stride=self.stride, bin_owner=owners,
                          bin_ptr=ptrs, placement=self.placement, quota=self.quota if tiered else None)
            L.bufs = M.SampleBuffers.allocate(self.B, self.fanout, n, device)
            if tiered and world > 1:
                # relays through other ranks: this lane's batch is ONE collective moment_step (the relay exchange
                # inside it; moment_ctx_set_exchange), into the exchange's registered output
                from paper_conf_sc_shi0s0x0w25_b200.exchange import PeerExchange

                px = PeerExchange(L.ctx, L.bufs.nodes.numel(), self.R, device, timeout_s=60.0)
                self.exchanges.append(px)
                L.rows = px.out
            else:
                L.rows = torch.empty((L.bufs.nodes.numel(), self.R), dtype=torch.uint8, device=device)
            L.stream = s_
            self.lanes.append(L)
        self.ctx, self.bufs, self.rows = self.lanes[0].ctx, self.lanes[0].bufs, self.lanes[0].rows
        self._batches = []
        self._epoch = 0

    def bins_of(self, nodes, nF):
        """Rows of a batch per owning bin (measurement bookkeeping, after the timed region)."""
        b = torch.bitwise_right_shift(self.placement[nodes[:nF]], 40)
        return torch.bincount(b, minlength=self.world)

    def queues_of(self, nodes, nF):
        """Rows of a batch per route queue q = bin * world + via (moment_bucket: HBM bins via their owner, host
        bins via the quota's relay rank), for the per-tier accounting after the timed region."""
        M, dev = self.M, nodes.device
        Q = self.n_bins * self.world
        route = torch.empty(max(1, nF), dtype=torch.int32, device=dev)
        qoff = torch.empty(Q + 1, dtype=torch.int64, device=dev)
        qpos = torch.empty(max(1, nF), dtype=torch.int64, device=dev)
        self.lanes[0].ctx.bucket(nodes, route, qoff, qpos, max_n=nF)
        return qoff[1:] - qoff[:-1]

    def close(self, dist):
        torch.cuda.synchronize()
        if dist is not None:
            dist.barrier()
        for px in self.exchanges:
            px.close()
        self.exchanges = []
        for base in self._imported:
            self.M.ipc_close(base)
        self._imported = []


def feature_check_ids(st, nodes):
    """Ids whose generated bytes a gathered row must equal (tiered layouts store feature(v mod r_phys))."""
    r_phys = getattr(st, "r_phys", None)
    return nodes % r_phys if r_phys else nodes


def build_state(name, device="cuda:0", rank=0, world=1, inflight=1, **kw):
    if kw.get("placement", "replicated") != "replicated":
        return PartState(name, device, rank, world, inflight, **kw)
    return State(name, device, rank, world, inflight)


class Clocks:
    """nvidia-smi clock / throttle sampling during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(index), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                       "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None

    def stop(self):
        if self.p is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.p.terminate()
        out, _ = self.p.communicate(timeout=10)
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in out.strip().splitlines():
            f = [x.strip() for x in line.split(",")]
            if len(f) < 8:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n_, v in zip(names, f[4:8]):
                if v.lower().startswith("active"):
                    reasons.add(n_)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def host_info():
    """CPU model, logical core count and one NUMA-0 core for the single-threaded oracle."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.startswith("Model name:"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    allowed = sorted(os.sched_getaffinity(0))
    node0 = None
    try:
        with open("/sys/devices/system/node/node0/cpulist") as f:
            node0 = set()
            for part in f.read().strip().split(","):
                a, _, b = part.partition("-")
                node0.update(range(int(a), int(b or a) + 1))
    except Exception:
        node0 = None
    cand = [c for c in allowed if node0 is None or c in node0] or allowed
    # the last allowed core of NUMA node 0 (core 0 tends to take the interrupts)
    return {"cpu_model": model, "os_cpu_count": os.cpu_count(), "allowed_cores": len(allowed),
            "core": cand[-1], "core_numa0": node0 is not None and cand[-1] in node0}


class PinnedCore:
    """Pin the calling thread to one core (the oracle's C code runs on it; `taskset -c core` in-process)."""

    def __init__(self, core):
        self.core = core

    def __enter__(self):
        self.old = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {self.core})
        return self

    def __exit__(self, *exc):
        os.sched_setaffinity(0, self.old)


def parity_subset(n_batches: int) -> list[int]:
    """the first 2 batches of the rank + 1 batch chosen by a counter hash."""
    first = list(range(min(2, n_batches)))
    if n_batches > 2:
        j = 2 + W.mix(RUN_SEED, 0xC0FFEE) % (n_batches - 2)
        first.append(int(j))
    return first


def oracle_baseline(st, pool, budget_s=10.0):
    """The CPU oracle as it stands (oracle/, single-threaded C, pinned to one NUMA-0 core) on a bounded
    sample of the bench's own batches: first the parity subset, each of which is also compared
    bit-exactly with the CUDA path's output for the same batch, then further batches of the pool until
    `budget_s` seconds of oracle time have been spent."""
    import oracle

    oracle.build()
    info = host_info()
    H = len(st.fanout)
    indptr = st.graph.indptr.cpu().numpy()
    indices = st.graph.indices.cpu().numpy()
    table = np.ascontiguousarray(st.table[:, :st.R].cpu().numpy())
    fan = list(st.fanout)
    subset = parity_subset(len(pool))
    # the parity subset first, then the pool in order, cycled until the budget is spent
    order = subset + [i % len(pool) for i in range(100 * len(pool)) if i >= len(pool) or i not in subset]
    t, seeds_done, n_b, checked = 0.0, 0, 0, []
    L = st.lanes[0]
    with PinnedCore(info["core"]):
        for i in order:
            seeds, rs = pool[i]
            s_np = seeds.cpu().numpy()
            t0 = time.perf_counter()
            r = oracle.sample(indptr, indices, s_np, fan, rs)
            rows = oracle.gather(table, r["nodes"])
            t += time.perf_counter() - t0
            seeds_done += len(s_np)
            n_b += 1
            if i in subset and i not in checked:
                # the CUDA path on the same batch (lane 0): every output compared, rows in full
                st.step(seeds, rs, lane=0)
                torch.cuda.synchronize()
                got = L.bufs.result()
                nF = int(r["counts"][H])
                ok = (np.array_equal(got["counts"], r["counts"]) and np.array_equal(got["nodes"], r["nodes"])
                      and all(np.array_equal(got["offsets"][h], r["offsets"][h]) and
                              np.array_equal(got["src"][h], r["src"][h]) for h in range(H))
                      and np.array_equal(L.rows[:nF].cpu().numpy(), rows.view(np.uint8).reshape(nF, -1)))
                if not ok:
                    raise AssertionError(f"bench batch {i}: CUDA path differs from the oracle")
                checked.append(i)
            if t >= budget_s and len(checked) == len(subset):
                break
    return {"value": seeds_done / t, "unit": "seeds/s", "cores": 1, "kind": "oracle",
            "sample": f"{n_b} batches x {st.B} seeds of {st.name} (the bench's own batches: parity subset "
                      f"{subset} first, then the pool in order, cycled, until {budget_s:g} s), sample + gather, "
                      f"single thread pinned to core {info['core']}",
            "host": info,
            "parity": {"batches": checked, "bit_exact": True,
                       "compared": "counts, F_H, per-hop offsets and src, every gathered row byte"}}


def partition_parity(st, pool):
    """Partitioned placement (no host copy of the table): the parity subset's samples are compared with the
    oracle's and every gathered row with its generated bytes (the oracle's gather is out[i] = table[ids[i]] with
    table[v] = featgen(v)); the oracle is timed on sampling only."""
    import oracle

    oracle.build()
    info = host_info()
    H = len(st.fanout)
    indptr = st.graph.indptr.cpu().numpy()
    indices = st.graph.indices.cpu().numpy()
    subset = parity_subset(len(pool))
    L = st.lanes[0]
    t, done = 0.0, 0
    with PinnedCore(info["core"]):
        for i in subset:
            seeds, rs = pool[i]
            t0 = time.perf_counter()
            r = oracle.sample(indptr, indices, seeds.cpu().numpy(), list(st.fanout), rs)
            t += time.perf_counter() - t0
            done += len(seeds)
            st.step(seeds, rs, lane=0)
            torch.cuda.synchronize()
            got = L.bufs.result()
            nF = int(r["counts"][H])
            ok = (np.array_equal(got["counts"], r["counts"]) and np.array_equal(got["nodes"], r["nodes"])
                  and all(np.array_equal(got["offsets"][h], r["offsets"][h]) and
                          np.array_equal(got["src"][h], r["src"][h]) for h in range(H)))
            ids = feature_check_ids(st, torch.as_tensor(r["nodes"], device=L.rows.device))
            for c0 in range(0, nF, 1 << 18):
                ok &= bool(torch.equal(L.rows[c0:min(nF, c0 + (1 << 18))],
                                       W.feature_rows(ids[c0:c0 + (1 << 18)], st.dim, st.dtype)))
            if not ok:
                raise AssertionError(f"bench batch {i}: CUDA path differs from the oracle")
    return {"value": done / t, "unit": "seeds/s (sampling only)", "cores": 1, "kind": "oracle",
            "sample": f"parity subset {subset} of {st.name}: oracle sampling timed (the partitioned table has no "
                      f"host copy to gather from), single thread pinned to core {info['core']}",
            "host": info,
            "parity": {"batches": subset, "bit_exact": True,
                       "compared": "counts, F_H, per-hop offsets and src; every gathered row vs its generated bytes"}}


def profile_summary(name):
    """The committed ncu summary of the gather kernel for `name` (per-launch DRAM bytes, launch shares)."""
    path = os.path.join(ROOT, "profiles", "ncu_gather_summary.json")
    try:
        with open(path) as f:
            return json.load(f).get(name, {})
    except Exception:
        return {}


# The sampler's bound is the DRAM random-access rate, not bytes: the random 64-byte atoms a batch must touch
# (indptr line per frontier node + distinct chunks of `indices` holding the chosen positions; tools/sampler_chunks.py,
# mean of 8 batches) and the measured rate of random loads (tools/exp_ld_granularity.cu, ld.global.nc.L2::64B).
SAMPLER_ATOMS = {"C2": (267750, "profiles/r02_sampler_chunks.txt"), "C3": (368168, "profiles/r02_sampler_chunks_C3.txt")}
ATOM_RATE = 36.96e9  # random loads/s, profiles/r02_sampler_experiments.txt


def step_floor(name, gather_bytes, peak_gbs, step_ms):
    """A floor for the whole step with sampling and gathering sharing DRAM: the gather's algorithmic bytes at the
    copy peak plus the sampler's random atoms at the random-access rate (null for configs without an atom count)."""
    if name not in SAMPLER_ATOMS:
        return None
    atoms, src = SAMPLER_ATOMS[name]
    g_us = gather_bytes / (peak_gbs * 1e9) * 1e6
    s_us = atoms / ATOM_RATE * 1e6
    return {"gather_us": g_us, "sampler_atoms": atoms, "atom_rate_G_per_s": ATOM_RATE / 1e9, "sampler_us": s_us,
            "floor_us": g_us + s_us, "step_us": step_ms * 1e3, "frac": (g_us + s_us) / (step_ms * 1e3),
            "how": f"gather alg bytes / copy peak + sampler random 64-byte atoms ({src}) / random-access rate; "
                   "frac = floor / the median region's time per step"}


def profile_traffic(name):
    """Per-launch DRAM bytes of the gather kernel from the committed ncu --set full summary, if any."""
    return profile_summary(name).get("dram_bytes_per_launch")


def run_reference(args, rank, world):
    """The tier's reference arm: the CPU oracle as it stands, on the host cores, same config/metric/unit.
    Under torchrun only rank 0 works; the other ranks exit 0."""
    if rank != 0:
        return
    cfg = W.CONFIGS[args.config]
    total_steps = args.steps + args.warmup
    # each step is a bounded slice of a batch so that the whole run stays within a few minutes
    budget = float(os.environ.get("MOMENT_REF_BUDGET_S", "150"))
    import oracle

    oracle.build()
    info = host_info()
    g = W.rmat_csr(cfg["n"], cfg["m"], device="cpu")
    indptr, indices = g.indptr.numpy(), g.indices.numpy()
    table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device="cpu").numpy()
    train = W.training_set(g, min_count=cfg["batch"])
    batches = W.epoch_batches(train, cfg["batch"], 0)
    fan = list(cfg["fanout"])
    with PinnedCore(info["core"]):
        t0 = time.perf_counter()
        r = oracle.sample(indptr, indices, batches[0][:16].numpy(), fan, 1)
        oracle.gather(table, r["nodes"])
        per_seed = (time.perf_counter() - t0) / 16
        s_per_step = int(max(1, min(cfg["batch"], budget / max(total_steps, 1) / max(per_seed, 1e-9))))
        t_meas, seeds_done = 0.0, 0
        for i in range(total_steps):
            seeds = batches[i % len(batches)][:s_per_step].numpy()
            t0 = time.perf_counter()
            r = oracle.sample(indptr, indices, seeds, fan, W.batch_rng_seed(RUN_SEED, 0, 0, i))
            oracle.gather(table, r["nodes"])
            dt = time.perf_counter() - t0
            if i >= args.warmup:
                t_meas += dt
                seeds_done += len(seeds)
    val = seeds_done / t_meas
    line = {"metric": METRIC, "value": val, "unit": "seeds/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": 1000 * t_meas / max(args.steps, 1), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": args.config, "desc": cfg["desc"], "global_batch": cfg["batch"],
                       "seeds_per_step": s_per_step, "fanout": fan, "parallelism": "oracle, 1 thread"},
            "impl": "reference",
            "cpu_baseline": {"value": val, "unit": "seeds/s", "cores": 1, "kind": "oracle",
                             "sample": f"{s_per_step} seeds per step x {args.steps} steps of {args.config}, "
                                       f"sample + gather, single thread pinned to core {info['core']}",
                             "host": info},
            "e2e": {"value": val, "unit": "seeds/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def spawn_ranks(n):
    """`bench.py --gpus N` outside torchrun: re-launch this command under torch.distributed.run, one rank per
    GPU on 127.0.0.1 (the driver's own N>1 launch sets WORLD_SIZE and never reaches this)."""
    import socket

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__)] + sys.argv[1:]
    os.execv(sys.executable, cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200, help="K: steps per timed region (exactly K batches per GPU)")
    ap.add_argument("--warmup", type=int, default=5, help="W: untimed warm-up steps per in-flight lane")
    ap.add_argument("--min-time", type=float, default=1.0,
                    help="seconds of timed regions: the K-step region is repeated (each bracketed by barrier + "
                         "synchronize) until this much device time is covered, and the median region is reported")
    ap.add_argument("--e2e-min-time", type=float, default=0.5)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="moment", choices=["moment", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0, help="seconds of oracle time for cpu_baseline")
    # 12-16 measured best on C2 (29.5-29.7 M seeds/s vs 27.7 at 8, 28.4 at 24)
    ap.add_argument("--inflight", type=int, default=0,
                    help="batches in flight per GPU (one stream each); 0 = auto: 16 for short regions (K <= 24: "
                         "fill and drain dominate, 20 lanes lose 1 %% at K = 20), 32 for longer ones when a lane's row "
                         "buffer is small (C2 K = 200: 38.8 vs 37.8 M seeds/s at 16), else 16")
    ap.add_argument("--placement", default="replicated", choices=["replicated", "ddak", "ddak-rep", "ddak-tiered"],
                    help="replicated: every GPU holds the whole table (C2 'all features in HBM'); ddak: the table "
                         "partitioned over the GPUs' HBM by DDAK (C3), peer rows read over NVLink; ddak-rep: the "
                         "same with the hottest --replicate-frac of the rows in every GPU (R25); ddak-tiered: a "
                         "--cache-gib HBM cache per GPU and one pinned host bin per socket (C4 / C5), host rows "
                         "routed by the plan's quotas and relayed through peer ranks (one-call exchange)")
    ap.add_argument("--cache-gib", type=float, default=32.0, help="ddak-tiered: HBM cache per GPU")
    ap.add_argument("--presample", type=int, default=64, help="pre-sample batches per rank for DDAK hotness (P2)")
    ap.add_argument("--replicate-frac", type=float, default=1 / 16)
    ap.add_argument("--layout", default=None, help="partitioned: save the DDAK layout here (rank 0), or check a saved one")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        spawn_ranks(args.gpus)
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    assert args.warmup >= 3, "W >= 3 warm-up steps"
    assert args.steps >= 1
    # MOMENT_BENCH_SHARED_GPU=1 (test only): every rank on cuda:0 with a gloo group, to exercise the
    # multi-rank code path on a one-GPU box (NCCL refuses two ranks on one device). Never a bench number.
    shared = os.environ.get("MOMENT_BENCH_SHARED_GPU") == "1"
    if shared:
        local = 0
    elif world > torch.cuda.device_count():
        raise SystemExit(f"bench.py: {world} ranks but only {torch.cuda.device_count()} visible GPUs")
    torch.cuda.set_device(local)
    dev = f"cuda:{local}"
    dist = None
    if world > 1:
        import torch.distributed as dist

        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device(dev))
    if args.inflight <= 0:
        cfg_ = W.CONFIGS[args.config]
        fb = cfg_["batch"]
        for k_ in cfg_["fanout"]:
            fb = min(fb + fb * k_, cfg_["n"])
        row_buf = fb * cfg_["dim"] * torch.empty(0, dtype=cfg_["dtype"]).element_size()
        args.inflight = 16 if args.steps <= 24 or row_buf > (1 << 30) else 32
    P = max(1, min(args.inflight, args.steps))
    global LANE_STEPS
    LANE_STEPS = args.steps  # the default lane priorities depend on the region length (lane_streams)
    part = args.placement != "replicated"
    kw = dict(placement=args.placement, dist=dist, shared=shared, presample=args.presample,
              replicate_frac=args.replicate_frac, layout=args.layout, cache_gib=args.cache_gib) if part else {}
    st = build_state(args.config, dev, rank, world, P, **kw)
    H = len(st.fanout)
    K = args.steps
    main_stream = torch.cuda.current_stream()

    def fork(ev):
        for L in st.lanes:
            if L.stream != main_stream:
                L.stream.wait_event(ev)

    def join():
        for L in st.lanes:
            if L.stream != main_stream:
                e = torch.cuda.Event()
                e.record(L.stream)
                main_stream.wait_event(e)

    def barrier():
        torch.cuda.synchronize()
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    # the batches: a pool of distinct batches of this rank (cycled epochs), timed steps cycle through it
    n_pool = max(64, min(K, 1024))
    pool = [st.batch(args.warmup * P + i) for i in range(n_pool)]
    warm = [st.batch(i) for i in range(args.warmup * P)]
    clocks = Clocks(local)  # sampled from the warm-up (also under load) through the timed regions
    # W warm-up steps on every lane (each lane's first step captures its CUDA graph)
    for i, b in enumerate(warm):
        st.step(*b, lane=i % P)
    barrier()

    def region(step_fn, first):
        """One timed region: exactly K steps, barrier + synchronize on both sides, device time (ms). Steps are
        issued P at a time (step first + j on lane j mod P): step_fn(i0, k) enqueues steps i0 .. i0 + k - 1 on
        lanes 0 .. k - 1 in one moment_step_batch call."""
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(main_stream)
        fork(e0)
        for j0 in range(0, K, P):
            step_fn(first + j0, min(P, K - j0))
        join()
        e1.record(main_stream)
        barrier()
        return e0.elapsed_time(e1)

    def repeats(step_fn, min_time):
        times, t, r = [], 0.0, 0
        while True:
            ms_ = region(step_fn, r * K)
            times.append(ms_)
            t += ms_
            r += 1
            done = r >= 3 and t >= min_time * 1000
            if dist:
                # every rank runs the same number of regions: rank 0 decides
                flag = torch.tensor([int(done)], device=dev if not shared else "cpu")
                dist.broadcast(flag, 0)
                done = bool(int(flag))
            if done:
                break
        tt = torch.tensor(times, dtype=torch.float64, device=dev if not shared else "cpu")
        if dist:
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)  # per region, the slowest rank
        return tt.cpu().tolist()

    pool_seeds, pool_rng = [b[0] for b in pool], [b[1] for b in pool]

    def pool_slice(i0, k):
        a = i0 % n_pool
        if a + k <= n_pool:
            return pool_seeds[a:a + k], pool_rng[a:a + k]
        idx = [(i0 + j) % n_pool for j in range(k)]
        return [pool_seeds[i] for i in idx], [pool_rng[i] for i in idx]

    # every lane's step prepared once; P steps per ctypes call (moment_step_batch)
    batch = st.M.StepBatch([L.ctx for L in st.lanes], st.graph.indptr, st.graph.indices, st.fanout,
                           [L.bufs for L in st.lanes], [L.rows for L in st.lanes], [L.stream for L in st.lanes])

    def dev_step(i0, k):
        batch.run(*pool_slice(i0, k))

    reg_ms = repeats(dev_step, args.min_time)
    ck = clocks.stop()
    n_regions = len(reg_ms)
    ms = statistics.median(reg_ms)
    # |F_H| of every pool batch (deterministic: identical to the timed steps), collected on the device
    L0 = st.lanes[0]
    cnt_dev = torch.empty((n_pool, 2 * H + 1), dtype=torch.int64, device=dev)
    for i in range(n_pool):
        L0.ctx.step(st.graph.indptr, st.graph.indices, pool[i][0], st.fanout, pool[i][1], L0.bufs, None,
                    stream=main_stream)
        cnt_dev[i].copy_(L0.bufs.counts)
    cnt_pool = cnt_dev.cpu().tolist()
    nF_pool = [c[H] for c in cnt_pool]
    med_r = min(range(n_regions), key=lambda r: abs(reg_ms[r] - ms))
    used = [(med_r * K + j) % n_pool for j in range(K)]
    nF_region = sum(nF_pool[i] for i in used)
    # algorithmic HBM bytes of a step: sampling = sum_{h<H} 16 |F_h| (indptr pair) + sum_h 8 E_h
    # (index read + src write) + 8 |F_H| (ids written); gather = |F_H| (8 placement/id + R read + R written)
    samp_bytes = sum(sum(16 * c[h] for h in range(H)) + sum(8 * e for e in c[H + 1:]) + 8 * c[H]
                     for c in (cnt_pool[i] for i in used))
    gath_bytes = nF_region * (2 * st.R + 8)
    tiers = None
    if part:
        # rows per owning bin of the median region's batches (deterministic: rerun on lane 0), then every
        # rank's counts, so each rank also knows how many of its bin's rows its peers read over NVLink
        tiered = st.placement_mode == "ddak-tiered"
        per_bin = torch.zeros(st.n_bins * world if tiered else world, dtype=torch.int64, device=dev)
        for i in sorted(set(used)):
            L0.ctx.step(st.graph.indptr, st.graph.indices, pool[i][0], st.fanout, pool[i][1], L0.bufs, None,
                        stream=main_stream)
            # tiered: rows per route queue (bin, via rank); else rows per owning HBM bin
            cnt = st.queues_of(L0.bufs.nodes, nF_pool[i]) if tiered else st.bins_of(L0.bufs.nodes, nF_pool[i])
            per_bin += cnt * used.count(i)
        # every rank: every row of one of its batches, gathered through the local and the peers' (CUDA-IPC
        # mapped) bins, equals the generated bytes of its id (the oracle's table[ids]; the sampler is per rank
        # and checked by the N = 1 parity subset)
        i0 = used[0]
        L0.ctx.step(st.graph.indptr, st.graph.indices, pool[i0][0], st.fanout, pool[i0][1], L0.bufs, L0.rows,
                    stream=main_stream)
        torch.cuda.synchronize()
        nf0 = nF_pool[i0]
        rows_ok = True
        for c0 in range(0, nf0, 1 << 18):
            c1 = min(nf0, c0 + (1 << 18))
            rows_ok &= bool(torch.equal(L0.rows[c0:c1],
                                        W.feature_rows(feature_check_ids(st, L0.bufs.nodes[c0:c1]), st.dim, st.dtype)))
        okt = torch.tensor([int(rows_ok)], dtype=torch.int64, device=dev if not shared else "cpu")
        if dist:
            dist.all_reduce(okt, op=dist.ReduceOp.MIN)
        if not int(okt):
            raise AssertionError("partitioned gather: rows differ from their generated bytes on some rank")
        allb = [torch.zeros_like(per_bin) for _ in range(world)]
        if dist:
            if shared:
                allc = [torch.zeros(per_bin.numel(), dtype=torch.int64) for _ in range(world)]
                dist.all_gather(allc, per_bin.cpu())
                allb = [c.to(dev) for c in allc]
            else:
                dist.all_gather(allb, per_bin)
        else:
            allb = [per_bin]
        mat = torch.stack(allb).cpu().numpy() / K  # [requester][owner] (tiered: [requester][bin * world + via])
        host_direct = relayed_in = served_relays = 0.0
        if tiered:
            q = lambda g, b, via: mat[g, b * world + via]  # noqa: E731
            local = q(rank, rank, rank)
            peer_in = sum(q(rank, b, b) for b in range(world) if b != rank)
            peer_out = sum(q(g, rank, rank) for g in range(world) if g != rank)
            hosts = range(world, st.n_bins)
            host_direct = sum(q(rank, j, rank) for j in hosts)
            relayed_in = sum(q(rank, j, h) for j in hosts for h in range(world) if h != rank)
            served_relays = sum(q(g, j, rank) for g in range(world) if g != rank for j in hosts)
        else:
            local = mat[rank, rank]
            peer_in = mat[rank].sum() - local
            peer_out = mat[:, rank].sum() - local
        nf_b = nF_region / K
        hbm_b = (local + peer_out) * st.R + nf_b * (st.R + 8) + samp_bytes / K
        t_hbm = hbm_b / (_peaks()[0] * 1e9)
        nv_in, nv_out = (peer_in + relayed_in) * st.R, (peer_out + served_relays) * st.R
        t_nvl = max(nv_in, nv_out) / (NVLINK_GBS * 1e9)
        pcie_b = (host_direct + served_relays) * st.R
        t_pcie = pcie_b / (PORT_GBS * 1e9)
        t_meas = ms / K / 1000
        t_all = {"hbm": t_hbm, "nvlink": t_nvl, "pcie": t_pcie}
        tiers = {"placement": st.placement_mode, "replicated_rows": st.replicated_rows, "bin_rows": st.bin_rows,
                 "rows_per_batch": {"local_hbm": local, "peer_in_nvlink": peer_in, "served_to_peers_nvlink": peer_out,
                                    "host_direct_pcie": host_direct, "host_relayed_to_me": relayed_in,
                                    "host_served_for_peers": served_relays},
                 "bytes_per_batch": {"hbm": hbm_b, "nvlink_in": nv_in, "nvlink_out": nv_out, "pcie_in": pcie_b},
                 "t_us": {"hbm": t_hbm * 1e6, "nvlink": t_nvl * 1e6, "pcie": t_pcie * 1e6, "measured": t_meas * 1e6},
                 "binding": max(t_all, key=t_all.get), "frac": max(t_all.values()) / t_meas,
                 "quota": st.quota.tolist() if tiered else None,
                 "peaks": {"hbm_gbs": _peaks()[0], "nvlink_gbs": NVLINK_GBS, "pcie_port_gbs": PORT_GBS,
                           "nvlink_source": "measured B200 peer copy per direction (B200_PROFILING.md; 900 nominal)"},
                 "plan": {"t_star_us": st.plan["t_star"], "t_nvlink_us": st.plan["t_nvlink"],
                          "t_hbm_us": st.plan["t_hbm"],
                          "note": "the plan predicts the gather per batch (P:L229-235, P:L339)"},
                 "offline_s": {"hotness": st.t_hotness, "ddak": st.t_place},
                 "rows_check": {"ranks": world, "rows_per_rank": "every row of one batch", "byte_exact": True}}
    # roofline pass: CUDA events around the dominant kernel (the gather) on its stream, one lane, one batch
    # at a time, over the pool
    n_roof = min(n_pool, 256)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n_roof)]
    for i in range(8):  # untimed: the first direct (non-graph) launches of this path
        st.step(*pool[i % n_pool], ev=evs[i % n_roof], lane=0)
    torch.cuda.synchronize()
    for i in range(n_roof):
        st.step(*pool[i], ev=evs[i], lane=0)
    torch.cuda.synchronize()
    launch_times = sorted(a.elapsed_time(b) for a, b in evs)
    gather_ms = sum(launch_times) / n_roof
    gather_ms_median = launch_times[n_roof // 2]
    nF_roof = nF_pool[:n_roof]
    # supplementary: the same gather kernel issued back to back (P sampled batches, one per lane, gathered in
    # rounds on one stream; > L2 per round), so launch latency overlaps the previous launch
    for i, L in enumerate(st.lanes):
        s_, r_ = pool[i % n_pool]
        L.ctx.sample(st.graph.indptr, st.graph.indices, s_, st.fanout, r_, L.bufs, stream=main_stream)
    torch.cuda.synchronize()
    nF_b2b = sum(int(L.bufs.counts[H]) for L in st.lanes) / P
    rounds = max(1, 200 // P)
    e_b0, e_b1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e_b0.record(main_stream)
    for _ in range(rounds):
        for L in st.lanes:
            L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(),
                         stream=main_stream)
    e_b1.record(main_stream)
    torch.cuda.synchronize()
    gather_ms_b2b = e_b0.elapsed_time(e_b1) / (rounds * P)
    # supplementary: the same gathers with the P lanes' launches concurrent (one stream per lane, as in the
    # timed region but without the sampling kernels)
    e_c0, e_c1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e_c0.record(main_stream)
    fork(e_c0)
    for _ in range(rounds):
        for L in st.lanes:
            L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(),
                         stream=L.stream)
    join()
    e_c1.record(main_stream)
    torch.cuda.synchronize()
    gather_ms_conc = e_c0.elapsed_time(e_c1) / (rounds * P)
    if dist:
        tot = torch.tensor([float(nF_region)], dtype=torch.float64, device=dev if not shared else "cpu")
        dist.all_reduce(tot)
        nF_total = float(tot)
    else:
        nF_total = float(nF_region)
    seeds_per_s = world * st.B * K / (ms / 1000)
    gather_gbs = nF_total * st.R / (ms / 1000) / 1e9
    # roofline of the dominant kernel (gather): algorithmic bytes = |F_H| (R read + R write + 8 id)
    alg_bytes = (sum(nF_roof) / n_roof) * (2 * st.R + 8)
    peak, peak_kind = _peaks()
    achieved = alg_bytes / (gather_ms / 1000) / 1e9
    # e2e: the same K-step regions through the C ABI with HOST buffers: each step's seeds copied H2D from
    # pinned memory and its counts read back D2H (moment_step_host), all copies inside the timed region
    seeds_pinned = torch.empty((n_pool, st.B), dtype=torch.int64).pin_memory()
    for i in range(n_pool):
        seeds_pinned[i].copy_(pool[i][0])
    counts_pinned = torch.zeros((K, 2 * H + 1), dtype=torch.int64).pin_memory()
    for i in range(P):
        st.step_host(seeds_pinned[i], pool[i][1], counts_pinned[i % K], lane=i)
    torch.cuda.synchronize()

    batch_h = st.M.StepBatch([L.ctx for L in st.lanes], st.graph.indptr, st.graph.indices, st.fanout,
                             [L.bufs for L in st.lanes], [L.rows for L in st.lanes], [L.stream for L in st.lanes],
                             host=True)
    pinned_list = [seeds_pinned[i] for i in range(n_pool)]
    counts_list = [counts_pinned[i] for i in range(K)]

    def host_step(i0, k):
        idx = [(i0 + j) % n_pool for j in range(k)]
        batch_h.run([pinned_list[i] for i in idx], [pool_rng[i] for i in idx],
                    [counts_list[(i0 + j) % K] for j in range(k)])

    e2e_ms_all = repeats(host_step, args.e2e_min_time)
    e2e_ms = statistics.median(e2e_ms_all)
    # the last region's counts: every step's |F_H| read back equals the device path's
    last = len(e2e_ms_all) - 1
    for j in range(K):
        assert int(counts_pinned[j][H]) == nF_pool[(last * K + j) % n_pool], "e2e counts differ from the device path"
    e2e_val = world * st.B * K / (e2e_ms / 1000)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_baseline(st, pool, args.cpu_budget) if not part else partition_parity(st, pool)
    if rank == 0:
        line = {
            "metric": METRIC, "value": seeds_per_s, "unit": "seeds/s", "n_gpus": world, "steps": K,
            "warmup": args.warmup, "ms_per_step": ms / K, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": args.config, "desc": st.cfg["desc"], "global_batch": st.B * world,
                       "fanout": list(st.fanout), "row_bytes": st.R, "inflight_batches_per_gpu": P,
                       "lane_priority": LANE_PRIO,
                       "parallelism": f"dp{world} (replicated graph+features, seeds sharded)",
                       "timing": f"each timed region = exactly {K} steps per GPU (barrier + synchronize on both "
                                 f"sides, CUDA events, max over ranks); {n_regions} regions (>= {args.min_time:g} s "
                                 f"of device time, so nvidia-smi samples the clocks inside them), median reported; "
                                 f"warm-up {args.warmup} steps on each of the {P} lanes; steps issued {P} per "
                                 f"moment_step_batch call (one per lane)",
                       "region_ms": {"median": ms, "min": min(reg_ms), "max": max(reg_ms), "n": n_regions},
                       "l2": "no flush: inputs larger than L2 (features %.2f GB, CSR %.2f GB)" % (
                           st.table.numel() / 1e9, (st.graph.indptr.numel() * 8 + st.graph.indices.numel() * 4) / 1e9),
                       "mean_F_H": nF_region / K,
                       **({"test_mode": "all ranks share cuda:0 over gloo: not a bench number"} if shared else {})},
            "gather_GBs": gather_gbs,
            "step_roofline": {"bound": "hbm", "alg_bytes_per_step": (samp_bytes + gath_bytes) / K,
                              "sampling_bytes_per_step": samp_bytes / K, "gather_bytes_per_step": gath_bytes / K,
                              "achieved": (samp_bytes + gath_bytes) / K / (ms / K / 1000) / 1e9, "peak": peak,
                              "unit": "GB/s",
                              "frac": (samp_bytes + gath_bytes) / K / (ms / K / 1000) / 1e9 / peak,
                              "how": "whole step (all 8(a) rows H1-H6): algorithmic bytes of the median region's "
                                     "batches / its device time, per GPU"},
            "step_floor": step_floor(args.config, gath_bytes / K, peak, ms / K),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": profile_traffic(args.config), "kernel": "gather_tma4_kernel",
                         "launch_shares": profile_summary(args.config).get("launch_shares"),
                         "why_this_kernel": profile_summary(args.config).get("why_gather"),
                         "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})",
                         "alg_bytes_per_launch": alg_bytes, "launch_ms": gather_ms, "launch_ms_median": gather_ms_median,
                         "how": f"CUDA events on the gather's stream around each of {n_roof} launches (one batch "
                                "at a time, lane 0, after 8 untimed), mean duration",
                         "gather_share_of_step": gather_ms / (ms / K),
                         "back_to_back": {
                             "launch_ms": gather_ms_b2b,
                             "achieved": nF_b2b * (2 * st.R + 8) / (gather_ms_b2b / 1000) / 1e9,
                             "frac": nF_b2b * (2 * st.R + 8) / (gather_ms_b2b / 1000) / 1e9 / peak,
                             "how": f"{rounds} rounds x {P} batches' gathers issued back to back on one stream, "
                                    "one event pair (launch latency overlapped)"},
                         "concurrent": {
                             "ms_per_launch": gather_ms_conc,
                             "achieved": nF_b2b * (2 * st.R + 8) / (gather_ms_conc / 1000) / 1e9,
                             "frac": nF_b2b * (2 * st.R + 8) / (gather_ms_conc / 1000) / 1e9 / peak,
                             "how": f"the same {rounds} x {P} gathers, each lane's on its own stream (as in the "
                                    "timed region, sampling absent): time per launch of the whole-GPU throughput"}},
            "cpu_baseline": cpu,
            "e2e": {"value": e2e_val, "unit": "seeds/s", "h2d_bytes_per_step": st.B * 8,
                    "d2h_bytes_per_step": (2 * H + 1) * 8,
                    "api": "moment_step_batch with host buffers (= moment_step_host per step, C ABI), same K-step "
                           "regions, median of "
                           f"{len(e2e_ms_all)}",
                    "copies_declared": "H2D: the step's 1024 int64 seeds, read from pinned host memory over PCIe "
                                       "by the first hop's kernel (zero-copy); D2H: the step's counts (|F_0..F_H|, "
                                       "E_0..E_{H-1}) stored into pinned host memory by the compaction's last block "
                                       "(pageable buffers would go through cudaMemcpyAsync). F_H, offsets, src and "
                                       "the gathered rows stay in HBM for the on-GPU consumer (the GNN layer, "
                                       "sage.py) and are not copied to the host"},
            "gpu_launches": st.launches_per_step() * K,
            "clocks": ck,
        }
        if part:
            tiers["plan"]["gather_us_measured"] = gather_ms * 1000
            line["tiers"] = tiers
            line["config"]["parallelism"] = f"dp{world}, features DDAK-partitioned over {world} HBM bins" + (
                f" + {st.replicated_rows} replicated rows" if st.replicated_rows else "") + (
                f" (HBM caches of {args.cache_gib:g} GiB) + {st.n_bins - world} pinned host bins (rings of "
                f"{st.r_phys} rows), quota-routed relays" if st.placement_mode == "ddak-tiered" else "")
            line["config"]["l2"] = "no flush: inputs larger than L2 (features %.2f GB over all GPUs, CSR %.2f GB)" % (
                st.graph.n * st.stride / 1e9, (st.graph.indptr.numel() * 8 + st.graph.indices.numel() * 4) / 1e9)
            line["roofline"]["kernel"] = ("gather_kernel (placement map; peer rows over NVLink)" +
                                          ("; host rows over PCIe, relayed by peers inside moment_step"
                                           if st.placement_mode == "ddak-tiered" else ""))
            line["roofline"]["traffic"] = None
            line["roofline"]["launch_shares"] = None
            line["roofline"]["why_this_kernel"] = None
        print(json.dumps(line), flush=True)
    if part:
        st.close(dist)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
