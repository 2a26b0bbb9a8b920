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
import math
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
        streams = [torch.cuda.current_stream(device)] + [torch.cuda.Stream(device) for _ in range(inflight - 1)]
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
        if ev is None:
            L.ctx.step(self.graph.indptr, self.graph.indices, seeds, self.fanout, rng_seed, L.bufs, L.rows, stream=s)
            return
        L.ctx.sample(self.graph.indptr, self.graph.indices, seeds, self.fanout, rng_seed, L.bufs, stream=s)
        ev[0].record(s)
        L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(), stream=s)
        ev[1].record(s)

    def step_host(self, seeds_host, rng_seed, counts_host, lane=0):
        """The same step through moment_step_host: host seeds in, host counts out (asynchronous)."""
        L = self.lanes[lane]
        L.ctx.step_host(self.graph.indptr, self.graph.indices, seeds_host, self.fanout, rng_seed, L.bufs, L.rows,
                        counts_host, stream=L.stream)

    def launches_per_step(self):
        # set_call, (sample, bitscan) per hop (the first hop's sampler also initialises the call), compact, gather
        return 1 + 2 * len(self.fanout) + 1 + 1


def build_state(name, device="cuda:0", rank=0, world=1, inflight=1):
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


def oracle_baseline(name, budget_s=15.0, seeds_cap=None, state=None):
    """Time the CPU oracle (as it stands, single-threaded) on a bounded sample of the workload."""
    import oracle

    oracle.build()
    cfg = W.CONFIGS[name]
    if state is not None:
        indptr = state.graph.indptr.cpu().numpy()
        indices = state.graph.indices.cpu().numpy()
        table = np.ascontiguousarray(state.table[:, :state.R].cpu().numpy())
        train = state.train.cpu()
    else:
        g = W.rmat_csr(cfg["n"], cfg["m"], device="cpu")
        indptr, indices = g.indptr.numpy(), g.indices.numpy()
        table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device="cpu").numpy()
        train = W.training_set(g, min_count=cfg["batch"])
    batches = W.epoch_batches(train, cfg["batch"], 0)
    fan = list(cfg["fanout"])
    # calibrate on a small slice, then size the sample to the budget
    t0 = time.perf_counter()
    r = oracle.sample(indptr, indices, batches[0][:16].numpy(), fan, 1)
    oracle.gather(table, r["nodes"])
    per_seed = (time.perf_counter() - t0) / 16
    n = int(max(16, min(seeds_cap or cfg["batch"], budget_s / max(per_seed, 1e-9))))
    done, t = 0, 0.0
    i = 0
    while done < n:
        seeds = batches[i % len(batches)][: min(cfg["batch"], n - done)].numpy()
        t0 = time.perf_counter()
        r = oracle.sample(indptr, indices, seeds, fan, W.batch_rng_seed(RUN_SEED, 0, 0, i))
        oracle.gather(table, r["nodes"])
        t += time.perf_counter() - t0
        done += len(seeds)
        i += 1
    return {"value": done / t, "unit": "seeds/s", "cores": 1, "kind": "oracle",
            "sample": f"{done} seeds of {name} ({i} batch slices of <= {cfg['batch']}), sample + gather, single thread"}


def profile_summary(name):
    """The committed ncu summary of the gather kernel for `name` (per-launch DRAM bytes, launch shares)."""
    path = os.path.join(ROOT, "profiles", "ncu_gather_summary.json")
    try:
        with open(path) as f:
            return json.load(f).get(name, {})
    except Exception:
        return {}


def profile_traffic(name):
    """Per-launch DRAM bytes of the gather kernel from the committed ncu --set full summary, if any."""
    return profile_summary(name).get("dram_bytes_per_launch")


def run_reference(args, rank, world):
    if rank != 0:
        return
    cfg = W.CONFIGS[args.config]
    total_steps = args.steps + args.warmup
    # each step is a bounded slice of a batch so that the whole run stays within a few minutes
    budget = float(os.environ.get("MOMENT_REF_BUDGET_S", "150"))
    import oracle

    oracle.build()
    g = W.rmat_csr(cfg["n"], cfg["m"], device="cpu")
    indptr, indices = g.indptr.numpy(), g.indices.numpy()
    table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device="cpu").numpy()
    train = W.training_set(g, min_count=cfg["batch"])
    batches = W.epoch_batches(train, cfg["batch"], 0)
    fan = list(cfg["fanout"])
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
                                       "sample + gather"},
            "e2e": {"value": val, "unit": "seeds/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20000)  # ~1 s timed: nvidia-smi samples the clocks in it
    ap.add_argument("--warmup", type=int, default=50)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--impl", default="moment", choices=["moment", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=4000)
    # 12-16 measured best on C2 (29.5-29.7 M seeds/s vs 27.7 at 8, 28.4 at 24)
    ap.add_argument("--inflight", type=int, default=16, help="batches in flight per GPU (one stream each)")
    args = ap.parse_args()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    assert args.warmup >= 3, "W >= 3 warm-up steps"
    # MOMENT_BENCH_SHARED_GPU=1 (test only): every rank on cuda:0 with a gloo group, to exercise the
    # multi-rank code path on a one-GPU box (NCCL refuses two ranks on one device). Never a bench number.
    shared = os.environ.get("MOMENT_BENCH_SHARED_GPU") == "1"
    if shared:
        local = 0
    torch.cuda.set_device(local)
    dev = f"cuda:{local}"
    dist = None
    if world > 1:
        import torch.distributed as dist

        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device(dev))
    st = build_state(args.config, dev, rank, world, args.inflight)
    H = len(st.fanout)
    P = len(st.lanes)
    main_stream = torch.cuda.current_stream()

    def fork(ev):
        for L in st.lanes[1:]:
            L.stream.wait_event(ev)

    def join():
        for L in st.lanes[1:]:
            e = torch.cuda.Event()
            e.record(L.stream)
            main_stream.wait_event(e)

    batches = [st.batch(args.warmup + i) for i in range(args.steps)]
    clocks = Clocks(local)  # sampled from the warm-up (also under load) through the timed region
    for i in range(args.warmup):
        st.step(*st.batch(i), lane=i % P)
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in range(min(args.steps, 1000))]
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    t_start, t_end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t_start.record(main_stream)
    fork(t_start)
    for i in range(args.steps):
        st.step(*batches[i], lane=i % P)
    join()
    t_end.record(main_stream)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    ck = clocks.stop()
    ms = t_start.elapsed_time(t_end)
    # roofline pass over (the first 1000 of) the same batches: CUDA events around the dominant kernel (the
    # gather) on its stream, one lane; then |F_H| of every timed step (deterministic, so identical to the
    # timed run), collected on the device and read once
    n_roof = min(args.steps, 1000)
    for i in range(n_roof):
        st.step(*batches[i], ev=evs[i], lane=0)
    torch.cuda.synchronize()
    gather_ms = sum(a.elapsed_time(b) for a, b in evs[:n_roof]) / n_roof
    # supplementary: the same gather kernel issued back to back (P sampled batches, one per lane, gathered in
    # rounds on one stream; 8 x 48 MB per round > L2), so launch latency overlaps the previous launch
    for i, L in enumerate(st.lanes):
        s_, r_ = batches[i % len(batches)]
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
    # timed region but without the sampling kernels): whole-GPU throughput of the kernel once the ramp and
    # tail of one launch overlap the others'
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
    nF_roof = []
    for i in range(n_roof):
        st.step(*batches[i], lane=0)
        nF_roof.append(int(st.lanes[0].bufs.counts[H]))
    L0 = st.lanes[0]
    nf_dev = torch.empty(args.steps, dtype=torch.int64, device=dev)
    for i in range(args.steps):
        L0.ctx.step(st.graph.indptr, st.graph.indices, batches[i][0], st.fanout, batches[i][1], L0.bufs, None,
                    stream=main_stream)
        nf_dev[i:i + 1].copy_(L0.bufs.counts[H:H + 1])
    nF = nf_dev.cpu().tolist()
    if dist:
        t = torch.tensor([ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t)
        tot = torch.tensor([float(sum(nF))], device=dev)
        dist.all_reduce(tot)
        nF_total = float(tot)
    else:
        nF_total = float(sum(nF))
    seeds_per_s = world * st.B * args.steps / (ms / 1000)
    gather_gbs = nF_total * st.R / (ms / 1000) / 1e9
    # roofline of the dominant kernel (gather): algorithmic bytes = |F_H| (R read + R write + 8 id)
    alg_bytes = (sum(nF_roof) / n_roof) * (2 * st.R + 8)
    peak, peak_kind = _peaks()
    achieved = alg_bytes / (gather_ms / 1000) / 1e9
    # e2e: the same steps through the C ABI with host buffers: pinned seeds H2D and counts D2H every step,
    # P steps in flight (one per lane), all copies inside the timed region
    n_e2e = max(3, args.e2e_steps)
    seeds_pinned = torch.empty((n_e2e, st.B), dtype=torch.int64).pin_memory()
    for i in range(n_e2e):
        seeds_pinned[i].copy_(batches[i % len(batches)][0])
    seeds_h = list(seeds_pinned)
    counts_pinned = torch.zeros((n_e2e, 2 * H + 1), dtype=torch.int64).pin_memory()
    counts_h = list(counts_pinned)
    for i in range(3):
        st.step_host(seeds_h[i], batches[i][1], counts_h[i], lane=i % P)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(main_stream)
    fork(e0)
    for i in range(args.e2e_steps):
        st.step_host(seeds_h[i], batches[i][1], counts_h[i], lane=i % P)
    join()
    e1.record(main_stream)
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1)
    assert all(int(c[H]) > 0 for c in counts_h[: args.e2e_steps])
    if dist:
        t = torch.tensor([e2e_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_ms = float(t)
    e2e_val = world * st.B * args.e2e_steps / (e2e_ms / 1000)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = oracle_baseline(args.config, state=st)
    if rank == 0:
        line = {
            "metric": METRIC, "value": seeds_per_s, "unit": "seeds/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": args.config, "desc": st.cfg["desc"], "global_batch": st.B * world,
                       "fanout": list(st.fanout), "row_bytes": st.R, "inflight_batches_per_gpu": P,
                       "parallelism": f"dp{world} (replicated graph+features)",
                       "l2": "inputs larger than L2 (features %.2f GB, CSR %.2f GB)" % (
                           st.table.numel() / 1e9, (st.graph.indptr.numel() * 8 + st.graph.indices.numel() * 4) / 1e9),
                       "mean_F_H": sum(nF) / args.steps,
                       **({"test_mode": "all ranks share cuda:0 over gloo: not a bench number"} if shared else {})},
            "gather_GBs": gather_gbs,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": profile_traffic(args.config), "kernel": "gather_tma4_kernel",
                         "launch_shares": profile_summary(args.config).get("launch_shares"),
                         "why_this_kernel": profile_summary(args.config).get("why_gather"),
                         "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_kind})",
                         "alg_bytes_per_launch": alg_bytes, "launch_ms": gather_ms,
                         "gather_share_of_step": gather_ms / (ms / args.steps),
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
                    "d2h_bytes_per_step": (2 * H + 1) * 8},
            "gpu_launches": st.launches_per_step() * args.steps,
            "clocks": ck,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
