"""Tiered gather on one B200: a partial HBM cache + pinned host DRAM (the out-of-core tier), placed by DDAK
(hot rows in HBM, from moment_hotness pre-sampling) or by the hash baseline, then the same
sample + gather batches through moment_sample + moment_gather. Reports seeds/s, per-tier bytes per batch,
host-link GB/s against the measured pinned H2D copy bandwidth, and DDAK's gain over hash.

    python tools/bench_tiers.py [--n 4000000] [--m 32000000] [--dim 768] [--hbm-frac 0.25] [--batches 40]

Features are fp16 x dim (C4: 768-d = 1536-byte rows). Prints one JSON line.
"""
import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402
import workloads as W  # noqa: E402


def h2d_peak(dev):
    n = 1 << 30
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    d = torch.empty(n, dtype=torch.uint8, device=dev)
    d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    best = 0.0
    for _ in range(5):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d.copy_(h, non_blocking=True)
        b.record()
        torch.cuda.synchronize()
        best = max(best, n / (a.elapsed_time(b) / 1e3) / 1e9)
    return best


def build_bins(table_dev, bin_of, slot_of, n_bins, host_bins, dev):
    bins = []
    b_t = torch.as_tensor(bin_of, device=dev)
    s_t = torch.as_tensor(slot_of, device=dev)
    for b in range(n_bins):
        sel = torch.nonzero(b_t == b).flatten()
        order = torch.argsort(s_t[sel])
        rows = table_dev.index_select(0, sel[order])
        if b in host_bins:
            h = torch.empty(rows.shape, dtype=torch.uint8).pin_memory()
            h.copy_(rows)
            bins.append(h)
        else:
            bins.append(rows.contiguous())
        del rows
    return bins


def run_mode(mode, g, table_dev, hot, args, batches, R, dev, fanout):
    n = g.n
    cap_hbm = int(args.hbm_frac * n)
    if mode == "ddak":
        # 1-GPU topology: HBM -> GPU (HBM bandwidth), host DRAM -> CPU -> GPU port (measured H2D)
        topo = M.topology([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 0),
                           (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0)],
                          [(0, 3, 6_469_000), (1, 2, 400_000), (2, 3, int(args.h2d * 1000))])
        bin_of, slot_of, acc, used, traffic = M.place(topo, hot, [cap_hbm, n])
    else:
        bin_of, slot_of, acc, used, traffic = M.place(None, hot, [cap_hbm, n], bin_tier=[1, 2], bin_traffic=[1, 1],
                                                      mode=M.PLACE_HASH)
    bins = build_bins(table_dev, bin_of, slot_of, 2, {1}, dev)
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=dev)
    ctx = M.Ctx(n_vertices=n, max_seeds=args.batch, max_fanout=fanout, device=0, row_bytes=R, bin_owner=[0, -1],
                bin_ptr=[b.data_ptr() for b in bins], placement=placement)
    bufs = M.SampleBuffers.allocate(args.batch, fanout, n, dev)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=dev)
    H = len(fanout)
    for s, r in batches[:3]:
        ctx.sample(g.indptr, g.indices, s, fanout, r, bufs)
        ctx.gather(bufs.nodes, rows, n_dev=bufs.counts[H:H + 1], max_n=bufs.nodes.numel())
    torch.cuda.synchronize()
    # per-tier request counts of every batch (untimed; deterministic)
    in_hbm = torch.as_tensor(bin_of == 0, device=dev)
    hbm_rows = host_rows = 0
    for s, r in batches:
        ctx.sample(g.indptr, g.indices, s, fanout, r, bufs)
        nF = int(bufs.counts[H])
        h = int(in_hbm[bufs.nodes[:nF]].sum())
        hbm_rows += h
        host_rows += nF - h
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    g0, g1 = [], []
    torch.cuda.synchronize()
    e0.record()
    for s, r in batches:
        ctx.sample(g.indptr, g.indices, s, fanout, r, bufs)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        ctx.gather(bufs.nodes, rows, n_dev=bufs.counts[H:H + 1], max_n=bufs.nodes.numel())
        b.record()
        g0.append(a)
        g1.append(b)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    gather_ms = sum(a.elapsed_time(b) for a, b in zip(g0, g1))
    nb = len(batches)
    host_bytes = host_rows * R
    # P5 prediction: the time-bisection plan of this batch's demand on the 1-GPU topology
    # (HBM bin -> GPU at the measured copy bandwidth, host bin -> CPU -> GPU port at the measured H2D),
    # against the measured gather time
    topo1 = M.topology([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 0),
                        (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0)],
                       [(0, 3, 6_469_000), (1, 2, 400_000), (2, 3, int(args.h2d * 1000))])
    N1 = topo1.info()[0]
    demand = np.zeros(N1, np.int64)
    demand[0] = int(hbm_rows * R / nb)
    demand[1] = int(host_bytes / nb)
    # HBM: each row is read once from the HBM bin and written once to the batch buffer (r + w bytes)
    plan = M.plan(topo1, [3], demand, 0, 6_469_000 // 2).info()
    out = {"placement": mode, "seeds_per_s": nb * args.batch / (ms / 1e3), "ms_per_batch": ms / nb,
           "gather_ms_per_batch": gather_ms / nb, "rows_per_batch": (hbm_rows + host_rows) / nb,
           "hbm_hit_rate": hbm_rows / max(1, hbm_rows + host_rows),
           "host_bytes_per_batch": host_bytes / nb, "hbm_bytes_per_batch": hbm_rows * R / nb,
           "host_link_GBs_in_gather": host_bytes / (gather_ms / 1e3) / 1e9,
           "host_link_frac_of_h2d": host_bytes / (gather_ms / 1e3) / 1e9 / args.h2d,
           "plan_t_star_us": plan["t_star"], "plan_t_ingest_us": plan["t_ingest"], "plan_t_hbm_us": plan["t_hbm"],
           "prediction_error": abs(plan["t_star"] - gather_ms / nb * 1e3) / (gather_ms / nb * 1e3),
           "bin_rows": [int(x) for x in used], "bin_traffic": [int(x) for x in traffic]}
    del bins, ctx
    torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=4_000_000)
    ap.add_argument("--m", type=int, default=32_000_000)
    ap.add_argument("--dim", type=int, default=768)
    ap.add_argument("--hbm-frac", type=float, default=0.25)
    ap.add_argument("--batch", type=int, default=1024)
    ap.add_argument("--batches", type=int, default=40)
    ap.add_argument("--presample", type=int, default=64)
    args = ap.parse_args()
    dev = "cuda:0"
    torch.cuda.set_device(0)
    fanout = [15, 10, 5]
    t0 = time.time()
    g = W.rmat_csr(args.n, args.m, device=dev)
    table_dev = W.feature_table(args.n, args.dim, torch.float16, device=dev)
    R = table_dev.shape[1]
    args.h2d = h2d_peak(dev)
    train = W.training_set(g, min_count=args.batch * (args.batches + args.presample))
    allb = W.epoch_batches(train, args.batch, 0)
    pre = [(allb[i % len(allb)], W.batch_rng_seed(1, 99, 0, i)) for i in range(args.presample)]
    batches = [(allb[i % len(allb)], W.batch_rng_seed(1, 0, 0, i)) for i in range(args.batches)]
    # P2 hotness by pre-sampling on the GPU (moment_hotness over F_H of the pre-sample batches)
    ctx = M.Ctx(n_vertices=g.n, max_seeds=args.batch, max_fanout=fanout, device=0)
    bufs = M.SampleBuffers.allocate(args.batch, fanout, g.n, dev)
    hot = torch.zeros(g.n, dtype=torch.int64, device=dev)
    for s, r in pre:
        ctx.sample(g.indptr, g.indices, s, fanout, r, bufs)
        ctx.hotness(bufs.nodes, hot, n_dev=bufs.counts[3:4], max_n=bufs.nodes.numel())
    hot_np = hot.cpu().numpy().astype(np.uint64)
    del ctx, bufs
    res = {"n": args.n, "m": args.m, "row_bytes": R, "hbm_frac": args.hbm_frac, "h2d_peak_GBs": args.h2d,
           "setup_s": time.time() - t0}
    res["ddak"] = run_mode("ddak", g, table_dev, hot_np, args, batches, R, dev, fanout)
    res["hash"] = run_mode("hash", g, table_dev, hot_np, args, batches, R, dev, fanout)
    res["ddak_speedup_over_hash"] = res["ddak"]["seeds_per_s"] / res["hash"]["seeds_per_s"]
    print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
