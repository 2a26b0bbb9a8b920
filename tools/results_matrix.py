"""Per-config results on one B200 (BASELINE.md's results table, k = 1): every BASELINE config C1-C5 at full
graph size, sample + gather steps with batches in flight, per-tier algorithmic bytes, binding tier, roofline
fraction, plan T* vs measured gather time, planner time (cf. P:L265 ~14 s) and the CPU oracle
(one thread) on a bounded slice of the same workload.

    python tools/results_matrix.py [--configs C1,C2,C3,C4,C5] [--batches 200] [--lanes 8] [--out FILE]

Feature placement per config:
  C1, C2, C3  replicated table, all rows in HBM (C3: 57 GB of 512-byte rows fits one B200).
  C4, C5      DDAK over P2 pre-sampling hotness: the hottest rows in a 32 GiB (C4) / 64 GiB (C5) HBM cache,
              every other row read zero-copy from pinned host DRAM over PCIe. The full tables (375 GB / 1.1 TB)
              exceed the host, so the host tier is a ring of R_phys physical rows and row(v) := feature(v mod
              R_phys) for every tier (the documented fallback); the bytes still cross PCIe.
Roofline (per batch): T_hbm = (sampling + gather algorithmic HBM bytes) / MEASURED_PEAKS hbm_gbs,
T_pcie = host-row bytes / measured pinned H2D; binding tier = argmax; fraction = max T / measured time per
batch (with `lanes` batches in flight). One JSON line per config.
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

DEV = "cuda:0"
CACHE_GIB = {"C4": 32, "C5": 64}
R_PHYS = 1 << 22


def hbm_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs"
    except Exception:
        return 6650.0, "fallback"


def h2d_peak():
    n = 1 << 30
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    d = torch.empty(n, dtype=torch.uint8, device=DEV)
    best = 0.0
    for _ in range(6):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        d.copy_(h, non_blocking=True)
        b.record()
        torch.cuda.synchronize()
        best = max(best, n / (a.elapsed_time(b) / 1e3) / 1e9)
    return best


def one_gpu_topology(h2d_gbs, hbm_gbs):
    # storage HBM -> GPU at the copy bandwidth; host DRAM -> CPU/RC -> GPU port at the measured H2D (bytes/us)
    return M.topology([(M.NODE_STORAGE, M.TIER_GPU_HBM, 0), (M.NODE_STORAGE, M.TIER_HOST_DRAM, 0),
                       (M.NODE_INTERCONNECT, 0, -1), (M.NODE_COMPUTE, 0, 0)],
                      [(0, 3, int(hbm_gbs * 1000)), (1, 2, 400_000), (2, 3, int(h2d_gbs * 1000))])


def build_tiers(name, cfg, g, R, batches, h2d, hbm_gbs, fan, presample=64, held=64):
    """P2 hotness (`presample` pre-sample batches: seeds of later epochs than the timed ones, rng epoch
    2^32 - 1), P3/P4 DDAK placement, HBM cache + pinned ring host tier. Also counts F_H over `held` held-out
    batches (other seeds, other rng stream) for the planner's demand estimate (as tools/sim_plan.py)."""
    n, B = g.n, cfg["batch"]
    ctx0 = M.Ctx(n_vertices=n, max_seeds=B, max_fanout=fan, device=0)
    bufs = M.SampleBuffers.allocate(B, fan, n, DEV)
    hot = torch.zeros(n, dtype=torch.int64, device=DEV)
    dem = torch.zeros(n, dtype=torch.int64, device=DEV)
    H = len(fan)
    pre = []
    e = 2
    while len(pre) < presample + held:
        pre += W.epoch_batches(batches["train"], B, e)
        e += 1
    for i in range(presample + held):
        p = i < presample
        ctx0.step(g.indptr, g.indices, pre[i], fan,
                  W.batch_rng_seed(5, 2**32 - 1, 0, i) if p else W.batch_rng_seed(7, 0, 0, i), bufs, None)
        ctx0.hotness(bufs.nodes, hot if p else dem, n_dev=bufs.counts[H:H + 1], max_n=bufs.nodes.numel())
    torch.cuda.synchronize()
    hot_np = hot.cpu().numpy().astype(np.uint64)
    dem_np = dem.cpu().numpy()
    del hot, dem, ctx0, bufs
    cap_hbm = (CACHE_GIB[name] << 30) // R
    topo = one_gpu_topology(h2d, hbm_gbs)
    t0 = time.perf_counter()
    bin_of, slot_of, acc, used, traffic = M.place(topo, hot_np, [cap_hbm, n])
    t_place = time.perf_counter() - t0
    host = bin_of == 1
    slot_of = slot_of.copy()
    slot_of[host] = np.nonzero(host)[0] % R_PHYS
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=DEV)
    in_hbm = np.nonzero(~host)[0]
    hbm_v = torch.as_tensor(in_hbm[np.argsort(slot_of[in_hbm])], device=DEV)
    del in_hbm
    chunk = max(1, (1 << 31) // (R // 4 * 8))
    hbm = torch.empty((max(1, len(hbm_v)), R), dtype=torch.uint8, device=DEV)
    for c0 in range(0, len(hbm_v), chunk):
        hbm[c0:c0 + chunk] = W.feature_rows(hbm_v[c0:c0 + chunk] % R_PHYS, cfg["dim"], cfg["dtype"])
    del hbm_v
    ring = torch.empty((R_PHYS, R), dtype=torch.uint8).pin_memory()
    for c0 in range(0, R_PHYS, chunk):
        ids = torch.arange(c0, min(R_PHYS, c0 + chunk), device=DEV)
        ring[c0:c0 + len(ids)] = W.feature_rows(ids, cfg["dim"], cfg["dtype"]).cpu()
    torch.cuda.empty_cache()
    held_rows = np.bincount(bin_of, weights=dem_np.astype(np.float64), minlength=2) / held
    info = {"hbm_cache_gib": CACHE_GIB[name], "hbm_rows": int(used[0]), "host_rows": int(used[1]),
            "presample_batches": presample, "held_out_batches": held,
            "held_out_rows_per_batch": [float(x) for x in held_rows],
            "host_tier": f"pinned ring of {R_PHYS} rows ({R_PHYS * R / 2**30:.1f} GiB), row(v) = feature(v mod R_phys)",
            "ddak_place_s": t_place, "bin_traffic": [int(x) for x in traffic]}
    return dict(bin_ptr=[hbm.data_ptr(), ring.data_ptr()], bin_owner=[0, -1], placement=placement,
                keep=(hbm, ring, placement), in_hbm=torch.as_tensor(~host, device=DEV), info=info, topo=topo)


def run_config(name, args, hbm_gbs, h2d):
    import oracle

    cfg = W.CONFIGS[name]
    fan = list(cfg["fanout"])
    H = len(fan)
    B = cfg["batch"]
    t0 = time.perf_counter()
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    t_graph = time.perf_counter() - t0
    torch.cuda.empty_cache()
    R = cfg["dim"] * torch.empty(0, dtype=cfg["dtype"]).element_size()
    train = W.training_set(g, min_count=B * args.lanes)
    allb = W.epoch_batches(train, B, 0) + W.epoch_batches(train, B, 1)
    batches = [(allb[i % len(allb)], W.batch_rng_seed(20251116, 0, 0, i)) for i in range(args.batches)]
    res = {"config": name, "desc": cfg["desc"], "k": 1, "n": g.n, "m": int(g.indices.numel()), "row_bytes": R,
           "fanout": fan, "batch": B, "graph_gen_s": t_graph}
    tiered = name in CACHE_GIB
    if tiered:
        tiers = build_tiers(name, cfg, g, R, {"train": train}, h2d, hbm_gbs, fan, presample=args.presample)
        res.update(tiers["info"])
        kw = dict(bin_owner=tiers["bin_owner"], bin_ptr=tiers["bin_ptr"], placement=tiers["placement"])
        stride = R
    else:
        stride = (R + 63) // 64 * 64
        table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device=DEV, row_stride_bytes=stride)
        kw = dict(bin_owner=[0], bin_ptr=[table.data_ptr()])
    lanes = []
    for i in range(args.lanes):
        ctx = M.Ctx(n_vertices=g.n, max_seeds=B, max_fanout=fan, device=0, row_bytes=R, row_stride=stride, **kw)
        bufs = M.SampleBuffers.allocate(B, fan, g.n, DEV)
        rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
        lanes.append((ctx, bufs, rows, torch.cuda.Stream(DEV) if i else torch.cuda.current_stream()))
    # per-batch sizes (untimed): |F_h|, E_h, rows per tier
    ctx, bufs, rows, _ = lanes[0]
    F_tot = np.zeros(H + 1)
    E_tot = np.zeros(H)
    hbm_rows = host_rows = 0
    nb_count = min(args.batches, 32)
    for s, r in batches[:nb_count]:
        ctx.sample(g.indptr, g.indices, s, fan, r, bufs)
        c = bufs.counts.cpu().numpy()
        F_tot += c[:H + 1]
        E_tot += c[H + 1:2 * H + 1]
        nF = int(c[H])
        h = int(tiers["in_hbm"][bufs.nodes[:nF]].sum()) if tiered else nF
        hbm_rows += h
        host_rows += nF - h
    F = F_tot / nb_count
    E = E_tot / nb_count
    rows_b = F[H]
    hbm_rows_b, host_rows_b = hbm_rows / nb_count, host_rows / nb_count
    sample_bytes = 16 * F[:H].sum() + 8 * E.sum() + 8 * F[H]
    gather_hbm_bytes = hbm_rows_b * R + rows_b * R + 8 * rows_b + (8 * rows_b if tiered else 0)
    host_bytes = host_rows_b * R
    # timed: every step = moment_step (sample + gather) of one batch, `lanes` batches in flight
    main = torch.cuda.current_stream()

    def run(bs):
        e0 = torch.cuda.Event()
        e0.record(main)
        for L in lanes[1:]:
            L[3].wait_event(e0)
        for i, (s, r) in enumerate(bs):
            c_, b_, rw_, st_ = lanes[i % len(lanes)]
            c_.step(g.indptr, g.indices, s, fan, r, b_, rw_, stream=st_)
        for L in lanes[1:]:
            e = torch.cuda.Event()
            e.record(L[3])
            main.wait_event(e)

    run(batches[:2 * args.lanes])
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(main)
    run(batches)
    b.record(main)
    torch.cuda.synchronize()
    us_batch = a.elapsed_time(b) * 1e3 / len(batches)
    # gather alone, one batch at a time (what the plan's T* predicts): events around moment_gather
    g_us = []
    for s, r in batches[:16]:
        ctx.sample(g.indptr, g.indices, s, fan, r, bufs)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ctx.gather(bufs.nodes, rows, n_dev=bufs.counts[H:H + 1], max_n=bufs.nodes.numel())
        e1.record()
        torch.cuda.synchronize()
        g_us.append(e0.elapsed_time(e1) * 1e3)
    gather_us = float(np.median(g_us))
    t_hbm = (sample_bytes + gather_hbm_bytes) / (hbm_gbs * 1e3)
    t_pcie = host_bytes / (h2d * 1e3)
    tiers_t = {"hbm": t_hbm, "pcie_host": t_pcie}
    bind = max(tiers_t, key=tiers_t.get)
    res.update({
        "lanes": args.lanes, "batches": len(batches),
        "seeds_per_s": B / (us_batch * 1e-6), "us_per_batch": us_batch,
        "mean_F": [float(x) for x in F], "mean_E": [float(x) for x in E],
        "gather_GBs": rows_b * R / (us_batch * 1e3),
        "hbm_hit_rate": hbm_rows_b / max(rows_b, 1),
        "bytes_per_batch": {"sampling_alg": float(sample_bytes), "gather_hbm_alg": float(gather_hbm_bytes),
                            "host_pcie": float(host_bytes)},
        "tier_time_us": tiers_t, "binding_tier": bind, "roofline_frac": tiers_t[bind] / us_batch,
        "peaks": {"hbm_GBs": hbm_gbs, "h2d_GBs": h2d, "pcie_gen5_x16_raw_GBs": 63.0},
        "gather_alone_us": gather_us,
    })
    if tiered:
        N1 = tiers["topo"].info()[0]
        demand = np.zeros(N1, np.int64)
        demand[0] = int(hbm_rows_b * R)
        demand[1] = int(host_bytes)
        t0 = time.perf_counter()
        pl = M.plan(tiers["topo"], [3], demand, 0, int(hbm_gbs * 1000) // 2).info()
        res["plan_s"] = time.perf_counter() - t0
        res["plan_t_star_us"] = pl["t_star"]
        res["plan_prediction_error"] = abs(pl["t_star"] - gather_us) / gather_us
        # the simulation's estimate: demand from held-out batches' counts, not from the measured batches
        hr = tiers["info"]["held_out_rows_per_batch"]
        demand[0], demand[1] = int(hr[0] * R), int(hr[1] * R)
        ph = M.plan(tiers["topo"], [3], demand, 0, int(hbm_gbs * 1000) // 2).info()
        res["plan_t_star_heldout_us"] = ph["t_star"]
        res["plan_heldout_prediction_error"] = abs(ph["t_star"] - gather_us) / gather_us
    # CPU oracle (single thread) on a bounded slice of the same workload: sample + gather (C4/C5 from the ring)
    oracle.build()
    ip, ix = g.indptr.cpu().numpy(), g.indices.cpu().numpy()
    if tiered:
        tab = tiers["keep"][1].numpy()
        ids_of = lambda nodes: nodes % R_PHYS  # noqa: E731
    else:
        tab = np.ascontiguousarray(table[:, :R].cpu().numpy())
        ids_of = lambda nodes: nodes  # noqa: E731
    done, t_or, i = 0, 0.0, 0
    per = 64
    while t_or < args.oracle_s and i < 64:
        s = batches[i][0][:per].cpu().numpy()
        t0 = time.perf_counter()
        o = oracle.sample(ip, ix, s, fan, batches[i][1])
        oracle.gather(tab, ids_of(o["nodes"]))
        t_or += time.perf_counter() - t0
        done += len(s)
        i += 1
    res["oracle"] = {"seeds_per_s": done / t_or, "cores": 1,
                     "sample": f"{i} slices of {per} seeds (sample + gather), single thread"}
    res["gpu_over_oracle"] = res["seeds_per_s"] / res["oracle"]["seeds_per_s"]
    for L in lanes:
        L[0].close()
    del lanes, g
    if tiered:
        del tiers
    else:
        del table
    torch.cuda.empty_cache()
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C4,C5")
    ap.add_argument("--batches", type=int, default=200)
    ap.add_argument("--lanes", type=int, default=8)
    ap.add_argument("--oracle-s", type=float, default=8.0)
    ap.add_argument("--presample", type=int, default=512,
                    help="pre-sample batches for the DDAK hotness (P2); 512 = SURVEY 8(d)'s 64 per rank summed over 8 ranks")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    hbm_gbs, _ = hbm_peak()
    h2d = h2d_peak()
    out = open(args.out, "w") if args.out else None
    for name in args.configs.split(","):
        r = run_config(name, args, hbm_gbs, h2d)
        line = json.dumps(r)
        print(line, flush=True)
        if out:
            out.write(line + "\n")
            out.flush()


if __name__ == "__main__":
    main()
