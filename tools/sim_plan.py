"""Planner simulation at k = 1, 2, 4, 8 B200: the time-bisection plan's predicted
per-batch gather time T* for DDAK placement with and without replicated hot rows (R25), on an HGX B200
topology graph (`boxes.hgx_b200`), from hotness pre-sampled on the GPU at full graph size.

The paper evaluates candidate layouts with its model instead of running every one and reports
its prediction error against measurement (8.61 %); the k = 1 rows here can be compared with the
measured gathers of profiles/r01_results_matrix.jsonl. k > 1 is a PREDICTION (the pool's boxes have one
GPU): NVLink at the measured 770 GB/s peer-copy rate per direction (900 nominal), host DRAM / UPI capacities
assumed (boxes.py).

    python tools/sim_plan.py [--configs C3,C4,C5] [--batches 512] [--switch 1] [--subsets] [--out FILE]

Per config and k: T*(r) for the candidate replica counts r, the best r, and the (T_ingest, T_nvlink, T_hbm)
breakdown of r = 0 and of the best r. Predicted seeds/s = k * batch / T*. Placement uses the pre-sample
hotness; the per-bin demand is counted on held-out batches (an in-sample estimate would credit the HBM bins
with every pre-sampled row and under-state the host traffic).
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
# HBM feature budget per GPU (GiB): C3 = the whole 57 GB table fits one B200 (leaves room for the CSR and
# workspaces); C4 / C5 = the SURVEY 8(d) cache sizes.
BUDGET_GIB = {"C2": 100, "C3": 120, "C4": 32, "C5": 64}


def counts(cfg, batches, held):
    """F_H appearance counts: `batches` pre-sample batches (placement hotness, R18: rng epoch 2^32 - 1) and
    `held` held-out training batches (other seeds, other rng stream) whose counts estimate the per-bin demand
    the placement will actually see."""
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    fan = list(cfg["fanout"])
    B = cfg["batch"]
    train = W.training_set(g, min_count=B)
    allb = []
    e = 0
    while len(allb) < batches + held:
        allb += W.epoch_batches(train, B, e)
        e += 1
    ctx = M.Ctx(n_vertices=g.n, max_seeds=B, max_fanout=fan, device=0)
    bufs = M.SampleBuffers.allocate(B, fan, g.n, DEV)
    hot = torch.zeros(g.n, dtype=torch.int64, device=DEV)
    dem = torch.zeros(g.n, dtype=torch.int64, device=DEV)
    H = len(fan)
    nF = 0
    for i in range(batches + held):
        pre = i < batches
        seed = W.batch_rng_seed(5, 2**32 - 1, 0, i) if pre else W.batch_rng_seed(1, 0, 0, i)
        seeds = allb[i] if pre else allb[len(allb) - 1 - (i - batches)]
        ctx.step(g.indptr, g.indices, seeds, fan, seed, bufs, None)
        ctx.hotness(bufs.nodes, hot if pre else dem, n_dev=bufs.counts[H:H + 1], max_n=bufs.nodes.numel())
        nF += int(bufs.counts[H]) if i < 8 else 0
    torch.cuda.synchronize()
    out = hot.cpu().numpy().astype(np.uint64), dem.cpu().numpy().astype(np.uint64)
    del g, ctx, bufs, hot, dem
    torch.cuda.empty_cache()
    return out[0], out[1], nF / 8


def breakdown(topo, box, active, hot, dem, caps, bin_node, R, held, r, nv, hbm, mode=M.PLACE_DDAK):
    b, s, A, U, T = M.place(topo, hot, caps, bin_node=bin_node, replicate_rows=r, traffic_mode=M.TRAFFIC_STANDALONE,
                            mode=mode)
    N = topo.info()[0]
    per_bin = np.bincount(b.astype(np.int64) + 2, weights=dem.astype(np.float64), minlength=len(bin_node) + 2)
    d = np.zeros(N, np.int64)
    for i, v in enumerate(bin_node):
        d[v] += int(per_bin[i + 2]) * R // held
    rep = int(per_bin[0])
    p = M.plan(topo, [box.gpu[g] for g in active], d, nv, hbm, replica_demand=rep * R // held).info()
    hbm_rows = int(U[:len(active)].sum())
    return {"t_star": p["t_star"], "t_ingest": p["t_ingest"], "t_nvlink": p["t_nvlink"], "t_hbm": p["t_hbm"],
            "partition_rows_hbm": hbm_rows, "host_rows": int(U[len(active):].sum()),
            "host_bytes_per_gpu_batch": int(sum(d[v] for v in box.host_bin)),
            "peer_bytes_per_gpu_batch": int(sum(d[box.hbm_bin[g]] for g in active) * (len(active) - 1) // len(active)),
            "replica_bytes_per_gpu_batch": rep * R // held,
            # the paper's QPI traffic: host bytes of all k GPUs' batches that cross sockets in
            # the plan's ingest flow (UPI links), per batch
            "upi_bytes_per_batch": box.upi_bytes(p["link_flow"]),
            "host_bytes_per_batch_all_gpus": int(sum(d[v] for v in box.host_bin)) * len(active)}


def evaluate(name, cfg, hot, dem, R, k, active, cap_gpu, a, hbm_gbs, nv_gbs, mean_fh, t_hot, gps, box_kw=None,
             provenance=None):
    n = len(hot)
    kw = dict(box_kw or {})
    kw.setdefault("hbm_gbs", hbm_gbs)
    hbm_gbs = kw["hbm_gbs"]
    box = M.boxes.hgx_b200(8, gpus_per_switch=gps, active=active, **kw)
    topo = box.topology()
    bin_node = [box.hbm_bin[g] for g in active] + box.host_bin
    caps = [cap_gpu] * k + [n, n]
    cand = sorted({0} | {min(n, cap_gpu * f // 64) for f in (1, 4, 8, 16, 32, 48, 64)})
    t1 = time.perf_counter()
    ts, best = M.replicate_search(topo, hot, caps, cand, gpu_node=[box.gpu[g] for g in active],
                                  nvlink_cap=int(nv_gbs * 1000), hbm_cap=int(hbm_gbs * 1000), row_bytes=R,
                                  hot_batches=a.batches, bin_node=bin_node, demand_counts=dem,
                                  demand_batches=a.held, traffic_mode=M.TRAFFIC_STANDALONE)
    t_search = time.perf_counter() - t1
    nv, hb = int(nv_gbs * 1000), int(hbm_gbs * 1000)
    b0 = breakdown(topo, box, active, hot, dem, caps, bin_node, R, a.held, 0, nv, hb)
    bb = breakdown(topo, box, active, hot, dem, caps, bin_node, R, a.held, cand[best], nv, hb)
    bh = breakdown(topo, box, active, hot, dem, caps, bin_node, R, a.held, 0, nv, hb, mode=M.PLACE_HASH)
    line = {"config": name, "k": k, "active_gpus": active, "gpus_per_switch": gps, "row_bytes": R,
            "n": n, "hbm_budget_rows_per_gpu": cap_gpu, "pre_sample_batches": a.batches, "held_out_batches": a.held,
            "mean_F_H": mean_fh, "candidates_r": cand, "t_star_us": [int(x) for x in ts],
            "best_r": cand[best], "ddak": b0, "ddak_replicated": bb, "hash": bh,
            "ddak_over_hash_t_star": bh["t_star"] / max(1, b0["t_star"]),
            "pred_seeds_per_s_ddak": k * cfg["batch"] / (b0["t_star"] * 1e-6),
            "pred_seeds_per_s_best": k * cfg["batch"] / (bb["t_star"] * 1e-6),
            "search_s": t_search, "hotness_s": t_hot,
            "capacities": {"nvlink_gbs": nv_gbs, "hbm_gbs": hbm_gbs,
                           **{kk: kw.get(kk, dflt) for kk, dflt in (("dram_gbs", 250.0), ("upi_gbs", 62.0),
                                                                    ("port_gbs", 55.6))}},
            "provenance": provenance or {"port_gbs": "measured r01 (55.6)", "hbm_gbs": "MEASURED_PEAKS.json",
                                         "nvlink_gbs": "B200_PROFILING.md peer copy", "dram_gbs": "assumed",
                                         "upi_gbs": "assumed"}}
    print(f"{name} k={k} gpus={active} per-switch={gps}: T*(r) {list(zip(cand, [int(x) for x in ts]))} best r={cand[best]}; "
          f"DDAK T*={b0['t_star']} (ing {b0['t_ingest']}, nv {b0['t_nvlink']}, hbm {b0['t_hbm']}) "
          f"-> +repl T*={bb['t_star']} (ing {bb['t_ingest']}, nv {bb['t_nvlink']}, hbm {bb['t_hbm']}); "
          f"pred {line['pred_seeds_per_s_ddak']/1e6:.2f} -> {line['pred_seeds_per_s_best']/1e6:.2f} M seeds/s; "
          f"hash T*={bh['t_star']} UPI {bh['upi_bytes_per_batch']/1e6:.1f} MB vs DDAK {b0['upi_bytes_per_batch']/1e6:.1f} MB "
          f"(search {t_search:.1f} s)", flush=True)
    return line


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C3,C4,C5")
    ap.add_argument("--batches", type=int, default=512, help="pre-sample batches (placement hotness)")
    ap.add_argument("--held", type=int, default=128, help="held-out batches (demand estimate)")
    ap.add_argument("--switch", default="1", help="GPUs per PCIe switch, a list (1 = direct to the socket)")
    ap.add_argument("--ks", default="1,2,4,8")
    ap.add_argument("--nvlink-gbs", type=float, default=770.0,
                    help="NVLink per direction per GPU: the measured B200 peer copy (B200_PROFILING; 900 nominal)")
    ap.add_argument("--subsets", action="store_true",
                    help="evaluate every class of active-GPU sets up to the box symmetry (P:L229-233)")
    ap.add_argument("--out", default="gpurun_out/plan_sim.jsonl")
    ap.add_argument("--probe", default=None, help="tools/probe_box.py JSON: measured capacities for the graph")
    a = ap.parse_args()
    box_kw, prov = None, None
    if a.probe:
        with open(a.probe) as f:
            box_kw, prov = M.boxes.from_probe(json.load(f))
        a.nvlink_gbs = prov.pop("nvlink_value")
    peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))) if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else {"hbm_gbs": 6543.4}
    hbm_gbs = float(peaks["hbm_gbs"])
    nv_gbs = a.nvlink_gbs
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    fout = open(a.out, "a")
    for name in a.configs.split(","):
        cfg = W.CONFIGS[name]
        R = cfg["dim"] * torch.tensor([], dtype=cfg["dtype"]).element_size()
        t0 = time.perf_counter()
        hot, dem, mean_fh = counts(cfg, a.batches, a.held)
        t_hot = time.perf_counter() - t0
        n = len(hot)
        cap_gpu = min(n, (BUDGET_GIB[name] << 30) // R)
        for gps, k in [(int(g), int(x)) for g in a.switch.split(",") for x in a.ks.split(",")]:
            subsets = (M.boxes.gpu_subset_classes(k, gpus_per_switch=gps) if a.subsets
                       else [M.boxes.spread_gpus(k, gpus_per_switch=gps)])
            for active in subsets:
                line = evaluate(name, cfg, hot, dem, R, k, active, cap_gpu, a, hbm_gbs, a.nvlink_gbs, mean_fh, t_hot,
                                gps, box_kw, prov)
                fout.write(json.dumps(line) + "\n")
                fout.flush()
        del hot, dem


if __name__ == "__main__":
    main()
