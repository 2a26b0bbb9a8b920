"""Offline planner cost at full vertex counts (cf. the paper's "~14 s" for Max-Flow + DDAK on UK):
the product's planner (Dinic + DDAK, C++, libmoment.so) beside the oracle (Edmonds-Karp + DDAK, plain
single-threaded C) on the same inputs, CPU only.

Inputs: the HGX B200 topology graph (`boxes.hgx_b200`, 8 GPUs), a power-law hotness over n vertices (the
shape pre-sampling gives on R-MAT graphs; seeded numpy), bins = 8 HBM caches (C3: ceil(n / 8) rows each, all
in HBM; C4 / C5: the SURVEY 8(d) 32 / 64 GiB caches) + 2 host DRAM bins. Both placements are checked equal.

    python tools/planner_times.py [--configs C3,C4,C5]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402

N = {"C3": 111_059_956, "C4": 244_160_499, "C5": 269_346_174}
ROW = {"C3": 512, "C4": 1536, "C5": 4096}
CACHE_GIB = {"C4": 32, "C5": 64}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C3,C4,C5")
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    oracle.build()
    rows = []
    for name in a.configs.split(","):
        n = N[name]
        rng = np.random.default_rng(1)
        hot = np.floor(rng.pareto(1.2, n) * 3).astype(np.uint64)  # most vertices 0-2, a heavy tail
        box = M.boxes.hgx_b200(8)
        topo = box.topology()
        bin_node = [box.hbm_bin[g] for g in range(8)] + box.host_bin
        if name == "C3":
            caps = [-(-n // 8)] * 8 + [0, 0]
        else:
            c = (CACHE_GIB[name] << 30) // ROW[name]
            caps = [c] * 8 + [n, n]
        t0 = time.perf_counter()
        F, flow = topo.maxflow()
        t_mf = time.perf_counter() - t0
        nodes, links, s, t = topo.export()
        traffic = []
        for v in bin_node:
            traffic.append(int(sum(f for (u, w, _), f in zip(links, flow) if u == s and w == v)))
        t0 = time.perf_counter()
        b, sl, *_ = M.place(topo, hot, caps, bin_node=bin_node, bin_traffic=traffic)
        t_ddak = time.perf_counter() - t0
        t0 = time.perf_counter()
        oF, oflow = oracle.maxflow(len(nodes), links, s, t)
        t_omf = time.perf_counter() - t0
        tiers = [0] * 8 + [1, 1]  # GPU tier first (R14)
        t0 = time.perf_counter()
        ob, osl, *_ = oracle.ddak(hot, tiers, caps, traffic, 100)
        t_oddak = time.perf_counter() - t0
        same = bool(np.array_equal(b, ob) and np.array_equal(sl, osl))
        line = {"config": name, "n_vertices": n, "bins": len(caps), "pool": 100,
                "product": {"maxflow_s": t_mf, "ddak_s": t_ddak, "total_s": t_mf + t_ddak},
                "oracle": {"maxflow_s": t_omf, "ddak_s": t_oddak, "total_s": t_omf + t_oddak},
                "maxflow_equal": F == oF, "placement_equal": same,
                "paper": "~14 s Max-Flow + DDAK on UK (P:L265), other hardware"}
        print(json.dumps(line), flush=True)
        rows.append(line)
        del hot, b, sl, ob, osl
    if a.out:
        with open(a.out, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
