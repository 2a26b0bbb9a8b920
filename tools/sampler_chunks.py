"""How many 64-byte DRAM atoms the C2 sampler must touch per batch (CPU, oracle-driven analysis).

For the first 8 batches of C2 (or --config): per hop, the frontier size, how many nodes take all their neighbours
(d <= k: one contiguous run) or draw Floyd positions (d > k), and the number of distinct 64-byte chunks of
`indices` those reads touch (Floyd positions simulated uniformly, the chunk count does not depend on which
k-subset it is); plus how much of the node visits a hub cache of the hottest adjacency lists would cover.
Output: profiles/r02_sampler_chunks.txt.
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
import workloads as W  # noqa: E402


def main():
    import argparse

    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--batches", type=int, default=8)
    ap.add_argument("--device", default="cpu", help="where to generate the graph (cuda: fast, then copied to host)")
    a = ap.parse_args()
    oracle.build()
    cfg = W.CONFIGS[a.config]
    t = time.time()
    g = W.rmat_csr(cfg["n"], cfg["m"], device=a.device)
    g = W.Graph(g.indptr.cpu(), g.indices.cpu(), g.n, g.m)
    print("graph built in %.1f s" % (time.time() - t))
    ip, ix = g.indptr.numpy(), g.indices.numpy()
    deg = np.diff(ip)
    bs = W.epoch_batches(W.training_set(g, min_count=1024), 1024, 0)
    rng = np.random.default_rng(0)
    fan = list(cfg["fanout"])
    tot, freq = {}, np.zeros(g.n, np.int64)
    nb = a.batches
    for b in range(nb):
        r = oracle.sample(ip, ix, bs[b].numpy(), fan, W.batch_rng_seed(1, 0, 0, b))
        c = r["counts"]
        F = c[: len(fan) + 1]
        nodes = r["nodes"]
        if b == 0:
            print("counts of batch 0 (|F_0..F_H|, E_0..E_H-1):", c.tolist())
        for h, k in enumerate(fan):
            v = nodes[: F[h]]
            d, lo = deg[v], ip[v]
            take = d <= k
            ch_take = ((lo[take] + d[take]) * 4 + 63) // 64 - (lo[take] * 4) // 64
            ch_take[d[take] == 0] = 0
            ch_f = [len(np.unique(((ll + rng.choice(dd, k, replace=False)) * 4) // 64))
                    for dd, ll in zip(d[~take], lo[~take])]
            tot.setdefault(h, np.zeros(6))
            tot[h] += [F[h], take.sum(), ch_take.sum(), (~take).sum(), sum(ch_f), F[h - 1] if h else 0]
            freq[v] += 1
    allc = 0
    for h, t_ in tot.items():
        t_ = t_ / nb
        allc += t_[2] + t_[4] + t_[0]
        print("hop %d: |F_h| %d, take-all %d (%d chunks), Floyd %d (%d chunks), re-sampled from F_h-1 %d" % tuple([h] + list(t_)))
    print("random 64-byte reads per batch (indptr + indices): %d = %.1f MB" % (allc, allc * 64 / 1e6))
    order = np.argsort(-freq)
    cum = np.cumsum(deg[order] * 4)
    for mb in (8, 16, 32, 64):
        m = int(np.searchsorted(cum, mb << 20))
        print("hub cache of %d MB: top %d vertices, %.3f of node visits" % (mb, m, freq[order[:m]].sum() / freq.sum()))


if __name__ == "__main__":
    main()
