"""Kernel efficiency vs batch size: one moment_step with B seeds (1 lane), edges sampled per us."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402
import workloads as W  # noqa: E402


def main():
    import argparse
    ap = argparse.ArgumentParser()
    ap.add_argument("--sizes", default="1024,2048,4096,8192,16384")
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    cfg = W.CONFIGS["C2"]
    g = W.rmat_csr(cfg["n"], cfg["m"], device="cuda:0")
    fan = list(cfg["fanout"])
    train = W.training_set(g, min_count=65536)
    perm = train[torch.randperm(len(train), generator=torch.Generator().manual_seed(0))]
    for B in [int(x) for x in a.sizes.split(",")]:
        ctx = M.Ctx(n_vertices=g.n, max_seeds=B, max_fanout=fan, device=0)
        bufs = M.SampleBuffers.allocate(B, fan, g.n, "cuda:0")
        seeds = [perm[(i * B) % (len(perm) - B):][:B].contiguous().cuda() for i in range(a.steps)]
        for i in range(3):
            ctx.step(g.indptr, g.indices, seeds[i % len(seeds)], fan, i, bufs, None)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(a.steps):
            ctx.step(g.indptr, g.indices, seeds[i], fan, 100 + i, bufs, None)
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / a.steps
        c = bufs.counts.cpu().tolist()
        E = sum(c[len(fan) + 1:])
        print(f"B={B:6d}: {us:7.1f} us/step  F_H={c[len(fan)]:8d}  E={E:8d}  {E / us:8.0f} edges/us  "
              f"{B / us:6.1f} seeds/us", flush=True)


if __name__ == "__main__":
    main()
