"""Is the gather kernel limited by itself or by random-row DRAM efficiency? Times one gather launch of m rows
of the C2 table (400-byte rows, 448-byte stride, 1.1 GB > L2) for different id orders: sequential rows,
sorted random rows, unsorted random rows; each warm back to back (one event pair over `reps` launches, so
dirty output lines of the previous launch are written back inside the next one, as in a bench step) and
with L2 flushed before a single launch. torch.index_select on the same rows is the library yardstick.
    python tools/exp_gather_locality.py [--rows 120000] [--reps 40]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as W  # noqa: E402
import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--rows", default="120000", help="comma-separated row counts")
    ap.add_argument("--orders", default="sequential,sorted random,unsorted random")
    ap.add_argument("--reps", type=int, default=40)
    a = ap.parse_args()
    cfg = W.CONFIGS["C2"]
    n = cfg["n"]
    R = cfg["dim"] * 4
    stride = (R + 63) // 64 * 64
    table = torch.empty((n, stride), dtype=torch.uint8, device="cuda")
    table.random_(0, 255)
    ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], rank=0, world=1, device=0, row_bytes=R,
                row_stride=stride, bin_owner=[0], bin_ptr=[table.data_ptr()])
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    for m in [int(x) for x in a.rows.split(",")]:
        run(a, ctx, table, flush, g, n, R, stride, m)


def run(a, ctx, table, flush, g, n, R, stride, m):
    outs = [torch.empty((m, R), dtype=torch.uint8, device="cuda") for _ in range(4)]
    peak = 6543.4
    orders = {
        "sequential": torch.arange(m, device="cuda", dtype=torch.int64),
        "sorted random": torch.randperm(n, device="cuda", generator=g)[:m].sort().values,
        "unsorted random": torch.randperm(n, device="cuda", generator=g)[:m],
    }
    alg = m * (2 * R + 8)
    print(f"rows {m}, R {R}, stride {stride}; alg bytes/launch {alg/1e6:.1f} MB; peak {peak} GB/s")
    print(f"{'order':>16s} {'warm b2b us':>12s} {'frac':>6s} {'flushed us':>11s} {'frac':>6s} {'index_select b2b us':>20s}")
    tab_view = table[:, :R]
    for name, ids in orders.items():
        if name not in a.orders.split(","):
            continue
        for _ in range(3):
            ctx.gather(ids, outs[0])
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for r in range(a.reps):
            ctx.gather(ids, outs[r & 3])
        e1.record()
        torch.cuda.synchronize()
        b2b = e0.elapsed_time(e1) * 1000 / a.reps
        ts = []
        for r in range(a.reps):
            flush.fill_(r & 0xff)
            f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            f0.record()
            ctx.gather(ids, outs[0])
            f1.record()
            torch.cuda.synchronize()
            ts.append(f0.elapsed_time(f1) * 1000)
        ts.sort()
        fl = ts[len(ts) // 2]
        e0.record()
        for r in range(a.reps):
            torch.index_select(tab_view, 0, ids, out=outs[r & 3])
        e1.record()
        torch.cuda.synchronize()
        isel = e0.elapsed_time(e1) * 1000 / a.reps
        print(f"{name:>16s} {b2b:12.2f} {alg/b2b/1e3/peak:6.3f} {fl:11.2f} {alg/fl/1e3/peak:6.3f} {isel:20.2f}",
              flush=True)


if __name__ == "__main__":
    main()
