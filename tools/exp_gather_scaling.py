"""Single-launch gather time vs number of rows (C2 table, 400-byte rows at a 448-byte stride): the slope is
the steady-state bandwidth, the intercept the fixed launch / ramp / tail cost. L2 is flushed before each
timed launch.   python tools/exp_gather_scaling.py [--reps 50]   (knobs via MOMENT_BULK / MOMENT_GATHER_PATH)
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
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--sizes", default="7500,15000,30000,60000,120000,240000,480000,960000")
    ap.add_argument("--row-bytes", type=int, default=0, help="bytes gathered per row (default: the C2 row, 400)")
    ap.add_argument("--stride", type=int, default=0, help="row stride in bytes (default: R rounded up to 64)")
    ap.add_argument("--overhead", action="store_true", help="also time launch overheads (tiny / repeated launches)")
    a = ap.parse_args()
    cfg = W.CONFIGS["C2"]
    n = cfg["n"]
    R = a.row_bytes or cfg["dim"] * 4
    stride = a.stride or (R + 63) // 64 * 64
    table = torch.empty((n, stride), dtype=torch.uint8, device="cuda")
    table.random_(0, 255)
    sizes = [int(s) for s in a.sizes.split(",")]
    ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], rank=0, world=1, device=0, row_bytes=R,
                row_stride=stride, bin_owner=[0], bin_ptr=[table.data_ptr()])
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    g = torch.Generator(device="cuda")
    g.manual_seed(1)
    out = torch.empty((max(sizes), R), dtype=torch.uint8, device="cuda")
    print(f"{'rows':>8s} {'us':>8s} {'GB/s alg':>9s}  (alg bytes = rows x (2R + 8))")
    pts = []
    for m in sizes:
        ids = torch.randperm(n, device="cuda", generator=g)[:m].sort().values
        ts = []
        for r in range(a.reps + 3):
            flush.fill_(r & 0xff)
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            ctx.gather(ids, out)
            e1.record()
            torch.cuda.synchronize()
            if r >= 3:
                ts.append(e0.elapsed_time(e1) * 1000)
        ts.sort()
        us = ts[len(ts) // 2]
        gbs = m * (2 * R + 8) / us / 1e3
        pts.append((m, us))
        print(f"{m:8d} {us:8.2f} {gbs:9.1f}", flush=True)
    # least squares on the three largest sizes: us = a + b * rows
    xs, ys = [p[0] for p in pts[-3:]], [p[1] for p in pts[-3:]]
    mx, my = sum(xs) / 3, sum(ys) / 3
    b = sum((x - mx) * (y - my) for x, y in zip(xs, ys)) / sum((x - mx) ** 2 for x in xs)
    if a.overhead:
        def t(fn, flush_first):
            ts = []
            for r in range(a.reps + 3):
                if flush_first:
                    flush.fill_(r & 0xff)
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                torch.cuda.synchronize()
                if r >= 3:
                    ts.append(e0.elapsed_time(e1) * 1000)
            return sum(ts) / len(ts)
        tiny = torch.zeros(1, device="cuda")
        ids32 = torch.arange(32, device="cuda", dtype=torch.int64)
        ids120 = torch.randperm(n, device="cuda", generator=g)[:120000].sort().values
        for fl in (False, True):
            print(f"flush={fl}: noop {t(lambda: tiny.add_(1), fl):.2f} us, gather32 {t(lambda: ctx.gather(ids32, out), fl):.2f} us, "
                  f"2x gather32 {t(lambda: (ctx.gather(ids32, out), ctx.gather(ids32, out)), fl):.2f} us, "
                  f"gather120k {t(lambda: ctx.gather(ids120, out), fl):.2f} us, "
                  f"2x gather120k {t(lambda: (ctx.gather(ids120, out), ctx.gather(ids120, out)), fl):.2f} us, "
                  f"noop+gather120k {t(lambda: (tiny.add_(1), ctx.gather(ids120, out)), fl):.2f} us", flush=True)
    print(f"fit (3 largest): intercept {my - b * mx:.2f} us, slope -> {(2 * R + 8) / b / 1e3:.1f} GB/s")


if __name__ == "__main__":
    main()
