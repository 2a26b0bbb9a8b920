"""Random-access rate of HBM: gathers of small rows (16/32/64 B) at uniformly random ids from tables of
0.25-8 GB, through the product's gather kernels (tile::gather4 with 64-byte L2 promotion, and LDG.128).
One gathered row = one random DRAM access once the table exceeds L2: rows/s bounds how many random
sampler loads (CSR indices, lidx) per second the memory system can serve.

    python tools/exp_random_access.py
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402


def run(table_bytes, R, path, n=1 << 23, reps=10):
    os.environ["MOMENT_GATHER_PATH"] = path
    rows = table_bytes // R
    table = torch.empty((rows, R), dtype=torch.uint8, device="cuda:0")
    ctx = M.Ctx(n_vertices=rows, max_seeds=1, max_fanout=[1], device=0, row_bytes=R, row_stride=R, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    g = torch.Generator(device="cuda:0").manual_seed(1)
    ids = [torch.randint(0, rows, (n,), device="cuda:0", generator=g) for _ in range(reps)]
    out = torch.empty((n, R), dtype=torch.uint8, device="cuda:0")
    for i in range(3):
        ctx.gather(ids[i], out)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(reps):
        ctx.gather(ids[i], out)
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / reps
    ctx.close()
    del table
    return n / us / 1e3  # G rows/s


def main():
    print(f"{'table':>8s} {'R':>4s} {'path':>6s} {'G rows/s':>9s} {'GB/s (64 B per row)':>20s}")
    for tb in (256 << 20, 2 << 30, 8 << 30):
        for R in (16, 64):
            for path in ("tma4", "ldg"):
                r = run(tb, R, path)
                print(f"{tb / 2**30:7.2f}G {R:4d} {path:>6s} {r:9.2f} {r * 64:20.0f}", flush=True)


if __name__ == "__main__":
    main()
