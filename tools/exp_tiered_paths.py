"""Tiered gather (local HBM bin + pinned host bin behind a placement map): LDG.128 vs TMA bulk copies.

The routed/tiered gather reads rows with LDG.128 (`gather_kernel`); `MOMENT_GATHER_PATH=bulk` forces the TMA
bulk-copy gather (one cp.async.bulk per row from wherever the placement points, host rows included). This
checks the bulk path is byte-exact on a host tier and times both at several host fractions.

    python tools/exp_tiered_paths.py
"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402
import workloads as W  # noqa: E402

DEV = "cuda:0"


def run(path, host_frac, n=1 << 22, R=512, m=1 << 18, reps=20):
    os.environ["MOMENT_GATHER_PATH"] = path
    rng = np.random.default_rng(3)
    bin_of = (rng.random(n) < host_frac).astype(np.int32)
    slot_of = np.zeros(n, np.int64)
    for b in (0, 1):
        sel = np.nonzero(bin_of == b)[0]
        slot_of[sel] = rng.permutation(len(sel))
    ids_all = torch.arange(n, device=DEV)
    feats = W.feature_rows(ids_all[: 1 << 16], R // 4, torch.float32)  # 64 k distinct rows, tiled
    table = feats[torch.arange(n, device=DEV) % (1 << 16)]
    bins = []
    for b in (0, 1):
        sel = torch.as_tensor(np.nonzero(bin_of == b)[0], device=DEV)
        buf = torch.empty((max(1, len(sel)), R), dtype=torch.uint8, device=DEV)
        if len(sel):
            buf[torch.as_tensor(slot_of[sel.cpu().numpy()], device=DEV)] = table[sel]
        if b == 1:
            h = torch.empty(buf.shape, dtype=torch.uint8).pin_memory()
            h.copy_(buf)
            buf = h
        bins.append(buf)
    placement = torch.as_tensor(M.place_pack(bin_of, slot_of).view(np.int64), device=DEV)
    ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], device=0, row_bytes=R, bin_owner=[0, -1],
                bin_ptr=[b.data_ptr() for b in bins], placement=placement)
    ids = torch.as_tensor(rng.integers(0, n, m), device=DEV)
    out = torch.empty((m, R), dtype=torch.uint8, device=DEV)
    ctx.gather(ids, out)
    torch.cuda.synchronize()
    ok = bool(torch.equal(out, table[ids]))
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        ctx.gather(ids, out)
    e1.record()
    torch.cuda.synchronize()
    us = e0.elapsed_time(e1) * 1e3 / reps
    host_rows = int((bin_of[ids.cpu().numpy()] == 1).sum())
    return {"path": path, "host_frac": host_frac, "byte_exact": ok, "us": us, "rows": m,
            "host_GBs": host_rows * R / us / 1e3, "total_GBs": m * R / us / 1e3}


def main():
    for hf in (0.0, 0.05, 0.25, 1.0):
        for path in ("ldg", "bulk"):
            print(json.dumps(run(path, hf)), flush=True)


if __name__ == "__main__":
    main()
