"""The sampler against its own bound: the DRAM random-access rate (64-byte atoms), not bytes.

Times C2 sampling alone (moment_step with no rows: H x (hop sample + bitscan) + compaction) with P batches in
flight, and the full step, through the bench's own State; the random atoms a C2 batch must touch come from
tools/sampler_chunks.py (profiles/r02_sampler_chunks.txt: 267 750 per batch = indptr line per resampled node +
distinct 64-byte chunks of `indices` per node), the atom rate roofline from tools/exp_random_access.py
(profiles/r01_random_access.txt: 35.8 G random 16-byte rows/s from an 8 GB table, each one DRAM atom).

    python tools/sampler_roofline.py [--lanes 16] [--batches 4000]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

ATOMS_PER_BATCH = 267750  # profiles/r02_sampler_chunks.txt
ATOM_RATE = 35.75e9       # profiles/r01_random_access.txt, LDG, 8 GB table, 16-byte rows


def timed(st, n, rows):
    P = len(st.lanes)
    main = torch.cuda.current_stream()
    for i in range(2 * P):
        L = st.lanes[i % P]
        s, r = st.batch(i)
        L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs, L.rows if rows else None, stream=L.stream)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    batches = [st.batch(i) for i in range(n)]
    e0.record(main)
    for L in st.lanes[1:]:
        L.stream.wait_event(e0)
    for i in range(n):
        L = st.lanes[i % P]
        s, r = batches[i]
        L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs, L.rows if rows else None, stream=L.stream)
    for L in st.lanes[1:]:
        ev = torch.cuda.Event()
        ev.record(L.stream)
        main.wait_event(ev)
    e1.record(main)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / n  # us per batch


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=16)
    ap.add_argument("--batches", type=int, default=4000)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--atoms", type=float, default=ATOMS_PER_BATCH, help="random atoms per batch of the config")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, a.lanes)
    us_s = timed(st, a.batches, False)
    us_f = timed(st, a.batches, True)
    floor = a.atoms / ATOM_RATE * 1e6
    print(json.dumps({"config": a.config, "lanes": a.lanes, "sampling_only_us_per_batch": us_s,
                      "full_step_us_per_batch": us_f, "random_atoms_per_batch": a.atoms,
                      "atom_rate_roofline_G_per_s": ATOM_RATE / 1e9,
                      "sampling_atom_floor_us": floor, "sampling_frac_of_atom_roofline": floor / us_s,
                      "achieved_G_atoms_per_s": a.atoms / us_s / 1e3}))


if __name__ == "__main__":
    main()
