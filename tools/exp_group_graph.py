"""Timing-only experiment: K steps on P lanes captured as ONE CUDA graph (each lane's step a branch; the
moment_step calls see a capturing stream and launch their kernels directly into it), replayed as one launch,
against the bench's K steps issued one moment_step graph launch per step. The replayed batches are fixed at
capture (timing only: the product API would re-parameterise each branch's call node per launch).

    python tools/exp_group_graph.py [--lanes 20] [--steps 20] [--regions 300]
"""
import argparse
import json
import os
import statistics
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, nargs="+", default=[16, 20])
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--regions", type=int, default=300)
    ap.add_argument("--config", default="C2")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, max(a.lanes))
    K = a.steps
    main_s = torch.cuda.current_stream()
    pool = [st.batch(i) for i in range(256)]
    out = {}
    for P in a.lanes:
        lanes = st.lanes[:P]
        for i in range(2 * P):
            st.step(*pool[i % 256], lane=i % P)
        torch.cuda.synchronize()

        def issue(first):
            e0 = torch.cuda.Event()
            e0.record(torch.cuda.current_stream())
            for L in lanes:
                L.stream.wait_event(e0)
            for j in range(K):
                st.step(*pool[(first + j) % 256], lane=j % P)
            cur = torch.cuda.current_stream()
            for L in lanes:
                e = torch.cuda.Event()
                e.record(L.stream)
                cur.wait_event(e)

        def region_direct(first):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(main_s)
            t0 = time.perf_counter()
            with torch.cuda.stream(main_s):
                issue(first)
            t = time.perf_counter() - t0
            e1.record(main_s)
            torch.cuda.synchronize()
            return e0.elapsed_time(e1), t * 1e6

        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            issue(0)
        torch.cuda.synchronize()
        g.replay()
        torch.cuda.synchronize()

        def region_graph():
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(main_s)
            t0 = time.perf_counter()
            g.replay()
            t = time.perf_counter() - t0
            e1.record(main_s)
            torch.cuda.synchronize()
            return e0.elapsed_time(e1), t * 1e6

        for rep in range(2):
            d = [region_direct(r * K) for r in range(a.regions)]
            gg = [region_graph() for _ in range(a.regions)]
            for name, v in (("per_step_launch", d), ("one_graph", gg)):
                ms = statistics.median(x[0] for x in v)
                out[f"P{P}_{name}_{rep}"] = {"region_ms": ms, "seeds_per_s_M": st.B * K / ms / 1e3,
                                             "host_us_per_region": statistics.median(x[1] for x in v)}
        del g
        torch.cuda.synchronize()
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
