"""Warm per-kernel timeline of bench steps (torch.profiler / CUPTI), CPU issue time and graph replay.

    python tools/step_timeline.py [--config C2] [--steps 20]

Prints, per kernel name, the mean warm device time and the mean idle gap before it, plus the host time
to issue one step and the device time of one step replayed from a CUDA graph.
"""
import argparse
import os
import sys
import time
from collections import defaultdict

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--steps", type=int, default=20)
    args = ap.parse_args()
    st = bench.build_state(args.config, "cuda:0", 0, 1)
    batches = [st.batch(i) for i in range(args.steps + 5)]
    for i in range(5):
        st.step(*batches[i])
    torch.cuda.synchronize()
    # host issue time per step (no sync inside)
    t0 = time.perf_counter()
    for i in range(args.steps):
        st.step(*batches[5 + i])
    t_issue = (time.perf_counter() - t0) / args.steps
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(args.steps):
        st.step(*batches[5 + i])
    e1.record()
    torch.cuda.synchronize()
    t_dev = e0.elapsed_time(e1) / args.steps * 1e3
    # graph replay of one step (same batch): device time without host launch overhead
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        st.step(*batches[5], stream=s)
        torch.cuda.synchronize()
        with torch.cuda.graph(g, stream=s):
            st.step(*batches[5], stream=s)
    torch.cuda.synchronize()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    e0.record()
    for _ in range(args.steps):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    t_graph = e0.elapsed_time(e1) / args.steps * 1e3
    print(f"host issue per step {t_issue * 1e6:.1f} us | stream device per step {t_dev:.1f} us | "
          f"graph replay per step {t_graph:.1f} us")
    from torch.profiler import ProfilerActivity, profile

    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for i in range(args.steps):
            st.step(*batches[5 + i])
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type.name == "CUDA"]
    evs.sort(key=lambda e: e.time_range.start)
    dur = defaultdict(list)
    gap = defaultdict(list)
    prev_end = None
    for e in evs:
        name = e.name.replace("(anonymous namespace)::", "").replace("moment::", "").replace("void ", "")
        name = name.split("(")[0][:48]
        dur[name].append(e.time_range.elapsed_us())
        if prev_end is not None:
            gap[name].append(max(0.0, e.time_range.start - prev_end))
        prev_end = e.time_range.end
    print(f"{'kernel':48s} {'n':>5s} {'mean_us':>8s} {'gap_us':>7s}")
    for k in sorted(dur, key=lambda k: -sum(dur[k])):
        gm = sum(gap[k]) / len(gap[k]) if gap[k] else 0.0
        print(f"{k:48s} {len(dur[k]):5d} {sum(dur[k]) / len(dur[k]):8.2f} {gm:7.2f}")


if __name__ == "__main__":
    main()
