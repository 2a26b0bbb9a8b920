"""Kernel durations with P lanes in flight (torch.profiler/CUPTI): how much each kernel stretches when
batches overlap, vs the same kernel with one lane.   python tools/lane_profile.py [--lanes 8] [--mode full]"""
import argparse
import os
import sys
from collections import defaultdict

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def profile(st, batches, P, mode):
    from torch.profiler import ProfilerActivity, profile as prof

    main = torch.cuda.current_stream()
    torch.cuda.synchronize()
    with prof(activities=[ProfilerActivity.CUDA]) as p:
        ev = torch.cuda.Event()
        ev.record(main)
        for L in st.lanes[1:P]:
            L.stream.wait_event(ev)
        for i, (s, r) in enumerate(batches):
            L = st.lanes[i % P]
            L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs, L.rows if mode == "full" else None,
                       stream=L.stream)
        torch.cuda.synchronize()
    evs = [e for e in p.events() if e.device_type.name == "CUDA"]
    t0 = min(e.time_range.start for e in evs)
    t1 = max(e.time_range.end for e in evs)
    dur = defaultdict(float)
    for e in evs:
        name = e.name.replace("(anonymous namespace)::", "").replace("moment::", "").replace("void ", "")
        dur[name.split("(")[0][:40]] += e.time_range.elapsed_us()
    return (t1 - t0) / len(batches), {k: v / len(batches) for k, v in dur.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=8)
    ap.add_argument("--mode", default="full")
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--config", default="C2")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, inflight=a.lanes)
    batches = [st.batch(i) for i in range(a.steps)]
    profile(st, batches[:16], a.lanes, a.mode)
    w1, d1 = profile(st, batches, 1, a.mode)
    wP, dP = profile(st, batches, a.lanes, a.mode)
    print(f"wall per batch: P=1 {w1:.1f} us, P={a.lanes} {wP:.1f} us")
    print(f"{'kernel':40s} {'P=1 us/batch':>12s} {'P us/batch':>12s} {'stretch':>8s}")
    for k in sorted(dP, key=lambda k: -dP[k]):
        print(f"{k:40s} {d1.get(k, 0):12.1f} {dP[k]:12.1f} {dP[k] / max(d1.get(k, 1e-9), 1e-9):8.2f}")
    print(f"{'sum':40s} {sum(d1.values()):12.1f} {sum(dP.values()):12.1f}")


if __name__ == "__main__":
    main()
