"""Whole-GPU counters of the saturated step (P lanes in flight) via ncu range replay: the batches between
cudaProfilerStart/Stop are measured as ONE range, concurrency included (kernel replay would serialise them).

  ncu --replay-mode app-range --profile-from-start off --metrics <list> python tools/exp_range_metrics.py \
      [--lanes 8] [--batches 256] [--mode full|sample|gather]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=8)
    ap.add_argument("--batches", type=int, default=256)
    ap.add_argument("--mode", default="full")
    ap.add_argument("--config", default="C2")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, inflight=a.lanes)
    batches = [st.batch(i) for i in range(a.batches)]
    H = len(st.fanout)

    def one(i, s, r):
        L = st.lanes[i % a.lanes]
        if a.mode == "gather":
            L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(), stream=L.stream)
        else:
            L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs,
                       L.rows if a.mode == "full" else None, stream=L.stream)

    for i, (s, r) in enumerate(batches[:64]):
        L = st.lanes[i % a.lanes]
        L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs, L.rows, stream=L.stream)
        one(i, s, r)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    for i, (s, r) in enumerate(batches):
        one(i, s, r)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    print(f"range: {a.batches} batches, mode {a.mode}, {a.lanes} lanes", flush=True)


if __name__ == "__main__":
    main()
