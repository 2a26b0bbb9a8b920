"""Which part saturates with batches in flight? Times full steps, sample-only and gather-only at P lanes.

    python tools/exp_saturation.py [--config C2] [--steps 400]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def run(st, batches, P, mode):
    H = len(st.fanout)
    main = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(main)
    for L in st.lanes[1:P]:
        L.stream.wait_event(e0)
    for i, (seeds, rng) in enumerate(batches):
        L = st.lanes[i % P]
        if mode == "full":
            L.ctx.step(st.graph.indptr, st.graph.indices, seeds, st.fanout, rng, L.bufs, L.rows, stream=L.stream)
        elif mode == "sample":
            L.ctx.step(st.graph.indptr, st.graph.indices, seeds, st.fanout, rng, L.bufs, None, stream=L.stream)
        else:
            L.ctx.gather(L.bufs.nodes, L.rows, n_dev=L.bufs.counts[H:H + 1], max_n=L.bufs.nodes.numel(),
                         stream=L.stream)
    for L in st.lanes[1:P]:
        e = torch.cuda.Event()
        e.record(L.stream)
        main.wait_event(e)
    e1.record(main)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) * 1e3 / len(batches)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--lanes", default="1,2,4,8,16")
    args = ap.parse_args()
    lanes = [int(x) for x in args.lanes.split(",")]
    st = bench.build_state(args.config, "cuda:0", 0, 1, inflight=max(lanes))
    batches = [st.batch(i) for i in range(args.steps)]
    for P in lanes:
        for L, b in zip(st.lanes[:P], batches):  # lanes hold a real F_H for gather-only
            L.ctx.step(st.graph.indptr, st.graph.indices, b[0], st.fanout, b[1], L.bufs, L.rows, stream=L.stream)
        torch.cuda.synchronize()
        res = {m: run(st, batches, P, m) for m in ("full", "sample", "gather")}
        for m in res:
            run(st, batches[:20], P, m)
        res = {m: run(st, batches, P, m) for m in ("full", "sample", "gather")}
        print(f"P={P}: " + "  ".join(f"{m} {v:6.1f} us/batch" for m, v in res.items()), flush=True)


if __name__ == "__main__":
    main()
