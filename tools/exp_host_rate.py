"""Is the saturated bench host-bound? Times the host enqueue of K moment_step calls (ctypes + graph launch)
against the device completion of the same K steps, at several lane counts.

  python tools/exp_host_rate.py [--config C2] [--steps 5000]
"""
import argparse
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--steps", type=int, default=5000)
    args = ap.parse_args()
    st = bench.build_state(args.config, "cuda:0", 0, 1, 16)
    P = len(st.lanes)
    batches = [st.batch(i) for i in range(64)]
    for lanes in (1, 4, 8, 16):
        for i in range(100):
            s, r = batches[i % 64]
            st.step(s, r, lane=i % lanes)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for i in range(args.steps):
            s, r = batches[i % 64]
            st.step(s, r, lane=i % lanes)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
        t2 = time.perf_counter()
        K = args.steps
        print(f"lanes {lanes:2d}: enqueue {1e6 * (t1 - t0) / K:6.2f} us/step  total {1e6 * (t2 - t0) / K:6.2f} us/step  "
              f"{K * st.B / (t2 - t0) / 1e6:6.2f} M seeds/s", flush=True)
    # the host cost alone: the ctypes call path on a step whose graph is replayed, K calls with the GPU idle
    # excluded is impossible (launch blocks when queues fill), so also report the raw C call rate on 1 lane
    L = st.lanes[0]
    s, r = batches[0]
    t0 = time.perf_counter()
    for i in range(1000):
        L.ctx.step(st.graph.indptr, st.graph.indices, s, st.fanout, r, L.bufs, L.rows, stream=L.stream)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    print(f"1 lane, 1000 calls: enqueue {1e3 * (t1 - t0):.2f} us/call (first calls do not wait on the queue)")


if __name__ == "__main__":
    main()
