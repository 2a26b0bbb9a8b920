"""Host time of the batched issue (StepBatch.run of P steps, C2 lanes) per step, with the GPU kept busy.
    python tools/exp_issue_batch.py [--lanes 16] [--calls 200]"""
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
    ap.add_argument("--lanes", type=int, default=16)
    ap.add_argument("--calls", type=int, default=200)
    a = ap.parse_args()
    st = bench.build_state("C2", "cuda:0", 0, 1, a.lanes)
    P = len(st.lanes)
    sb = st.M.StepBatch([L.ctx for L in st.lanes], st.graph.indptr, st.graph.indices, st.fanout,
                        [L.bufs for L in st.lanes], [L.rows for L in st.lanes], [L.stream for L in st.lanes])
    pool = [st.batch(i) for i in range(P)]
    seeds, rngs = [p[0] for p in pool], [p[1] for p in pool]
    for _ in range(3):
        sb.run(seeds, rngs)
    torch.cuda.synchronize()
    t = []
    for _ in range(a.calls):
        t0 = time.perf_counter()
        sb.run(seeds, rngs)
        t.append((time.perf_counter() - t0) * 1e6 / P)
        torch.cuda.synchronize()
    print(json.dumps({"lanes": P, "host_us_per_step_median": statistics.median(t), "min": min(t)}))


if __name__ == "__main__":
    main()
