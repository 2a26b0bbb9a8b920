"""DRAM utilisation (nvidia-smi dmon) while a mode runs for a few seconds with P lanes in flight:
full / sample-only / gather-only.   python tools/exp_dram_util.py [--lanes 8] [--secs 4]"""
import argparse
import os
import subprocess
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from exp_saturation import run  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=8)
    ap.add_argument("--secs", type=float, default=4.0)
    a = ap.parse_args()
    st = bench.build_state("C2", "cuda:0", 0, 1, inflight=a.lanes)
    batches = [st.batch(i) for i in range(400)]
    for L, b in zip(st.lanes, batches):
        L.ctx.step(st.graph.indptr, st.graph.indices, b[0], st.fanout, b[1], L.bufs, L.rows, stream=L.stream)
    torch.cuda.synchronize()
    for mode in ("full", "sample", "gather"):
        us = run(st, batches, a.lanes, mode)
        reps = max(1, int(a.secs * 1e6 / (us * len(batches))))
        p = subprocess.Popen(["nvidia-smi", "dmon", "-s", "u", "-d", "1"], stdout=subprocess.PIPE, text=True)
        time.sleep(1.5)
        t0 = time.time()
        for _ in range(reps):
            run(st, batches, a.lanes, mode)
        dt = time.time() - t0
        time.sleep(0.5)
        p.terminate()
        out = p.communicate()[0].strip().splitlines()
        rows = [l.split() for l in out if l.strip() and not l.startswith("#")]
        print(f"{mode}: {us:.1f} us/batch over {dt:.1f} s; dmon (sm% mem%): " +
              " ".join(f"{r[1]}/{r[2]}" for r in rows if len(r) > 2), flush=True)


if __name__ == "__main__":
    main()
