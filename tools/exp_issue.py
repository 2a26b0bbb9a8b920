"""How much of a short (K = 20) bench region is host issue: the driver's K-step region against the same region
with every step already enqueued when it starts (the lanes wait on a host-released gate,
cuStreamWaitValue32, and the start event is recorded after the gate), plus the host time per step of the
bench's `st.step` and of the bare ctypes call with prebuilt arguments.

    python tools/exp_issue.py [--lanes 16] [--steps 20] [--regions 300]
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
    from cuda.bindings import driver as drv

    ap = argparse.ArgumentParser()
    ap.add_argument("--lanes", type=int, default=16)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--regions", type=int, default=300)
    ap.add_argument("--config", default="C2")
    a = ap.parse_args()
    st = bench.build_state(a.config, "cuda:0", 0, 1, a.lanes)
    P, K = len(st.lanes), a.steps
    main_s = torch.cuda.current_stream()
    pool = [st.batch(i) for i in range(256)]
    for i in range(3 * P):
        st.step(*pool[i % 256], lane=i % P)
    torch.cuda.synchronize()
    gate = torch.zeros(4, dtype=torch.int32, pin_memory=True)
    gptr = gate.data_ptr()

    def region(first, gated):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        if gated:
            gate[0] = 0
            (err,) = drv.cuStreamWaitValue32(drv.CUstream(main_s.cuda_stream), drv.CUdeviceptr(gptr), 1,
                                             drv.CUstreamWaitValue_flags.CU_STREAM_WAIT_VALUE_GEQ)
            assert err == drv.CUresult.CUDA_SUCCESS, err
        e0.record(main_s)
        for L in st.lanes:
            if L.stream != main_s:
                L.stream.wait_event(e0)
        t0 = time.perf_counter()
        for j in range(K):
            st.step(*pool[(first + j) % 256], lane=j % P)
        t_issue = time.perf_counter() - t0
        for L in st.lanes:
            if L.stream != main_s:
                e = torch.cuda.Event()
                e.record(L.stream)
                main_s.wait_event(e)
        e1.record(main_s)
        if gated:
            gate[0] = 1
        torch.cuda.synchronize()
        return e0.elapsed_time(e1), t_issue * 1e6 / K

    res = {}
    for rep in range(2):
        for gated in (False, True):
            ms, iss = [], []
            for r in range(a.regions):
                m, i_ = region(r * K, gated)
                ms.append(m)
                iss.append(i_)
            med = statistics.median(ms)
            res[f"{'gated' if gated else 'driver'}_{rep}"] = {
                "region_ms": med, "seeds_per_s_M": st.B * K / med / 1e3, "host_us_per_step": statistics.median(iss)}
    # host cost per call: the bench's st.step, and the bare ctypes call with prebuilt arguments
    L = st.lanes[0]
    M = st.M
    n = 400
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for j in range(n):
        st.step(*pool[j % 256], lane=j % P)
    t_step = (time.perf_counter() - t0) * 1e6 / n
    torch.cuda.synchronize()
    lib = M.moment.lib()
    pre = []
    for j in range(P):
        Lj = st.lanes[j]
        ar = Lj.ctx._args(st.graph.indptr, st.graph.indices, st.fanout, 0, Lj.bufs)
        pre.append((Lj.ctx.handle, ar, Lj.rows.data_ptr(), Lj.stream.cuda_stream))
    seeds = [(s.data_ptr(), s.numel(), r) for s, r in pool]
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for j in range(n):
        h, ar, rows, sp = pre[j % P]
        sp_, ns, r = seeds[j % 256]
        ar[1].rng_seed = r & 0xFFFFFFFFFFFFFFFF
        lib.moment_step(h, ar[4], sp_, ns, ar[5], ar[6], rows, sp)
    t_raw = (time.perf_counter() - t0) * 1e6 / n
    torch.cuda.synchronize()
    res["host_us_per_call"] = {"st.step": t_step, "bare ctypes moment_step": t_raw}
    print(json.dumps(res))


if __name__ == "__main__":
    main()
