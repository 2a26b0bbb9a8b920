"""Box probe (the paper builds its capacity graph from profiled link limits):
measures the capacities the planner's topology graph needs on THIS box and writes them as JSON that
`boxes.from_probe` turns into `boxes.hgx_b200` arguments (each capacity tagged measured / assumed).

    python tools/probe_box.py [--out gpurun_out/probe.json]

Measured here (CUDA events, best of several):
  * hbm_gbs          device copy, read + write bytes (the HBM bin -> GPU link)
  * port_gbs         pinned host -> device copy per GPU with the host buffer on the GPU's own NUMA node
                     (the GPU's PCIe port), alone; port_concurrent_gbs: every GPU at once (a shared uplink or
                     socket DRAM limit shows as a lower per-GPU rate)
  * port_remote_gbs  the same with the buffer on another NUMA node (crosses UPI), if the box has > 1 node
  * zero_copy_gbs    SM-issued zero-copy reads of pinned host rows by the library's own gather (the tier the
                     product reads host rows through)
  * nvlink_gbs       peer copy GPU 0 -> GPU 1 per direction, if the box has > 1 GPU
Not measurable from a process (assumed unless the box shows them): socket DRAM bandwidth and UPI capacity
beyond what port_remote_gbs bounds.
"""
import argparse
import json
import os
import subprocess
import sys
import threading

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:  # noqa: BLE001
        return f"ERR {e}"


def numa_nodes():
    base = "/sys/devices/system/node"
    nodes = {}
    try:
        for d in sorted(os.listdir(base)):
            if d.startswith("node") and d[4:].isdigit():
                cpus = set()
                with open(os.path.join(base, d, "cpulist")) as f:
                    for part in f.read().strip().split(","):
                        if part:
                            a, _, b = part.partition("-")
                            cpus.update(range(int(a), int(b or a) + 1))
                if cpus:
                    nodes[int(d[4:])] = sorted(cpus)
    except OSError:
        pass
    return nodes or {0: sorted(os.sched_getaffinity(0))}


def gpu_numa(i):
    """NUMA node of GPU i's PCIe function (sysfs), 0 if unknown."""
    bus = sh(f"nvidia-smi -i {i} --query-gpu=pci.bus_id --format=csv,noheader").strip().lower()
    if bus and not bus.startswith("err"):
        if bus.count(":") == 2 and len(bus.split(":")[0]) == 8:
            bus = bus[4:]
        try:
            with open(f"/sys/bus/pci/devices/{bus}/numa_node") as f:
                return max(int(f.read().strip()), 0)
        except (OSError, ValueError):
            pass
    return 0


def timed(fn, nbytes, dev, reps=8):
    with torch.cuda.device(dev):
        fn()
        torch.cuda.synchronize(dev)
        best = 1e30
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize(dev)
            best = min(best, a.elapsed_time(b))
    return nbytes / (best * 1e-3) / 1e9


def pinned_on(node_cpus, nbytes):
    """A pinned host buffer whose pages were first touched from a core of the given NUMA node."""
    old = os.sched_getaffinity(0)
    try:
        os.sched_setaffinity(0, set(node_cpus))
        h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
        h.fill_(1)
    finally:
        os.sched_setaffinity(0, old)
    return h


def zero_copy_gbs(dev, host_rows, R=512):
    """The library's gather reading every row zero-copy from a pinned host table (bin 0 on the host)."""
    import paper_conf_sc_shi0s0x0w25_b200 as M

    n = host_rows.shape[0]
    ctx = M.Ctx(n_vertices=n, max_seeds=1, max_fanout=[1], device=dev.index or 0, row_bytes=R, bin_owner=[-1],
                bin_ptr=[host_rows.data_ptr()])
    m = 1 << 18
    ids = torch.randint(0, n, (m,), device=dev, dtype=torch.int64)
    out = torch.empty((m, R), dtype=torch.uint8, device=dev)
    return timed(lambda: ctx.gather(ids, out), m * R, dev)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/probe.json")
    ap.add_argument("--mib", type=int, default=1024)
    a = ap.parse_args()
    nb = a.mib << 20
    nodes = numa_nodes()
    k = torch.cuda.device_count()
    res = {"gpus": k, "numa_nodes": len(nodes), "cpu_count": os.cpu_count(),
           "cpu_model": next((l.split(":", 1)[1].strip() for l in sh("lscpu").splitlines()
                              if l.startswith("Model name:")), None),
           "gpu_name": torch.cuda.get_device_name(0), "gpu_numa": [gpu_numa(i) for i in range(k)],
           "sm_count": torch.cuda.get_device_properties(0).multi_processor_count,
           "smi_topo": sh("nvidia-smi topo -m")}
    d0 = torch.device("cuda:0")
    x = torch.empty(nb, dtype=torch.uint8, device=d0)
    y = torch.empty_like(x)
    res["hbm_gbs"] = timed(lambda: y.copy_(x), 2 * nb, d0)
    del y
    port, remote = [], []
    for i in range(k):
        di = torch.device(f"cuda:{i}")
        xi = torch.empty(nb, dtype=torch.uint8, device=di)
        loc = res["gpu_numa"][i] if res["gpu_numa"][i] in nodes else next(iter(nodes))
        h = pinned_on(nodes[loc], nb)
        port.append(timed(lambda: xi.copy_(h, non_blocking=True), nb, di))
        others = [j for j in nodes if j != loc]
        if others:
            hr = pinned_on(nodes[others[0]], nb)
            remote.append(timed(lambda: xi.copy_(hr, non_blocking=True), nb, di))
            del hr
        del h, xi
    res["port_gbs_per_gpu"] = port
    res["port_gbs"] = min(port)
    res["port_remote_gbs"] = min(remote) if remote else None
    if k > 1:  # every GPU's port at once: per-GPU rate under contention
        bufs = []
        for i in range(k):
            di = torch.device(f"cuda:{i}")
            loc = res["gpu_numa"][i] if res["gpu_numa"][i] in nodes else next(iter(nodes))
            bufs.append((di, torch.empty(nb, dtype=torch.uint8, device=di), pinned_on(nodes[loc], nb)))
        rates = [0.0] * k

        def run(i):
            di, xi, hi = bufs[i]
            rates[i] = timed(lambda: xi.copy_(hi, non_blocking=True), nb, di, reps=4)

        th = [threading.Thread(target=run, args=(i,)) for i in range(k)]
        for t in th:
            t.start()
        for t in th:
            t.join()
        res["port_concurrent_gbs"] = rates
        del bufs
        d1 = torch.device("cuda:1")
        z = torch.empty(nb, dtype=torch.uint8, device=d1)
        res["nvlink_gbs"] = timed(lambda: z.copy_(x), nb, d0)
        del z
    else:
        res["port_concurrent_gbs"] = None
        res["nvlink_gbs"] = None
    rows = (256 << 20) // 512
    host_rows = torch.empty((rows, 512), dtype=torch.uint8, pin_memory=True)
    res["zero_copy_gbs"] = zero_copy_gbs(d0, host_rows)
    res["measured"] = [key for key in ("hbm_gbs", "port_gbs", "port_remote_gbs", "nvlink_gbs", "zero_copy_gbs")
                       if res.get(key) is not None]
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps({kk: v for kk, v in res.items() if kk != "smi_topo"}))


if __name__ == "__main__":
    main()
