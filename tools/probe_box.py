"""Box probe: host/GPU topology facts and link bandwidths.

Writes gpurun_out/probe.json. Not part of the product; plain torch only.
"""
import json, os, subprocess, time
import torch

def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:  # noqa
        return f"ERR {e}"

out = {}
out["lscpu"] = sh("lscpu")
out["meminfo"] = sh("head -5 /proc/meminfo")
out["numa"] = sh("numactl -H 2>/dev/null || ls /sys/devices/system/node/")
out["nproc"] = os.cpu_count()
out["smi_topo"] = sh("nvidia-smi topo -m")
out["smi_q"] = sh("nvidia-smi -q | grep -iE 'Product Name|Bus Id|Link Width|PCIe Generation|Max|Current' | head -60")
out["hugepages"] = sh("grep -i huge /proc/meminfo")
dev = torch.device("cuda:0")
props = torch.cuda.get_device_properties(0)
out["sm_count"] = props.multi_processor_count
out["total_mem"] = props.total_memory

def bw(fn, nbytes, reps=10):
    fn(); torch.cuda.synchronize()
    s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    best = 1e9
    for _ in range(reps):
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e))
    return nbytes / (best * 1e-3) / 1e9

N = 1 << 30
h = torch.empty(N, dtype=torch.uint8, pin_memory=True)
d = torch.empty(N, dtype=torch.uint8, device=dev)
out["h2d_pinned_GBs"] = bw(lambda: d.copy_(h, non_blocking=True), N)
out["d2h_pinned_GBs"] = bw(lambda: h.copy_(d, non_blocking=True), N)
d2 = torch.empty_like(d)
out["d2d_copy_GBs_rw"] = bw(lambda: d2.copy_(d), 2 * N)
# random row gather in HBM (torch index_select), 400 B rows
tab = torch.empty((2_449_029, 100), dtype=torch.float32, device=dev)
idx = torch.randint(0, tab.shape[0], (700_000,), device=dev)
o = torch.empty((idx.numel(), 100), dtype=torch.float32, device=dev)
out["torch_index_select_400B_GBs_rw"] = bw(lambda: torch.index_select(tab, 0, idx, out=o), 2 * idx.numel() * 400)
# zero-copy: gather from pinned host via index_select on a mapped view is not expressible in torch; use UVA via cuda-python later
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
print(json.dumps({k: v for k, v in out.items() if not isinstance(v, str)}, indent=1))
