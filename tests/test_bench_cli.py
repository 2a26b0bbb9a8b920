"""bench.py end to end with the driver's own argument shapes (`--steps 20 --warmup 5` crashed
after the timed region). The reference arm runs on CPU; the CUDA arm needs a GPU."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None, timeout=900):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                       timeout=timeout, cwd=ROOT, env=e)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_reference_arm_driver_args():
    line = _run(["--impl", "reference", "--config", "C1", "--gpus", "1", "--steps", "20", "--warmup", "5"],
                env={"MOMENT_REF_BUDGET_S": "3"})
    assert line["impl"] == "reference" and line["steps"] == 20 and line["warmup"] == 5
    assert line["value"] > 0 and line["unit"] == "seeds/s"
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["cpu_baseline"]["kind"] == "oracle"
    assert line["cpu_baseline"]["cores"] == 1


@pytest.mark.gpu
@pytest.mark.parametrize("steps,warmup", [(20, 5), (1, 3), (3, 3)])
def test_bench_driver_args_c1(steps, warmup):
    line = _run(["--config", "C1", "--gpus", "1", "--steps", str(steps), "--warmup", str(warmup), "--min-time", "0.2",
                 "--e2e-min-time", "0.1", "--cpu-budget", "1"])
    assert line["steps"] == steps and line["warmup"] == warmup and line["n_gpus"] == 1
    assert line["value"] > 0 and line["e2e"]["value"] > 0
    for k in ("roofline", "cpu_baseline", "e2e", "clocks", "gpu_launches", "step_roofline"):
        assert line[k] is not None, k
    assert 0 < line["roofline"]["frac"] < 1.5
    assert line["cpu_baseline"]["parity"]["bit_exact"]
    assert line["config"]["region_ms"]["n"] >= 3


def _run_torchrun(nproc, args, env=None, timeout=900):
    import socket

    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    e = dict(os.environ)
    e.update(env or {})
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.join(ROOT, "bench.py")] + args
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT, env=e)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


@pytest.mark.gpu
@pytest.mark.parametrize("placement", ["ddak", "ddak-rep"])
def test_bench_partitioned_one_rank(placement):
    """N = 1: the partitioned path (placement map, DDAK over one HBM bin) with the parity subset checked."""
    line = _run(["--config", "C1", "--placement", placement, "--steps", "20", "--warmup", "3", "--min-time", "0.2",
                 "--e2e-min-time", "0.1", "--presample", "8"])
    assert line["cpu_baseline"]["parity"]["bit_exact"]
    t = line["tiers"]
    assert t["rows_per_batch"]["peer_in_nvlink"] == 0 and t["rows_per_batch"]["local_hbm"] > 0
    assert t["plan"]["t_star_us"] >= 0


@pytest.mark.gpu
@pytest.mark.parametrize("placement", ["ddak", "ddak-rep"])
def test_bench_partitioned_two_ranks_shared_gpu(placement):
    """N = 2 ranks sharing cuda:0 over gloo (MOMENT_BENCH_SHARED_GPU: the multi-rank code path on a one-GPU box,
    never a bench number): the table is split over the two ranks' bins, each maps the other's by CUDA IPC,
    and every batch reads peer rows; DDAK's bins partition the non-replicated rows."""
    line = _run_torchrun(2, ["--gpus", "2", "--config", "C1", "--placement", placement, "--steps", "10",
                             "--warmup", "3", "--min-time", "0.1", "--e2e-min-time", "0.05", "--presample", "8"],
                         env={"MOMENT_BENCH_SHARED_GPU": "1"})
    assert line["n_gpus"] == 2 and "test_mode" in line["config"]
    t = line["tiers"]
    assert t["rows_per_batch"]["peer_in_nvlink"] > 0 and t["rows_per_batch"]["served_to_peers_nvlink"] > 0
    assert sum(t["bin_rows"]) == (1 << 16) - t["replicated_rows"]  # a partition of the non-replicated rows
    if placement == "ddak-rep":
        assert t["replicated_rows"] > 0


@pytest.mark.gpu
def test_bench_replicated_two_ranks_self_launched():
    """`bench.py --gpus 2` outside torchrun re-launches itself under torch.distributed.run (here both ranks on
    cuda:0 over gloo, MOMENT_BENCH_SHARED_GPU): one JSON line, n_gpus = 2, global batch 2 x 1024."""
    line = _run(["--gpus", "2", "--config", "C1", "--steps", "10", "--warmup", "3", "--min-time", "0.1",
                 "--e2e-min-time", "0.05"], env={"MOMENT_BENCH_SHARED_GPU": "1"})
    assert line["n_gpus"] == 2 and line["config"]["global_batch"] == 2048 and "test_mode" in line["config"]
    assert line["cpu_baseline"] is None  # rank 0 at N = 1 only


def test_bench_refuses_more_ranks_than_gpus():
    import torch

    if torch.cuda.is_available() and torch.cuda.device_count() >= 2:
        pytest.skip("box has 2+ GPUs")
    e = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    e.pop("MOMENT_BENCH_SHARED_GPU", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--config", "C1"],
                       capture_output=True, text=True, timeout=300, cwd=ROOT, env=e)
    assert r.returncode != 0 and "visible GPUs" in (r.stderr + r.stdout)


@pytest.mark.gpu
def test_bench_partitioned_layout_reuse(tmp_path):
    """--layout: the first run saves the DDAK layout (placement + topology hash), a second run checks that it
    recomputes the identical placement (plan reuse)."""
    lay = str(tmp_path / "c1.npz")
    args = ["--config", "C1", "--placement", "ddak-rep", "--steps", "5", "--warmup", "3", "--min-time", "0.05",
            "--e2e-min-time", "0.02", "--presample", "8", "--no-cpu-baseline", "--layout", lay]
    _run(args)
    assert os.path.exists(lay)
    _run(args)


@pytest.mark.gpu
def test_bench_tiered_one_rank():
    """N = 1, ddak-tiered: a small HBM cache + pinned host bins read zero-copy; every gathered row of the parity
    subset byte-exact; host rows accounted over PCIe."""
    line = _run(["--config", "C1", "--placement", "ddak-tiered", "--cache-gib", "0.008", "--steps", "10", "--warmup",
                 "3", "--min-time", "0.1", "--e2e-min-time", "0.05", "--presample", "8"])
    assert line["cpu_baseline"]["parity"]["bit_exact"]
    t = line["tiers"]
    assert t["rows_per_batch"]["host_direct_pcie"] > 0 and t["rows_per_batch"]["local_hbm"] > 0
    assert t["rows_per_batch"]["host_relayed_to_me"] == 0


@pytest.mark.gpu
def test_bench_tiered_two_ranks_shared_gpu():
    """N = 2 ranks sharing cuda:0 (test mode): HBM caches + host bins, the plan's quotas, relays through the peer
    rank inside every collective moment_step (moment_ctx_set_exchange); every rank's rows of one batch
    byte-exact; relayed rows one rank receives are the rows the other serves."""
    line = _run_torchrun(2, ["--gpus", "2", "--config", "C1", "--placement", "ddak-tiered", "--cache-gib", "0.004",
                             "--steps", "6", "--warmup", "3", "--inflight", "2", "--min-time", "0.05",
                             "--e2e-min-time", "0.02", "--presample", "64"],
                         env={"MOMENT_BENCH_SHARED_GPU": "1"})
    t = line["tiers"]
    assert t["rows_check"]["byte_exact"] and line["n_gpus"] == 2
    r = t["rows_per_batch"]
    assert r["peer_in_nvlink"] > 0
    # the two GPUs sit on different sockets (spread_gpus): the plan ingests each socket's host bin through its
    # own GPU's port, so rank 0 reads host bin 0 directly and gets host bin 1's rows relayed by rank 1
    q = t["quota"]
    assert len(q) == 4 and q[2][0] > 0 and q[2][1] == 0 and q[3][0] == 0 and q[3][1] > 0
    assert r["host_direct_pcie"] > 0 and r["host_relayed_to_me"] > 0 and r["host_served_for_peers"] > 0


def test_step_floor_arithmetic():
    """bench.step_floor: the gather's bytes at the copy peak plus the sampler's random atoms at the measured
    random-access rate (C2: 97.6 MB at 6536 GB/s = 14.93 us, 267 750 atoms at 36.96 G/s = 7.24 us)."""
    sys.path.insert(0, ROOT)
    import bench

    f = bench.step_floor("C2", 97.6e6, 6536.0, 0.0246)
    assert abs(f["gather_us"] - 97.6e6 / 6536e9 * 1e6) < 1e-9
    assert abs(f["sampler_us"] - 267750 / 36.96e9 * 1e6) < 1e-9
    assert abs(f["floor_us"] - (f["gather_us"] + f["sampler_us"])) < 1e-9
    assert abs(f["frac"] - f["floor_us"] / 24.6) < 1e-9 and 0.8 < f["frac"] < 1.0
    assert bench.step_floor("C1", 1e6, 6536.0, 0.01) is None
