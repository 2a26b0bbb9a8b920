"""GraphSAGE training on the sampled + gathered batches (the consumer) on one B200.

The paper's model and loader settings: GraphSAGE, hidden 256, 2-hop fan-outs [25, 10], batch 8000; here
on the C2 (ogbn-products-shaped) graph with its 100-d fp32 features and 47 classes, synthetic labels. One
training step = moment_step (sample + gather, one CUDA graph) -> counts to the host (tensor shapes) ->
forward (bf16 autocast GEMMs + moment_sage_mean) -> cross-entropy -> backward (moment_sage_mean_backward) ->
Adam. Reported: seeds/s of the loader alone and of the full step, the step's time split, and the same model
with torch's own mean aggregation (index_add_) in place of the kernels.

    python tools/bench_train.py [--config C2] [--batch 8000] [--fanout 25,10] [--steps 50]
"""
import argparse
import json
import os
import sys
import time

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_sc_shi0s0x0w25_b200 as M  # noqa: E402
from paper_conf_sc_shi0s0x0w25_b200 import sage as S  # noqa: E402
import workloads as W  # noqa: E402

DEV = "cuda:0"


def torch_mean(x, offsets, src, n_dst):
    """The library path: mean aggregation with torch ops (repeat_interleave + index_add_)."""
    deg = (offsets[1:n_dst + 1] - offsets[:n_dst])
    dst = torch.repeat_interleave(torch.arange(n_dst, device=x.device), deg)
    out = torch.zeros((n_dst, x.shape[1]), device=x.device, dtype=torch.float32)
    out.index_add_(0, dst, x[src.long()].float())
    return (out / deg.clamp(min=1).unsqueeze(1)).to(x.dtype)


class TorchSAGE(S.GraphSAGE):
    def forward(self, x, blocks):
        h = x
        H = len(blocks)
        for l, layer in enumerate(self.layers):
            off, src, n_dst = blocks[H - 1 - l]
            last = l + 1 == len(self.layers)
            n_pad = n_dst if last else max(n_dst, min(h.shape[0], -(-n_dst // self.bucket) * self.bucket))
            agg = torch.nn.functional.pad(torch_mean(h, off, src, n_dst), (0, 0, 0, n_pad - n_dst))
            h = layer.self_lin(h[:n_pad]) + layer.neigh_lin(agg)
            if not last:
                h = torch.relu(h)
        return h


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--batch", type=int, default=8000)
    ap.add_argument("--fanout", default="25,10")
    ap.add_argument("--hidden", type=int, default=256)
    ap.add_argument("--classes", type=int, default=47)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--out", default=None)
    ap.add_argument("--profile", action="store_true", help="print the top CUDA kernels of 5 steps (torch.profiler)")
    ap.add_argument("--impls", default="moment,torch", help="order of the aggregation implementations")
    ap.add_argument("--bucket", type=int, default=2048, help="GEMM row bucket (0 = exact shapes)")
    a = ap.parse_args()
    cfg = W.CONFIGS[a.config]
    fan = [int(f) for f in a.fanout.split(",")]
    B = a.batch
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    R = cfg["dim"] * 4
    stride = (R + 63) // 64 * 64
    table = W.feature_table(cfg["n"], cfg["dim"], cfg["dtype"], device=DEV, row_stride_bytes=stride)
    # features as fp32 numbers in [-1, 1): the generator's random words scaled (no NaN bit patterns)
    tv = table[:, :R].view(torch.int32)
    table[:, :R] = (tv.float() * 2.0 ** -31).view(torch.uint8).view(cfg["n"], R)
    del tv
    train = W.training_set(g, min_count=B)
    batches = []
    e = 0
    while len(batches) < a.steps + a.warmup:
        batches += W.epoch_batches(train, B, e)
        e += 1
    labels = torch.randint(0, a.classes, (cfg["n"],), device=DEV, generator=torch.Generator(DEV).manual_seed(0))
    ctx = M.Ctx(n_vertices=g.n, max_seeds=B, max_fanout=fan, device=0, row_bytes=R, row_stride=stride,
                bin_owner=[0], bin_ptr=[table.data_ptr()])
    bufs = M.SampleBuffers.allocate(B, fan, g.n, DEV)
    rows = torch.empty((bufs.nodes.numel(), R), dtype=torch.uint8, device=DEV)
    counts_h = torch.empty(bufs.counts.numel(), dtype=torch.int64).pin_memory()
    results = {}
    for impl in a.impls.split(","):
        torch.manual_seed(0)
        model = (S.GraphSAGE if impl == "moment" else TorchSAGE)(cfg["dim"], a.hidden, a.classes, len(fan),
                                                                bucket=a.bucket).to(DEV)
        opt = torch.optim.Adam(model.parameters(), lr=1e-3)
        ev = {k: [] for k in ("load", "train")}

        def step(i, timed):
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record()
            ctx.step(g.indptr, g.indices, batches[i], fan, W.batch_rng_seed(3, 0, 0, i), bufs, rows)
            e1.record()
            counts_h.copy_(bufs.counts, non_blocking=True)
            torch.cuda.current_stream().synchronize()
            c = counts_h.numpy()
            nF = int(c[len(fan)])
            x = rows[:nF].view(torch.float32)
            with torch.autocast("cuda", dtype=torch.bfloat16):
                logits = model(x, S.blocks_of(bufs, c))
                loss = torch.nn.functional.cross_entropy(logits.float(), labels[bufs.nodes[:B]])
            opt.zero_grad(set_to_none=True)
            loss.backward()
            opt.step()
            e2.record()
            if timed:
                ev["load"].append((e0, e1))
                ev["train"].append((e1, e2))
            return loss

        for i in range(a.warmup):
            step(i, False)
        torch.cuda.synchronize()
        if a.profile:
            from torch.profiler import profile, ProfilerActivity
            with profile(activities=[ProfilerActivity.CUDA]) as prof:
                for i in range(5):
                    step(i, False)
                torch.cuda.synchronize()
            print(f"== {impl}")
            print(prof.key_averages().table(sort_by="cuda_time_total", row_limit=14))
            import cProfile
            import pstats
            pr = cProfile.Profile()
            pr.enable()
            for i in range(5):
                step(i, False)
            torch.cuda.synchronize()
            pr.disable()
            pstats.Stats(pr).sort_stats("tottime").print_stats(12)
        t0 = torch.cuda.Event(enable_timing=True)
        t1 = torch.cuda.Event(enable_timing=True)
        w0 = time.perf_counter()
        t0.record()
        for i in range(a.warmup, a.warmup + a.steps):
            loss = step(i, True)
        t1.record()
        torch.cuda.synchronize()
        wall = time.perf_counter() - w0
        ms = t0.elapsed_time(t1) / a.steps
        load_ms = sum(x.elapsed_time(y) for x, y in ev["load"]) / a.steps
        train_ms = sum(x.elapsed_time(y) for x, y in ev["train"]) / a.steps
        results[impl] = {"seeds_per_s": B / (ms / 1e3), "ms_per_step": ms, "load_ms": load_ms, "train_ms": train_ms,
                         "loader_only_seeds_per_s": B / (load_ms / 1e3), "wall_s": wall, "final_loss": float(loss.detach())}
        print(f"{impl}: {B / (ms / 1e3) / 1e6:.3f} M seeds/s, {ms:.3f} ms/step (sample+gather {load_ms:.3f} ms, "
              f"fwd+bwd+adam {train_ms:.3f} ms), loss {float(loss.detach()):.3f}", flush=True)
    line = {"config": a.config, "model": "GraphSAGE (mean)", "hidden": a.hidden, "classes": a.classes, "batch": B,
            "fanout": fan, "steps": a.steps, "dtype": "bf16 GEMMs (autocast), fp32/bf16 aggregation",
            "data": "synthetic (R-MAT graph, generated features, random labels)", "results": results,
            "kernel_over_torch": (results["moment"]["seeds_per_s"] / results["torch"]["seeds_per_s"]
                                  if len(results) == 2 else None)}
    print(json.dumps(line))
    if a.out:
        with open(a.out, "a") as f:
            f.write(json.dumps(line) + "\n")


if __name__ == "__main__":
    main()
