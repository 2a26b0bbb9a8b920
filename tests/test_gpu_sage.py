"""GPU parity of the consumer's aggregation kernels (moment_sage_mean / _backward, through the C ABI) against the
oracle's fp64 definition. Tolerances: fp32 accumulation of <= deg terms (forward rtol 1e-5 of the sum of
|terms| / deg); bf16 output adds one bf16 rounding (2^-8 relative); backward fp32 atomics in any order."""
import numpy as np
import pytest
import torch

import paper_conf_sc_shi0s0x0w25_b200 as M
import workloads as W

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _block(rng, n_dst, n_src, max_deg):
    deg = rng.integers(0, max_deg + 1, n_dst)
    if n_dst > 3:
        deg[1] = 0
        deg[2] = max_deg + 37  # > 32 edges: the 32-edge chunk loop
    off = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    src = rng.integers(0, n_src, int(off[-1])).astype(np.int32)
    return off, src


@pytest.mark.parametrize("dim,dtype,ld_pad", [(4, torch.float32, 0), (100, torch.float32, 0), (100, torch.float32, 12),
                                             (256, torch.float32, 0), (512, torch.float32, 0),
                                             (8, torch.bfloat16, 0), (256, torch.bfloat16, 8),
                                             (1024, torch.bfloat16, 0)])
@pytest.mark.parametrize("n_dst", [0, 1, 7, 3000])
def test_sage_mean_vs_oracle(orc, dim, dtype, ld_pad, n_dst):
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    rng = np.random.default_rng(dim + n_dst)
    n_src = 5000
    off, src = _block(rng, n_dst, n_src, 12)
    xb = torch.randn((n_src, dim + ld_pad), device=DEV).to(dtype)
    x = xb[:, :dim]
    out = torch.full((max(n_dst, 1), dim), float("nan"), device=DEV, dtype=dtype)
    off_d = torch.as_tensor(off, device=DEV)
    src_d = torch.as_tensor(src, device=DEV)
    M.sage_mean(x, off_d, src_d, n_dst, out)
    x64 = x.float().cpu().numpy().astype(np.float64)
    want = orc.sage_mean(x64, off, src)
    got = out[:n_dst].float().cpu().numpy()
    deg = np.maximum(np.diff(off), 1)[:, None]
    scale = orc.sage_mean(np.abs(x64), off, src)  # mean of |terms|
    tol = scale * (1e-5 + (2.0 ** -8 if dtype == torch.bfloat16 else 0)) + 1e-7
    assert np.all(np.abs(got - want) <= tol)
    # backward: grad_x = A^T grad_out, fp32 atomics
    g = torch.randn((max(n_dst, 1), dim), device=DEV).to(dtype)
    gx = torch.zeros((n_src, dim), device=DEV, dtype=torch.float32)
    M.sage_mean_backward(g, off_d, src_d, n_dst, gx)
    g64 = g[:n_dst].float().cpu().numpy().astype(np.float64)
    want_b = orc.sage_mean_backward(g64, off, src, n_src)
    mag = orc.sage_mean_backward(np.abs(g64), off, src, n_src)
    assert np.all(np.abs(gx.cpu().numpy() - want_b) <= 1e-5 * mag + 1e-7)
    del deg


def test_sage_mean_errors():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    off = torch.zeros(2, dtype=torch.int64, device=DEV)
    src = torch.zeros(1, dtype=torch.int32, device=DEV)
    with pytest.raises(M.MomentError):  # 3 x 4 bytes: not a multiple of 16
        M.sage_mean(torch.zeros((4, 3), device=DEV), off, src, 1, torch.zeros((1, 3), device=DEV))
    with pytest.raises(M.MomentError):  # fp16 unsupported
        M.sage_mean(torch.zeros((4, 8), device=DEV, dtype=torch.float16), off, src, 1,
                    torch.zeros((1, 8), device=DEV, dtype=torch.float16))
    with pytest.raises(M.MomentError):  # rows above 2048 bytes
        M.sage_mean(torch.zeros((4, 1024), device=DEV), off, src, 1, torch.zeros((1, 1024), device=DEV))


def test_sage_mean_on_sampled_gathered_batch(orc):
    """The consumer pipeline on C1: moment_sample -> moment_gather -> moment_sage_mean over each hop's block,
    against the oracle's sample, the oracle's gather and its fp64 mean."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    cfg = W.CONFIGS["C1"]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    table = W.feature_table(g.n, 128, torch.float32, device=DEV)
    fan = [10, 5]
    seeds = W.epoch_batches(W.training_set(g, min_count=1024), 1024, 0)[0]
    ctx = M.Ctx(n_vertices=g.n, max_seeds=1024, max_fanout=fan, device=0, row_bytes=512, bin_owner=[0],
                bin_ptr=[table.data_ptr()])
    bufs = M.SampleBuffers.allocate(1024, fan, g.n, DEV)
    rows = torch.empty((bufs.nodes.numel(), 512), dtype=torch.uint8, device=DEV)
    ctx.step(g.indptr, g.indices, seeds, fan, 1234, bufs, rows)
    res = bufs.result()
    want = orc.sample(g.indptr.cpu().numpy(), g.indices.cpu().numpy(), seeds.cpu().numpy(), fan, 1234)
    assert np.array_equal(res["nodes"], want["nodes"])
    nF = len(want["nodes"])
    # feature words are random bits (NaN patterns as fp32): read them as int32 scaled to [-1, 1) on both sides
    X = rows[:nF].view(torch.int32).float() * 2.0 ** -31
    x64 = (orc.gather(table.cpu().numpy(), want["nodes"]).view(np.int32).astype(np.float32) * np.float32(2.0 ** -31)
           ).astype(np.float64)
    for h in range(2):
        off_d = torch.as_tensor(res["offsets"][h], device=DEV)
        src_d = torch.as_tensor(res["src"][h], device=DEV)
        n_dst = len(res["offsets"][h]) - 1
        out = torch.empty((n_dst, 128), device=DEV)
        M.sage_mean(X, off_d, src_d, n_dst, out)
        ref = orc.sage_mean(x64, want["offsets"][h], want["src"][h])
        scale = orc.sage_mean(np.abs(x64), want["offsets"][h], want["src"][h])
        assert np.all(np.abs(out.cpu().numpy() - ref) <= 1e-5 * scale + 1e-7), h


def test_graphsage_forward_backward_vs_dense_fp64():
    """GraphSAGE (the consumer) on a C1 batch: logits and every weight gradient against the same model in fp64
    on the CPU with the block means written as dense row-normalised adjacency matrices (A[i, src[e]] += 1/deg_i)."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_sc_shi0s0x0w25_b200 import sage as S
    cfg = W.CONFIGS["C1"]
    g = W.rmat_csr(cfg["n"], cfg["m"], device=DEV)
    fan = [10, 5]
    seeds = W.epoch_batches(W.training_set(g, min_count=1024), 1024, 0)[0][:256]
    ctx = M.Ctx(n_vertices=g.n, max_seeds=256, max_fanout=fan, device=0)
    bufs = M.SampleBuffers.allocate(256, fan, g.n, DEV)
    ctx.sample(g.indptr, g.indices, seeds, fan, 77, bufs)
    counts = bufs.counts.cpu().numpy()
    nF = int(counts[2])
    torch.manual_seed(0)
    x = torch.randn((nF, 32), device=DEV)
    model = S.GraphSAGE(32, 64, 10, 2).to(DEV)
    labels = torch.randint(0, 10, (256,), device=DEV)
    blocks = S.blocks_of(bufs, counts)
    logits = model(x, blocks)
    loss = torch.nn.functional.cross_entropy(logits, labels)
    loss.backward()
    # fp64 reference
    ref = S.GraphSAGE(32, 64, 10, 2).double()
    ref.load_state_dict({k: v.double().cpu() for k, v in model.state_dict().items()})
    res = bufs.result()

    def dense(h):
        off, src = res["offsets"][h], res["src"][h]
        A = torch.zeros((len(off) - 1, len(res["nodes"]) if h == 1 else int(counts[1])), dtype=torch.float64)
        for i in range(len(off) - 1):
            for e in range(off[i], off[i + 1]):
                A[i, src[e]] += 1.0 / (off[i + 1] - off[i])
        return A

    A1, A0 = dense(1), dense(0)
    h = x.double().cpu()
    l0, l1 = ref.layers
    h1 = torch.relu(l0.self_lin(h[:A1.shape[0]]) + l0.neigh_lin(A1 @ h))
    out = l1.self_lin(h1[:A0.shape[0]]) + l1.neigh_lin(A0 @ h1)
    assert torch.allclose(logits.double().cpu(), out, rtol=1e-4, atol=1e-5)
    torch.nn.functional.cross_entropy(out, labels.cpu()).backward()
    for (n, p), (_, q) in zip(model.named_parameters(), ref.named_parameters()):
        assert torch.allclose(p.grad.double().cpu(), q.grad, rtol=1e-3, atol=1e-6), n
