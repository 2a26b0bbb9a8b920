"""Consumer of the sampled + gathered batches: GraphSAGE with mean aggregation, the model
the paper trains (hidden 256, fan-outs [25, 10], batch 8000; Eq. 1).

Layer l (0-based, L layers, H = L hops) computes the rows of F_{H-1-l} from those of F_{H-l}:
    h_v = act( h_v^{prev} W_self + mean_{u in sampled N(v)} h_u^{prev} W_neigh + b )
where the mean runs over hop H-1-l's block of `moment_sample` (offsets over F_{H-1-l}, src indices into
F_{H-l}) and h^{prev} of F_{H-1-l} is the prefix of h^{prev} of F_{H-l} (F_h is a prefix of F_{h+1}, R6).
The sparse mean is `moment_sage_mean` / `_backward` (sm_100a kernels); the weight GEMMs are cuBLAS through
torch (bf16 autocast) — plain library GEMMs.
"""
import torch

from . import moment as M


class SageMean(torch.autograd.Function):
    """mean over a block: [n_src, dim] -> [n_dst, dim] (fp32 or bf16), backward by the adjoint kernel."""

    @staticmethod
    def forward(ctx, x, offsets, src, n_dst: int):
        out = torch.empty((n_dst, x.shape[1]), device=x.device, dtype=x.dtype)
        M.sage_mean(x, offsets, src, n_dst, out)
        ctx.save_for_backward(offsets, src)
        ctx.n_dst, ctx.n_src, ctx.x_dtype = n_dst, x.shape[0], x.dtype
        return out

    @staticmethod
    def backward(ctx, grad_out):
        offsets, src = ctx.saved_tensors
        if not ctx.needs_input_grad[0]:
            return None, None, None, None
        g = grad_out.contiguous()
        gx = torch.zeros((ctx.n_src, g.shape[1]), device=g.device, dtype=torch.float32)
        M.sage_mean_backward(g, offsets, src, ctx.n_dst, gx)
        return gx.to(ctx.x_dtype), None, None, None


def sage_mean(x, offsets, src, n_dst: int):
    return SageMean.apply(x, offsets, src, n_dst)


class SAGELayer(torch.nn.Module):
    def __init__(self, d_in: int, d_out: int):
        super().__init__()
        self.self_lin = torch.nn.Linear(d_in, d_out)
        self.neigh_lin = torch.nn.Linear(d_in, d_out, bias=False)

    def forward(self, h, block, bucket: int = 0):
        """Rows [0, n_dst) are the layer's output. bucket > 0: the GEMMs run on n_pad = n_dst rounded up to a
        multiple of `bucket` (at most h's rows) so that batches of different sizes share a few GEMM shapes —
        every new shape costs the library a heuristic search (measured: ~5 ms per training step when every
        batch brings new ones). Rows [n_dst, n_pad) are don't-care: the mean part is zero there, no later
        layer reads them (src < n_dst) and the loss never does, so they get zero gradient."""
        offsets, src, n_dst = block
        n_pad = min(h.shape[0], -(-n_dst // bucket) * bucket) if bucket > 0 else n_dst
        n_pad = max(n_pad, n_dst)
        agg = sage_mean(h, offsets, src, n_dst)
        if n_pad > n_dst:
            agg = torch.nn.functional.pad(agg, (0, 0, 0, n_pad - n_dst))
        return self.self_lin(h[:n_pad]) + self.neigh_lin(agg)


class GraphSAGE(torch.nn.Module):
    def __init__(self, d_in: int, hidden: int, n_classes: int, n_layers: int, bucket: int = 2048):
        super().__init__()
        dims = [d_in] + [hidden] * (n_layers - 1) + [n_classes]
        self.layers = torch.nn.ModuleList(SAGELayer(dims[i], dims[i + 1]) for i in range(n_layers))
        self.bucket = bucket

    def forward(self, x, blocks):
        """x: rows of F_H (fp32); blocks: [(offsets, src, n_dst)] per hop 0..H-1 (moment_sample's layout)."""
        h = x
        H = len(blocks)
        for l, layer in enumerate(self.layers):
            last = l + 1 == len(self.layers)
            h = layer(h, blocks[H - 1 - l], 0 if last else self.bucket)
            if not last:
                h = torch.relu(h)
        return h


def blocks_of(bufs: "M.SampleBuffers", counts):
    """Per-hop (offsets, src, n_dst) views of a SampleBuffers batch; counts = host copy of bufs.counts."""
    H = len(bufs.fanout)
    F, E = [int(c) for c in counts[:H + 1]], [int(c) for c in counts[H + 1:2 * H + 1]]
    out, ob, eb = [], 0, 0
    for h in range(H):
        out.append((bufs.offsets[ob: ob + F[h] + 1], bufs.src[eb: eb + E[h]], F[h]))
        ob += F[h] + 1
        eb += E[h]
    return out
