"""Seeded synthetic inputs shaped like the paper's workloads (shared by tests, bench and smoke).

This module holds input generators only — none of the method's arithmetic (no Philox, no sampling,
no gather, no flow): a splitmix64 counter hash drives an R-MAT edge generator, a feature-row generator
and the training-seed selection. Everything is plain torch, so it runs on the GPU box (fast) and on CPU
(tests, the reference arm) with bit-identical results.

Recipe:
* Graph: R-MAT (a, b, c, d) = (0.57, 0.19, 0.19, 0.05) (Graph500) over 2^L >= n ids, one hash per edge
  per level; ids scaled to [0, n) by v * n >> L, then relabelled by the bijection v -> (A v + B) mod n to
  decouple id from degree; exactly m directed edges (a multigraph: duplicates and self-loops kept);
  CSR over the source, each adjacency sorted by destination.
* Features: row v, 32-bit word w = low 32 bits of splitmix64(feature_seed ^ (v * words + w) * K).
* Training set: 1 % of the vertices with degree >= 1, at least `min_count`, chosen by hash order;
  each epoch a hash-ordered permutation; rank r takes batches from its contiguous 1/k slice.
"""
from __future__ import annotations

import math
from dataclasses import dataclass

import torch

MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15

CONFIGS = {
    # BASELINE.json configs[0..4]; n, m = CSR entries, R = row bytes (dim * dtype size), fanout, batch.
    "C1": dict(n=1 << 16, m=1 << 20, dim=128, dtype=torch.float32, fanout=(10, 5), batch=1024,
               desc="R-MAT 2^16, avg degree 16, 128-d fp32, fanout [10,5], batch 1024, 1 GPU"),
    # experiment only (not a BASELINE config): C2's per-vertex shape on a graph whose CSR fits in L2
    "X_L2": dict(n=1 << 18, m=1 << 22, dim=100, dtype=torch.float32, fanout=(15, 10, 5), batch=1024,
                 desc="experiment: R-MAT 2^18 / 2^22 edges (CSR 18 MB, L2-resident), C2 fanout and rows"),
    "C2": dict(n=2_449_029, m=61_859_140, dim=100, dtype=torch.float32, fanout=(15, 10, 5), batch=1024,
               desc="ogbn-products-shaped: 2.45M vertices, 61.9M edges, 100-d fp32, fanout [15,10,5], batch 1024, "
                    "all features in HBM"),
    "C3": dict(n=111_059_956, m=1_615_685_872, dim=128, dtype=torch.float32, fanout=(15, 10, 5), batch=1024,
               desc="ogbn-papers100M-shaped: 111M vertices, 1.6B edges, 128-d fp32"),
    "C4": dict(n=244_160_499, m=1_728_364_232, dim=768, dtype=torch.float16, fanout=(15, 10, 5), batch=1024,
               desc="MAG240M-shaped: 244M vertices, 1.7B edges, 768-d fp16"),
    "C5": dict(n=269_346_174, m=3_995_777_033, dim=1024, dtype=torch.float32, fanout=(15, 10, 5), batch=1024,
               desc="IGB-260M-shaped: 269M vertices, 4.0B edges, 1024-d fp32"),
}


def _i64(x: int) -> int:
    x &= MASK64
    return x - (1 << 64) if x >= 1 << 63 else x


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 (torch's >> is arithmetic)."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    """splitmix64 finaliser on int64 tensors (wrapping arithmetic)."""
    x = x + _i64(GOLDEN)
    x = (x ^ _srl(x, 30)) * _i64(0xBF58476D1CE4E5B9)
    x = (x ^ _srl(x, 27)) * _i64(0x94D049BB133111EB)
    return x ^ _srl(x, 31)


def mix(*vals: int) -> int:
    """Host-side splitmix64 chain of integers (per-batch rng seeds, derived keys)."""
    h = 0
    for v in vals:
        x = (h ^ (v & MASK64)) + GOLDEN
        x &= MASK64
        x = ((x ^ (x >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
        x = ((x ^ (x >> 27)) * 0x94D049BB133111EB) & MASK64
        h = x ^ (x >> 31)
    return h


@dataclass
class Graph:
    indptr: torch.Tensor  # int64 [n + 1]
    indices: torch.Tensor  # int32 [m]
    n: int
    m: int

    def degree(self) -> torch.Tensor:
        return self.indptr[1:] - self.indptr[:-1]

    def stats(self) -> dict:
        d = self.degree()
        return {"n": self.n, "m": self.m, "max_degree": int(d.max()), "isolated_frac": float((d == 0).float().mean())}


def rmat_csr(n: int, m: int, seed: int = 0x4D4F4D454E54, device="cpu", a=0.57, b=0.19, c=0.19,
             chunk: int = 1 << 23, max_edges_in_memory: int = 1 << 31) -> Graph:
    L = max(1, math.ceil(math.log2(n)))
    ta = int(a * 2**32)
    tb = int((a + b) * 2**32)
    tc = int((a + b + c) * 2**32)
    key = _i64(mix(seed, 1))
    A = mix(seed, 2) % n
    while math.gcd(A, n) != 1 or A == 0:
        A = (A + 1) % n
    B = mix(seed, 3) % n
    def edges(e0, e1):
        e = torch.arange(e0, e1, device=device, dtype=torch.int64)
        s = torch.zeros_like(e)
        d = torch.zeros_like(e)
        for lvl in range(L):
            r = splitmix64((e * L + lvl) ^ key) & 0xFFFFFFFF
            q_b = (r >= ta) & (r < tb)
            q_c = (r >= tb) & (r < tc)
            q_d = r >= tc
            s = (s << 1) | (q_c | q_d).to(torch.int64)
            d = (d << 1) | (q_b | q_d).to(torch.int64)
        s = (s * n) >> L
        d = (d * n) >> L
        return (s * A + B) % n, (d * A + B) % n

    if m > max_edges_in_memory:
        return _rmat_csr_partitioned(n, m, edges, chunk, max_edges_in_memory, device)
    srcs, dsts = [], []
    for e0 in range(0, m, chunk):
        s, d = edges(e0, min(m, e0 + chunk))
        srcs.append(s)
        dsts.append(d)
    src = torch.cat(srcs)
    dst = torch.cat(dsts)
    del srcs, dsts
    keyv = src * n + dst
    del src, dst
    keyv, _ = torch.sort(keyv)
    src = torch.div(keyv, n, rounding_mode="floor")
    indices = (keyv - src * n).to(torch.int32)
    del keyv
    counts = torch.bincount(src, minlength=n)
    del src
    indptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    indptr[1:] = torch.cumsum(counts, 0)
    return Graph(indptr, indices, n, m)


def _rmat_csr_partitioned(n, m, edges, chunk, budget, device) -> Graph:
    """The same canonical CSR for graphs too large to sort at once: one pass for the degrees, then one pass
    per source range of <= `budget` edges, each regenerating every edge and keeping its range's."""
    counts = torch.zeros(n, dtype=torch.int64, device=device)
    for e0 in range(0, m, chunk):
        s, _ = edges(e0, min(m, e0 + chunk))
        counts += torch.bincount(s, minlength=n)
    indptr = torch.zeros(n + 1, dtype=torch.int64, device=device)
    indptr[1:] = torch.cumsum(counts, 0)
    del counts
    indices = torch.empty(m, dtype=torch.int32, device=device)
    lo = 0
    while lo < n:
        # largest hi with indptr[hi] - indptr[lo] <= budget (at least one vertex)
        hi = int(torch.searchsorted(indptr, indptr[lo] + budget, right=True)) - 1
        hi = max(lo + 1, min(hi, n))
        keys = []
        for e0 in range(0, m, chunk):
            s, d = edges(e0, min(m, e0 + chunk))
            sel = (s >= lo) & (s < hi)
            keys.append((s[sel] - lo) * n + d[sel])
        kv = torch.cat(keys)
        del keys
        kv, _ = torch.sort(kv)
        indices[int(indptr[lo]):int(indptr[hi])] = (kv % n).to(torch.int32)
        del kv
        lo = hi
    return Graph(indptr, indices, n, m)


def feature_table(n: int, dim: int, dtype=torch.float32, seed: int = 0xFEA7, device="cpu", row_stride_bytes=None,
                  chunk_rows: int = 1 << 18) -> torch.Tensor:
    """uint8 view [n, row_stride] of feature rows; row v's bytes are a function of (seed, v) only."""
    R = dim * torch.empty(0, dtype=dtype).element_size()
    assert R % 4 == 0
    stride = row_stride_bytes or R
    words = R // 4
    out = torch.zeros((n, stride), dtype=torch.uint8, device=device)
    key = _i64(mix(seed, 7))
    col = torch.arange(words, device=device, dtype=torch.int64)
    for r0 in range(0, n, chunk_rows):
        r1 = min(n, r0 + chunk_rows)
        v = torch.arange(r0, r1, device=device, dtype=torch.int64)
        w = splitmix64((v[:, None] * words + col[None, :]) ^ key) & 0xFFFFFFFF
        w = w.to(torch.int32)  # wraps to the same 32 bits
        out[r0:r1, :R] = w.view(torch.uint8).view(r1 - r0, R)
    return out


def feature_rows(ids: torch.Tensor, dim: int, dtype=torch.float32, seed: int = 0xFEA7) -> torch.Tensor:
    """The bytes of rows `ids` (uint8 [len, R]) without materialising the table."""
    R = dim * torch.empty(0, dtype=dtype).element_size()
    words = R // 4
    key = _i64(mix(seed, 7))
    col = torch.arange(words, device=ids.device, dtype=torch.int64)
    w = splitmix64((ids.to(torch.int64)[:, None] * words + col[None, :]) ^ key) & 0xFFFFFFFF
    return w.to(torch.int32).view(torch.uint8).view(len(ids), R)


def training_set(g: Graph, frac: float = 0.01, min_count: int = 0, seed: int = 0x7EED) -> torch.Tensor:
    """1 % of the vertices with degree >= 1, at least min_count, in hash order."""
    cand = torch.nonzero(g.degree() > 0).flatten()
    cnt = max(int(math.ceil(frac * g.n)), min_count)
    cnt = min(cnt, len(cand))
    h = splitmix64(cand ^ _i64(mix(seed, 11)))
    order = torch.argsort(h)
    return cand[order[:cnt]].contiguous()


def epoch_batches(train: torch.Tensor, batch: int, epoch: int, rank: int = 0, world: int = 1,
                  seed: int = 0x7EED) -> list[torch.Tensor]:
    """Rank r's batches of one epoch: a hash permutation of the training set, contiguous 1/k slice."""
    idx = torch.arange(len(train), device=train.device, dtype=torch.int64)
    perm = torch.argsort(splitmix64(idx ^ _i64(mix(seed, 13, epoch))))
    per_rank = len(train) // world
    mine = train[perm[rank * per_rank:(rank + 1) * per_rank]]
    return [mine[i:i + batch].contiguous() for i in range(0, per_rank - batch + 1, batch)]


def batch_rng_seed(run_seed: int, epoch: int, rank: int, batch: int) -> int:
    """Per-batch Philox key (R1): splitmix64(run seed, epoch, rank, batch)."""
    return mix(run_seed, epoch, rank, batch)
