"""CPU oracle for the Moment hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl reference``
legs may import this package. The product package (``paper_conf_sc_shi0s0x0w25_b200``) never imports it,
and this package imports nothing from the product: the two share no code.

The arithmetic lives in ``moment_oracle.c`` (plain single-threaded C, each function citing the
PAPER.md passage it follows). This module only compiles it with gcc and marshals numpy arrays.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "moment_oracle.c")
LIB = os.path.join(HERE, "_build", "liboracle.so")

OK, EINVAL, ENOMEM, EINFEASIBLE, EOVERFLOW = 0, -1, -2, -5, -6
INF = np.iinfo(np.int64).max


class OracleError(RuntimeError):
    def __init__(self, status: int, what: str):
        super().__init__(f"oracle {what} failed with status {status}")
        self.status = status


def build(force: bool = False) -> str:
    """Compile the oracle (gcc, single-threaded, no product headers)."""
    os.makedirs(os.path.dirname(LIB), exist_ok=True)
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.run(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", LIB, SRC], check=True)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        _setup(_lib)
    return _lib


P = C.c_void_p
I32, I64, U64, U32 = C.c_int32, C.c_int64, C.c_uint64, C.c_uint32


def _setup(L):
    L.orc_philox4x32_10.argtypes = [P, P, P]
    L.orc_philox4x32_10.restype = None
    L.orc_draw.argtypes = [U64, I64, I32, I64]
    L.orc_draw.restype = U32
    L.orc_uniform.argtypes = [U32, U64]
    L.orc_uniform.restype = U64
    L.orc_floyd.argtypes = [I64, I32, P, P]
    L.orc_floyd.restype = I64
    L.orc_sample_node.argtypes = [U64, I64, I32, I64, I32, I32, P]
    L.orc_sample_node.restype = I64
    L.orc_sample.argtypes = [P, P, I64, P, I64, P, I32, U64, I32, I64, I64, P, P, P, P]
    L.orc_sample.restype = C.c_int
    L.orc_gather.argtypes = [P, I64, P, I64, P]
    L.orc_gather.restype = None
    L.orc_maxflow.argtypes = [I32, I32, P, P, P, I32, I32, P, P]
    L.orc_maxflow.restype = C.c_int
    L.orc_time_bisect.argtypes = [I32, I32, P, P, P, P, I32, I32, P, P]
    L.orc_time_bisect.restype = C.c_int
    L.orc_plan_closed_forms.argtypes = [I32, I32, P, P, P, I64, I64, I64, P, P]
    L.orc_plan_closed_forms.restype = C.c_int
    L.orc_quota.argtypes = [I32, I32, P, P, P, I32, I32, I32, P, P]
    L.orc_quota.restype = C.c_int
    L.orc_hash_place.argtypes = [I64, I32, P, P, P, P]
    L.orc_hash_place.restype = C.c_int
    L.orc_bucket.argtypes = [I32, I32, I32, P, P, P, I64, P, P, P]
    L.orc_bucket.restype = C.c_int
    L.orc_ddak.argtypes = [I64, P, I32, P, P, P, I64, P, P, P, P]
    L.orc_ddak.restype = C.c_int
    L.orc_ddak_replicate.argtypes = [I64, P, I32, P, P, P, I64, I64, P, P, P, P, P]
    L.orc_ddak_replicate.restype = C.c_int
    L.orc_sage_mean.argtypes = [P, I64, P, P, I64, P]
    L.orc_sage_mean.restype = None
    L.orc_sage_mean_backward.argtypes = [P, I64, P, P, I64, P]
    L.orc_sage_mean_backward.restype = None


def _p(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _c(a, dtype):
    return np.ascontiguousarray(np.asarray(a, dtype=dtype))


def philox4x32_10(ctr, key) -> np.ndarray:
    c = _c(ctr, np.uint32)
    k = _c(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(_p(c), _p(k), _p(out))
    return out


def draw(rng_seed: int, v: int, h: int, i: int) -> int:
    return int(lib().orc_draw(rng_seed, v, h, i))


def uniform(r: int, m: int) -> int:
    return int(lib().orc_uniform(r, m))


def floyd(d: int, k: int, t) -> list[int]:
    tt = _c(t, np.int64)
    out = np.zeros(max(k, 1), np.int64)
    c = lib().orc_floyd(d, k, _p(tt), _p(out))
    return [int(x) for x in out[:c]]


def sample_node(rng_seed: int, v: int, h: int, d: int, k: int, replace: bool = False) -> list[int]:
    out = np.zeros(max(k, d, 1), np.int64)
    c = lib().orc_sample_node(rng_seed, v, h, d, k, int(replace), _p(out))
    return [int(x) for x in out[:c]]


def sample_bounds(n_seeds: int, fanout, n_vertices: int) -> tuple[int, int]:
    """Upper bounds on |F_H| and sum_h E_h without dedup (|F_{h+1}| <= |F_h| (1 + f_h))."""
    f, e = n_seeds, 0
    for k in fanout:
        e += f * k
        f = min(f + f * k, n_vertices)
    return f, e


def sample(indptr, indices, seeds, fanout, rng_seed: int, replace: bool = False):
    """Returns dict(nodes, offsets=[per-hop arrays], src=[per-hop arrays], counts)."""
    indptr = _c(indptr, np.int64)
    indices = _c(indices, np.int32)
    seeds = _c(seeds, np.int64)
    fan = _c(fanout, np.int32)
    n = indptr.shape[0] - 1
    H = len(fanout)
    cap_nodes, cap_edges = sample_bounds(len(seeds), fanout, n)
    cap_nodes = max(cap_nodes, len(seeds), 1)
    nodes = np.zeros(cap_nodes, np.int64)
    offsets_len = 0
    f = len(seeds)
    for k in fanout:
        offsets_len += f + 1
        f = min(f + f * k, n)
    offsets = np.zeros(max(offsets_len, 1), np.int64)
    src = np.zeros(max(cap_edges, 1), np.int32)
    counts = np.zeros(2 * H + 1, np.int64)
    st = lib().orc_sample(_p(indptr), _p(indices), n, _p(seeds), len(seeds), _p(fan), H, rng_seed, int(replace),
                          cap_nodes, cap_edges, _p(nodes), _p(offsets), _p(src), _p(counts))
    if st != OK:
        raise OracleError(st, "sample")
    F = counts[: H + 1]
    E = counts[H + 1:]
    offs, srcs = [], []
    ob, eb = 0, 0
    for h in range(H):
        offs.append(offsets[ob: ob + F[h] + 1].copy())
        srcs.append(src[eb: eb + E[h]].copy())
        ob += F[h] + 1
        eb += E[h]
    return {"nodes": nodes[: F[H]].copy(), "offsets": offs, "src": srcs, "counts": counts}


def gather(table: np.ndarray, ids) -> np.ndarray:
    table = np.ascontiguousarray(table)
    R = table.strides[0] if table.ndim > 1 else table.itemsize
    ids = _c(ids, np.int64)
    out = np.empty((len(ids),) + table.shape[1:], table.dtype)
    lib().orc_gather(_p(table), R, _p(ids), len(ids), _p(out))
    return out


def maxflow(n_nodes: int, links, s: int, t: int):
    """links: sequence of (from, to, cap). Returns (value, flow per link)."""
    fr = _c([l[0] for l in links], np.int32)
    to = _c([l[1] for l in links], np.int32)
    cap = _c([l[2] for l in links], np.int64)
    val = np.zeros(1, np.int64)
    flow = np.zeros(max(len(links), 1), np.int64)
    st = lib().orc_maxflow(n_nodes, len(links), _p(fr), _p(to), _p(cap), s, t, _p(val), _p(flow))
    if st != OK:
        raise OracleError(st, "maxflow")
    return int(val[0]), flow[: len(links)]


def time_bisect(n_nodes: int, links, is_supply, s: int, t: int):
    fr = _c([l[0] for l in links], np.int32)
    to = _c([l[1] for l in links], np.int32)
    cap = _c([l[2] for l in links], np.int64)
    sup = _c(is_supply, np.uint8)
    ts = np.zeros(1, np.int64)
    flow = np.zeros(max(len(links), 1), np.int64)
    st = lib().orc_time_bisect(n_nodes, len(links), _p(fr), _p(to), _p(cap), _p(sup), s, t, _p(ts), _p(flow))
    if st != OK:
        raise OracleError(st, "time_bisect")
    return int(ts[0]), flow[: len(links)]


def plan_closed_forms(k: int, hbm_owner, d, x, nvlink_cap: int, hbm_cap: int, replica_d: int = 0):
    own = _c(hbm_owner, np.int32)
    dd = _c(d, np.int64)
    xx = _c(x, np.int64).reshape(-1)
    tn = np.zeros(1, np.int64)
    th = np.zeros(1, np.int64)
    st = lib().orc_plan_closed_forms(k, len(own), _p(own), _p(dd), _p(xx), nvlink_cap, hbm_cap, replica_d, _p(tn),
                                     _p(th))
    if st != OK:
        raise OracleError(st, "plan_closed_forms")
    return int(tn[0]), int(th[0])


def quota(n_nodes: int, links, flow, s: int, t: int, gpu_nodes):
    """Path decomposition of a given ingest flow (R11): x[n_nodes][k], k = len(gpu_nodes) (rank order)."""
    fr = _c([l[0] for l in links], np.int32)
    to = _c([l[1] for l in links], np.int32)
    fl = _c(flow, np.int64)
    k = len(gpu_nodes)
    rank = np.full(n_nodes, -1, np.int32)
    for r, v in enumerate(gpu_nodes):
        rank[v] = r
    x = np.zeros((n_nodes, k), np.int64)
    st = lib().orc_quota(n_nodes, len(links), _p(fr), _p(to), _p(fl), s, t, k, _p(rank), _p(x))
    if st != OK:
        raise OracleError(st, "quota")
    return x


def hash_place(n: int, cap_rows):
    """Hash-partitioning baseline (R24): (bin_of int32[n], slot_of int64[n], used int64[n_bins])."""
    cap = _c(cap_rows, np.int64)
    bin_of = np.full(max(n, 1), -1, np.int32)
    slot_of = np.full(max(n, 1), -1, np.int64)
    used = np.zeros(len(cap), np.int64)
    st = lib().orc_hash_place(n, len(cap), _p(cap), _p(bin_of), _p(slot_of), _p(used))
    if st != OK:
        raise OracleError(st, "hash_place")
    return bin_of[:n], slot_of[:n], used


def bucket(g: int, k: int, hbm_owner, x, bin_of_id):
    own = _c(hbm_owner, np.int32)
    xx = _c(x, np.int64).reshape(-1)
    b = _c(bin_of_id, np.int32)
    n = len(b)
    route = np.zeros(max(n, 1), np.int32)
    Q = len(own) * k
    qoff = np.zeros(Q + 1, np.int64)
    qpos = np.zeros(max(n, 1), np.int64)
    st = lib().orc_bucket(g, k, len(own), _p(own), _p(xx), _p(b), n, _p(route), _p(qoff), _p(qpos))
    if st != OK:
        raise OracleError(st, "bucket")
    return route[:n], qoff, qpos[:n]


def ddak(hotness, tier_rank, cap_rows, traffic, pool: int = 100):
    hot = _c(hotness, np.uint64)
    tr = _c(tier_rank, np.int32)
    cap = _c(cap_rows, np.int64)
    traf = _c(traffic, np.int64)
    n = len(hot)
    nb = len(tr)
    bin_of = np.full(max(n, 1), -1, np.int32)
    slot_of = np.full(max(n, 1), -1, np.int64)
    A = np.zeros(nb, np.uint64)
    U = np.zeros(nb, np.int64)
    st = lib().orc_ddak(n, _p(hot), nb, _p(tr), _p(cap), _p(traf), pool, _p(bin_of), _p(slot_of), _p(A), _p(U))
    if st != OK:
        raise OracleError(st, "ddak")
    return bin_of[:n], slot_of[:n], A, U


def ddak_replicate(hotness, tier_rank, cap_rows, traffic, r: int, pool: int = 100):
    """R25: (bin_of with -2 = replica, slot_of, A, U, replica_access)."""
    hot = _c(hotness, np.uint64)
    tr = _c(tier_rank, np.int32)
    cap = _c(cap_rows, np.int64)
    traf = _c(traffic, np.int64)
    n = len(hot)
    nb = len(tr)
    bin_of = np.full(max(n, 1), -1, np.int32)
    slot_of = np.full(max(n, 1), -1, np.int64)
    A = np.zeros(nb, np.uint64)
    U = np.zeros(nb, np.int64)
    rep = np.zeros(1, np.uint64)
    st = lib().orc_ddak_replicate(n, _p(hot), nb, _p(tr), _p(cap), _p(traf), pool, r, _p(bin_of), _p(slot_of), _p(A),
                                  _p(U), _p(rep))
    if st != OK:
        raise OracleError(st, "ddak_replicate")
    return bin_of[:n], slot_of[:n], A, U, int(rep[0])


def sage_mean(x, offsets, src):
    """fp64 mean aggregation over a block (Eq. 1): out[i] = mean of x[src[e]], e in [offsets[i], offsets[i+1])."""
    x = _c(x, np.float64)
    off = _c(offsets, np.int64)
    sr = _c(src, np.int32)
    n_dst = len(off) - 1
    dim = x.shape[1]
    out = np.zeros((max(n_dst, 1), dim), np.float64)
    lib().orc_sage_mean(_p(x), dim, _p(off), _p(sr), n_dst, _p(out))
    return out[:n_dst]


def sage_mean_backward(g, offsets, src, n_src: int):
    """fp64 adjoint of sage_mean: gx[src[e]] += g[i] / deg_i."""
    g = _c(g, np.float64)
    off = _c(offsets, np.int64)
    sr = _c(src, np.int32)
    n_dst = len(off) - 1
    dim = g.shape[1]
    gx = np.zeros((max(n_src, 1), dim), np.float64)
    lib().orc_sage_mean_backward(_p(g), dim, _p(off), _p(sr), n_dst, _p(gx))
    return gx[:n_src]
