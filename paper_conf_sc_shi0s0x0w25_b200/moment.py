"""Thin Python binding of include/moment.h (ctypes; argument marshalling only).

Every computation runs in libmoment.so: the host planner in C++, the hot path in sm_100a kernels.
PyTorch is used for device memory and streams only. There is no fallback: if the library is missing or
fails to load, every call raises.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("MOMENT_LIB_PATH") or os.path.join(_PKG, "lib", "libmoment.so")

OK, EINVAL, ENOMEM, ECUDA, ENCCL, EINFEASIBLE, EOVERFLOW, EUNSUPPORTED, ETIMEDOUT = 0, -1, -2, -3, -4, -5, -6, -7, -8
CAP_INF = np.iinfo(np.int64).max
NODE_SOURCE, NODE_SINK, NODE_STORAGE, NODE_INTERCONNECT, NODE_COMPUTE = range(5)
TIER_NONE, TIER_GPU_HBM, TIER_HOST_DRAM, TIER_SSD = range(4)
PLACE_DDAK, PLACE_HASH = 0, 1
BIN_REPLICA = -2
TRAFFIC_RATE_FLOW, TRAFFIC_STANDALONE = 0, 1
DTYPE_F32, DTYPE_BF16 = 0, 1
SAMPLE_REPLACE, SAMPLE_CHECK = 1, 2
MAX_BINS = 64

EXPORTED = [
    "moment_last_error", "moment_version", "moment_topology", "moment_topology_info", "moment_topology_export",
    "moment_topology_free", "moment_maxflow", "moment_place", "moment_place_pack", "moment_place_pack_rank", "moment_plan",
    "moment_plan_info", "moment_plan_free", "moment_replicate_search", "moment_ctx_create", "moment_ctx_free", "moment_ctx_workspace_bytes", "moment_sample_bounds",
    "moment_sample", "moment_sample_check", "moment_hotness", "moment_bucket", "moment_gather", "moment_gather_group",
    "moment_step", "moment_step_host", "moment_step_batch", "moment_gather_routed", "moment_relay_pack", "moment_relay_serve",
    "moment_relay_scatter", "moment_relay_push", "moment_relay_serve_push", "moment_ipc_export", "moment_ipc_import",
    "moment_ipc_close", "moment_sage_mean", "moment_sage_mean_backward", "moment_signal_barrier",
    "moment_ctx_set_exchange", "moment_exchange_status",
]
MAX_WORLD = 64


class MomentError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"[moment status {status}] {msg}")
        self.status = status


class Node(C.Structure):
    _fields_ = [("kind", C.c_int32), ("tier", C.c_int32), ("device", C.c_int32), ("reserved", C.c_int32)]


class Link(C.Structure):
    _fields_ = [("from_", C.c_int32), ("to", C.c_int32), ("cap", C.c_int64)]


class PlaceArgs(C.Structure):
    _fields_ = [("n_vertices", C.c_int64), ("hotness", C.c_void_p), ("n_bins", C.c_int32), ("bin_node", C.c_void_p),
                ("bin_tier", C.c_void_p), ("bin_capacity_rows", C.c_void_p), ("bin_traffic", C.c_void_p),
                ("pool", C.c_int64), ("mode", C.c_int32), ("replicate_rows", C.c_int64),
                ("traffic_mode", C.c_int32)]


class PlaceOut(C.Structure):
    _fields_ = [("bin_of", C.c_void_p), ("slot_of", C.c_void_p), ("bin_access", C.c_void_p),
                ("bin_rows_used", C.c_void_p), ("bin_traffic_used", C.c_void_p), ("replica_access", C.c_void_p)]


class PlanArgs(C.Structure):
    _fields_ = [("k", C.c_int32), ("gpu_node", C.c_void_p), ("bin_demand_bytes", C.c_void_p),
                ("nvlink_cap", C.c_int64), ("hbm_cap", C.c_int64), ("replica_demand_bytes", C.c_int64)]


class ReplicateArgs(C.Structure):
    _fields_ = [("place", C.c_void_p), ("k", C.c_int32), ("gpu_node", C.c_void_p), ("nvlink_cap", C.c_int64),
                ("hbm_cap", C.c_int64), ("row_bytes", C.c_int64), ("hot_batches", C.c_int64),
                ("demand_counts", C.c_void_p), ("demand_batches", C.c_int64),
                ("n_candidates", C.c_int32), ("candidates", C.c_void_p)]


class CtxArgs(C.Structure):
    _fields_ = [("rank", C.c_int32), ("world", C.c_int32), ("device", C.c_int32), ("n_vertices", C.c_int64),
                ("max_seeds", C.c_int64), ("max_hops", C.c_int32), ("max_fanout", C.c_void_p),
                ("row_bytes", C.c_int64), ("row_stride", C.c_int64), ("n_bins", C.c_int32),
                ("bin_owner", C.c_void_p), ("bin_ptr", C.c_void_p), ("placement", C.c_void_p), ("quota", C.c_void_p)]


class ExchangeArgs(C.Structure):
    _fields_ = [("cap", C.c_int64), ("inbox", C.c_void_p), ("inbox_count", C.c_void_p), ("flags", C.c_void_p),
                ("out", C.c_void_p), ("peer_inbox", C.c_void_p * 64), ("peer_count", C.c_void_p * 64),
                ("peer_out", C.c_void_p * 64), ("peer_flag", C.c_void_p * 64), ("timeout_ns", C.c_int64)]


class Csr(C.Structure):
    _fields_ = [("indptr", C.c_void_p), ("indices", C.c_void_p), ("n_vertices", C.c_int64), ("n_edges", C.c_int64)]


class SampleParams(C.Structure):
    _fields_ = [("n_hops", C.c_int32), ("fanout", C.c_void_p), ("rng_seed", C.c_uint64), ("flags", C.c_uint32)]


class SampleOut(C.Structure):
    _fields_ = [("nodes", C.c_void_p), ("offsets", C.c_void_p), ("src", C.c_void_p), ("counts", C.c_void_p),
                ("cap_nodes", C.c_int64), ("cap_offsets", C.c_int64), ("cap_edges", C.c_int64)]


_lib = None
P = C.c_void_p
I32, I64, U64 = C.c_int32, C.c_int64, C.c_uint64


def lib():
    """Load libmoment.so (raises if it is missing: there is no fallback path)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise MomentError(EUNSUPPORTED, f"{LIB_PATH} is missing: run __graft_entry__.build()")
        L = C.CDLL(LIB_PATH)
        sig = {
            "moment_last_error": ([], C.c_char_p),
            "moment_version": ([], I32),
            "moment_topology": ([P, I32, P, I32, P], I32),
            "moment_topology_info": ([P, P, P, P, P], I32),
            "moment_topology_export": ([P, P, P], I32),
            "moment_topology_free": ([P], I32),
            "moment_maxflow": ([P, P, P], I32),
            "moment_place": ([P, P, P], I32),
            "moment_place_pack": ([I64, P, P, P], I32),
            "moment_place_pack_rank": ([I64, P, P, I32, P], I32),
            "moment_replicate_search": ([P, P, P, P], I32),
            "moment_plan": ([P, P, P], I32),
            "moment_plan_info": ([P, P, P, P, P, P, P], I32),
            "moment_plan_free": ([P], I32),
            "moment_ctx_create": ([P, P], I32),
            "moment_ctx_free": ([P], I32),
            "moment_ctx_workspace_bytes": ([P, P], I32),
            "moment_sample_bounds": ([I64, P, I32, I64, P, P, P], I32),
            "moment_sample": ([P, P, P, I64, P, P, P], I32),
            "moment_sample_check": ([P, P], I32),
            "moment_hotness": ([P, P, P, I64, P, P], I32),
            "moment_bucket": ([P, P, P, I64, P, P, P, P], I32),
            "moment_gather": ([P, P, P, I64, P, P], I32),
            "moment_gather_group": ([P, I32, P, P, I64, P, P], I32),
            "moment_step": ([P, P, P, I64, P, P, P, P], I32),
            "moment_step_host": ([P, P, P, I64, P, P, P, P, P], I32),
            "moment_step_batch": ([I32, P, P, P, I64, P, P, P, P, P, P], I32),
            "moment_gather_routed": ([P, P, P, I64, P, P, P], I32),
            "moment_relay_pack": ([P, P, I64, P, P, P, P, P], I32),
            "moment_relay_serve": ([P, P, P, I64, P, P], I32),
            "moment_relay_scatter": ([P, P, P, I64, P, P, P], I32),
            "moment_relay_push": ([P, P, I64, P, P, P, P, P], I32),
            "moment_relay_serve_push": ([P, P, P, I64, P, P], I32),
            "moment_ipc_export": ([P, P, P], I32),
            "moment_ipc_import": ([P, P], I32),
            "moment_ipc_close": ([P], I32),
            "moment_sage_mean": ([P, I64, I32, I64, P, P, I64, P, I64, P], I32),
            "moment_signal_barrier": ([I32, I32, P, P, U64, I64, P, P], I32),
            "moment_sage_mean_backward": ([P, I64, I32, I64, P, P, I64, P, I64, P], I32),
            "moment_ctx_set_exchange": ([P, P], I32),
            "moment_exchange_status": ([P, P], I32),
        }
        for name, (args, res) in sig.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = res
        _lib = L
    return _lib


def _check(status: int):
    if status != OK:
        raise MomentError(status, lib().moment_last_error().decode())


def _np(a, dtype):
    return np.ascontiguousarray(np.asarray(a, dtype=dtype))


def _ptr(a) -> int:
    """Address of a numpy array or torch tensor (None -> NULL)."""
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        return a.ctypes.data
    return a.data_ptr()


def _stream(stream) -> int | None:
    if stream is None:
        import torch

        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


# ---------------------------------------------------------------------------------------------- P1
class Topology:
    def __init__(self, nodes, links):
        """nodes: [(kind, tier, device)], links: [(from, to, cap)] (cap = CAP_INF for infinite)."""
        na = (Node * len(nodes))(*[Node(k, t, d, 0) for (k, t, d) in nodes])
        la = (Link * max(1, len(links)))(*[Link(f, t, c) for (f, t, c) in links])
        h = C.c_void_p()
        _check(lib().moment_topology(C.cast(na, P), len(nodes), C.cast(la, P), len(links), C.byref(h)))
        self.handle = h

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:
            _lib.moment_topology_free(self.handle)
            self.handle = None

    def info(self):
        n, m, s, t = C.c_int32(), C.c_int32(), C.c_int32(), C.c_int32()
        _check(lib().moment_topology_info(self.handle, C.byref(n), C.byref(m), C.byref(s), C.byref(t)))
        return n.value, m.value, s.value, t.value

    def export(self):
        n, m, s, t = self.info()
        na = (Node * n)()
        la = (Link * max(1, m))()
        _check(lib().moment_topology_export(self.handle, C.cast(na, P), C.cast(la, P)))
        nodes = [(x.kind, x.tier, x.device) for x in na]
        links = [(x.from_, x.to, x.cap) for x in la[:m]]
        return nodes, links, s, t

    def maxflow(self):
        """P3: (value, per-link flow) of the rate max-flow (Dinic)."""
        _, m, _, _ = self.info()
        v = C.c_int64()
        flow = np.zeros(max(m, 1), np.int64)
        _check(lib().moment_maxflow(self.handle, C.byref(v), _ptr(flow)))
        return v.value, flow[:m]


def topology(nodes, links) -> Topology:
    return Topology(nodes, links)


# ---------------------------------------------------------------------------------------------- P4
def place(topo: Topology | None, hotness, capacity_rows, *, bin_node=None, bin_tier=None, bin_traffic=None,
          pool: int = 100, mode: int = PLACE_DDAK, replicate_rows: int = 0, return_replica_access: bool = False,
          traffic_mode: int = TRAFFIC_RATE_FLOW):
    """DDAK placement. Returns (bin_of int32[n], slot_of int64[n], access uint64[nb], used int64[nb],
    traffic int64[nb]) [+ replica_access]. replicate_rows > 0: the hottest rows are copied into every GPU bin
    (bin_of = BIN_REPLICA, R25)."""
    hot = _np(hotness, np.uint64)
    cap = _np(capacity_rows, np.int64)
    nb = len(cap)
    n = len(hot)
    keep = []

    def opt(a, dt):
        if a is None:
            return None
        arr = _np(a, dt)
        keep.append(arr)
        return arr.ctypes.data

    args = PlaceArgs(n, hot.ctypes.data, nb, opt(bin_node, np.int32), opt(bin_tier, np.int32), cap.ctypes.data,
                     opt(bin_traffic, np.int64), pool, mode, replicate_rows, traffic_mode)
    bin_of = np.zeros(max(n, 1), np.int32)
    slot_of = np.zeros(max(n, 1), np.int64)
    acc = np.zeros(nb, np.uint64)
    used = np.zeros(nb, np.int64)
    traf = np.zeros(nb, np.int64)
    rep = np.zeros(1, np.uint64)
    out = PlaceOut(bin_of.ctypes.data, slot_of.ctypes.data, acc.ctypes.data, used.ctypes.data, traf.ctypes.data,
                   rep.ctypes.data)
    _check(lib().moment_place(topo.handle if topo is not None else None, C.byref(args), C.byref(out)))
    if return_replica_access:
        return bin_of[:n], slot_of[:n], acc, used, traf, int(rep[0])
    return bin_of[:n], slot_of[:n], acc, used, traf


def place_pack(bin_of, slot_of) -> np.ndarray:
    b = _np(bin_of, np.int32)
    s = _np(slot_of, np.int64)
    out = np.zeros(max(len(b), 1), np.uint64)
    _check(lib().moment_place_pack(len(b), b.ctypes.data, s.ctypes.data, out.ctypes.data))
    return out[: len(b)]


def place_pack_rank(bin_of, slot_of, replica_bin: int) -> np.ndarray:
    """One rank's device map: replicated vertices point at that rank's own HBM bin `replica_bin`."""
    b = _np(bin_of, np.int32)
    s = _np(slot_of, np.int64)
    out = np.zeros(max(len(b), 1), np.uint64)
    _check(lib().moment_place_pack_rank(len(b), b.ctypes.data, s.ctypes.data, replica_bin, out.ctypes.data))
    return out[: len(b)]


# ---------------------------------------------------------------------------------------------- P5
class Plan:
    def __init__(self, topo: Topology, gpu_node, demand_bytes, nvlink_cap: int, hbm_cap: int, replica_demand: int = 0):
        g = _np(gpu_node, np.int32)
        d = _np(demand_bytes, np.int64)
        n, m, _, _ = topo.info()
        if len(d) != n:
            raise MomentError(EINVAL, f"demand has {len(d)} entries, topology has {n} nodes")
        self.k, self.n_nodes, self.n_links = len(g), n, m
        args = PlanArgs(len(g), g.ctypes.data, d.ctypes.data, nvlink_cap, hbm_cap, replica_demand)
        h = C.c_void_p()
        _check(lib().moment_plan(topo.handle, C.byref(args), C.byref(h)))
        self.handle = h

    def __del__(self):
        if getattr(self, "handle", None) and _lib is not None:
            _lib.moment_plan_free(self.handle)
            self.handle = None

    def info(self):
        ts, ti, tn, th = C.c_int64(), C.c_int64(), C.c_int64(), C.c_int64()
        flow = np.zeros(max(self.n_links, 1), np.int64)
        quota = np.zeros(self.n_nodes * self.k, np.int64)
        _check(lib().moment_plan_info(self.handle, C.byref(ts), C.byref(ti), C.byref(tn), C.byref(th), _ptr(flow),
                                      _ptr(quota)))
        return {"t_star": ts.value, "t_ingest": ti.value, "t_nvlink": tn.value, "t_hbm": th.value,
                "link_flow": flow[: self.n_links], "quota": quota.reshape(self.n_nodes, self.k)}


def plan(topo, gpu_node, demand_bytes, nvlink_cap, hbm_cap, replica_demand: int = 0) -> Plan:
    return Plan(topo, gpu_node, demand_bytes, nvlink_cap, hbm_cap, replica_demand)


def replicate_search(topo: Topology, hotness, capacity_rows, candidates, *, gpu_node, nvlink_cap: int, hbm_cap: int,
                     row_bytes: int, hot_batches: int, bin_node=None, bin_tier=None, bin_traffic=None, pool: int = 100,
                     demand_counts=None, demand_batches: int = 0, traffic_mode: int = TRAFFIC_RATE_FLOW):
    """T*(r) of the plan for every candidate replicate_rows r (R25). Returns (t_star int64[n_cand] with -1 =
    infeasible, best index or -1). demand_counts / demand_batches: held-out F_H counts for the per-bin demand
    (default: the placement's own hotness)."""
    hot = _np(hotness, np.uint64)
    cap = _np(capacity_rows, np.int64)
    keep = []

    def opt(a, dt):
        if a is None:
            return None
        arr = _np(a, dt)
        keep.append(arr)
        return arr.ctypes.data

    pa = PlaceArgs(len(hot), hot.ctypes.data, len(cap), opt(bin_node, np.int32), opt(bin_tier, np.int32),
                   cap.ctypes.data, opt(bin_traffic, np.int64), pool, PLACE_DDAK, 0, traffic_mode)
    g = _np(gpu_node, np.int32)
    cand = _np(candidates, np.int64)
    ts = np.zeros(max(len(cand), 1), np.int64)
    best = C.c_int32()
    dem = opt(demand_counts, np.uint64)
    args = ReplicateArgs(C.addressof(pa), len(g), g.ctypes.data, nvlink_cap, hbm_cap, row_bytes, hot_batches,
                         dem, demand_batches, len(cand), cand.ctypes.data)
    _check(lib().moment_replicate_search(topo.handle, C.byref(args), ts.ctypes.data, C.byref(best)))
    return ts[: len(cand)], best.value


# ---------------------------------------------------------------------------------------------- ctx
def sample_bounds(n_seeds: int, fanout, n_vertices: int):
    f = _np(fanout, np.int32)
    a, b, c = C.c_int64(), C.c_int64(), C.c_int64()
    _check(lib().moment_sample_bounds(n_seeds, f.ctypes.data, len(f), n_vertices, C.byref(a), C.byref(b), C.byref(c)))
    return a.value, b.value, c.value


@dataclass
class SampleBuffers:
    nodes: object
    offsets: object
    src: object
    counts: object
    fanout: tuple

    @staticmethod
    def allocate(n_seeds: int, fanout, n_vertices: int, device):
        import torch

        mn, mo, me = sample_bounds(n_seeds, fanout, n_vertices)
        H = len(fanout)
        return SampleBuffers(torch.empty(max(mn, 1), dtype=torch.int64, device=device),
                             torch.empty(max(mo, 1), dtype=torch.int64, device=device),
                             torch.empty(max(me, 1), dtype=torch.int32, device=device),
                             torch.zeros(2 * H + 1, dtype=torch.int64, device=device), tuple(fanout))

    def struct(self) -> SampleOut:
        return SampleOut(self.nodes.data_ptr(), self.offsets.data_ptr(), self.src.data_ptr(), self.counts.data_ptr(),
                         self.nodes.numel(), self.offsets.numel(), self.src.numel())

    def result(self):
        """Host copy split per hop, in the oracle's layout (synchronises)."""
        H = len(self.fanout)
        counts = self.counts.cpu().numpy()
        F, E = counts[: H + 1], counts[H + 1:]
        nodes = self.nodes[: F[H]].cpu().numpy()
        offs_all = self.offsets.cpu().numpy()
        src_all = self.src.cpu().numpy()
        offs, srcs, ob, eb = [], [], 0, 0
        for h in range(H):
            offs.append(offs_all[ob: ob + F[h] + 1])
            srcs.append(src_all[eb: eb + E[h]])
            ob += F[h] + 1
            eb += E[h]
        return {"nodes": nodes, "offsets": offs, "src": srcs, "counts": counts}


class StepBatch:
    """moment_step_batch over a fixed set of ctxs (one per batch in flight) with their sample buffers, row
    buffers and streams, prepared once: run(seeds, rng_seeds[, counts_host]) issues len(seeds) <= len(ctxs)
    steps on the first ctxs in one ctypes call (host=True: moment_step_host, seeds in pinned host memory)."""

    def __init__(self, ctxs, indptr, indices, fanout, outs, rows, streams, *, flags: int = 0, host: bool = False):
        n = len(ctxs)
        if not (n == len(outs) == len(rows) == len(streams)) or n == 0:
            raise ValueError("StepBatch: one out, rows buffer and stream per ctx")
        f = _np(fanout, np.int32)
        self._csr = Csr(indptr.data_ptr(), indices.data_ptr(), indptr.numel() - 1, indices.numel())
        self._params = SampleParams(len(f), f.ctypes.data, 0, flags)
        self._ctxs = (P * n)(*[c.handle.value for c in ctxs])
        self._outs = (SampleOut * n)(*[o.struct() for o in outs])
        self._rows = (P * n)(*[_ptr(r) for r in rows])
        self._streams = (P * n)(*[_stream(s) for s in streams])
        self._seeds, self._rng, self._counts = (P * n)(), (U64 * n)(), (P * n)()
        self._refs = (C.byref(self._csr), C.byref(self._params))
        self._host, self._n = host, n
        self._keep = (list(ctxs), list(outs), list(rows), list(streams), f, indptr, indices)
        self._fn = lib().moment_step_batch

    def run(self, seeds, rng_seeds, counts_host=None):
        k = len(seeds)
        if k > self._n or len(rng_seeds) != k or (self._host != (counts_host is not None)):
            raise ValueError("StepBatch.run: at most one batch per ctx, one rng seed per batch, counts iff host")
        sp, rs = self._seeds, self._rng
        n_seeds = seeds[0].numel()
        for i in range(k):
            if seeds[i].numel() != n_seeds:
                raise ValueError("StepBatch.run: batches of different sizes")
            sp[i] = seeds[i].data_ptr()
            rs[i] = rng_seeds[i] & 0xFFFFFFFFFFFFFFFF
        ch = None
        if counts_host is not None:
            ch = self._counts
            for i in range(k):
                ch[i] = counts_host[i].data_ptr()
        st = self._fn(k, self._ctxs, self._refs[0], sp, n_seeds, self._refs[1], rs, self._outs, self._rows, ch,
                      self._streams)
        if st:
            _check(st)


class Ctx:
    """Device context of one rank (moment_ctx_create)."""

    def __init__(self, *, n_vertices: int, max_seeds: int, max_fanout, rank: int = 0, world: int = 1, device: int = 0,
                 row_bytes: int = 0, row_stride: int | None = None, bin_owner=(), bin_ptr=(), placement=None,
                 quota=None):
        mf = _np(max_fanout, np.int32)
        owners = _np(bin_owner, np.int32) if len(bin_owner) else np.zeros(1, np.int32)
        ptrs = (C.c_void_p * max(1, len(bin_ptr)))(*[C.c_void_p(int(p)) for p in bin_ptr])
        q = _np(quota, np.int64) if quota is not None else None
        self._keep = (mf, owners, ptrs, q, placement)
        args = CtxArgs(rank, world, device, n_vertices, max_seeds, len(mf), mf.ctypes.data, row_bytes,
                       row_stride if row_stride is not None else row_bytes, len(bin_ptr), owners.ctypes.data,
                       C.cast(ptrs, P), _ptr(placement), q.ctypes.data if q is not None else None)
        h = C.c_void_p()
        _check(lib().moment_ctx_create(C.byref(args), C.byref(h)))
        self.handle = h
        self.rank, self.world, self.device, self.row_bytes = rank, world, device, row_bytes
        self.n_vertices = n_vertices

    def close(self):
        if getattr(self, "handle", None) and _lib is not None:
            _lib.moment_ctx_free(self.handle)
            self.handle = None

    def __del__(self):
        self.close()

    def workspace_bytes(self) -> int:
        b = C.c_int64()
        _check(lib().moment_ctx_workspace_bytes(self.handle, C.byref(b)))
        return b.value

    def sample(self, indptr, indices, seeds, fanout, rng_seed: int, out: SampleBuffers, *, flags: int = 0,
               stream=None):
        csr = Csr(indptr.data_ptr(), indices.data_ptr(), indptr.numel() - 1, indices.numel())
        f = _np(fanout, np.int32)
        params = SampleParams(len(f), f.ctypes.data, rng_seed & 0xFFFFFFFFFFFFFFFF, flags)
        so = out.struct()
        _check(lib().moment_sample(self.handle, C.byref(csr), seeds.data_ptr(), seeds.numel(), C.byref(params),
                                   C.byref(so), _stream(stream)))
        return out

    def sample_check(self, stream=None):
        _check(lib().moment_sample_check(self.handle, _stream(stream)))

    def gather(self, ids, out, *, n_dev=None, max_n: int | None = None, stream=None):
        mn = ids.numel() if max_n is None else max_n
        _check(lib().moment_gather(self.handle, ids.data_ptr(), _ptr(n_dev), mn, out.data_ptr(), _stream(stream)))
        return out

    def bucket(self, ids, route, qoff, qpos, *, n_dev=None, max_n: int | None = None, stream=None):
        mn = ids.numel() if max_n is None else max_n
        _check(lib().moment_bucket(self.handle, ids.data_ptr(), _ptr(n_dev), mn, route.data_ptr(), qoff.data_ptr(),
                                   qpos.data_ptr(), _stream(stream)))

    def hotness(self, ids, hot, *, n_dev=None, max_n: int | None = None, stream=None):
        mn = ids.numel() if max_n is None else max_n
        _check(lib().moment_hotness(self.handle, ids.data_ptr(), _ptr(n_dev), mn, hot.data_ptr(), _stream(stream)))

    def _args(self, indptr, indices, fanout, flags, out):
        """ctypes argument structs for one (graph, fanout, flags, buffers) shape, built once and reused."""
        key = (indptr.data_ptr(), indptr.numel(), indices.data_ptr(), tuple(int(x) for x in fanout), flags, id(out),
               out.nodes.data_ptr())
        cache = self.__dict__.setdefault("_arg_cache", {})
        hit = cache.get(key)
        if hit is None:
            f = _np(fanout, np.int32)
            csr = Csr(indptr.data_ptr(), indices.data_ptr(), indptr.numel() - 1, indices.numel())
            params = SampleParams(len(f), f.ctypes.data, 0, flags)
            so = out.struct()
            hit = (csr, params, so, f, C.byref(csr), C.byref(params), C.byref(so))
            cache[key] = hit
        return hit

    def step(self, indptr, indices, seeds, fanout, rng_seed: int, out: SampleBuffers, rows, *, flags: int = 0,
             stream=None):
        """moment_step: sample + gather of one batch, replayed from the ctx's cached CUDA graph."""
        a = self._args(indptr, indices, fanout, flags, out)
        a[1].rng_seed = rng_seed & 0xFFFFFFFFFFFFFFFF
        _check(lib().moment_step(self.handle, a[4], seeds.data_ptr(), seeds.numel(), a[5], a[6], _ptr(rows),
                                 _stream(stream)))
        return out

    def bind_step(self, indptr, indices, fanout, out: SampleBuffers, rows, *, flags: int = 0, stream=None,
                  host: bool = False):
        """moment_step (host=False: run(seeds, rng_seed)) or moment_step_host (host=True: run(seeds_host,
        rng_seed, counts_host)) prepared for one (graph, fanout, buffers, rows, stream): the returned callable
        marshals only the per-batch pointers and the rng seed (the argument structs are built once), so issuing
        a step costs one ctypes call."""
        a = self._args(indptr, indices, fanout, flags, out)
        params, csr_r, par_r, so_r = a[1], a[4], a[5], a[6]
        h, rows_p, sp = self.handle, _ptr(rows), _stream(stream)
        if host:
            fn = lib().moment_step_host

            def run(seeds_host, rng_seed: int, counts_host):
                params.rng_seed = rng_seed & 0xFFFFFFFFFFFFFFFF
                st = fn(h, csr_r, seeds_host.data_ptr(), seeds_host.numel(), par_r, so_r, rows_p,
                        counts_host.data_ptr(), sp)
                if st:
                    _check(st)
        else:
            fn = lib().moment_step

            def run(seeds, rng_seed: int):
                params.rng_seed = rng_seed & 0xFFFFFFFFFFFFFFFF
                st = fn(h, csr_r, seeds.data_ptr(), seeds.numel(), par_r, so_r, rows_p, sp)
                if st:
                    _check(st)

        run.keep = (self, a, out, rows)  # the prepared structs, buffers and ctx live as long as the callable
        return run

    def step_host(self, indptr, indices, seeds_host, fanout, rng_seed: int, out: SampleBuffers, rows, counts_host,
                  *, flags: int = 0, stream=None):
        """moment_step_host: host seeds in, host counts out, all asynchronous on `stream`."""
        a = self._args(indptr, indices, fanout, flags, out)
        a[1].rng_seed = rng_seed & 0xFFFFFFFFFFFFFFFF
        _check(lib().moment_step_host(self.handle, a[4], seeds_host.data_ptr(), seeds_host.numel(), a[5], a[6],
                                      _ptr(rows), counts_host.data_ptr(), _stream(stream)))


    # ---- H5 exchange for one process per GPU (see exchange.py for the orchestration) ----
    def gather_routed(self, ids, route, out, *, n_dev=None, max_n: int | None = None, stream=None):
        mn = ids.numel() if max_n is None else max_n
        _check(lib().moment_gather_routed(self.handle, ids.data_ptr(), _ptr(n_dev), mn, route.data_ptr(),
                                          out.data_ptr(), _stream(stream)))

    def relay_pack(self, ids, qoff, qpos, words, send_counts, *, max_n: int | None = None, stream=None):
        mn = ids.numel() if max_n is None else max_n
        _check(lib().moment_relay_pack(self.handle, ids.data_ptr(), mn, qoff.data_ptr(), qpos.data_ptr(),
                                       words.data_ptr(), send_counts.data_ptr(), _stream(stream)))

    def relay_serve(self, words, rows, *, n: int, stream=None):
        _check(lib().moment_relay_serve(self.handle, words.data_ptr(), None, n, rows.data_ptr(), _stream(stream)))

    def relay_scatter(self, words, rows, out, *, n: int, stream=None):
        _check(lib().moment_relay_scatter(self.handle, words.data_ptr(), None, n, rows.data_ptr(), out.data_ptr(),
                                          _stream(stream)))

    # ---- one-call collective exchange (moment_ctx_set_exchange; exchange.PeerExchange sets it up) ----
    def set_exchange(self, *, cap: int, inbox, inbox_count, flags, out, peer_inbox: list[int], peer_count: list[int],
                     peer_out: list[int], peer_flag: list[int], timeout_ns: int = 10**10):
        """Register this rank's inbox / counts / flags / output and the peers' mapped addresses: moment_gather
        and moment_step then run the relay exchange as one enqueue (collective over the ctx's world)."""
        a = ExchangeArgs()
        a.cap, a.inbox, a.inbox_count, a.flags, a.out = cap, inbox.data_ptr(), inbox_count.data_ptr(), \
            flags.data_ptr(), out.data_ptr()
        for h in range(self.world):
            a.peer_inbox[h] = peer_inbox[h] or None
            a.peer_count[h] = peer_count[h] or None
            a.peer_out[h] = peer_out[h] or None
            a.peer_flag[h] = peer_flag[h] or None
        a.timeout_ns = timeout_ns
        _check(lib().moment_ctx_set_exchange(self.handle, C.byref(a)))
        self._keep_ex = (inbox, inbox_count, flags, out)

    def exchange_status(self, stream=None):
        """Raise MomentError(ETIMEDOUT) if a device barrier of this ctx expired (synchronises the stream)."""
        _check(lib().moment_exchange_status(self.handle, _stream(stream)))

    # ---- the same exchange over peer memory, phase by phase (see exchange.PeerExchange) ----
    def relay_push(self, ids, qoff, qpos, peer_inbox: list[int], peer_count: list[int], *, max_n: int | None = None,
                   stream=None):
        """peer_inbox[h] / peer_count[h]: device addresses of rank h's inbox / count slot for this rank."""
        mn = ids.numel() if max_n is None else max_n
        inb = (C.c_void_p * len(peer_inbox))(*[p or None for p in peer_inbox])
        cnt = (C.c_void_p * len(peer_count))(*[p or None for p in peer_count])
        _check(lib().moment_relay_push(self.handle, ids.data_ptr(), mn, qoff.data_ptr(), qpos.data_ptr(),
                                       C.cast(inb, P), C.cast(cnt, P), _stream(stream)))

    def relay_serve_push(self, inbox, inbox_count, cap: int, peer_out: list[int], *, stream=None):
        """Serve every source's inbox into its output (peer_out[g]: device address of rank g's output)."""
        outs = (C.c_void_p * len(peer_out))(*[p or None for p in peer_out])
        _check(lib().moment_relay_serve_push(self.handle, inbox.data_ptr(), inbox_count.data_ptr(), cap,
                                             C.cast(outs, P), _stream(stream)))


def signal_barrier(world: int, rank: int, peer_flags: list[int], flags, epoch: int, *, timeout_ns: int = 10**10,
                   status=None, stream=None):
    """Device-side barrier over peer-mapped flag words (moment_signal_barrier); enqueued, no host sync."""
    arr = (C.c_void_p * world)(*[p or None for p in peer_flags])
    _check(lib().moment_signal_barrier(world, rank, arr, _ptr(flags), epoch, timeout_ns, _ptr(status),
                                       _stream(stream)))


IPC_HANDLE_BYTES = 64


def ipc_export(tensor) -> tuple[bytes, int]:
    """(64-byte CUDA IPC handle of the allocation holding `tensor`, byte offset of the tensor in it)."""
    h = (C.c_uint8 * IPC_HANDLE_BYTES)()
    off = C.c_int64()
    _check(lib().moment_ipc_export(tensor.data_ptr(), C.cast(h, P), C.byref(off)))
    return bytes(h), off.value


def ipc_import(handle: bytes) -> int:
    """Map another process's device allocation into this one; returns its base address (add the offset)."""
    h = (C.c_uint8 * IPC_HANDLE_BYTES).from_buffer_copy(handle)
    ptr = C.c_void_p()
    _check(lib().moment_ipc_import(C.cast(h, P), C.byref(ptr)))
    return ptr.value


def ipc_close(ptr: int):
    _check(lib().moment_ipc_close(ptr))


def gather_group(ctxs, ids, out, *, n_dev=None, max_n: int, stream=None):
    """moment_gather_group: logical ranks driven from one stream (all pointers addressable)."""
    k = len(ctxs)
    hs = (C.c_void_p * k)(*[c.handle for c in ctxs])
    ip = (C.c_void_p * k)(*[t.data_ptr() for t in ids])
    op = (C.c_void_p * k)(*[t.data_ptr() for t in out])
    nd = (C.c_void_p * k)(*[t.data_ptr() for t in n_dev]) if n_dev is not None else None
    _check(lib().moment_gather_group(C.cast(hs, P), k, C.cast(ip, P), C.cast(nd, P) if nd is not None else None,
                                     max_n, C.cast(op, P), _stream(stream)))


# ---------------------------------------------------------------------------------------------- consumer
def _dtype_code(t) -> int:
    import torch

    if t.dtype == torch.float32:
        return DTYPE_F32
    if t.dtype == torch.bfloat16:
        return DTYPE_BF16
    raise MomentError(EINVAL, f"unsupported dtype {t.dtype}")


def sage_mean(x, offsets, src, n_dst: int, out, *, stream=None):
    """out[i] = mean of x[src[e]] over the block's edges of row i (moment_sage_mean). x, out: 2-D tensors of the
    same dtype (fp32 / bf16) with unit column stride."""
    if x.stride(1) != 1 or out.stride(1) != 1 or out.dtype != x.dtype:
        raise MomentError(EINVAL, "sage_mean: x and out need unit column stride and one dtype")
    _check(lib().moment_sage_mean(x.data_ptr(), x.stride(0), _dtype_code(x), x.shape[1], offsets.data_ptr(),
                                  src.data_ptr(), n_dst, out.data_ptr(), out.stride(0), _stream(stream)))
    return out


def sage_mean_backward(grad_out, offsets, src, n_dst: int, grad_x, *, stream=None):
    """grad_x[src[e]] += grad_out[i] / deg_i (fp32 grad_x, caller-zeroed)."""
    if grad_out.stride(1) != 1 or grad_x.stride(1) != 1:
        raise MomentError(EINVAL, "sage_mean_backward: unit column stride needed")
    _check(lib().moment_sage_mean_backward(grad_out.data_ptr(), grad_out.stride(0), _dtype_code(grad_out),
                                           grad_out.shape[1], offsets.data_ptr(), src.data_ptr(), n_dst,
                                           grad_x.data_ptr(), grad_x.stride(0), _stream(stream)))
    return grad_x
