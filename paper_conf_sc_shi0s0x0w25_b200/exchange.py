"""H5 exchange for one process per GPU: the per-batch relay of host rows through peer ranks.

Orchestration only (torch.distributed is the transport, every byte is computed by libmoment.so kernels):

  moment_bucket          routes (local / peer HBM / host direct / host via relay rank h), stable queues
  moment_gather_routed   every row this rank reads itself (overlaps the exchange below)
  moment_relay_pack      (placement word, output position) of each request routed through another rank
  all-to-all             counts, then request words (2 x int64 per request)
  moment_relay_serve     the relay rank reads the requested host rows over ITS PCIe link
  all-to-all             rows back to the requesters (same splits, in rows)
  moment_relay_scatter   rows into the requester's output positions

With NCCL the collectives run on the GPU stream; with gloo (CPU tests, or several processes sharing one
GPU) they are staged through host memory. `alltoallv` is the transport helper both use.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import torch
import torch.distributed as dist


def _is_gloo(group) -> bool:
    return dist.get_backend(group) == "gloo"


def alltoallv(send: torch.Tensor, send_splits: list[int], recv_splits: list[int], group=None) -> torch.Tensor:
    """Variable-size all-to-all of the leading dimension. Returns a tensor of sum(recv_splits) rows on
    send's device (staged through host memory for gloo)."""
    out_shape = (sum(recv_splits),) + tuple(send.shape[1:])
    if _is_gloo(group) and send.is_cuda:
        recv = torch.empty(out_shape, dtype=send.dtype)
        dist.all_to_all_single(recv, send.cpu().contiguous(), recv_splits, send_splits, group=group)
        return recv.to(send.device, non_blocking=False)
    recv = torch.empty(out_shape, dtype=send.dtype, device=send.device)
    dist.all_to_all_single(recv, send.contiguous(), recv_splits, send_splits, group=group)
    return recv


def exchange_counts(send_counts: torch.Tensor, group=None) -> list[int]:
    """Each rank's number of requests for every other rank -> how many this rank will serve from each."""
    world = dist.get_world_size(group)
    send = send_counts.to(torch.int64).reshape(world)
    recv = alltoallv(send.reshape(world, 1), [1] * world, [1] * world, group)
    return [int(x) for x in recv.reshape(world).cpu()]


@dataclass
class ExchangeBuffers:
    """Device buffers of one rank's exchange, sized once for max_n requests (receive buffers grow)."""

    max_n: int
    row_bytes: int
    n_queues: int
    device: torch.device
    route: torch.Tensor = field(init=False)
    qoff: torch.Tensor = field(init=False)
    qpos: torch.Tensor = field(init=False)
    words: torch.Tensor = field(init=False)
    send_counts: torch.Tensor = field(init=False)

    def __post_init__(self):
        d = self.device
        self.route = torch.empty(max(self.max_n, 1), dtype=torch.int32, device=d)
        self.qoff = torch.empty(self.n_queues + 1, dtype=torch.int64, device=d)
        self.qpos = torch.empty(max(self.max_n, 1), dtype=torch.int64, device=d)
        self.words = torch.empty(2 * max(self.max_n, 1), dtype=torch.int64, device=d)
        self.send_counts = torch.zeros(64, dtype=torch.int64, device=d)


def gather_exchange(ctx, ids: torch.Tensor, out: torch.Tensor, bufs: ExchangeBuffers, *, n: int, group=None,
                    stream=None) -> dict:
    """Collective: out[:n] = rows of ids[:n] for every rank of `group` (ctx.rank == group rank).
    Returns the per-batch traffic (requests sent to / served for each rank)."""
    world = ctx.world
    s = stream if stream is not None else torch.cuda.current_stream(ids.device)
    with torch.cuda.stream(s):
        ctx.bucket(ids, bufs.route, bufs.qoff, bufs.qpos, max_n=n, stream=s)
        ctx.gather_routed(ids, bufs.route, out, max_n=n, stream=s)
        ctx.relay_pack(ids, bufs.qoff, bufs.qpos, bufs.words, bufs.send_counts, max_n=n, stream=s)
        send = [int(x) for x in bufs.send_counts[:world].cpu()]  # synchronises the stream
        recv = exchange_counts(torch.tensor(send, dtype=torch.int64), group)
        n_send, n_recv = sum(send), sum(recv)
        words_in = alltoallv(bufs.words[: 2 * n_send].view(n_send, 2), send, recv, group).reshape(-1)
        rows_srv = torch.empty((max(n_recv, 1), ctx.row_bytes), dtype=torch.uint8, device=ids.device)
        if n_recv:
            ctx.relay_serve(words_in, rows_srv, n=n_recv, stream=s)
        rows_back = alltoallv(rows_srv[:n_recv], recv, send, group)
        if n_send:
            ctx.relay_scatter(bufs.words, rows_back, out, n=n_send, stream=s)
    return {"sent": send, "served": recv}


class PeerExchange:
    """H5 over peer memory (one process per GPU, no all-to-all): requests are stored straight into the
    relay rank's inbox and served rows straight into the requester's output, both by libmoment.so kernels
    through CUDA-IPC-mapped peer pointers (NVLink loads/stores between the GPUs of one node).

    Setup is collective over `group`: this rank allocates its inbox (int64 [world][cap][2]), inbox counts
    (int64 [world]), barrier flags and batch output (uint8 [cap][R]), exports them, and maps every peer's.

    one_call=True (default): the pointers are registered with the ctx (moment_ctx_set_exchange), and a batch
    is ONE library call: `gather` = moment_gather, `step` = moment_step (sample + the whole exchange,
    replayed from the ctx's CUDA graph), with device-side signal barriers between the phases and no host
    synchronisation. This class is then setup only.
    one_call=False: the phases are sequenced from here (bucket -> routed gather -> relay_push -> barrier ->
    relay_serve_push -> barrier); device_barrier=False: each barrier is a stream synchronize + process barrier
    (NCCL: device collective, gloo: host); device_barrier=True: `moment_signal_barrier` on the stream.
    `check()` reports a watchdog timeout of a device barrier.
    """

    def __init__(self, ctx, max_n: int, row_bytes: int, device, group=None, device_barrier: bool = False,
                 timeout_s: float = 10.0, one_call: bool = True):
        import paper_conf_sc_shi0s0x0w25_b200 as M

        self.M, self.ctx, self.group = M, ctx, group
        self.world, self.rank = ctx.world, ctx.rank
        self.cap = max(1, int(max_n))
        dev = torch.device(device)
        self.inbox = torch.zeros((self.world, self.cap, 2), dtype=torch.int64, device=dev)
        self.count = torch.zeros(self.world, dtype=torch.int64, device=dev)
        self.out = torch.zeros((self.cap, row_bytes), dtype=torch.uint8, device=dev)
        self.route = torch.empty(self.cap, dtype=torch.int32, device=dev)
        self.qoff = torch.empty(64 * self.world + 1, dtype=torch.int64, device=dev)
        self.qpos = torch.empty(self.cap, dtype=torch.int64, device=dev)
        self.device_barrier, self.timeout_ns, self.epoch = device_barrier, int(timeout_s * 1e9), 0
        self.flags = torch.zeros(self.world, dtype=torch.int64, device=dev)  # uint64 flag words
        self.status = torch.zeros(1, dtype=torch.int32, device=dev)
        mine = [M.ipc_export(t) for t in (self.inbox, self.count, self.out, self.flags)]
        everyone = [None] * self.world
        dist.all_gather_object(everyone, mine, group=group)
        self._bases = []
        self.peer_inbox = [0] * self.world
        self.peer_count = [0] * self.world
        self.peer_out = [0] * self.world
        self.peer_flag = [0] * self.world
        slot_bytes = self.cap * 2 * 8
        for h in range(self.world):
            if h == self.rank:
                continue
            addr = []
            for handle, off in everyone[h]:
                base = M.ipc_import(handle)
                self._bases.append(base)
                addr.append(base + off)
            self.peer_inbox[h] = addr[0] + self.rank * slot_bytes  # rank h's inbox slot for this rank
            self.peer_count[h] = addr[1] + self.rank * 8
            self.peer_out[h] = addr[2]
            self.peer_flag[h] = addr[3] + self.rank * 8  # rank h's flag word for this rank
        self.one_call = one_call
        if one_call:
            ctx.set_exchange(cap=self.cap, inbox=self.inbox, inbox_count=self.count, flags=self.flags, out=self.out,
                             peer_inbox=self.peer_inbox, peer_count=self.peer_count, peer_out=self.peer_out,
                             peer_flag=self.peer_flag, timeout_ns=self.timeout_ns)
        dist.barrier(group=group)

    def _barrier(self, s):
        self.epoch += 1
        self.M.signal_barrier(self.world, self.rank, self.peer_flag, self.flags, self.epoch,
                              timeout_ns=self.timeout_ns, status=self.status, stream=s)

    def check(self):
        """Raise if a device barrier timed out (synchronises)."""
        if self.one_call:
            self.ctx.exchange_status()
            return
        st = int(self.status.item())
        if st != 0:
            raise self.M.MomentError(st, "PeerExchange: device barrier watchdog expired")

    def gather(self, ids: torch.Tensor, n: int, stream=None) -> torch.Tensor:
        """Collective: returns this rank's output view [n, R] = rows of ids[:n]."""
        assert n <= self.cap
        s = stream if stream is not None else torch.cuda.current_stream(ids.device)
        ctx = self.ctx
        if self.one_call:
            ctx.gather(ids, self.out, max_n=n, stream=s)
            return self.out[:n]
        with torch.cuda.stream(s):
            ctx.bucket(ids, self.route, self.qoff, self.qpos, max_n=n, stream=s)
            ctx.gather_routed(ids, self.route, self.out, max_n=n, stream=s)
            ctx.relay_push(ids, self.qoff, self.qpos, self.peer_inbox, self.peer_count, max_n=n, stream=s)
            if self.device_barrier:
                self._barrier(s)  # every rank's requests are in its relays' inboxes
                ctx.relay_serve_push(self.inbox, self.count, self.cap, self.peer_out, stream=s)
                self._barrier(s)  # every relayed row is in its requester's output
        if self.device_barrier:
            return self.out[:n]
        s.synchronize()
        dist.barrier(group=self.group)  # every rank's requests are in its relays' inboxes
        with torch.cuda.stream(s):
            ctx.relay_serve_push(self.inbox, self.count, self.cap, self.peer_out, stream=s)
        s.synchronize()
        dist.barrier(group=self.group)  # every relayed row is in its requester's output
        return self.out[:n]

    def step(self, indptr, indices, seeds, fanout, rng_seed: int, bufs, stream=None):
        """Collective (one_call only): sample `seeds` and gather F_H with the relay exchange, all in ONE
        moment_step call replayed from the ctx's CUDA graph; the rows land in self.out[:|F_H|]."""
        assert self.one_call
        self.ctx.step(indptr, indices, seeds, fanout, rng_seed, bufs, self.out, stream=stream)
        return self.out

    def close(self):
        """Collective: unmap the peers' buffers once every rank is done with them."""
        torch.cuda.synchronize(self.out.device)
        dist.barrier(group=self.group)
        for b in self._bases:
            self.M.ipc_close(b)
        self._bases = []
