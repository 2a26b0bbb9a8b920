"""P1 topology graph of an 8-GPU B200 box (HGX B200 class) for the planner.

The paper builds its capacity graph from the machine's physical topology: storage nodes (GPU HBM, host DRAM
per NUMA node, SSDs), interconnect nodes (CPU root complexes, PCIe switches) and computation nodes, each link
carrying its profiled throughput upper limit. This module writes that graph for a two-socket box
with k_total GPUs: host DRAM bin per socket -> socket root complex -> (optional PCIe switch shared by
`gpus_per_switch` GPUs) -> GPU port; an HBM bin per GPU; the sockets joined by UPI in both directions.
NVLink / NVSwitch is not a graph link: the plan treats it as the forwarding fabric and checks it in closed
form (R11, `nvlink_cap` of moment_plan).

Capacities are bytes/us (= MB/s). Defaults: `port_gbs` and `hbm_gbs` are measured on this pool's B200
(pinned H2D copy 55.6 GB/s, device copy `MEASURED_PEAKS.json`); `dram_gbs`, `upi_gbs` and the switch layout
are ASSUMPTIONS for a DGX/HGX B200 host (two Xeon sockets, 4 GPUs per socket) that the 1-GPU boxes of this
pool cannot measure — callers pass their own probe values.
"""
from dataclasses import dataclass, field

from . import moment as M


@dataclass
class Box:
    nodes: list
    links: list
    host_bin: list = field(default_factory=list)   # node of the host DRAM bin of socket j
    hbm_bin: list = field(default_factory=list)    # node of GPU g's HBM bin
    gpu: list = field(default_factory=list)        # computation node of GPU g
    socket_of_gpu: list = field(default_factory=list)
    rc: list = field(default_factory=list)         # interconnect node of socket j's root complex
    upi_links: list = field(default_factory=list)  # indices (in `links`) of the socket-to-socket links

    def upi_bytes(self, link_flow) -> int:
        """Bytes a plan's flow moves across sockets (the paper's QPI traffic): the flow on the
        UPI links (link indices are those of `links`, which the topology export keeps)."""
        return int(sum(int(link_flow[i]) for i in self.upi_links))

    def topology(self) -> M.Topology:
        return M.topology(self.nodes, self.links)


def hgx_b200(k_total: int = 8, *, port_gbs: float = 55.6, hbm_gbs: float = 6543.4, dram_gbs: float = 250.0,
             upi_gbs: float = 62.0, gpus_per_switch: int = 1, uplink_gbs: float | None = None,
             sockets: int = 2, active=None) -> Box:
    """Two-socket box, GPUs split evenly over the sockets. gpus_per_switch = 1: every GPU port hangs off its
    socket's root complex; > 1: that many GPUs share a PCIe switch whose uplink (default: one port) is the
    contended link the paper's PLX discussion is about. active: the GPUs in use (default all);
    the others are left out of the graph (no HBM bin, port or computation node; their entries are None), so
    the rate max-flow that sets Bin_traffic only counts the GPUs that read."""
    if k_total % sockets or (k_total // sockets) % gpus_per_switch:
        raise ValueError("GPUs must split evenly over sockets and switches")
    cap = lambda gbs: int(round(gbs * 1000))  # noqa: E731  GB/s -> bytes/us
    uplink_gbs = port_gbs if uplink_gbs is None else uplink_gbs
    nodes, links = [], []
    b = Box(nodes, links)
    for j in range(sockets):
        b.host_bin.append(len(nodes))
        nodes.append((M.NODE_STORAGE, M.TIER_HOST_DRAM, j))
    rc = []
    for j in range(sockets):
        rc.append(len(nodes))
        nodes.append((M.NODE_INTERCONNECT, M.TIER_NONE, -1))
    act = set(range(k_total) if active is None else active)
    for g in range(k_total):
        b.hbm_bin.append(len(nodes) if g in act else None)
        if g in act:
            nodes.append((M.NODE_STORAGE, M.TIER_GPU_HBM, g))
    for g in range(k_total):
        b.gpu.append(len(nodes) if g in act else None)
        if g in act:
            nodes.append((M.NODE_COMPUTE, M.TIER_NONE, g))
    for j in range(sockets):
        links.append((b.host_bin[j], rc[j], cap(dram_gbs)))
    b.rc = rc
    for j in range(sockets):
        for i in range(sockets):
            if i != j:
                b.upi_links.append(len(links))
                links.append((rc[j], rc[i], cap(upi_gbs)))
    per_socket = k_total // sockets
    for g in range(k_total):
        j = g // per_socket
        b.socket_of_gpu.append(j)
        if gpus_per_switch == 1:
            if g in act:
                links.append((rc[j], b.gpu[g], cap(port_gbs)))
        elif g % gpus_per_switch == 0 and any(g + q in act for q in range(gpus_per_switch)):
            sw = len(nodes)
            nodes.append((M.NODE_INTERCONNECT, M.TIER_NONE, -1))
            links.append((rc[j], sw, cap(uplink_gbs)))
            for q in range(gpus_per_switch):
                if g + q in act:
                    links.append((sw, b.gpu[g + q], cap(port_gbs)))
        if g in act:
            links.append((b.hbm_bin[g], b.gpu[g], cap(hbm_gbs)))
    return b


def spread_gpus(k: int, k_total: int = 8, sockets: int = 2, gpus_per_switch: int = 1) -> list:
    """A balanced choice of k active GPUs: round-robin over sockets, then over switches within a socket."""
    per_socket = k_total // sockets
    n_sw = per_socket // gpus_per_switch
    order = []
    for q in range(gpus_per_switch):
        for s in range(n_sw):
            for j in range(sockets):
                order.append(j * per_socket + s * gpus_per_switch + q)
    return sorted(order[:k])


def gpu_subset_classes(k: int, k_total: int = 8, sockets: int = 2, gpus_per_switch: int = 1) -> list:
    """Candidate sets of k active GPUs up to the box's symmetry (the paper prunes isomorphic hardware
    placements before evaluating them). The symmetries of the two-socket box permute sockets,
    the switches of a socket and the GPUs of a switch, so a subset's class is the multiset over sockets of the
    multiset over switches of how many of its GPUs are active. Returns one representative per class
    (the lexicographically smallest subset), sorted."""
    from itertools import combinations
    per_socket = k_total // sockets
    n_sw = per_socket // gpus_per_switch
    reps = {}
    for sub in combinations(range(k_total), k):
        cnt = [[0] * n_sw for _ in range(sockets)]
        for g in sub:
            cnt[g // per_socket][(g % per_socket) // gpus_per_switch] += 1
        sig = tuple(sorted(tuple(sorted(c, reverse=True)) for c in cnt))
        if sig not in reps:
            reps[sig] = list(sub)
    return sorted(reps.values())


# Capacities of hgx_b200 that this pool's boxes cannot measure (one GPU, one socket): assumptions for a
# two-socket HGX B200 host.
ASSUMED = {"dram_gbs": 250.0, "upi_gbs": 62.0}


def from_probe(probe: dict) -> tuple[dict, dict]:
    """hgx_b200 keyword arguments from a tools/probe_box.py JSON (capacities are profiled limits),
    and the provenance of each: {"port_gbs": "measured", "upi_gbs": "assumed", ...}.
    port = the slowest GPU's local-NUMA pinned H2D copy (or, when every GPU copied at once, the slowest
    concurrent rate); hbm = the device copy (read + write); nvlink = the peer copy when the box has 2+ GPUs
    (else the B200_PROFILING.md figure, 770 GB/s); UPI = the remote-NUMA H2D rate when the box has 2+ NUMA
    nodes (a lower bound on what one GPU can pull across sockets), else assumed; socket DRAM assumed."""
    kw, src = {}, {}
    conc = probe.get("port_concurrent_gbs")
    kw["port_gbs"] = float(min(conc)) if conc else float(probe["port_gbs"])
    src["port_gbs"] = "measured (concurrent)" if conc else "measured (one GPU at a time)"
    kw["hbm_gbs"] = float(probe["hbm_gbs"])
    src["hbm_gbs"] = "measured"
    if probe.get("port_remote_gbs"):
        kw["upi_gbs"] = float(probe["port_remote_gbs"])
        src["upi_gbs"] = "measured (remote-NUMA H2D, lower bound)"
    else:
        kw["upi_gbs"] = ASSUMED["upi_gbs"]
        src["upi_gbs"] = "assumed"
    kw["dram_gbs"] = ASSUMED["dram_gbs"]
    src["dram_gbs"] = "assumed"
    nv = probe.get("nvlink_gbs")
    src["nvlink_gbs"] = "measured (peer copy)" if nv else "B200_PROFILING.md peer copy (770 GB/s)"
    return kw, dict(src, nvlink_value=float(nv) if nv else 770.0)
