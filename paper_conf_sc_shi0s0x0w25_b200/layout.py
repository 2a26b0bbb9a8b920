"""Plan reuse (the offline Max-Flow + DDAK step "runs once per model/hardware configuration and
is reused across runs"): a placement (bin_of, slot_of per vertex, from moment_place) and the plan that goes
with it (per-link flow, quota matrix, T*), saved to one .npz file and loaded back, bound to the topology graph
they were computed on.

The file stores the arrays as produced by the library and a JSON header: format version, vertex and bin
counts, the bins' storage nodes and capacities, the replica count, and a sha256 of the topology (nodes and
links as exported by moment_topology_export, so the s/t augmentation is included). `load` refuses a file whose
topology hash differs from the topology the caller passes (a layout planned for another box), or whose arrays
are inconsistent with the header. Argument marshalling and file I/O only: the placement and the plan are the
library's.
"""
from __future__ import annotations

import hashlib
import json

import numpy as np

from . import moment as M

FORMAT = 1


def topology_hash(topo: M.Topology) -> str:
    nodes, links, s, t = topo.export()
    h = hashlib.sha256()
    h.update(json.dumps({"nodes": [list(x) for x in nodes], "links": [[int(a), int(b), int(c)] for a, b, c in links],
                         "s": s, "t": t}, sort_keys=True).encode())
    return h.hexdigest()


def save(path: str, topo: M.Topology, *, bin_of, slot_of, bin_node, capacity_rows, replicate_rows: int = 0,
         plan: dict | None = None, note: str = "") -> None:
    """Write a layout (and optionally its plan: the dict of moment_plan_info) to `path` (.npz)."""
    bin_of = np.ascontiguousarray(bin_of, np.int32)
    slot_of = np.ascontiguousarray(slot_of, np.int64)
    if bin_of.shape != slot_of.shape:
        raise M.MomentError(M.EINVAL, "layout.save: bin_of and slot_of differ in length")
    hdr = {"format": FORMAT, "n_vertices": int(len(bin_of)), "n_bins": len(bin_node),
           "bin_node": [int(x) for x in bin_node], "capacity_rows": [int(x) for x in capacity_rows],
           "replicate_rows": int(replicate_rows), "topology_sha256": topology_hash(topo), "note": note,
           "plan": None}
    arrays = {"bin_of": bin_of, "slot_of": slot_of}
    if plan is not None:
        hdr["plan"] = {k: int(plan[k]) for k in ("t_star", "t_ingest", "t_nvlink", "t_hbm")}
        arrays["link_flow"] = np.ascontiguousarray(plan["link_flow"], np.int64)
        arrays["quota"] = np.ascontiguousarray(plan["quota"], np.int64)
    with open(path, "wb") as f:
        np.savez(f, header=np.frombuffer(json.dumps(hdr).encode(), np.uint8), **arrays)


def load(path: str, topo: M.Topology | None = None) -> dict:
    """Read a layout; with `topo`, check it was planned on that topology graph. Returns the header fields
    plus bin_of, slot_of (and link_flow, quota when a plan was saved)."""
    with np.load(path, allow_pickle=False) as z:
        hdr = json.loads(bytes(z["header"]).decode())
        if hdr.get("format") != FORMAT:
            raise M.MomentError(M.EINVAL, f"layout.load: format {hdr.get('format')} (expected {FORMAT})")
        out = dict(hdr)
        for k in z.files:
            if k != "header":
                out[k] = z[k]
    if topo is not None and topology_hash(topo) != hdr["topology_sha256"]:
        raise M.MomentError(M.EINVAL, "layout.load: the layout was planned on another topology graph")
    n, nb = hdr["n_vertices"], hdr["n_bins"]
    b, s = out["bin_of"], out["slot_of"]
    if len(b) != n or len(s) != n:
        raise M.MomentError(M.EINVAL, "layout.load: array lengths disagree with the header")
    part = b >= 0
    if n and ((b[part] >= nb).any() or ((b < 0) & (b != M.BIN_REPLICA)).any() or (s < 0).any()):
        raise M.MomentError(M.EINVAL, "layout.load: bin or slot out of range")
    counts = np.bincount(b[part], minlength=nb) if n else np.zeros(nb, np.int64)
    if (counts > np.asarray(hdr["capacity_rows"])).any() or int((b == M.BIN_REPLICA).sum()) != hdr["replicate_rows"]:
        raise M.MomentError(M.EINVAL, "layout.load: bin fill or replica count disagrees with the header")
    if hdr["plan"] is not None:
        out["plan"] = dict(hdr["plan"], link_flow=out.pop("link_flow"), quota=out.pop("quota"))
    return out
