"""Plan reuse: a DDAK placement and its plan saved and loaded back bit-identically, bound to
the topology graph they were planned on."""
import numpy as np
import pytest

import paper_conf_sc_shi0s0x0w25_b200 as M


def _layout(k=4, n=5000, r=0):
    box = M.boxes.hgx_b200(8, active=M.boxes.spread_gpus(k))
    topo = box.topology()
    act = M.boxes.spread_gpus(k)
    bin_node = [box.hbm_bin[g] for g in act] + box.host_bin
    rng = np.random.default_rng(5)
    hot = (rng.pareto(1.0, n) * 3).astype(np.uint64)
    caps = [r + n // (2 * k)] * k + [n, n]
    b, s, A, U, T = M.place(topo, hot, caps, bin_node=bin_node, replicate_rows=r)
    N = topo.info()[0]
    d = np.zeros(N, np.int64)
    for i, v in enumerate(bin_node):
        d[v] = int(A[i]) * 512 // 10
    plan = M.plan(topo, [box.gpu[g] for g in act], d, 770_000, 6_500_000).info()
    return topo, b, s, bin_node, caps, plan, box


@pytest.mark.parametrize("r", [0, 300])
def test_layout_roundtrip(tmp_path, r):
    topo, b, s, bin_node, caps, plan, _ = _layout(r=r)
    p = str(tmp_path / "layout.npz")
    M.layout.save(p, topo, bin_of=b, slot_of=s, bin_node=bin_node, capacity_rows=caps, replicate_rows=r, plan=plan)
    got = M.layout.load(p, topo)
    assert np.array_equal(got["bin_of"], b) and np.array_equal(got["slot_of"], s)
    assert got["replicate_rows"] == r and got["bin_node"] == [int(x) for x in bin_node]
    for k in ("t_star", "t_ingest", "t_nvlink", "t_hbm"):
        assert got["plan"][k] == plan[k]
    assert np.array_equal(got["plan"]["quota"], plan["quota"]) and np.array_equal(got["plan"]["link_flow"], plan["link_flow"])
    # the device map packs the same from the loaded arrays
    assert np.array_equal(M.place_pack_rank(got["bin_of"], got["slot_of"], 0), M.place_pack_rank(b, s, 0))


def test_layout_refuses_other_topology_and_bad_files(tmp_path):
    topo, b, s, bin_node, caps, plan, _ = _layout()
    p = str(tmp_path / "layout.npz")
    M.layout.save(p, topo, bin_of=b, slot_of=s, bin_node=bin_node, capacity_rows=caps)
    other = M.boxes.hgx_b200(8, port_gbs=40.0).topology()  # another box: other capacities
    with pytest.raises(M.MomentError):
        M.layout.load(p, other)
    assert M.layout.load(p)["plan"] is None  # no topology given: no check, loads
    bad = b.copy()
    bad[0] = 99  # a bin that does not exist
    M.layout.save(p, topo, bin_of=bad, slot_of=s, bin_node=bin_node, capacity_rows=caps)
    with pytest.raises(M.MomentError):
        M.layout.load(p, topo)
    with pytest.raises(M.MomentError):
        M.layout.save(p, topo, bin_of=b[:-1], slot_of=s, bin_node=bin_node, capacity_rows=caps)
