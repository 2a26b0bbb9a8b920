"""Input generators: the partitioned CSR builder (graphs too large to sort at once) yields exactly the
canonical CSR of the in-memory builder; feature rows are reproducible without the table."""
import torch

import workloads as W


def test_partitioned_csr_equals_in_memory():
    g1 = W.rmat_csr(5000, 60000, device="cpu")
    g2 = W.rmat_csr(5000, 60000, device="cpu", chunk=7000, max_edges_in_memory=9000)
    assert torch.equal(g1.indptr, g2.indptr)
    assert torch.equal(g1.indices, g2.indices)
    # adjacency sorted by destination, CSR over the source
    d = g1.indptr[1:] - g1.indptr[:-1]
    assert int(d.sum()) == 60000
    for v in range(0, 5000, 97):
        a = g1.indices[g1.indptr[v]:g1.indptr[v + 1]]
        assert torch.all(a[1:] >= a[:-1])


def test_feature_rows_match_table():
    t = W.feature_table(300, 24, torch.float32, row_stride_bytes=128)
    ids = torch.tensor([0, 7, 299, 150])
    assert torch.equal(t[ids, :96], W.feature_rows(ids, 24, torch.float32))
    assert not t[:, 96:].any()
