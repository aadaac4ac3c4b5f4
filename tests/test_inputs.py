"""Input generators: determinism, CSR well-formedness, device independence."""
import numpy as np
import pytest
import torch

from glp_inputs import graphs, rng
from glp_inputs.csr import from_edges


def test_splitmix_matches_python():
    xs = [0, 1, 12345, 2 ** 40 + 7, 2 ** 62 - 1]
    t = rng.splitmix64(torch.tensor(xs, dtype=torch.int64))
    for x, y in zip(xs, t.tolist()):
        assert (y & ((1 << 64) - 1)) == rng.splitmix64_int(x)


def test_uniform_range_and_mean():
    u = rng.uniform(1, 2, torch.arange(200000, dtype=torch.int64))
    assert float(u.min()) >= 0.0 and float(u.max()) < 1.0
    assert abs(float(u.mean()) - 0.5) < 0.005
    r = rng.randint(1, 3, torch.arange(100000, dtype=torch.int64), 7)
    assert int(r.min()) == 0 and int(r.max()) == 6


def _check_csr(csr):
    off, col = csr.numpy()
    assert off[0] == 0 and off[-1] == col.size and (np.diff(off) >= 0).all()
    assert col.size == 0 or (col.min() >= 0 and col.max() < csr.n)
    # symmetric, no self loops, no duplicates
    rows = np.repeat(np.arange(csr.n), np.diff(off))
    fwd = set(zip(rows.tolist(), col.tolist()))
    assert len(fwd) == col.size
    assert all(a != b for a, b in fwd)
    assert all((b, a) in fwd for a, b in fwd)


def test_generators_wellformed():
    for csr in [graphs.karate(), graphs.bowtie(), graphs.rmat(9), graphs.sbm(n=1000, k=10, m=5000),
                graphs.taobao(users=800, items=200, pairs=3000, rings=4)[0], graphs.cliques([3, 4]),
                graphs.gnp(20, 0.2, 1), graphs.star(5), graphs.empty(3)]:
        _check_csr(csr)
    k = graphs.karate()
    assert k.n == 34 and k.nnz == 156


def test_deterministic():
    a = graphs.rmat(10, seed=4)
    b = graphs.rmat(10, seed=4)
    assert a.sha256() == b.sha256()
    assert graphs.rmat(10, seed=5).sha256() != a.sha256()


def test_taobao_seeds():
    csr, seeds = graphs.taobao(users=10000, items=2000, pairs=50000, rings=2, seed=7)
    s = seeds.numpy()
    assert s.size == 10 and len(set(s.tolist())) == s.size  # 0.1% of users
    assert (np.diff(s) > 0).all() and s.min() >= 0 and s.max() < csr.n


def test_from_edges_dedupe():
    src = torch.tensor([0, 1, 1, 2, 2])
    dst = torch.tensor([1, 0, 1, 0, 0])
    c = from_edges(3, src, dst)
    assert c.row_offsets.tolist() == [0, 2, 3, 4]
    assert c.col_idx.tolist() == [1, 2, 0, 0]


@pytest.mark.gpu
def test_cuda_generation_matches_cpu():
    for mk in [lambda d: graphs.rmat(12, seed=3, device=d),
               lambda d: graphs.sbm(n=5000, k=50, m=40000, device=d),
               lambda d: graphs.taobao(users=4000, items=1000, pairs=20000, rings=10, device=d)[0]]:
        assert mk("cpu").sha256() == mk("cuda").sha256()


def test_rmat_bucketed_build_matches_plain():
    """The memory-bounded RMAT-28 builder (row buckets) yields the same CSR."""
    from glp_inputs import graphs
    for scale in (9, 12):
        a = graphs.rmat(scale, seed=1)
        for buckets in (2, 5, 16):
            b = graphs.rmat(scale, seed=1, buckets=buckets)
            assert torch.equal(a.row_offsets, b.row_offsets)
            assert torch.equal(a.col_idx, b.col_idx)


@pytest.mark.gpu
def test_taobao_generation_repeatable_on_gpu():
    """Two generations of a mid-size TaoBao window are identical (the
    inverse-CDF tables once came from a device float scan whose rounding
    order varied run to run)."""
    import torch
    a, sa = graphs.taobao(users=20_000_000, items=5_000_000, pairs=40_000_000, rings=100, device="cuda")
    b, sb = graphs.taobao(users=20_000_000, items=5_000_000, pairs=40_000_000, rings=100, device="cuda")
    assert torch.equal(a.row_offsets, b.row_offsets) and torch.equal(a.col_idx, b.col_idx)
    assert torch.equal(sa, sb)
