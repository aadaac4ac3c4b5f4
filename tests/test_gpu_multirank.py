"""libglp's partitioned path (P > 1 ranks, 1-D vertex ranges [P:103]) vs the
CPU oracle, run on ONE GPU through an in-process rank group
(glp_local_group): P Graph instances, one host thread each, exchange labels
through each other's device buffers.  Everything but the NCCL calls
themselves executes: per-rank layout and internal ids, the pos/orig
all-gather, the label all-gather (equal and unequal slices), the counter
all-reduce (every rank takes the same stop / frontier decision), the
frontier-mark merge of sparse iterations, and the sharded LLP histogram.

Synchronous LP is partition-independent, so every rank's labels, the
iteration count and the per-iteration change counts must equal the oracle's
bit for bit, for any P and any bounds.
"""
import numpy as np
import pytest
import torch

import oracle
from glp_inputs import graphs

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")
from paper_conf_sigmod_yelhls21_b200.dist import LocalGroup, shard_bounds  # noqa: E402


def run_group(csr, P, variant, max_iters, seeds=None, gamma=0.0, edge_balanced=False, bounds=None, **kw):
    with LocalGroup(csr, P, edge_balanced=edge_balanced, bounds=bounds) as grp:
        infos = grp.run(variant, max_iters, seeds, gamma=gamma, **kw)
        labs = [grp.labels(r).numpy().copy() for r in range(P)]
        st = [grp.iter_stats(r) for r in range(P)]
        ks = [grp.graphs[r].kernel_stats() for r in range(P)]
        b = list(grp.bounds)
    return labs, infos, st, ks, b


def check(csr, P, variant, max_iters, seeds=None, gamma=0.0, **kw):
    vid = glp.VARIANTS[variant]
    ref = oracle.run(csr, vid, max_iters, seeds=None if seeds is None else np.asarray(seeds), gamma=gamma,
                     threads=8)
    labs, infos, st, ks, b = run_group(csr.to("cuda"), P, variant, max_iters, seeds, gamma, **kw)
    for r in range(P):
        assert infos[r].iterations == ref.iterations, (r, infos[r], ref)
        assert infos[r].stop_reason == ref.stop_reason
        assert [s["changed"] for s in st[r]] == list(ref.changed), r
        mism = np.flatnonzero(labs[r] != ref.labels)
        assert mism.size == 0, f"rank {r}: {mism.size} labels differ, first {mism[:10]}"
    return ref, labs, infos, st, ks, b


@pytest.mark.parametrize("P", [2, 3, 4])
@pytest.mark.parametrize("edge_balanced", [False, True])
def test_classic_rmat(P, edge_balanced):
    csr = graphs.rmat(14, seed=8)
    ref, labs, infos, st, ks, b = check(csr, P, "classic", 20, edge_balanced=edge_balanced)
    if edge_balanced:
        assert b != shard_bounds(csr.n, P)  # unequal slices: grouped/unequal all-gather
    # the run reached sparse (frontier) iterations, so the mark merge ran
    assert any(not s["dense"] for s in st[0])


@pytest.mark.parametrize("P", [2, 4])
def test_llp_sharded_and_replicated(P):
    csr = graphs.rmat(13, seed=9)
    for gamma in (1.0, 0.37):
        for mode in (2, 1):
            ref, labs, infos, st, ks, b = check(csr, P, "llp", 10, gamma=gamma, llp_hist=mode)
            hist = [next(k for k in ks[r] if k["name"] == "llp_hist") for r in range(P)]
            per_it = [h["arcs"] / max(infos[r].iterations - 1, 1) for r, h in enumerate(hist)]
            if mode == 2:
                # sharded: each rank histograms only its own rows (<= ceil(n/P) labels)
                for r in range(P):
                    assert per_it[r] <= b[r + 1] - b[r] + 1e-9, (r, per_it[r])
            else:
                assert all(abs(x - csr.n) < 1e-9 for x in per_it)


def test_llp_modularity_floor():
    """north_star's LLP floor at P = 3: modularity within 1e-9, >= 99.99 %
    agreement (bit-exact in fact)."""
    csr = graphs.sbm(n=30_008, k=31, m=400_000, mu=0.2, seed=3)  # n % 3 == 2
    ref, labs, *_ = check(csr, 3, "llp", 12, gamma=1.0)
    assert abs(oracle.modularity(csr, labs[0]) - oracle.modularity(csr, ref.labels)) <= 1e-9


@pytest.mark.parametrize("P", [2, 3])
def test_seeded_sparse_frontier(P):
    csr, seeds = graphs.taobao(users=40_000, items=10_000, pairs=200_000, rings=40, seed=5)
    ref, labs, infos, st, *_ = check(csr, P, "seeded", 30, seeds=seeds.numpy())
    assert any(not s["dense"] for s in st[0])
    s = seeds.numpy()
    assert (labs[0][s] == s).all()


def test_n_not_divisible_by_P():
    """n % P != 0 (P = 4, 7): padded label arrays, a short last slice."""
    csr = graphs.sbm(n=20_010, k=30, m=200_000, mu=0.1, seed=2)
    for P in (4, 7):
        check(csr, P, "classic", 30)
    check(graphs.karate(), 3, "classic", 20)


def test_explicit_uneven_bounds_and_empty_slice():
    """Hand-picked bounds: a rank owning no rows and one owning nearly all."""
    csr = graphs.rmat(12, seed=4)
    n = csr.n
    check(csr, 3, "classic", 20, bounds=[0, 17, 17, n])
    check(csr, 3, "llp", 6, gamma=1.0, bounds=[0, n - 100, n - 100, n])


def test_group_ranks_agree_with_single_gpu_stats():
    """Iterations and per-iteration changes of a 4-rank run equal the 1-GPU
    run's.  (Scanned vertices and arcs may differ: a low-degree chunk is
    scanned whole when any of its vertices is active, and chunks are packed
    per rank; a block stops on a strict majority when its warps poll.)"""
    csr = graphs.rmat(13, seed=21)
    c = csr.to("cuda")
    with glp.Graph(c) as g:
        info1 = g.run("classic", 20)
        st1 = g.iter_stats()
    labs, infos, st, ks, b = run_group(c, 4, "classic", 20)
    assert infos[0].iterations == info1.iterations
    assert [s["changed"] for s in st[0]] == [s["changed"] for s in st1]
    assert [s["dense"] for s in st[0]] == [s["dense"] for s in st1]


def test_failed_rank_releases_group():
    """A rank whose run fails (bad seed) aborts the group: the other ranks
    return an error instead of waiting at the exchange forever."""
    csr = graphs.rmat(11, seed=2).to("cuda")
    grp = LocalGroup(csr, 2)
    try:
        def body(r):
            seeds = [5, 10**9] if r == 1 else [5, 7]
            return grp.graphs[r].run("seeded", 10, seeds)
        with pytest.raises(glp.GlpError):
            grp._all(body)
    finally:
        grp.close()


@pytest.mark.parametrize("mode", [1, -1])
@pytest.mark.parametrize("P", [2, 3])
def test_sparse_exchange(mode, P):
    """§8(f)1: only the changed vertices' (id, label) pairs of t-1 and t are
    exchanged (forced every iteration, or automatically once few vertices
    change); labels and iteration counts stay bit-exact."""
    for csr, variant, seeds, mi in [(graphs.rmat(14, seed=8), "classic", None, 20),
                                    (graphs.sbm(n=20_010, k=30, m=200_000, mu=0.1, seed=2), "classic", None, 30),
                                    (graphs.taobao(users=40_000, items=10_000, pairs=200_000, rings=40, seed=5)[0],
                                     "seeded", np.array([3, 500, 40_000, 45_000], dtype=np.int32), 30)]:
        ref, labs, infos, st, ks, b = check(csr, P, variant, mi, seeds=seeds, sparse_exchange=mode)
        ex = [s["exchange"] for s in st[0]]
        if mode == 1:
            assert set(ex) == {2}
        else:
            assert 2 in ex and 1 in ex  # dense early, sparse once changes are few
