"""§8(f)3 weighted LP on the GPU (mfl_weighted.cuh) vs the weighted oracle,
bit for bit: a label's frequency is the sum of its arcs' weights
(LoadNeighbor's weight [P:110, P:145])."""
import numpy as np
import pytest
import torch

import oracle
from glp_inputs import graphs
from glp_inputs.csr import from_arrays, from_edges

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


def weights_for(csr, seed, hi=8):
    return torch.from_numpy(np.random.default_rng(seed).integers(1, hi + 1, csr.nnz).astype(np.int32))


def check(csr, w, variant, max_iters, seeds=None, on_device=True):
    ref = oracle.run_weighted(csr, w.numpy().astype(np.uint32), glp.VARIANTS[variant], max_iters, seeds=seeds,
                              threads=8)
    c = csr.to("cuda") if on_device else csr
    with glp.Graph(c, weights=w.to("cuda") if on_device else w) as g:
        info = g.run(variant, max_iters, seeds)
        lab = g.labels("cpu").numpy()
        st = g.iter_stats()
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason), (info, ref)
    assert [s["changed"] for s in st] == list(ref.changed)
    mism = np.flatnonzero(lab != ref.labels)
    assert mism.size == 0, f"{mism.size} labels differ, first {mism[:10]}"
    return st


@pytest.mark.parametrize("variant", ["classic", "seeded"])
@pytest.mark.parametrize("on_device", [True, False])
def test_weighted_rmat(variant, on_device):
    csr = graphs.rmat(14, seed=3)
    seeds = np.array([5, 700, 9000, 16000], dtype=np.int32) if variant == "seeded" else None
    st = check(csr, weights_for(csr, 1), variant, 25, seeds, on_device)
    assert any(not s["dense"] for s in st)  # symmetric: sparse (frontier) iterations ran


def test_weighted_long_rows_partitioned():
    """Hub rows of 5k..60k arcs with all-distinct labels at t = 2: the block
    kernel's label partitions (and their retries) must stay exact."""
    g = np.random.default_rng(7)
    n_priv = 70_000
    leaves = n_priv + np.arange(n_priv)
    src = [np.arange(n_priv)]
    dst = [leaves]
    for h, d in enumerate(list(g.integers(5000, 15000, 20)) + list(g.integers(20000, 60000, 6))):
        src.append(np.full(d, 2 * n_priv + h))
        dst.append(g.choice(leaves, d, replace=False))
    csr = from_edges(2 * n_priv + 26, torch.from_numpy(np.concatenate(src)), torch.from_numpy(np.concatenate(dst)))
    check(csr, weights_for(csr, 2, hi=1000), "classic", 6)


def test_multiplicity_weights_equal_multigraph():
    """GPU weighted run on the deduplicated graph == GPU unweighted run on the
    multigraph whose repeated arcs the weights count."""
    g = np.random.default_rng(11)
    n, m = 5000, 200_000
    src = g.integers(0, n, m)
    dst = (g.zipf(1.5, m) % n)
    key = np.unique(np.concatenate([src * n + dst, dst * n + src]), return_counts=False)
    rep = np.concatenate([key, key[g.integers(0, key.size, key.size // 2)]])
    rep = np.sort(rep)
    rows, cols = rep // n, rep % n
    keep = rows != cols
    rows, cols = rows[keep], cols[keep]
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(np.bincount(rows, minlength=n))
    multi = from_arrays(n, off, cols.astype(np.int32))
    uk, mult = np.unique(rows * n + cols, return_counts=True)
    off2 = np.zeros(n + 1, dtype=np.int64)
    off2[1:] = np.cumsum(np.bincount(uk // n, minlength=n))
    simple = from_arrays(n, off2, (uk % n).astype(np.int32))
    with glp.Graph(multi.to("cuda")) as gm:
        gm.run("classic", 30)
        a = gm.labels("cpu").numpy()
    with glp.Graph(simple.to("cuda"), weights=torch.from_numpy(mult.astype(np.int32)).cuda()) as gs:
        gs.run("classic", 30)
        b = gs.labels("cpu").numpy()
    assert (a == b).all()


def test_weighted_errors():
    csr = graphs.karate()
    w = torch.ones(csr.nnz, dtype=torch.int32)
    with glp.Graph(csr.to("cuda"), weights=w.cuda()) as g:
        with pytest.raises(glp.GlpError) as e:
            g.run("llp", 5, gamma=1.0)
        assert e.value.status == 6
    w0 = w.clone()
    w0[3] = 0
    with pytest.raises(glp.GlpError) as e:
        glp.Graph(csr.to("cuda"), weights=w0.cuda())
    assert e.value.status == 2


@pytest.mark.parametrize("P", [2, 3])
def test_weighted_local_group(P):
    from paper_conf_sigmod_yelhls21_b200.dist import LocalGroup
    csr = graphs.rmat(13, seed=6)
    w = weights_for(csr, 4)
    ref = oracle.run_weighted(csr, w.numpy().astype(np.uint32), oracle.CLASSIC, 20, threads=8)
    with LocalGroup(csr.to("cuda"), P, weights=w) as grp:
        infos = grp.run("classic", 20)
        labs = [grp.labels(r).numpy() for r in range(P)]
    for r in range(P):
        assert infos[r].iterations == ref.iterations and (labs[r] == ref.labels).all()


@pytest.mark.parametrize("variant", ["classic", "seeded"])
@pytest.mark.parametrize("giant_kernel", ["1", "0"])
def test_weighted_giant_rows(variant, giant_kernel, monkeypatch):
    """Rows past kGiantMin (65536 arcs) with weights: the segmented giant
    kernels add each arc's weight into the per-row global tables (default),
    or one block per row (GLP_WT_GIANT=0); both equal the weighted oracle."""
    monkeypatch.setenv("GLP_WT_GIANT", giant_kernel)
    rng = np.random.default_rng(11)
    n_leaf = 90_000
    hubs = [70_000, 80_000, 66_000]
    src, dst = [], []
    for h, d in enumerate(hubs):  # hub h -> d leaves (distinct), leaves cross-linked
        leaves = rng.choice(n_leaf, d, replace=False) + len(hubs)
        src.append(np.full(d, h)); dst.append(leaves)
    a = rng.integers(len(hubs), len(hubs) + n_leaf, 150_000)
    b = rng.integers(len(hubs), len(hubs) + n_leaf, 150_000)
    src.append(a); dst.append(b)
    csr = from_edges(len(hubs) + n_leaf, torch.from_numpy(np.concatenate(src).astype(np.int64)),
                     torch.from_numpy(np.concatenate(dst).astype(np.int64)), "wgiant")
    w = weights_for(csr, 4)
    seeds = np.array([0, 5, 17, 400, 9000], dtype=np.int32) if variant == "seeded" else None
    check(csr, w, variant, 15, seeds=seeds)


@pytest.mark.parametrize("variant", ["classic", "seeded"])
@pytest.mark.parametrize("low_kernel", ["1", "0"])
def test_weighted_low_rows(variant, low_kernel, monkeypatch):
    """Vertices of degree <= 32 with weights: the packed-warp kernel sums the
    weights of equal labels per segment (default) or the warp-per-vertex
    kernel (GLP_WT_LOW=0); every low degree 1..32 occurs."""
    monkeypatch.setenv("GLP_WT_LOW", low_kernel)
    rng = np.random.default_rng(21)
    n = 60_000
    deg = rng.integers(1, 33, n)
    src = np.repeat(np.arange(n), deg)
    dst = rng.integers(0, n // 8, src.size)  # few targets: labels repeat inside segments
    csr = from_edges(n, torch.from_numpy(src.astype(np.int64)), torch.from_numpy(dst.astype(np.int64)), "wlow")
    w = weights_for(csr, 9, hi=50)
    seeds = np.array([1, 2, 3, 50, 700, 5000], dtype=np.int32) if variant == "seeded" else None
    check(csr, w, variant, 20, seeds=seeds)
