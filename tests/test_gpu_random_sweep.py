"""A seeded sweep of random small graphs through every variant and mode,
against the oracle, bit for bit: power-law and uniform degrees, repeated arcs,
self-loops, directed and symmetric input, isolated vertices, hub rows past
the W / M / L / giant class limits, forced re-queues (debug_pred_cap), the
sparse exchange, the HT + CMS path, weights, SLP, a 2- or 3-rank group.  Each
case is small, so the sweep covers many shapes in a few seconds."""
import numpy as np
import pytest
import torch

import oracle
from glp_inputs.csr import from_arrays

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")
from paper_conf_sigmod_yelhls21_b200.dist import LocalGroup  # noqa: E402


def random_graph(seed):
    g = np.random.default_rng(seed)
    n = int(g.integers(50, 6000))
    m = int(g.integers(n, 20 * n))
    skew = float(g.uniform(0.0, 1.4))
    w = 1.0 / np.arange(1, n + 1) ** skew
    w /= w.sum()
    perm = g.permutation(n)
    src = perm[g.choice(n, m, p=w)]
    dst = perm[g.choice(n, m, p=w)]
    if g.random() < 0.3:  # a hub row past the class limits
        h = int(g.integers(0, n))
        d = int(g.integers(3000, 80000))
        src = np.concatenate([src, np.full(d, h)])
        dst = np.concatenate([dst, g.integers(0, n, d)])
    directed = g.random() < 0.3
    if not g.random() < 0.5:  # simple graph: no loops, no repeats
        keep = src != dst
        key = np.unique(src[keep].astype(np.int64) * n + dst[keep])
        src, dst = key // n, key % n
    if not directed:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    o = np.lexsort((dst, src))
    src, dst = src[o], dst[o]
    if g.random() < 0.5:  # arbitrary arc order inside rows
        o = np.lexsort((g.random(src.size), src))
        src, dst = src[o], dst[o]
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(np.bincount(src, minlength=n))
    return from_arrays(n, off, dst.astype(np.int32), symmetric=not directed), g


@pytest.mark.parametrize("seed", range(96))
def test_random_sweep(seed):
    csr, g = random_graph(1000 + seed)
    n = csr.n
    variant = ["classic", "seeded", "llp", "classic", "slp", "weighted"][seed % 6]
    kw, okw = {}, {}
    seeds = None
    if variant == "seeded":
        seeds = np.unique(g.integers(0, n, int(g.integers(1, 20)))).astype(np.int32)
    if variant == "llp":
        kw["gamma"] = okw["gamma"] = float(g.choice([0.0, 0.25, 1.0, 0.37]))
    run_kw = dict(kw)
    if g.random() < 0.4:
        run_kw["debug_pred_cap"] = int(g.integers(1, 64))
    if variant == "classic" and g.random() < 0.5:
        run_kw["tail_cms"] = True
        run_kw["cms_ht_slots"] = int(g.choice([0, 64, 512]))
    mi = 20
    if variant == "slp":
        K, r = int(g.integers(1, 6)), float(g.choice([0.0, 0.1]))
        ml, mc, sp = oracle.run_slp(csr, K=K, r=r, max_iters=12, threads=8)
        with glp.Graph(csr.to("cuda")) as G:
            G.run("slp", 12, slp_max_labels=K, slp_threshold=r)
            assert (G.labels("cpu").numpy() == sp).all()
            gl, gc = G.slp_memory(K)
        assert (gl.numpy() == ml).all() and (gc.numpy() == mc).all()
        return
    if variant == "weighted":
        wts = g.integers(1, 50, csr.nnz).astype(np.int32)
        ref = oracle.run_weighted(csr, wts.astype(np.uint32), oracle.CLASSIC, mi, threads=8)
        with glp.Graph(csr.to("cuda"), weights=torch.from_numpy(wts).cuda()) as G:
            info = G.run("classic", mi, **run_kw)
            lab = G.labels("cpu").numpy()
        assert info.iterations == ref.iterations and (lab == ref.labels).all()
        return
    ref = oracle.run(csr, glp.VARIANTS[variant], mi, seeds=seeds, threads=8, **okw)
    P = int(g.choice([1, 1, 2, 3]))
    if P == 1:
        with glp.Graph(csr.to("cuda")) as G:
            info = G.run(variant, mi, seeds, **run_kw)
            lab = G.labels("cpu").numpy()
            st = G.iter_stats()
    else:
        run_kw["sparse_exchange"] = int(g.choice([-1, 1]))
        with LocalGroup(csr.to("cuda"), P, edge_balanced=bool(g.random() < 0.5)) as grp:
            info = grp.run(variant, mi, seeds, **run_kw)[0]
            lab = grp.labels(P - 1).numpy()
            st = grp.iter_stats(0)
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason), (variant, P, run_kw)
    assert [s["changed"] for s in st] == list(ref.changed)
    mism = np.flatnonzero(lab != ref.labels)
    assert mism.size == 0, f"{variant} P={P} {run_kw}: {mism.size} labels differ, first {mism[:10]}"
