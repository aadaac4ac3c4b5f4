"""Inputs the C ABI accepts but the generators never produce, vs the oracle.

glp.h promises that a row may list a neighbour twice (two votes, R3), that
self-loops are ordinary arcs (v votes with its own previous label when the
CSR says v is its own neighbour), and that directed input (symmetric = 0,
"incoming neighbours" [P:68], directed datasets [P:255-264]) runs with full
sweeps.  The oracle counts CSR entries exactly as listed, so labels must be
bit-exact.  Also: the concurrent static-L / redo-L launches with many
partitioned rows (the staging regions of ADVICE r1).
"""
import numpy as np
import pytest
import torch

import oracle
from glp_inputs.csr import from_arrays, from_edges

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


def raw_csr(n, src, dst, symmetric, shuffle_seed=None):
    """CSR listing every (src, dst) pair as given: duplicates and self-loops kept."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    if shuffle_seed is not None:  # arbitrary arc order inside rows
        g = np.random.default_rng(shuffle_seed)
        key = src * 2 ** 20 + g.integers(0, 2 ** 20, src.size)
        o = np.argsort(key, kind="stable")
        src, dst = src[o], dst[o]
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(np.bincount(src, minlength=n))
    return from_arrays(n, off, dst.astype(np.int32), symmetric=symmetric)


def multigraph(n, m, seed, directed, loops=0.02, dup=0.3, skew=1.2):
    """Power-law-ish endpoints (hub rows), a fraction of repeated arcs and of
    self-loops."""
    g = np.random.default_rng(seed)
    w = 1.0 / np.arange(1, n + 1) ** (skew / 2)
    w /= w.sum()
    perm = g.permutation(n)
    src = perm[g.choice(n, m, p=w)]
    dst = perm[g.choice(n, m, p=w)]
    k = int(loops * m)
    dst[:k] = src[:k]  # self-loops
    r = int(dup * m)
    i = g.integers(0, m, r)
    src = np.concatenate([src, src[i]])  # repeated arcs
    dst = np.concatenate([dst, dst[i]])
    if not directed:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    return raw_csr(n, src, dst, symmetric=not directed, shuffle_seed=seed)


def gpu_vs_oracle(csr, variant, max_iters, seeds=None, gamma=0.0, **kw):
    ref = oracle.run(csr, glp.VARIANTS[variant], max_iters, seeds=seeds, gamma=gamma, threads=8)
    with glp.Graph(csr.to("cuda")) as g:
        info = g.run(variant, max_iters, seeds, gamma=gamma, **kw)
        lab = g.labels("cpu").numpy()
        st = g.iter_stats()
    assert info.iterations == ref.iterations and info.stop_reason == ref.stop_reason, (info, ref)
    assert [s["changed"] for s in st] == list(ref.changed)
    mism = np.flatnonzero(lab != ref.labels)
    assert mism.size == 0, f"{mism.size} labels differ, first {mism[:10]}"
    return lab, st


def test_duplicate_arc_is_two_votes():
    """Row 0 lists 2 twice and 1 once: counts {2: 2, 1: 1}, so label 2 wins
    (a set view of N(0) would tie and give the smaller label 1)."""
    csr = raw_csr(3, [0, 0, 0, 1, 2], [2, 2, 1, 0, 0], symmetric=False)
    lab, _ = gpu_vs_oracle(csr, "classic", 1)
    assert lab[0] == 2


def test_self_loop_votes_own_label():
    # row 0: [0, 0, 5]: own label (0) twice beats 5; row 5: [0]
    csr = raw_csr(6, [0, 0, 0, 5], [0, 0, 5, 0], symmetric=False)
    lab, _ = gpu_vs_oracle(csr, "classic", 1)
    assert lab[0] == 0 and lab[5] == 0


@pytest.mark.parametrize("directed", [True, False])
@pytest.mark.parametrize("variant", ["classic", "seeded", "llp"])
def test_multigraph_runs(directed, variant):
    csr = multigraph(4000, 120_000, seed=7 + directed, directed=directed)
    assert csr.symmetric == (not directed)
    seeds = np.array([3, 77, 1500, 3999], dtype=np.int32) if variant == "seeded" else None
    gamma = 0.5 if variant == "llp" else 0.0
    mi = 10 if variant == "llp" else 25
    lab, st = gpu_vs_oracle(csr, variant, mi, seeds=seeds, gamma=gamma)
    if directed or variant == "llp":
        assert all(s["dense"] for s in st)  # no frontier without symmetry


def test_directed_hubs_all_row_classes():
    """Directed graph with long rows (M / L / giant classes) full of repeats."""
    g = np.random.default_rng(11)
    n = 200_000
    hubs = [5000, 9000, 20000, 70000, 150000]
    src, dst = [], []
    for i, d in enumerate(hubs):
        src.append(np.full(d, i))
        dst.append(g.integers(0, 3000 + 20 * i, d))  # few distinct targets: many repeats
    m = 600_000
    src.append(g.integers(0, n, m))
    dst.append(g.integers(0, n, m))
    csr = raw_csr(n, np.concatenate(src), np.concatenate(dst), symmetric=False, shuffle_seed=3)
    gpu_vs_oracle(csr, "classic", 8)
    gpu_vs_oracle(csr, "llp", 5, gamma=1.0)


def many_hubs(n_priv, hub_degs, seed):
    """Leaf i touches private vertex i (smaller id) and some hubs: at t = 1 it
    takes label i, so at t = 2 every hub row sees all-distinct labels and the
    long ones need the L kernel's partitioned (staged) count."""
    g = np.random.default_rng(seed)
    H = len(hub_degs)
    leaves = n_priv + np.arange(n_priv)
    src = [np.arange(n_priv)]
    dst = [leaves]
    for h, d in enumerate(hub_degs):
        src.append(np.full(d, 2 * n_priv + h))
        dst.append(g.choice(leaves, d, replace=False))
    src = torch.from_numpy(np.concatenate(src))
    dst = torch.from_numpy(np.concatenate(dst))
    return from_edges(2 * n_priv + H, src, dst, "many_hubs")


@pytest.mark.parametrize("cap", [0, 48])
def test_concurrent_static_and_redo_L(cap):
    """Hundreds of partitioned rows in the static L launch while re-queued
    rows (W -> M -> L, forced by clamping the predictions) run the redo L
    launch beside it: both stage labels, in separate regions."""
    g = np.random.default_rng(5)
    degs = list(g.integers(5000, 15000, 160)) + list(g.integers(17000, 60000, 40))
    csr = many_hubs(70_000, degs, seed=9)
    gpu_vs_oracle(csr, "classic", 5, debug_pred_cap=cap)
    gpu_vs_oracle(csr, "llp", 4, gamma=0.25, debug_pred_cap=cap)
