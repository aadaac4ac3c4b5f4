"""Pins of the weighted oracle (§8(f)3: LoadNeighbor returns (l, weight)
[P:110, P:145]; a label's frequency is the sum of its arcs' weights).

Each pin is independent of the oracle's sort-and-scan:
  * multiplicity equivalence: a multigraph's repeated arcs (unweighted oracle,
    already pinned) == the deduplicated graph weighted by multiplicity;
  * unit weights == the unweighted oracle;
  * iteration-1 closed form on unique labels: L_1[v] = the neighbour of
    maximum arc weight, smallest id on ties (numpy lexsort);
  * brute force (pure-Python dict sums, no sorting) on tiny graphs;
  * scaling every weight by a constant changes nothing;
  * a hand-derived star where the weights reverse the unweighted choice.
"""
import numpy as np
import pytest

import oracle
from glp_inputs import graphs
from glp_inputs.csr import from_arrays


def raw_csr(n, src, dst, symmetric=False):
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    o = np.lexsort((dst, src))
    src, dst = src[o], dst[o]
    off = np.zeros(n + 1, dtype=np.int64)
    off[1:] = np.cumsum(np.bincount(src, minlength=n))
    return from_arrays(n, off, dst.astype(np.int32), symmetric=symmetric)


def random_multigraph(n, m, seed, directed=True):
    g = np.random.default_rng(seed)
    src = g.integers(0, n, m)
    dst = g.integers(0, min(n, 40), m)  # few targets: many repeats
    keep = src != dst
    src, dst = src[keep], dst[keep]
    if not directed:
        src, dst = np.concatenate([src, dst]), np.concatenate([dst, src])
    return src, dst


def dedup_weighted(n, src, dst):
    key = np.asarray(src, dtype=np.int64) * n + np.asarray(dst, dtype=np.int64)
    uk, mult = np.unique(key, return_counts=True)
    return raw_csr(n, uk // n, uk % n), mult.astype(np.uint32)


@pytest.mark.parametrize("variant", [oracle.CLASSIC, oracle.SEEDED])
@pytest.mark.parametrize("directed", [True, False])
def test_multiplicity_equivalence(variant, directed):
    n = 300
    src, dst = random_multigraph(n, 6000, seed=3 + directed, directed=directed)
    multi = raw_csr(n, src, dst)
    simple, w = dedup_weighted(n, src, dst)
    seeds = np.array([0, 5, 17, 250], dtype=np.int32) if variant == oracle.SEEDED else None
    a = oracle.run(multi, variant, 25, seeds=seeds, trace=True)
    b = oracle.run_weighted(simple, w, variant, 25, seeds=seeds, trace=True)
    assert a.iterations == b.iterations and a.stop_reason == b.stop_reason
    assert (a.trace == b.trace).all()


@pytest.mark.parametrize("variant", [oracle.CLASSIC, oracle.SEEDED])
def test_unit_weights_equal_unweighted(variant):
    csr = graphs.rmat(11, seed=4)
    seeds = np.array([1, 100, 999], dtype=np.int32) if variant == oracle.SEEDED else None
    a = oracle.run(csr, variant, 20, seeds=seeds, trace=True)
    b = oracle.run_weighted(csr, np.ones(csr.nnz, dtype=np.uint32), variant, 20, seeds=seeds, trace=True)
    assert a.iterations == b.iterations and (a.trace == b.trace).all()


def test_iteration1_closed_form():
    csr = graphs.rmat(12, seed=9)
    off, col = csr.numpy()
    w = np.random.default_rng(1).integers(1, 6, csr.nnz).astype(np.uint32)
    res = oracle.run_weighted(csr, w, oracle.CLASSIC, 1)
    rows = np.repeat(np.arange(csr.n), np.diff(off))
    # per row: max weight, then smallest neighbour id (labels are unique ids)
    o = np.lexsort((col, -w.astype(np.int64), rows))
    first = np.ones(o.size, dtype=bool)
    first[1:] = rows[o][1:] != rows[o][:-1]
    exp = np.arange(csr.n, dtype=np.int32)
    exp[rows[o][first]] = col[o][first]
    assert (res.labels == exp).all()


def test_hand_star():
    """Centre 0 with leaves 1, 2, 3; arc 0->3 has weight 5: L_1[0] = 3
    (unweighted: 1).  Leaves see only 0."""
    csr = raw_csr(4, [0, 0, 0, 1, 2, 3], [1, 2, 3, 0, 0, 0])
    w = np.array([1, 1, 5, 1, 1, 1], dtype=np.uint32)  # arc order: (0,1) (0,2) (0,3) (1,0) (2,0) (3,0)
    r = oracle.run_weighted(csr, w, oracle.CLASSIC, 1)
    assert r.labels.tolist() == [3, 0, 0, 0]
    assert oracle.run(csr, oracle.CLASSIC, 1).labels.tolist() == [1, 0, 0, 0]


def brute(n, off, col, w, max_iters, seeds=None):
    L = list(range(n)) if seeds is None else [v if v in set(seeds) else -1 for v in range(n)]
    S = set() if seeds is None else set(int(s) for s in seeds)
    prev2, trace = None, []
    for t in range(max_iters):
        nxt = []
        for v in range(n):
            if v in S:
                nxt.append(L[v]); continue
            acc = {}
            for e in range(off[v], off[v + 1]):
                lab = L[col[e]]
                if lab != -1:
                    acc[lab] = acc.get(lab, 0) + int(w[e])
            if not acc:
                nxt.append(L[v]); continue
            top = max(acc.values())
            nxt.append(min(k for k, s in acc.items() if s == top))
        trace.append(nxt)
        changed = sum(a != b for a, b in zip(nxt, L))
        stop = changed == 0 or (prev2 is not None and nxt == prev2)
        prev2, L = L, nxt
        if stop:
            break
    return trace


@pytest.mark.parametrize("seed", range(8))
def test_bruteforce_tiny(seed):
    g = np.random.default_rng(100 + seed)
    n = int(g.integers(3, 11))
    src, dst = random_multigraph(n, int(g.integers(5, 40)), seed, directed=bool(seed % 2))
    csr, w = dedup_weighted(n, src, dst)
    w = (w * g.integers(1, 4, w.size)).astype(np.uint32)
    off, col = csr.numpy()
    seeds = None if seed % 3 else [0, n - 1]
    r = oracle.run_weighted(csr, w, oracle.SEEDED if seeds else oracle.CLASSIC, 12, seeds=seeds, trace=True)
    assert r.trace.tolist() == brute(n, off, col, w, 12, seeds)


def test_scale_invariance():
    csr = graphs.sbm(n=3000, k=30, m=30000, mu=0.2, seed=5)
    w = np.random.default_rng(2).integers(1, 9, csr.nnz).astype(np.uint32)
    a = oracle.run_weighted(csr, w, oracle.CLASSIC, 20, trace=True)
    b = oracle.run_weighted(csr, 3 * w, oracle.CLASSIC, 20, trace=True)
    assert a.iterations == b.iterations and (a.trace == b.trace).all()
