"""§8(f)2 the paper's HT + Count-Min Sketch single scan for long rows
(PAPER §4.1 Procedure SharedMemBigNodes [P:132-182], analysis [P:186-213]).

1. Exactness: with tail_cms the labels equal the oracle's bit for bit, for
   any HT capacity and sketch depth -- the HT's best is taken only when it
   beats every sketch estimate strictly (R15), else the row is recounted.
2. The fallback rate against Theorem 1 [P:213]: on rows shaped as the
   analysis assumes (one label of frequency f_max, every other label once,
   random order, m distinct labels, m <= (f_max - 1) / 2), the fraction of
   rows that needed the exact recount (the paper's global-memory access) is
   at most m * 2^-d + e^-h (Lemma 1 + Lemma 2), with binomial slack.
"""
import math

import numpy as np
import pytest
import torch

import oracle
from glp_inputs import graphs
from glp_inputs.csr import from_edges

pytestmark = pytest.mark.gpu

glp = pytest.importorskip("paper_conf_sigmod_yelhls21_b200")


def check(csr, variant, max_iters, gamma=0.0, seeds=None, **kw):
    ref = oracle.run(csr, glp.VARIANTS[variant], max_iters, seeds=seeds, gamma=gamma, threads=8)
    with glp.Graph(csr.to("cuda")) as g:
        info = g.run(variant, max_iters, seeds, gamma=gamma, tail_cms=True, **kw)
        lab = g.labels("cpu").numpy()
        st = g.iter_stats()
    assert (info.iterations, info.stop_reason) == (ref.iterations, ref.stop_reason)
    assert [s["changed"] for s in st] == list(ref.changed)
    mism = np.flatnonzero(lab != ref.labels)
    assert mism.size == 0, f"{mism.size} labels differ, first {mism[:10]}"
    return st


@pytest.mark.parametrize("ht,depth", [(0, 4), (256, 4), (64, 8), (1024, 1)])
def test_cms_exact_rmat(ht, depth):
    csr = graphs.rmat(16, seed=2)
    st = check(csr, "classic", 20, cms_ht_slots=ht, cms_depth=depth)
    if ht:  # a small HT sends labels to the sketch
        assert sum(s["cms_rows"] for s in st) > 0
    check(csr, "llp", 6, gamma=1.0, cms_ht_slots=ht, cms_depth=depth)
    check(csr, "seeded", 20, seeds=np.array([3, 77, 5000, 60000], dtype=np.int32), cms_ht_slots=ht,
          cms_depth=depth)


def lemma_rows(H, f_max, m, seed):
    """H hubs; at t = 2 hub h sees label a_h on f_max arcs and m - 1 other
    labels once each, in random arc order (PAPER Lemma 1's setting)."""
    g = np.random.default_rng(seed)
    n_small = H * m  # per hub: one anchor + m - 1 private vertices (small ids)
    n_leaf = H * (f_max + m - 1)
    leaf_ids = n_small + g.permutation(n_leaf)  # random order inside the hub rows
    hub0 = n_small + n_leaf
    src, dst = [], []
    li = 0
    for h in range(H):
        anchor = h * m
        privs = h * m + 1 + np.arange(m - 1)
        lf = leaf_ids[li:li + f_max]
        li += f_max
        ls = leaf_ids[li:li + m - 1]
        li += m - 1
        src += [lf, ls, lf, ls]
        dst += [np.full(f_max, anchor), privs, np.full(f_max, hub0 + h), np.full(m - 1, hub0 + h)]
    src = torch.from_numpy(np.concatenate(src))
    dst = torch.from_numpy(np.concatenate(dst))
    return from_edges(hub0 + H, src, dst, "lemma_rows")


@pytest.mark.parametrize("h,d,m,f_max", [(64, 8, 100, 2001), (32, 6, 40, 2101), (128, 8, 200, 1901)])
def test_fallback_rate_within_theorem1(h, d, m, f_max):
    H = 300
    csr = lemma_rows(H, f_max, m, seed=h + d)
    with glp.Graph(csr.to("cuda")) as g:
        g.run("classic", 2, tail_cms=True, cms_ht_slots=h, cms_depth=d)
        st = g.iter_stats()
        lab = g.labels("cpu").numpy()
    ref = oracle.run(csr, oracle.CLASSIC, 2, threads=8)
    assert (lab == ref.labels).all()
    it2 = st[1]
    assert it2["cms_rows"] == H  # every hub row overflowed its h-slot HT into the sketch
    rate = it2["cms_fallbacks"] / H
    bound = m * 2.0 ** -d + math.exp(-h)
    assert bound < 1.0
    slack = 3.0 * math.sqrt(bound * (1 - bound) / H)
    assert rate <= bound + slack, (rate, bound)
