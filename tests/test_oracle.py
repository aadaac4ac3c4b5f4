"""Pins for the CPU oracle (no GPU).  Each test pins the oracle to something
other than itself: the hand-derived bowtie trajectories, closed forms,
brute-force recount on tiny graphs, textbook BFS and networkx modularity.
"""
import json
import os

import networkx as nx
import numpy as np
import pytest

import oracle
from glp_inputs import graphs
from glp_inputs.csr import from_arrays

from . import bruteforce


def _np(csr):
    off, col = csr.numpy()
    return csr.n, off, col


# --------------------------------------------------------------------------- golden
@pytest.mark.parametrize("case,variant", [("classic", oracle.CLASSIC), ("llp_gamma_1", oracle.LLP),
                                          ("seeded_4", oracle.SEEDED), ("seeded_1_4", oracle.SEEDED)])
def test_bowtie_golden(golden_dir, case, variant):
    g = json.load(open(os.path.join(golden_dir, "bowtie.json")))
    csr = from_arrays(g["graph"]["n"], g["graph"]["row_offsets"], g["graph"]["col_idx"])
    exp = g[case]
    r = oracle.run(csr, variant, max_iters=20, seeds=exp.get("seeds"), gamma=exp.get("gamma", 0.0),
                   trace=True)
    assert r.trace.tolist() == exp["trajectory"]
    assert list(r.changed) == exp["changed"]
    assert r.iterations == exp["iterations"] and r.stop_reason == exp["stop_reason"]


def test_bowtie_llp_gamma_half_same_trajectory(golden_dir):
    # gamma = 0.5 gives the same trajectory as gamma = 1 on the bowtie.
    g = json.load(open(os.path.join(golden_dir, "bowtie.json")))
    csr = from_arrays(g["graph"]["n"], g["graph"]["row_offsets"], g["graph"]["col_idx"])
    n, off, col = _np(csr)
    hist, changed, reason = bruteforce.run(n, off, col, 2, 20, gamma=0.5)
    r = oracle.run(csr, oracle.LLP, gamma=0.5, trace=True)
    assert r.trace.tolist() == hist and r.stop_reason == reason == 2


# --------------------------------------------------------------------------- closed forms
def test_first_iteration_is_min_neighbour():
    """Unique labels => every count is 1 => L_1[v] = min N(v) [P:68] + R4."""
    for csr in [graphs.rmat(10, seed=3), graphs.gnp(60, 0.1, seed=5), graphs.karate()]:
        n, off, col = _np(csr)
        for variant, gamma in [(oracle.CLASSIC, 0.0), (oracle.LLP, 1.0), (oracle.LLP, 0.37)]:
            r = oracle.run(csr, variant, max_iters=1, gamma=gamma)
            exp = np.arange(n, dtype=np.int32)
            for v in range(n):
                if off[v + 1] > off[v]:
                    exp[v] = col[off[v]:off[v + 1]].min()
            assert (r.labels == exp).all()


def test_seeded_first_iteration_min_seed_neighbour():
    csr, seeds = graphs.taobao(users=4000, items=1000, pairs=20000, rings=10, seed=3)
    n, off, col = _np(csr)
    S = set(int(s) for s in seeds.tolist())
    r = oracle.run(csr, oracle.SEEDED, max_iters=1, seeds=seeds.numpy())
    for v in range(n):
        nb = [int(u) for u in col[off[v]:off[v + 1]] if int(u) in S]
        if v in S:
            assert r.labels[v] == v
        elif nb:
            assert r.labels[v] == min(nb)
        else:
            assert r.labels[v] == -1


@pytest.mark.parametrize("sizes", [[3], [4], [3, 5, 7], [10, 3, 6]])
def test_disjoint_cliques(sizes):
    """K_k, k>=3: t=1 every vertex changes (min vertex takes 2nd smallest id,
    the rest take the min); t=2 only the min vertex changes back; t=3 fixed."""
    csr = graphs.cliques(sizes)
    r = oracle.run(csr, oracle.CLASSIC, max_iters=20)
    exp, base = [], 0
    for k in sizes:
        exp += [base] * k
        base += k
    assert r.labels.tolist() == exp
    assert list(r.changed) == [sum(sizes), len(sizes), 0]
    assert r.iterations == 3 and r.stop_reason == oracle.STOP_FIXED_POINT


def test_k2_two_cycle():
    """K2: labels swap every iteration; L_2 == L_0 -> two-cycle at t=2."""
    r = oracle.run(graphs.path(2), oracle.CLASSIC, trace=True)
    assert r.trace.tolist() == [[1, 0], [0, 1]]
    assert r.iterations == 2 and r.stop_reason == oracle.STOP_TWO_CYCLE


@pytest.mark.parametrize("leaves", [1, 2, 5, 40])
def test_star_two_cycle(leaves):
    """Star: L1=[1,0..0], L2=[0,1..1], L3=L1 -> two-cycle at t=3 (t=2 if 1 leaf)."""
    r = oracle.run(graphs.star(leaves), oracle.CLASSIC, trace=True)
    l1 = [1] + [0] * leaves
    l2 = [0] + [1] * leaves
    if leaves == 1:
        assert r.trace.tolist() == [l1, l2] and r.iterations == 2
    else:
        assert r.trace.tolist() == [l1, l2, l1] and r.iterations == 3
    assert r.stop_reason == oracle.STOP_TWO_CYCLE


def test_no_2cycle_stop_runs_to_max_iters():
    r = oracle.run(graphs.path(2), oracle.CLASSIC, max_iters=7, stop_on_2cycle=False)
    assert r.iterations == 7 and r.stop_reason == oracle.STOP_MAX_ITERS
    assert r.labels.tolist() == [1, 0]


def test_isolated_and_zero_iters():
    r = oracle.run(graphs.empty(5), oracle.CLASSIC)
    assert r.labels.tolist() == list(range(5)) and r.iterations == 1
    assert r.stop_reason == oracle.STOP_FIXED_POINT
    r = oracle.run(graphs.karate(), oracle.CLASSIC, max_iters=0)
    assert r.labels.tolist() == list(range(34)) and r.iterations == 0


# --------------------------------------------------------------------------- brute force
@pytest.mark.parametrize("seed", range(12))
def test_bruteforce_tiny_random(seed):
    n = 4 + seed % 9
    csr = graphs.gnp(n, 0.35, seed=seed)
    nn, off, col = _np(csr)
    seeds = [v for v in range(n) if (v * 7 + seed) % 5 == 0]
    for variant, gamma, sd in [(0, 0.0, ()), (2, 1.0, ()), (2, 0.3, ()), (2, 0.125, ()),
                               (1, 0.0, seeds)]:
        hist, changed, reason = bruteforce.run(n, off, col, variant, 12, seeds=sd, gamma=gamma)
        r = oracle.run(csr, variant, max_iters=12, seeds=list(sd) if variant == 1 else None,
                       gamma=gamma, trace=True)
        assert r.trace.tolist() == hist, (variant, gamma)
        assert list(r.changed) == changed and r.stop_reason == reason


def test_bruteforce_multiedge_free_bipartite_and_path():
    for csr in [graphs.complete_bipartite(3, 4), graphs.path(6), graphs.bowtie(), graphs.star(6)]:
        n, off, col = _np(csr)
        hist, changed, reason = bruteforce.run(n, off, col, 0, 20)
        r = oracle.run(csr, oracle.CLASSIC, trace=True)
        assert r.trace.tolist() == hist and r.stop_reason == reason


def test_known_two_cycles():
    # K_{3,4} 2-cycles at t=3 and P6 at t=6 (re-derived by brute force above)
    r = oracle.run(graphs.complete_bipartite(3, 4), oracle.CLASSIC)
    assert (r.iterations, r.stop_reason) == (3, oracle.STOP_TWO_CYCLE)
    r = oracle.run(graphs.path(6), oracle.CLASSIC)
    assert (r.iterations, r.stop_reason) == (6, oracle.STOP_TWO_CYCLE)


# --------------------------------------------------------------------------- invariants
def _check_mfl_invariant(csr, prev, cur, variant=0, gamma=0.0, seeds=()):
    """cur[v] has max score among the labels in N(v); no smaller label ties."""
    n, off, col = _np(csr)
    S = set(int(s) for s in seeds)
    V = np.bincount(prev[prev >= 0], minlength=n) if variant == 2 else None
    for v in range(n):
        nb = prev[col[off[v]:off[v + 1]]]
        nb = nb[nb >= 0]
        if (variant == 1 and v in S) or nb.size == 0:
            assert cur[v] == prev[v]
            continue
        labs, ks = np.unique(nb, return_counts=True)
        if variant == 2:
            sc = ks.astype(np.float64) - gamma * (V[labs].astype(np.float64) - ks.astype(np.float64))
        else:
            sc = ks
        best = sc.max()
        assert labs[sc == best].min() == cur[v]


def test_mfl_invariant_rmat_sbm():
    for csr in [graphs.rmat(11, seed=2), graphs.sbm(n=3000, k=30, m=30000, seed=4)]:
        r = oracle.run(csr, oracle.CLASSIC, max_iters=6, trace=True)
        prev = np.arange(csr.n, dtype=np.int32)
        for t in range(r.iterations):
            _check_mfl_invariant(csr, prev, r.trace[t])
            prev = r.trace[t]
        r = oracle.run(csr, oracle.LLP, gamma=0.25, max_iters=4, trace=True)
        prev = np.arange(csr.n, dtype=np.int32)
        for t in range(r.iterations):
            _check_mfl_invariant(csr, prev, r.trace[t], 2, 0.25)
            prev = r.trace[t]


def test_llp_gamma0_equals_classic():
    """gamma = 0 turns val = k - gamma*(v-k) into val = k [P:119]."""
    for csr in [graphs.rmat(12, seed=7), graphs.karate(), graphs.sbm(n=2000, k=20, m=20000, seed=1)]:
        a = oracle.run(csr, oracle.CLASSIC, max_iters=15, trace=True)
        b = oracle.run(csr, oracle.LLP, gamma=0.0, max_iters=15, trace=True)
        assert (a.trace == b.trace).all() and a.iterations == b.iterations


def test_fixed_point_is_self_consistent():
    csr = graphs.cliques([5, 6, 3])
    r = oracle.run(csr, oracle.CLASSIC)
    assert r.stop_reason == oracle.STOP_FIXED_POINT
    r1 = oracle.run(csr, oracle.CLASSIC, max_iters=r.iterations + 3)
    assert (r1.labels == r.labels).all()


# --------------------------------------------------------------------------- seeded BFS pin
def test_seeded_bfs_reach():
    """SEEDED: v is labelled after t iterations iff dist(v, S) <= t (BFS);
    seeds keep their own id; the labelled set only grows."""
    csr, seeds = graphs.taobao(users=3000, items=800, pairs=6000, rings=5, seed=11)
    n, off, col = _np(csr)
    G = nx.Graph()
    G.add_nodes_from(range(n))
    for v in range(n):
        for u in col[off[v]:off[v + 1]]:
            G.add_edge(v, int(u))
    S = [int(s) for s in seeds.tolist()]
    dist = nx.multi_source_dijkstra_path_length(G, S)
    r = oracle.run(csr, oracle.SEEDED, seeds=S, max_iters=30, trace=True)
    for t in range(r.iterations):
        lab = r.trace[t] >= 0
        exp = np.array([dist.get(v, 10 ** 9) <= t + 1 for v in range(n)])
        assert (lab == exp).all(), t
        assert all(r.trace[t][s] == s for s in S)


# --------------------------------------------------------------------------- modularity
def test_modularity_networkx():
    G = nx.karate_club_graph()
    k = graphs.karate()
    parts = [{v for v in G if graphs.KARATE_CLUB[v] == c} for c in (0, 1)]
    q_nx = nx.algorithms.community.modularity(G, parts, weight=None)
    assert abs(oracle.modularity(k, graphs.KARATE_CLUB) - q_nx) < 1e-12
    assert abs(oracle.modularity(k, [0] * 34)) < 1e-15
    csr = graphs.sbm(n=2000, k=20, m=20000, seed=9)
    n, off, col = _np(csr)
    Gs = nx.Graph()
    Gs.add_nodes_from(range(n))
    for v in range(n):
        for u in col[off[v]:off[v + 1]]:
            Gs.add_edge(v, int(u))
    r = oracle.run(csr, oracle.CLASSIC)
    comms = {}
    for v, l in enumerate(r.labels.tolist()):
        comms.setdefault(l, set()).add(v)
    q_nx = nx.algorithms.community.modularity(Gs, list(comms.values()), weight=None)
    assert abs(oracle.modularity(csr, r.labels) - q_nx) < 1e-9


# --------------------------------------------------------------------------- regression / determinism
def test_karate_regression():
    """Regression value (probe; not a paper number): 11 iterations,
    fixed point, all labels 0.  The include-own-label reading (R2) gives 4."""
    r = oracle.run(graphs.karate(), oracle.CLASSIC)
    assert r.iterations == 11 and r.stop_reason == oracle.STOP_FIXED_POINT
    assert list(r.changed) == [34, 21, 17, 14, 13, 13, 14, 11, 9, 2, 0]
    assert (r.labels == 0).all()


def test_threads_do_not_change_results():
    csr = graphs.rmat(13, seed=5)
    a = oracle.run(csr, oracle.CLASSIC, threads=1, trace=True)
    b = oracle.run(csr, oracle.CLASSIC, threads=4, trace=True)
    assert (a.trace == b.trace).all()
    a = oracle.run(csr, oracle.LLP, gamma=1.0, max_iters=5, threads=1, trace=True)
    b = oracle.run(csr, oracle.LLP, gamma=1.0, max_iters=5, threads=3, trace=True)
    assert (a.trace == b.trace).all()
