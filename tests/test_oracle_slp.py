"""Pins of the SLP oracle (§8(f)3: speaker-listener LP [P:120], 5 labels and
20 iterations [P:270]; readings R19 in DESIGN.md).

  * one memory slot, no threshold: the speakers follow the classic LP
    trajectory exactly (the pinned classic oracle), iteration by iteration;
  * count conservation: without threshold and with room for every label, a
    vertex with neighbours gains exactly one count per iteration;
  * a threshold above one half leaves exactly one label per vertex;
  * brute force (pure-Python memories) on tiny graphs, several K and r.
"""
import numpy as np
import pytest

import oracle
from glp_inputs import graphs


@pytest.mark.parametrize("T", [1, 2, 3, 5, 8])
def test_one_slot_is_classic(T):
    csr = graphs.rmat(11, seed=7)
    ml, mc, sp = oracle.run_slp(csr, K=1, r=0.0, max_iters=T)
    ref = oracle.run(csr, oracle.CLASSIC, T, stop_on_2cycle=False)
    assert (sp == ref.labels).all()
    assert (ml[:, 0] == sp).all()


def test_count_conservation():
    csr = graphs.sbm(n=2000, k=20, m=20000, mu=0.2, seed=3)
    T = 7
    ml, mc, sp = oracle.run_slp(csr, K=T + 1, r=0.0, max_iters=T)
    deg = np.diff(csr.numpy()[0])
    tot = np.where(ml >= 0, mc, 0).sum(1)
    assert (tot[deg > 0] == T + 1).all() and (tot[deg == 0] == 1).all()


def test_high_threshold_keeps_one_label():
    csr = graphs.rmat(10, seed=2)
    ml, mc, sp = oracle.run_slp(csr, K=5, r=0.6, max_iters=10)
    assert ((ml >= 0).sum(1) == 1).all()
    assert (ml.max(1) == sp).all()


def brute(n, off, col, K, r, T):
    mem = [[(v, 1)] + [None] * (K - 1) for v in range(n)]

    def speak(m):
        live = [x for x in m if x is not None]
        top = max(c for _, c in live)
        return min(l for l, c in live if c == top)
    for t in range(1, T + 1):
        S = [speak(mem[v]) for v in range(n)]
        for v in range(n):
            nb = [S[col[e]] for e in range(off[v], off[v + 1])]
            if nb:
                cnt = {}
                for x in nb:
                    cnt[x] = cnt.get(x, 0) + 1
                top = max(cnt.values())
                m = min(l for l, c in cnt.items() if c == top)
                slots = mem[v]
                hit = [k for k, x in enumerate(slots) if x is not None and x[0] == m]
                if hit:
                    slots[hit[0]] = (m, slots[hit[0]][1] + 1)
                elif None in slots:
                    slots[slots.index(None)] = (m, 1)
                else:
                    low = min(range(K), key=lambda k: (slots[k][1], -slots[k][0]))
                    slots[low] = (m, 1)
            slots = mem[v]
            live = [k for k, x in enumerate(slots) if x is not None]
            keep = min(live, key=lambda k: (-slots[k][1], slots[k][0]))
            for k in live:
                if k != keep and slots[k][1] < r * (t + 1):
                    slots[k] = None
    ml = np.array([[-1 if x is None else x[0] for x in m] for m in mem], dtype=np.int32)
    mc = np.array([[0 if x is None else x[1] for x in m] for m in mem], dtype=np.int32)
    return ml, mc


@pytest.mark.parametrize("seed", range(6))
def test_bruteforce_tiny(seed):
    g = np.random.default_rng(seed)
    n = int(g.integers(4, 12))
    csr = graphs.gnp(n, 0.4, seed)
    off, col = csr.numpy()
    K = int(g.integers(1, 4))
    r = [0.0, 0.3, 0.15][seed % 3]
    T = 9
    ml, mc, sp = oracle.run_slp(csr, K=K, r=r, max_iters=T)
    bl, bc = brute(n, off, col, K, r, T)
    assert (ml == bl).all() and (mc == bc).all()
