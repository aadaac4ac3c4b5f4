"""Brute-force LP for tiny graphs: an independent check of the oracle.

Written from the definition in PAPER.md [P:68 §2.1] (MFL among neighbours) and
[P:119 §3.1] (LLP score) with readings R2/R4/R5/R8/R12 -- but by a different
method than the oracle: for every vertex it enumerates every possible label
value and counts it with a Python loop (O(n * deg) per vertex), with no sort.
Use only on graphs with n <= ~64.
"""
from __future__ import annotations


def neighbours(off, col, v):
    return [int(col[e]) for e in range(int(off[v]), int(off[v + 1]))]


def step(n, off, col, L, variant, gamma=0.0, seeds=()):
    seeds = set(int(s) for s in seeds)
    V = {}
    if variant == 2:
        for lab in range(-1, n):
            V[lab] = sum(1 for w in range(n) if L[w] == lab)
    out = list(L)
    for v in range(n):
        if variant == 1 and v in seeds:
            continue
        nb = neighbours(off, col, v)
        best = None  # (score, label)
        for lab in range(0, n):           # every possible label value
            k = 0
            for u in nb:
                if L[u] == lab:
                    k += 1
            if k == 0:
                continue                  # only labels present among neighbours compete
            if variant == 2:
                score = float(k) - gamma * (float(V[lab]) - float(k))
            else:
                score = k
            if best is None or score > best[0]:   # labels visited ascending: first max = min label
                best = (score, lab)
        if best is not None:
            out[v] = best[1]
    return out


def run(n, off, col, variant=0, max_iters=20, seeds=(), gamma=0.0, stop_on_2cycle=True):
    if variant == 1:
        L = [v if v in set(seeds) else -1 for v in range(n)]
    else:
        L = list(range(n))
    hist = [L]
    changed = []
    reason = 0
    for t in range(1, max_iters + 1):
        nxt = step(n, off, col, hist[-1], variant, gamma, seeds)
        changed.append(sum(1 for v in range(n) if nxt[v] != hist[-1][v]))
        hist.append(nxt)
        if changed[-1] == 0:
            reason = 1
            break
        if stop_on_2cycle and t >= 2 and nxt == hist[-3]:
            reason = 2
            break
    return hist[1:], changed, reason
