"""Seeded synthetic graphs with the shapes of the paper's workloads.

Recipes (also in DESIGN.md §Inputs):

* ``karate``      Zachary's karate club, 34 v / 78 e (BASELINE.json configs[0]);
                  edge list stored below in networkx ordering.
* ``bowtie``      two triangles sharing vertex 2 (hand-checkable).
* ``cliques``     disjoint K_k, ``path``, ``complete_bipartite``, ``star``,
                  ``gnp`` (tiny random graphs for brute-force pins).
* ``sbm``         planted partition: k contiguous blocks, m sampled pairs, a
                  fraction (1-mu) drawn inside a uniform block, mu uniform over
                  all vertices (configs[1]: 1M v, 1k blocks, 20M pairs, mu=0.1).
                  The paper's "community property" premise [P:52, P:130].
* ``rmat``        Graph500 Kronecker (a,b,c,d)=(0.57,0.19,0.19,0.05), 2^s
                  vertices, ef*2^s pairs, Graph500-style vertex scramble
                  (configs[2]: s=24, ef=16; configs[4]: s=28).  Power-law skew
                  like twitter/uk-2002 [P:255-264].
* ``taobao``      bipartite user-item transaction window (configs[3]): Chung-Lu
                  pairs with truncated power-law weights, planted complete
                  bipartite fraud rings, 0.1 % of users as black-listed seeds
                  [P:33, Table 4 P:337-347].

Everything is a deterministic function of (parameters, seed) through
``glp_inputs.rng`` and runs on CPU or CUDA with identical results.  No
label-propagation arithmetic lives here.
"""
from __future__ import annotations

import math

import torch

from . import rng
from .csr import CSR, from_edges

KARATE_EDGES = [
    (0, 1), (0, 2), (0, 3), (0, 4), (0, 5), (0, 6), (0, 7), (0, 8), (0, 10), (0, 11), (0, 12),
    (0, 13), (0, 17), (0, 19), (0, 21), (0, 31), (1, 2), (1, 3), (1, 7), (1, 13), (1, 17),
    (1, 19), (1, 21), (1, 30), (2, 3), (2, 7), (2, 8), (2, 9), (2, 13), (2, 27), (2, 28), (2, 32),
    (3, 7), (3, 12), (3, 13), (4, 6), (4, 10), (5, 6), (5, 10), (5, 16), (6, 16), (8, 30), (8, 32),
    (8, 33), (9, 33), (13, 33), (14, 32), (14, 33), (15, 32), (15, 33), (18, 32), (18, 33),
    (19, 33), (20, 32), (20, 33), (22, 32), (22, 33), (23, 25), (23, 27), (23, 29), (23, 32),
    (23, 33), (24, 25), (24, 27), (24, 31), (25, 31), (26, 29), (26, 33), (27, 33), (28, 31),
    (28, 33), (29, 32), (29, 33), (30, 32), (30, 33), (31, 32), (31, 33), (32, 33),
]
# Zachary's two factions ("Mr. Hi" = 0, "Officer" = 1), networkx ordering.
KARATE_CLUB = [0, 0, 0, 0, 0, 0, 0, 0, 0, 1, 0, 0, 0, 0, 1, 1, 0, 0, 1, 0, 1, 0, 1, 1, 1, 1, 1,
               1, 1, 1, 1, 1, 1, 1]


def _edges(n, pairs, name, device="cpu") -> CSR:
    if pairs:
        t = torch.tensor(pairs, dtype=torch.int64, device=device)
        return from_edges(n, t[:, 0], t[:, 1], name)
    z = torch.zeros(0, dtype=torch.int64, device=device)
    return from_edges(n, z, z, name)


def karate(device="cpu") -> CSR:
    return _edges(34, KARATE_EDGES, "karate", device)


def bowtie(device="cpu") -> CSR:
    """Two triangles {0,1,2} and {2,3,4} sharing vertex 2."""
    return _edges(5, [(0, 1), (0, 2), (1, 2), (2, 3), (2, 4), (3, 4)], "bowtie", device)


def cliques(sizes, device="cpu") -> CSR:
    pairs, base = [], 0
    for k in sizes:
        pairs += [(base + i, base + j) for i in range(k) for j in range(i + 1, k)]
        base += k
    return _edges(base, pairs, f"cliques{list(sizes)}", device)


def path(n, device="cpu") -> CSR:
    return _edges(n, [(i, i + 1) for i in range(n - 1)], f"path{n}", device)


def complete_bipartite(a, b, device="cpu") -> CSR:
    return _edges(a + b, [(i, a + j) for i in range(a) for j in range(b)], f"K{a},{b}", device)


def star(leaves, device="cpu") -> CSR:
    return _edges(leaves + 1, [(0, i + 1) for i in range(leaves)], f"star{leaves}", device)


def empty(n, device="cpu") -> CSR:
    return _edges(n, [], f"empty{n}", device)


def gnp(n: int, p: float, seed: int, device="cpu") -> CSR:
    """Erdos-Renyi G(n, p) (tiny graphs for brute-force pins)."""
    iu = torch.triu_indices(n, n, offset=1, device=device)
    idx = torch.arange(iu.shape[1], dtype=torch.int64, device=device)
    keep = rng.uniform(seed, 11, idx) < p
    return from_edges(n, iu[0][keep], iu[1][keep], f"gnp{n},{p},{seed}")


def random_multidegree(n: int, m: int, seed: int, device="cpu") -> CSR:
    """m uniform random pairs over n vertices (a simple test graph)."""
    idx = torch.arange(m, dtype=torch.int64, device=device)
    src = rng.randint(seed, 21, idx, n)
    dst = rng.randint(seed, 22, idx, n)
    return from_edges(n, src, dst, f"rand{n},{m},{seed}")


def sbm(n: int = 1_000_000, k: int = 1000, m: int = 20_000_000, mu: float = 0.1,
        seed: int = 42, device="cpu") -> CSR:
    """Planted partition: k contiguous blocks of n//k ids (configs[1])."""
    assert n % k == 0
    bs = n // k
    idx = torch.arange(m, dtype=torch.int64, device=device)
    intra = rng.uniform(seed, 1, idx) >= mu
    blk = rng.randint(seed, 2, idx, k)
    a_in = blk * bs + rng.randint(seed, 3, idx, bs)
    b_in = blk * bs + rng.randint(seed, 4, idx, bs)
    a_out = rng.randint(seed, 5, idx, n)
    b_out = rng.randint(seed, 6, idx, n)
    src = torch.where(intra, a_in, a_out)
    dst = torch.where(intra, b_in, b_out)
    del a_in, b_in, a_out, b_out, blk, intra
    return from_edges(n, src, dst, f"sbm{n},{k},{m},{mu}")


def rmat_pairs(scale: int, edge_factor: int = 16, seed: int = 1, a=0.57, b=0.19, c=0.19,
               device="cpu", chunk: int = 1 << 26, scramble: bool = True):
    """Graph500 Kronecker generator: (src, dst) int64 of edge_factor*2^scale pairs.

    At each of ``scale`` levels a quadrant is drawn with probabilities
    (a, b, c, 1-a-b-c); the row bit is set for quadrants c,d and the column
    bit for b,d.  Vertex ids are then scrambled by a seeded permutation.
    (Graph500's per-level probability noise is not applied.)
    """
    n = 1 << scale
    m = edge_factor * n
    ab, abc = a + b, a + b + c
    src = torch.empty(m, dtype=torch.int64, device=device)
    dst = torch.empty(m, dtype=torch.int64, device=device)
    for s0 in range(0, m, chunk):
        s1 = min(m, s0 + chunk)
        idx = torch.arange(s0, s1, dtype=torch.int64, device=device)
        r = torch.zeros_like(idx)
        cc = torch.zeros_like(idx)
        for lvl in range(0, scale, 2):
            u0, u1 = rng.uniform_pair(seed, 100 + lvl // 2, idx)
            for j, u in enumerate((u0, u1)):
                if lvl + j >= scale:
                    break
                bit = 1 << (lvl + j)
                rbit = u >= ab                      # quadrants c, d
                cbit = ((u >= a) & (u < ab)) | (u >= abc)  # quadrants b, d
                r |= rbit.to(torch.int64) * bit
                cc |= cbit.to(torch.int64) * bit
        src[s0:s1] = r
        dst[s0:s1] = cc
    if scramble:
        perm = rng.permutation(seed, 99, n, device)
        src = perm[src]
        dst = perm[dst]
    return n, src, dst


def _rmat_chunk(scale, lo, hi, seed, a, ab, abc, device):
    """(row, col) of Kronecker pairs [lo, hi) before the scramble (rmat_pairs' draws)."""
    idx = torch.arange(lo, hi, dtype=torch.int64, device=device)
    r = torch.zeros_like(idx)
    cc = torch.zeros_like(idx)
    for lvl in range(0, scale, 2):
        u0, u1 = rng.uniform_pair(seed, 100 + lvl // 2, idx)
        for j, u in enumerate((u0, u1)):
            if lvl + j >= scale:
                break
            bit = 1 << (lvl + j)
            r |= (u >= ab).to(torch.int64) * bit
            cc |= (((u >= a) & (u < ab)) | (u >= abc)).to(torch.int64) * bit
    return r, cc


def rmat(scale: int, edge_factor: int = 16, seed: int = 1, device="cpu", scramble=True,
         buckets: int = 0) -> CSR:
    """RMAT CSR = from_edges(rmat_pairs(...)).  buckets > 1 builds the same CSR
    in row buckets (pairs generated chunk by chunk, each directed arc kept as a
    bucket-local int64 key) so that scale 28 (2^32 pairs, ~8.5e9 arcs) fits in
    one GPU's memory; the result is identical to the unbucketed build."""
    if buckets <= 1:
        n, src, dst = rmat_pairs(scale, edge_factor, seed, device=device, scramble=scramble)
        return from_edges(n, src, dst, f"rmat{scale}ef{edge_factor}")
    n = 1 << scale
    m = edge_factor * n
    a, b, c = 0.57, 0.19, 0.19
    perm = rng.permutation(seed, 99, n, device) if scramble else None
    width = (n + buckets - 1) // buckets
    keys = [[] for _ in range(buckets)]
    chunk = 1 << 26
    for s0 in range(0, m, chunk):
        r, cc = _rmat_chunk(scale, s0, min(m, s0 + chunk), seed, a, a + b, a + b + c, device)
        if perm is not None:
            r, cc = perm[r], perm[cc]
        keep = r != cc
        r, cc = r[keep], cc[keep]
        src, dst = torch.cat([r, cc]), torch.cat([cc, r])  # symmetrise (R1)
        del r, cc, keep
        bk = torch.div(src, width, rounding_mode="floor")
        order = torch.argsort(bk, stable=True)
        src, dst, bk = src[order], dst[order], bk[order]
        cnt = torch.bincount(bk, minlength=buckets).tolist()
        pos = 0
        for i, k in enumerate(cnt):
            if k:
                keys[i].append((src[pos:pos + k] - i * width) * n + dst[pos:pos + k])
            pos += k
        del src, dst, bk, order
    off = torch.zeros(n + 1, dtype=torch.int64, device=device)
    cols = []
    base = 0
    for i in range(buckets):
        r0, r1 = i * width, min(n, (i + 1) * width)
        if keys[i]:
            key = torch.unique(torch.cat(keys[i]))  # sorted, deduplicated
        else:
            key = torch.zeros(0, dtype=torch.int64, device=device)
        keys[i] = None
        rows = torch.div(key, n, rounding_mode="floor")
        cols.append((key - rows * n).to(torch.int32))
        counts = torch.bincount(rows, minlength=r1 - r0)
        off[r0 + 1:r1 + 1] = base + torch.cumsum(counts, 0)
        base += int(key.numel())
        del key, rows, counts
    col = torch.cat(cols) if len(cols) > 1 else cols[0]
    del cols
    return CSR(n, off, col.contiguous(), f"rmat{scale}ef{edge_factor}", True)


def _trunc_powerlaw_quantiles(count: int, alpha: float, lo: float, hi: float, device):
    """Deterministic weights: quantiles of a power law p(x) ~ x^-alpha on [lo, hi]."""
    q = (torch.arange(count, dtype=torch.float64, device=device) + 0.5) / count
    e = 1.0 - alpha
    a, b = lo ** e, hi ** e
    return (a + q * (b - a)) ** (1.0 / e)


def _cdf(w: torch.Tensor):
    """Normalised running sum of w, accumulated sequentially (numpy)."""
    import numpy as np
    c = np.cumsum(w.numpy())
    return c / c[-1]


def taobao(users: int = 80_000_000, items: int = 20_000_000, pairs: int = 1_000_000_000,
           rings: int = 10_000, ring_users: int = 20, ring_items: int = 5,
           seeds_per_ring: int = 4, seed_frac: float = 0.001, seed: int = 7,
           device="cpu", chunk: int = 1 << 26):
    """TaoBao-shaped bipartite transaction window (configs[3]).

    Users 0..U-1 and items U..U+I-1 before scrambling.  ``pairs`` (user,item)
    pairs are drawn Chung-Lu style: user ~ w_u (power law, exponent 2.5 on
    [1, 2000]) and item ~ w_i (exponent 2.0 on [1, 5e6]) by inverse-CDF search.
    ``rings`` complete bipartite fraud rings (ring_users x ring_items) are
    planted on users [r*ring_users, ...) and items [r*ring_items, ...).
    Seeds: ``seeds_per_ring`` users of every ring plus uniform users up to
    ``seed_frac`` of all users.  Returns (CSR, seeds int32 tensor).
    """
    n = users + items
    # the inverse-CDF tables are built on the host (sequential float64
    # cumsum): a parallel device scan rounds in a run-dependent order, which
    # made the 100M-vertex graph differ from run to run
    cu = torch.from_numpy(_cdf(_trunc_powerlaw_quantiles(users, 2.5, 1.0, 2000.0, "cpu").flip(0))).to(device)
    ci = torch.from_numpy(_cdf(_trunc_powerlaw_quantiles(items, 2.0, 1.0, 5e6, "cpu").flip(0))).to(device)
    srcs, dsts = [], []
    for s0 in range(0, pairs, chunk):
        s1 = min(pairs, s0 + chunk)
        idx = torch.arange(s0, s1, dtype=torch.int64, device=device)
        uu, ui = rng.uniform_pair(seed, 1, idx)
        u = torch.searchsorted(cu, uu, right=True).clamp_(max=users - 1)
        it = torch.searchsorted(ci, ui, right=True).clamp_(max=items - 1) + users
        srcs.append(u)
        dsts.append(it)
    rings = min(rings, users // ring_users, items // ring_items)
    if rings > 0:
        r = torch.arange(rings, dtype=torch.int64, device=device)
        ru = torch.arange(ring_users, dtype=torch.int64, device=device)
        ri = torch.arange(ring_items, dtype=torch.int64, device=device)
        ring_u = (r[:, None, None] * ring_users + ru[None, :, None]).expand(rings, ring_users, ring_items)
        ring_i = (users + r[:, None, None] * ring_items + ri[None, None, :]).expand(rings, ring_users, ring_items)
        srcs.append(ring_u.reshape(-1))
        dsts.append(ring_i.reshape(-1))
    src = torch.cat(srcs)
    dst = torch.cat(dsts)
    del srcs, dsts
    # seeds (pre-scramble ids)
    n_seeds_total = max(1, int(round(seed_frac * users)))
    ring_seeds = []
    if rings > 0:
        ring_seeds = (torch.arange(rings, dtype=torch.int64, device=device)[:, None] * ring_users
                      + torch.arange(min(seeds_per_ring, ring_users), dtype=torch.int64, device=device)[None, :]).reshape(-1)
    n_uniform = max(0, n_seeds_total - (len(ring_seeds) if rings > 0 else 0))
    first_free = rings * ring_users
    pool = users - first_free
    uni = torch.zeros(0, dtype=torch.int64, device=device)
    if n_uniform > 0 and pool > 0:
        h = rng.hash64(seed, 2, torch.arange(pool, dtype=torch.int64, device=device))
        uni = torch.sort(h, stable=True).indices[:n_uniform] + first_free
    seeds = torch.cat([ring_seeds, uni]) if rings > 0 else uni
    perm = rng.permutation(seed, 99, n, device)
    src = perm[src]
    dst = perm[dst]
    seeds = torch.sort(perm[seeds]).values.to(torch.int32)
    csr = from_edges(n, src, dst, f"taobao{users},{items},{pairs}")
    return csr, seeds


CONFIGS = {
    "karate": dict(kind="karate"),
    "sbm1m": dict(kind="sbm", n=1_000_000, k=1000, m=20_000_000, mu=0.1, seed=42),
    "rmat24": dict(kind="rmat", scale=24, edge_factor=16, seed=1),
    "taobao100m": dict(kind="taobao", users=80_000_000, items=20_000_000, pairs=1_000_000_000, seed=7),
    "rmat28": dict(kind="rmat", scale=28, edge_factor=16, seed=1, buckets=16),
}


def make(name_or_kind: str, device="cpu", **kw):
    """Build a named config (``CONFIGS``) or a generator kind with overrides.

    Returns (CSR, seeds-or-None).
    """
    spec = dict(CONFIGS.get(name_or_kind, dict(kind=name_or_kind)))
    spec.update(kw)
    kind = spec.pop("kind")
    if kind == "karate":
        return karate(device), None
    if kind == "sbm":
        return sbm(device=device, **spec), None
    if kind == "rmat":
        return rmat(device=device, **spec), None
    if kind == "taobao":
        return taobao(device=device, **spec)
    raise ValueError(f"unknown graph kind {kind}")


def lcg_degrees_hint(csr: CSR) -> dict:
    """Degree-bin summary (arcs and vertices per bin) for reports."""
    deg = csr.degrees()
    out = {}
    edges = [0, 1, 33, 257, 4097, 1 << 62]
    names = ["0", "1-32", "33-256", "257-4096", ">4096"]
    for nm, lo, hi in zip(names, edges[:-1], edges[1:]):
        msk = (deg >= lo) & (deg < hi)
        out[nm] = dict(vertices=int(msk.sum()), arcs=int(deg[msk].sum()))
    out["max_degree"] = int(deg.max()) if deg.numel() else 0
    out["log2_n"] = math.log2(max(csr.n, 1))
    return out


def edge_weights(csr: CSR, seed: int = 5, hi: int = 8) -> torch.Tensor:
    """Integer arc weights in [1, hi] (weighted LP, §8(f)3), symmetric: arc
    (u, v) and arc (v, u) get the same weight (a counter-based hash of the
    unordered pair).  int32 tensor on the CSR's device."""
    off = csr.row_offsets
    deg = off[1:] - off[:-1]
    rows = torch.repeat_interleave(torch.arange(csr.n, device=off.device), deg)
    cols = csr.col_idx.to(torch.int64)
    key = torch.minimum(rows, cols) * csr.n + torch.maximum(rows, cols)
    return (rng.hash64(seed, 31, key) % hi + 1).to(torch.int32)
