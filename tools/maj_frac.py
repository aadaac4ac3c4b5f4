"""Fraction of rows (and of arcs) whose own label L_{t-1}[v] is a strict
majority of their neighbours' labels L_{t-1}[N(v)], per iteration (design probe)."""
import sys, torch
sys.path.insert(0, '.')
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
wl = sys.argv[1] if len(sys.argv) > 1 else 'rmat24'
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
csr, seeds = bench.make_graph(spec, 'cuda')
g = glp.Graph(csr)
off = csr.row_offsets
deg = off[1:] - off[:-1]
n = csr.n
row = torch.repeat_interleave(torch.arange(n, device='cuda'), deg)
col = csr.col_idx.long()
for t in range(1, 8):
    # L_{t-1}: labels after t-1 iterations
    if t == 1:
        L = torch.arange(n, device='cuda', dtype=torch.int32) if variant != 'seeded' else None
        if L is None: continue
    else:
        g.run(variant, t - 1, seeds, gamma=gamma)
        L = g.labels('cuda')
    eq = (L[col] == L[row]).to(torch.int32)
    c = torch.zeros(n, dtype=torch.int32, device='cuda').index_add_(0, row, eq)
    maj = (2 * c > deg) & (deg > 32)
    big = deg > 32
    print(t, 'rows>32', int(big.sum()), 'maj rows', round(float(maj.sum()) / max(int(big.sum()), 1), 3),
          'maj arcs', round(float(deg[maj].sum()) / max(float(deg[big].sum()), 1), 3),
          'low maj', round(float(((2 * c > deg) & (deg <= 32) & (deg > 0)).sum()) / max(int(((deg <= 32) & (deg > 0)).sum()), 1), 3), flush=True)
    del eq, c
