import sys, torch
sys.path.insert(0, '.')
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
spec, variant, max_iters, gamma = bench.WORKLOADS['taobao100m']
csr, seeds = bench.make_graph(spec, 'cuda')
g = glp.Graph(csr)
deg = (csr.row_offsets[1:] - csr.row_offsets[:-1])
for t in range(1, 9):
    info = g.run(variant, t, seeds, gamma=gamma)
    lab = g.labels('cuda')
    m = lab >= 0
    # fraction of arcs whose source label is valid (gathered label >= 0): sum of degree of labelled vertices / nnz
    print(t, info.iterations, int(m.sum()), round(float(m.float().mean()), 4), round(float(deg[m].sum()) / csr.nnz, 4), flush=True)
