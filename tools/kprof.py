"""Per-iteration kernel breakdown of a bench workload (profiled runs of
1..T iterations, differences of the per-kernel CUDA-event totals)."""
import os, sys, json, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
wl = sys.argv[1] if len(sys.argv) > 1 else 'rmat24'
T = int(sys.argv[2]) if len(sys.argv) > 2 else 5
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
csr, seeds = bench.make_graph(spec, 'cuda')
torch.cuda.synchronize(); torch.cuda.empty_cache()
g = glp.Graph(csr, weights=bench.workload_weights(wl, csr))
info = g.run(variant, max_iters, seeds, gamma=gamma, profile=True)
print(info)
print({k['name']: round(k['ms'], 3) for k in g.kernel_stats() if k['launches']})
prev = {}
for t in range(1, min(T, info.iterations) + 1):
    g.run(variant, t, seeds, gamma=gamma, profile=True)
    cur = {k['name']: k['ms'] for k in g.kernel_stats()}
    st = g.iter_stats()[-1]
    print('iter', t, 'dense' if st['dense'] else 'sparse', 'arcs %.1fM' % (st['active_arcs'] / 1e6),
          {k: round(cur[k] - prev.get(k, 0), 3) for k in cur if cur[k] - prev.get(k, 0) > 0.001})
    prev = cur
