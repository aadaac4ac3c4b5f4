"""Quick timing probe: generate a graph on the GPU, run LP, print per-iteration stats."""
import sys, time, json, torch
sys.path.insert(0, '.')
import paper_conf_sigmod_yelhls21_b200 as glp
from glp_inputs import graphs
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 20
import os
VAR = os.environ.get('GLP_VARIANT', 'classic')
GAMMA = float(os.environ.get('GLP_GAMMA', '1.0' if VAR == 'llp' else '0'))
t0 = time.time()
_seeds = None
if os.environ.get('GLP_GRAPH'):
    csr, _seeds = graphs.make(os.environ['GLP_GRAPH'], device='cuda')
else:
    csr = graphs.rmat(scale, seed=1, device='cuda', buckets=16 if scale >= 27 else 0)
torch.cuda.synchronize()
print('gen', scale, csr.nnz, round(time.time() - t0, 2), 's', flush=True)
g = glp.Graph(csr)
print(json.dumps(g.info()), flush=True)
for rep in range(int(os.environ.get('GLP_REPS', '3'))):
    info = g.run(VAR, 20, _seeds if VAR == 'seeded' else None, gamma=GAMMA, profile=(rep == 2))
    print(info, flush=True)
for s in g.iter_stats():
    print({k: (round(v, 4) if isinstance(v, float) else v) for k, v in s.items()})
for k in g.kernel_stats():
    if k['launches']:
        print(k['name'], k['launches'], round(k['ms'], 3), 'ms', round(k['bytes'] / max(k['ms'], 1e-9) / 1e6, 1), 'GB/s alg',
              round(k['arcs'] / max(k['ms'], 1e-9) / 1e6, 2), 'Garcs/s')
# per-iteration kernel breakdown (profiled runs of 1..4 iterations, differences)
prev, preva = {}, {}
for t in range(1, int(sys.argv[2]) + 1 if len(sys.argv) > 2 else 5):
    g.run(VAR, t, _seeds if VAR == 'seeded' else None, gamma=GAMMA, profile=True)
    cur = {k['name']: k['ms'] for k in g.kernel_stats()}
    cura = {k['name']: k['arcs'] for k in g.kernel_stats()}
    print('iter', t, {k: round(cur[k] - prev.get(k, 0), 3) for k in cur if cur[k] - prev.get(k, 0) > 0})
    print('arcs', t, {k: round((cura[k] - preva.get(k, 0)) / 1e6, 1) for k in cura if cura[k] - preva.get(k, 0) > 0})
    prev, preva = cur, cura
