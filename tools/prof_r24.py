"""One classic LP run on RMAT-S for ncu (kernels named mfl_*)."""
import sys, torch
sys.path.insert(0, '.')
import paper_conf_sigmod_yelhls21_b200 as glp
from glp_inputs import graphs
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 5
csr = graphs.rmat(scale, seed=1, device='cuda')
g = glp.Graph(csr)
print(g.run('classic', iters))
