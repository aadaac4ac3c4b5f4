"""One profiled window for ncu (--profile-from-start off): a run of WORKLOAD
with ITERS iterations after a warm-up run; class kernels serialised."""
import os, sys, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
wl = sys.argv[1] if len(sys.argv) > 1 else 'rmat24'
iters = int(sys.argv[2]) if len(sys.argv) > 2 else 2
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
csr, seeds = bench.make_graph(spec, 'cuda')
torch.cuda.synchronize(); torch.cuda.empty_cache()
g = glp.Graph(csr)
print(g.run(variant, iters, seeds, gamma=gamma))
torch.cuda.synchronize()
torch.cuda.profiler.start()
print(g.run(variant, iters, seeds, gamma=gamma, profile=True))
torch.cuda.synchronize()
torch.cuda.profiler.stop()
