"""Host-CSR create time of a bench workload (pinned buffers), for A/B of
libglp builds (GLP_LIB):  python tools/create_ab.py WORKLOAD [reps]"""
import os, sys, time, statistics, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
wl = sys.argv[1] if len(sys.argv) > 1 else "rmat24"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
csr, seeds = bench.make_graph(spec, "cuda")
off_h = csr.row_offsets.cpu().pin_memory(); col_h = csr.col_idx.cpu().pin_memory()
n, sym = csr.n, csr.symmetric
del csr
torch.cuda.synchronize(); torch.cuda.empty_cache()
ts = []
for r in range(reps + 2):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g = glp.Graph(n=n, row_offsets=off_h, col_idx=col_h, symmetric=sym)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    g.close()
    if r >= 2: ts.append(1e3 * (t1 - t0))
print(os.environ.get("GLP_LIB", "in-tree"), wl, "create ms median", round(statistics.median(ts), 2), [round(x, 1) for x in ts])
