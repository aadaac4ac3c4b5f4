"""glp_graph_create phase trace (GLP_TRACE_CREATE=1) from pinned host CSR of a
bench workload:  python tools/create_trace.py WORKLOAD [reps]"""
import os, sys, time, torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["GLP_TRACE_CREATE"] = "1"
import bench
import paper_conf_sigmod_yelhls21_b200 as glp
wl = sys.argv[1] if len(sys.argv) > 1 else "taobao100m"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
spec, variant, max_iters, gamma = bench.WORKLOADS[wl]
csr, seeds = bench.make_graph(spec, "cuda")
off_h = csr.row_offsets.cpu().pin_memory()
col_h = csr.col_idx.cpu().pin_memory()
n = csr.n
del csr
torch.cuda.synchronize(); torch.cuda.empty_cache()
for r in range(reps):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g = glp.Graph(n=n, row_offsets=off_h, col_idx=col_h, symmetric=True)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    g.close()
    print(f"rep {r}: host create {1e3 * (t1 - t0):.1f} ms", flush=True)
