"""Time the e2e phases through the C ABI with pinned host buffers (create / run / labels D2H)."""
import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_sigmod_yelhls21_b200 as glp
from glp_inputs import graphs
csr = graphs.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 24, seed=1, device='cuda')
off_h = csr.row_offsets.cpu().pin_memory(); col_h = csr.col_idx.cpu().pin_memory()
out_h = torch.empty(csr.n, dtype=torch.int32).pin_memory()
stream = torch.cuda.current_stream()
for r in range(4):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g2 = glp.Graph(n=csr.n, row_offsets=off_h, col_idx=col_h, stream=stream)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    ri = g2.run('classic', 20)
    t2 = time.perf_counter()
    glp.glp_labels_get(g2.handle, out_h)
    t3 = time.perf_counter()
    g2.close(); t4 = time.perf_counter()
    print(f'create {1e3*(t1-t0):.1f} run {1e3*(t2-t1):.1f} (dev {ri.elapsed_ms:.1f}) get {1e3*(t3-t2):.1f} close {1e3*(t4-t3):.1f} ms', flush=True)
