"""Time glp_graph_create from host CSR vs device CSR on RMAT-24."""
import sys, time, torch
sys.path.insert(0, '.')
import paper_conf_sigmod_yelhls21_b200 as glp
from glp_inputs import graphs
csr = graphs.rmat(int(sys.argv[1]) if len(sys.argv) > 1 else 24, seed=1, device='cuda')
off_h = csr.row_offsets.cpu().pin_memory(); col_h = csr.col_idx.cpu().pin_memory()
for rep in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g = glp.Graph(n=csr.n, row_offsets=off_h, col_idx=col_h)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    g.close(); t2 = time.perf_counter()
    g = glp.Graph(csr)
    torch.cuda.synchronize(); t3 = time.perf_counter()
    g.close(); t4 = time.perf_counter()
    print(f'host-create {1e3*(t1-t0):.1f} ms destroy {1e3*(t2-t1):.1f} ms | device-create {1e3*(t3-t2):.1f} ms destroy {1e3*(t4-t3):.1f} ms')
