"""Create-time variance probe: N host-buffer creates of one workload's graph
(pinned host CSR), printing create / run / destroy times per step.
  python tools/e2e_var.py sbm1m 8 [empty_cache|run|smi]"""
import os, sys, time, torch
sys.path.insert(0, '.')
os.environ.setdefault("GLP_POOL_KEEP_GB", "64")
import paper_conf_sigmod_yelhls21_b200 as glp
from glp_inputs import graphs
name = sys.argv[1]; steps = int(sys.argv[2])
csr, seeds = graphs.make(name, device='cuda')
off_h = csr.row_offsets.cpu().pin_memory(); col_h = csr.col_idx.cpu().pin_memory()
n = csr.n
del csr
mode = sys.argv[3] if len(sys.argv) > 3 else ""
torch.cuda.empty_cache() if mode == "empty_cache" else None
if mode == "smi":  # a short nvidia-smi sampling window first, as bench.py's clock sampler
    import subprocess
    p = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv", "-lms", "200"],
                         stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
    time.sleep(0.1); p.terminate(); p.wait()
stream = torch.cuda.current_stream()
print(name, 'torch reserved GB', round(torch.cuda.memory_reserved() / 2**30, 2), flush=True)
for r in range(steps):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    g2 = glp.Graph(n=n, row_offsets=off_h, col_idx=col_h, stream=stream)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    if mode in ("run", "smi"):
        g2.run("classic", 20)
    g2.close(); torch.cuda.synchronize(); t2 = time.perf_counter()
    free, tot = torch.cuda.mem_get_info()
    print(f'{r} create {1e3*(t1-t0):.1f} destroy {1e3*(t2-t1):.1f} ms  free {free/2**30:.1f} GB', flush=True)
