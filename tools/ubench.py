"""Run tools/ubench.cu ceilings on RMAT-S (default 24): HBM stream, random gather, smem atomics, match_any."""
import ctypes, os, subprocess, sys, torch
sys.path.insert(0, '.')
from glp_inputs import graphs
here = os.path.dirname(os.path.abspath(__file__))
so = os.path.join(here, 'libubench.so')
subprocess.check_call(['nvcc', '-gencode', 'arch=compute_100a,code=sm_100a', '-O3', '-Xcompiler', '-fPIC', '-shared', '-o', so, os.path.join(here, 'ubench.cu')])
lib = ctypes.CDLL(so)
for f in ['ub_stream', 'ub_gather', 'ub_atoms', 'ub_match', 'ub_atoms2']:
    getattr(lib, f).restype = ctypes.c_float
P, I64, I32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
lib.ub_stream.argtypes = [P, I64, P, I32]; lib.ub_gather.argtypes = [P, I64, P, P, I32, I32]
lib.ub_atoms.argtypes = [I32, P, I32]; lib.ub_atoms2.argtypes = [I32, P, I32]; lib.ub_match.argtypes = [P, P, I32]
scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
csr = graphs.rmat(scale, seed=1, device='cuda', buckets=16 if scale >= 27 else 0)
sms = torch.cuda.get_device_properties(0).multi_processor_count
out = torch.zeros(1, dtype=torch.int64, device='cuda')
col = csr.col_idx[: (csr.nnz // 4) * 4].contiguous()
nnz = col.numel()
L = torch.arange(csr.n, dtype=torch.int32, device='cuda')
ms = lib.ub_stream(col.data_ptr(), nnz, out.data_ptr(), sms)
print(f'stream col: {ms:.3f} ms  {4*nnz/ms/1e6:.1f} GB/s')
for u in (1, 2, 4):
    ms = lib.ub_gather(col.data_ptr(), nnz, L.data_ptr(), out.data_ptr(), sms, u)
    print(f'gather L[col] U={u}: {ms:.3f} ms  {nnz/ms/1e6:.1f} Garcs/s  ({4*nnz/ms/1e6:.1f} GB/s col)')
# the library's internal vertex order (degree-descending ids): hub labels cluster
deg = (csr.row_offsets[1:] - csr.row_offsets[:-1])
order = torch.argsort(deg, descending=True, stable=True)
newid = torch.empty_like(order)
newid[order] = torch.arange(csr.n, device='cuda')
del order, deg
for c0 in range(0, nnz, 1 << 28):  # relabel in place, chunked
    col[c0:c0 + (1 << 28)] = newid[col[c0:c0 + (1 << 28)].long()].to(torch.int32)
del newid
ms = lib.ub_gather(col.data_ptr(), nnz, L.data_ptr(), out.data_ptr(), sms, 4)
print(f'gather L[col] degree-ordered ids: {ms:.3f} ms  {nnz/ms/1e6:.1f} Garcs/s')
if scale < 27:
    # sorted (coalesced) gather for contrast
    cs = torch.sort(col).values
    ms = lib.ub_gather(cs.data_ptr(), nnz, L.data_ptr(), out.data_ptr(), sms, 4)
    print(f'gather sorted col: {ms:.3f} ms  {nnz/ms/1e6:.1f} Garcs/s')
    del cs
for d in (1, 0):
    ms = lib.ub_atoms(d, out.data_ptr(), sms)
    ops = sms * 4 * 512 * 1024
    print(f'smem atomicAdd distinct={d}: {ms:.3f} ms  {ops/ms/1e6/sms:.2f} Gops/s/SM = {ops/ms/1e6/sms/1.9:.2f} /clk/SM')
ms = lib.ub_match(L.data_ptr(), out.data_ptr(), sms)
ops = sms * 4 * 16 * 1024
print(f'match_any: {ms:.3f} ms  {ops/ms/1e6/sms/1.9:.3f} warp-ops/clk/SM')
for mode, name in [(0, 'LDS hashed'), (1, 'atomicAdd hashed, return used'), (2, 'atomicCAS hashed'), (3, 'atomicAdd hashed, no return')]:
    ms = lib.ub_atoms2(mode, out.data_ptr(), sms)
    ops = sms * 4 * 512 * 1024
    print(f'smem {name}: {ms:.3f} ms  {ops/ms/1e6/sms/1.965:.2f} lane-ops/clk/SM')
