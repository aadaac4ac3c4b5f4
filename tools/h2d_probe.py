import torch, time
x = torch.empty(2_000_000_000, dtype=torch.int32).pin_memory()
y = torch.empty_like(x, device='cuda')
for r in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter(); y.copy_(x, non_blocking=True); torch.cuda.synchronize(); t1 = time.perf_counter()
    print('h2d 8 GB', round(8e9 / (t1 - t0) / 1e9, 1), 'GB/s', flush=True)
