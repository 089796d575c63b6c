import torch, time
n = 738_000_000
dev = 'cuda'
src = torch.arange(n, dtype=torch.int32, device=dev)
out = torch.empty(n, dtype=torch.int32, device=dev)
for tile in [1<<20, 1<<22, 1<<23, 14_000_000, 1<<25, 1<<27, n]:
    # random permutation within tiles
    idx = torch.empty(n, dtype=torch.int64, device=dev)
    for t0 in range(0, n, tile):
        m = min(tile, n - t0)
        idx[t0:t0+m] = torch.randperm(m, device=dev) + t0
    torch.cuda.synchronize()
    for rep in range(3):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); out.index_put_((idx,), src); e1.record(); torch.cuda.synchronize()
        sc = e0.elapsed_time(e1)
        e0.record(); g = src[idx]; e1.record(); torch.cuda.synchronize()
        ga = e0.elapsed_time(e1)
    print(f"tile {tile:>10d} ({tile*4/2**20:8.1f} MB): scatter {sc:7.2f} ms  gather {ga:7.2f} ms", flush=True)
    del idx, g
