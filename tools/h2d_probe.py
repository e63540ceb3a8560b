import torch, time
n = 1_000_000_000
a = torch.empty(n, dtype=torch.int32, pin_memory=True); b = torch.empty(n, dtype=torch.int32, pin_memory=True)
da = torch.empty(n, dtype=torch.int32, device='cuda'); db = torch.empty(n, dtype=torch.int32, device='cuda')
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
for rep in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    da.copy_(a, non_blocking=True); db.copy_(b, non_blocking=True); torch.cuda.synchronize()
    t1 = time.perf_counter()
    with torch.cuda.stream(s1): da.copy_(a, non_blocking=True)
    with torch.cuda.stream(s2): db.copy_(b, non_blocking=True)
    torch.cuda.synchronize(); t2 = time.perf_counter()
    # chunked interleaved on 4 streams
    ss = [torch.cuda.Stream() for _ in range(4)]
    ch = n // 8
    for i in range(8):
        with torch.cuda.stream(ss[i % 4]):
            da[i*ch:(i+1)*ch].copy_(a[i*ch:(i+1)*ch], non_blocking=True)
            db[i*ch:(i+1)*ch].copy_(b[i*ch:(i+1)*ch], non_blocking=True)
    torch.cuda.synchronize(); t3 = time.perf_counter()
    print(f"seq {8e9/(t1-t0)/1e9:.1f} GB/s  2 streams {8e9/(t2-t1)/1e9:.1f} GB/s  4 streams chunked {8e9/(t3-t2)/1e9:.1f} GB/s")
