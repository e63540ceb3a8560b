"""How many distinct (kernel, t) values a config has (sizing the value-level ROOT)."""
import sys, os
sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
import torch
import tracegen as G
name = sys.argv[1] if len(sys.argv) > 1 else "C5"
sp = G.spec(name)
ds = G.DeviceSpec(sp, "cuda")
n = sp.n
kid = torch.empty(n, dtype=torch.int32, device="cuda")
t = torch.empty(n, dtype=torch.int32, device="cuda")
G.generate_cuda(ds, kid, t)
key = (kid.to(torch.int64) << 32) | (t.to(torch.int64) & 0xFFFFFFFF)
del t
key, _ = torch.sort(key)
new = torch.ones(n, dtype=torch.bool, device="cuda")
new[1:] = key[1:] != key[:-1]
D = int(new.sum())
k = (key >> 32)
cnt = torch.bincount(k, minlength=sp.n_kernels)
dk = torch.bincount(k[new], minlength=sp.n_kernels)
big = cnt >= 1 << 20
print(name, "rows", n, "distinct", D, "ratio", n / D)
print("kernels >= 2^20 rows:", int(big.sum()), "rows", int(cnt[big].sum()), "distinct", int(dk[big].sum()))
top = torch.argsort(cnt, descending=True)[:10]
for i in top.tolist():
    print(" kernel", i, "rows", int(cnt[i]), "distinct", int(dk[i]))
