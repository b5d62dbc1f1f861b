import torch, time
dev='cuda'
n=27467757
g=torch.Generator(device=dev); g.manual_seed(1)
# zipf-ish keys: mix hot and cold
k=torch.randint(0, 1<<26, (n,), device=dev, dtype=torch.int32)
hot=torch.randint(0, 1000, (n,), device=dev, dtype=torch.int32)
mask=torch.rand(n, device=dev) < 0.5
k=torch.where(mask, hot*52000, k)
v=torch.arange(n, device=dev, dtype=torch.int32)
for name, fn in [('sort stable int32 (keys+idx)', lambda: torch.sort(k, stable=True)),
                 ('sort int64 combined', lambda: torch.sort((k.long()<<32)|v.long()))]:
    for _ in range(3): fn()
    torch.cuda.synchronize()
    e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): fn()
    e1.record(); torch.cuda.synchronize()
    print(name, e0.elapsed_time(e1)/10, 'ms')
