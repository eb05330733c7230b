"""Probe: random 8-byte gathers over a buffer of S MB (torch index kernel) -> effective L2 size."""
import torch, time
torch.cuda.init()
N = 1 << 26
for mb in [8, 16, 32, 48, 56, 64, 72, 80, 96, 112, 128, 160, 256]:
    n = mb * (1 << 20) // 8
    x = torch.randn(n, dtype=torch.float64, device="cuda")
    idx = torch.randint(0, n, (N,), device="cuda")
    out = torch.empty(N, dtype=torch.float64, device="cuda")
    for _ in range(3):
        torch.index_select(x, 0, idx, out=out)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10):
        torch.index_select(x, 0, idx, out=out)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    print(f"{mb:4d} MB  {ms:.3f} ms  {N/ms/1e6:.2f} Ggather/s", flush=True)
