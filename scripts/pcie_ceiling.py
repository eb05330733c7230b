"""Host link ceiling for the e2e leg: pinned H2D alone, D2H alone, and both at once (two streams),
16.8 MB per copy (one C2 FP64 x / y vector), best of 20, CUDA events."""
import json
import torch

n = 2097152
h_in = torch.empty(n, dtype=torch.float64).pin_memory()
h_out = torch.empty(n, dtype=torch.float64).pin_memory()
d_in = torch.empty(n, dtype=torch.float64, device="cuda")
d_out = torch.empty(n, dtype=torch.float64, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
nb = n * 8


def timed(fn, reps=20):
    best = 1e9
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


def both():
    cur = torch.cuda.current_stream()
    s1.wait_stream(cur)
    s2.wait_stream(cur)
    with torch.cuda.stream(s1):
        d_in.copy_(h_in, non_blocking=True)
    with torch.cuda.stream(s2):
        h_out.copy_(d_out, non_blocking=True)
    cur.wait_stream(s1)
    cur.wait_stream(s2)


h2d = timed(lambda: d_in.copy_(h_in, non_blocking=True))
d2h = timed(lambda: h_out.copy_(d_out, non_blocking=True))
bo = timed(both)
print(json.dumps({"bytes": nb, "h2d_ms": h2d, "h2d_gbs": nb / h2d / 1e6, "d2h_ms": d2h, "d2h_gbs": nb / d2h / 1e6,
                  "both_ms": bo, "both_gbs_each": nb / bo / 1e6}))
