"""Host link probe: pinned H2D of 100 MB (one C3 FP64 x) split over 1 / 2 / 4 concurrent streams, and
H2D + D2H together; best of 10, CUDA events on the issuing stream (other streams joined)."""
import json
import torch

n = 12_500_000
h = torch.empty(n, dtype=torch.float64).pin_memory()
h2 = torch.empty(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device="cuda")
d2 = torch.empty(n, dtype=torch.float64, device="cuda")
streams = [torch.cuda.Stream() for _ in range(4)]


def run(k, with_d2h=False):
    cur = torch.cuda.current_stream()
    best = 1e9
    for _ in range(10):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(cur)
        chunk = (n + k - 1) // k
        for i in range(k):
            s = streams[i]
            s.wait_stream(cur)
            with torch.cuda.stream(s):
                d[i * chunk:(i + 1) * chunk].copy_(h[i * chunk:(i + 1) * chunk], non_blocking=True)
        if with_d2h:
            s = streams[3]
            s.wait_stream(cur)
            with torch.cuda.stream(s):
                h2.copy_(d2, non_blocking=True)
        for i in range(k):
            cur.wait_stream(streams[i])
        if with_d2h:
            cur.wait_stream(streams[3])
        b.record(cur)
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


out = {}
for k in (1, 2, 3):
    ms = run(k)
    out[f"h2d_{k}streams"] = {"ms": ms, "gbs": n * 8 / ms / 1e6}
    ms = run(k, True)
    out[f"h2d_{k}streams+d2h"] = {"ms": ms}
print(json.dumps(out))
