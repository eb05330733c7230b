"""Host->device ceiling probe: one cudaMemcpyAsync vs the copy split over k streams vs SM loads from
pinned host memory (zero-copy, UVA). 16.8 MB (one C2 FP64 x vector), best of 20, CUDA events."""
import ctypes, json, os
import torch

lib = ctypes.CDLL(os.path.join(os.path.dirname(os.path.abspath(__file__)), "libzc.so"))
n = 2097152
nb = n * 8
h = torch.randn(n, dtype=torch.float64).pin_memory()
d = torch.empty(n, dtype=torch.float64, device="cuda")
streams = [torch.cuda.Stream() for _ in range(8)]


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


def split(k):
    def f():
        cur = torch.cuda.current_stream()
        c = n // k
        for i in range(k):
            s = streams[i]
            s.wait_stream(cur)
            with torch.cuda.stream(s):
                d[i * c:(i + 1) * c].copy_(h[i * c:(i + 1) * c], non_blocking=True)
        for i in range(k):
            cur.wait_stream(streams[i])
    return f


def zc(blocks, threads):
    def f():
        rc = lib.zc_copy(ctypes.c_void_p(h.data_ptr()), ctypes.c_void_p(d.data_ptr()), ctypes.c_int64(nb),
                         blocks, threads, ctypes.c_void_p(torch.cuda.current_stream().cuda_stream))
        assert rc == 0, rc
    return f


out = {"bytes": nb}
for k in (1, 2, 4, 8):
    t = timed(split(k))
    out[f"memcpy_x{k}_gbs"] = nb / t / 1e6
for blocks in (148, 296, 592, 1184, 2368):
    for threads in (256, 512):
        d.zero_()
        t = timed(zc(blocks, threads))
        assert torch.equal(d.cpu(), h), "zero-copy result differs"
        out[f"zc_b{blocks}_t{threads}_gbs"] = nb / t / 1e6
print(json.dumps(out))
