"""Set-associative LRU simulation (scripts/probe/l2sim.c) of the long-row kernel x sector accesses of C3
in unit execution order, for the current long format (S=1) and column-segmented long rows (S parts, each
row padded per part): x sector misses at 48 / 96 MB of cache.  Result: profiles/r02b/long_segment_sim.txt."""
import os
import ctypes, numpy as np, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import synth
import os, subprocess
HERE = os.path.dirname(os.path.abspath(__file__))
SO = '/tmp/l2sim.so'
subprocess.check_call(['gcc', '-O2', '-shared', '-fPIC', '-o', SO, os.path.join(HERE, 'l2sim.c')])
lib = ctypes.CDLL(SO)
lib.simulate.restype = ctypes.c_int64
lib.simulate.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_int64]
A = synth.generate(synth.config('c3'))
L = np.diff(A.row_ptr)
longr = np.nonzero(L > 256)[0]
n = A.n
G, U = 64, 256
def region(S):
    segs = []
    for s in range(S):
        for r in longr:
            c = A.col[A.row_ptr[r]:A.row_ptr[r+1]]
            if S > 1:
                c = c[(c.astype(np.int64) * S) // n == s]
            if len(c) == 0: continue
            pad = (-len(c)) % G
            segs.append(c)
            if pad: segs.append(np.full(pad, -1, np.int32))
    reg = np.concatenate(segs)
    pad = (-len(reg)) % U
    reg = np.concatenate([reg, np.full(pad, -1, np.int32)])
    return reg
def order(reg, buckets):
    nu = len(reg) // U
    first = reg[::U].astype(np.int64)
    b = np.where(first < 0, buckets - 1, first * buckets // n)
    o = np.argsort(b, kind='stable')
    return reg.reshape(nu, U)[o].ravel().copy()
for S in (1, 2, 4):
    t = time.time()
    reg = region(S)
    for buckets in (16, 256):
        seq = order(reg, buckets)
        for mb in (48, 96):
            sectors = mb * 2**20 // 32
            ways = 16
            miss = lib.simulate(seq.ctypes.data, len(seq), sectors // ways, ways, 8, 0)
            print(f"S={S} buckets={buckets} cache={mb}MB slots={len(reg)/1e6:.1f}M misses={miss/1e6:.2f}M sectors ({miss*32/1e6:.0f} MB)", flush=True)
    print('t', time.time() - t, flush=True)
