"""Probe: can an HBM-bound copy (compaction-like traffic) overlap the hash bins?
Times MxM alone, a 2x10 GB copy alone, and both concurrently (copy on a side
stream of given priority launched right before the MxM)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp
sp.Initialize(0)
n = 1 << 22
r, c = spgen.rmat_pairs(22, 32, 0.4, 0.2, 0.2, seed=5, device="cuda")
A = sp.Matrix.from_pairs(n, n, r, c); del r, c
C = sp.Matrix.new(n, n)
src = torch.empty(5 << 30 >> 2, dtype=torch.int32, device="cuda")  # 5 GB
dst = torch.empty_like(src)
main = torch.cuda.current_stream()
NC = int(os.environ.get("NC", "16"))
def ev(): return torch.cuda.Event(enable_timing=True)
def run(mode, prio):
    side = torch.cuda.Stream(priority=prio)
    torch.cuda.synchronize()
    e0, e1, c0, c1 = ev(), ev(), ev(), ev()
    if mode in ("copy", "both"):
        side.wait_stream(main)
        with torch.cuda.stream(side):
            c0.record(side)
            for _ in range(NC): dst.copy_(src)   # NC x (5 GB read + 5 GB write)
            c1.record(side)
    e0.record(main)
    if mode in ("mxm", "both"):
        sp.MxM(C, A, A)
    e1.record(main)
    torch.cuda.synchronize()
    m = e0.elapsed_time(e1)
    cp = c0.elapsed_time(c1) if mode != "mxm" else 0
    return m, cp
for mode in ("mxm", "copy", "both"):
    for prio in (0, -1):
        for it in range(2):
            m, cp = run(mode, prio)
        print(f"{mode:5s} side-prio {prio:2d}: mxm-stream {m:7.2f} ms   copy {cp:7.2f} ms", flush=True)
