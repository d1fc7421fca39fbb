"""Scratch probe (not the bench contract): run the configs[3] closure with the
library's SPBLA_TRACE phases and print the trace of the slowest steps."""
import os, sys, time, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp
sp.Initialize(0)
n = 1 << 18
(a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
U = sp.ewise_add(sp.Matrix.from_pairs(n, n, a0, b0), sp.Matrix.from_pairs(n, n, a1, b1))
torch.cuda.synchronize()
for i in range(12):
    C = U.duplicate()
    t = time.perf_counter()
    print(f"=== step {i}", file=sys.stderr, flush=True)
    sp.TransitiveClosure(C)
    torch.cuda.synchronize()
    print(f"=== step {i} {1e3*(time.perf_counter()-t):.1f} ms", file=sys.stderr, flush=True)
    C.free()
