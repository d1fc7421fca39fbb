"""Scratch probe of the configs[3] closure's host overhead (not the bench
contract): per closure step, device time (events) vs host wall time, with and
without kernel timing / the L2 flush (run with SPBLA_TRACE=1 for the
library's per-phase trace)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp

sp.Initialize(0)
n = 1 << 18
(a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
L0 = sp.Matrix.from_pairs(n, n, a0, b0)
L1 = sp.Matrix.from_pairs(n, n, a1, b1)
U = sp.ewise_add(L0, L1)
st = torch.cuda.current_stream()
flush = torch.empty(1 << 26, dtype=torch.float32, device="cuda")


def step():
    C = U.duplicate()
    it = sp.TransitiveClosure(C)
    C.free()
    return it


for mode in ("plain", "ktime", "flush", "ktime+flush"):
    sp.set_kernel_timing("ktime" in mode)
    out = []
    for i in range(12):
        if "flush" in mode:
            flush.zero_()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        t0 = time.perf_counter()
        e0.record(st)
        step()
        e1.record(st)
        t1 = time.perf_counter()
        e1.synchronize()
        out.append((round(e0.elapsed_time(e1), 2), round((t1 - t0) * 1e3, 2)))
    print(mode, "(device ms, host ms):", out, flush=True)
    sp.set_kernel_timing(False)
if os.environ.get("SPBLA_TRACE"):
    step()
