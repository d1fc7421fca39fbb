"""Scratch probe (not the bench contract): host stalls of the configs[3]
closure loop vs hypervisor steal time and Python GC."""
import gc, os, sys, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp


def steal():
    with open("/proc/stat") as f:
        p = f.readline().split()
    return int(p[8])  # cpu aggregate: user nice system idle iowait irq softirq steal


def ctxsw():
    with open(f"/proc/{os.getpid()}/status") as f:
        d = dict(l.split(":", 1) for l in f if ":" in l)
    return int(d["voluntary_ctxt_switches"]), int(d["nonvoluntary_ctxt_switches"])


sp.Initialize(0)
n = 1 << 18
(a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
U = sp.ewise_add(sp.Matrix.from_pairs(n, n, a0, b0), sp.Matrix.from_pairs(n, n, a1, b1))
st = torch.cuda.current_stream()
for mode in ("gc-on", "gc-off"):
    if mode == "gc-off":
        gc.disable()
    ms, bad = [], []
    for i in range(60):
        C = U.duplicate()
        s0, c0, t0 = steal(), ctxsw(), time.perf_counter()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(st)
        sp.TransitiveClosure(C)
        e1.record(st); e1.synchronize()
        t1, s1, c1 = time.perf_counter(), steal(), ctxsw()
        d = e0.elapsed_time(e1)
        ms.append(d)
        if d > 12:
            bad.append((i, round(d, 1), round(1e3 * (t1 - t0), 1), s1 - s0, c1[0] - c0[0], c1[1] - c0[1]))
        C.free()
    print(mode, "median", round(statistics.median(ms), 2), "max", round(max(ms), 1), "slow steps (i, dev ms, host ms, steal jiffies, vol cs, invol cs):", bad, flush=True)
    gc.enable()
