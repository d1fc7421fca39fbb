"""Scratch probe (not the bench contract): does in-process NVML sampling stall
the host-sync-heavy closure loop, and which query is responsible?"""
import os, sys, threading, time, statistics
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import pynvml
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp

sp.Initialize(0)
n = 1 << 18
(a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
L0 = sp.Matrix.from_pairs(n, n, a0, b0)
L1 = sp.Matrix.from_pairs(n, n, a1, b1)
U = sp.ewise_add(L0, L1)
st = torch.cuda.current_stream()
pynvml.nvmlInit()
h = pynvml.nvmlDeviceGetHandleByIndex(0)
calls = {
    "none": [],
    "clock": [lambda: pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)],
    "reasons": [lambda: pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)],
    "both": [lambda: pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM),
             lambda: pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)],
}
for period in (0.1, 0.5):
    for name, fns in calls.items():
        stop = threading.Event()
        dur = []

        def run():
            while not stop.is_set():
                for f in fns:
                    t = time.perf_counter()
                    f()
                    dur.append(time.perf_counter() - t)
                stop.wait(period)
        th = threading.Thread(target=run, daemon=True)
        th.start()
        ms = []
        for i in range(25):
            C = U.duplicate()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(st)
            sp.TransitiveClosure(C)
            e1.record(st); e1.synchronize()
            ms.append(e0.elapsed_time(e1))
            C.free()
        stop.set(); th.join()
        print(f"period {period} {name:8s} median {statistics.median(ms):6.2f} max {max(ms):7.2f} "
              f"nvml call ms: max {1e3*max(dur) if dur else 0:.2f} mean {1e3*statistics.mean(dur) if dur else 0:.3f}", flush=True)
