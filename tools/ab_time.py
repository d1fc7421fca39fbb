"""Scratch A/B timing (not the bench contract): configs[4] A.A with the
per-kernel groups, for the package found under argv[1]."""
import os, sys, statistics
sys.path.insert(0, sys.argv[1])
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp
print("package:", sp.__file__)
sp.Initialize(0)
r, c = spgen.rmat_pairs(22, 32, 0.4, 0.2, 0.2, seed=5, device="cuda")
n = 1 << 22
A = sp.Matrix.from_pairs(n, n, r, c)
del r, c
groups = ("mxm_ub", "warp_bins", "H0", "H1", "H2", "H3", "H4", "H5", "H6", "dense", "compact")
st = torch.cuda.current_stream()
C = sp.Matrix.new(n, n)
for i in range(3):
    sp.MxM(C, A, A)
sp.set_kernel_timing(True)
ms = []
for i in range(6):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(st); sp.MxM(C, A, A); e1.record(st); e1.synchronize()
    ms.append(e0.elapsed_time(e1))
print("step ms", [round(x, 2) for x in ms], "median", round(statistics.median(ms), 2))
print({k: round(sp.kernel_timing(k)[0] / 6, 2) for k in groups})
