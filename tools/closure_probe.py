"""Scratch probe of the configs[3] closure (not the bench contract): per
iteration, the rows per ub bin, their duplication (ub / distinct), column
span, and the kernel-group times of that iteration's MxM."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp

sp.Initialize(0)
n = 1 << 18
(a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
L0 = sp.Matrix.from_pairs(n, n, a0, b0)
L1 = sp.Matrix.from_pairs(n, n, a1, b1)
C = sp.ewise_add(L0, L1)
groups = ("mxm_ub", "warp_bins", "H0", "H1", "H2", "H3", "H4", "H5", "H6", "dense", "dense_ovf", "compact")
edges = [0, 1, 257, 513, 1025, 2049, 4097, 8193, 20481, 40961, 1 << 62]
for it in range(8):
    rp, ci = C.device_tensors()
    lens = rp[1:] - rp[:-1]
    rows_of = torch.repeat_interleave(torch.arange(n, device="cuda"), lens)
    ub = lens.clone().index_add_(0, rows_of, lens[ci.long()])
    first = torch.where(lens > 0, ci[rp[:-1].clamp(max=max(ci.numel() - 1, 0))].long(), 0)
    prev = C.nvals
    sp.set_kernel_timing(True)
    torch.cuda.synchronize()
    sp.MxM(C, C, C, accumulate=True, closure_step=True)
    torch.cuda.synchronize()
    kt = {k: round(sp.kernel_timing(k)[0], 3) for k in groups}
    sp.set_kernel_timing(False)
    rp2, ci2 = C.device_tensors()
    lens2 = rp2[1:] - rp2[:-1]
    # span of the new rows (new rows contain the old ones; span of the result)
    lo = torch.where(lens2 > 0, ci2[rp2[:-1].clamp(max=ci2.numel() - 1)].long(), 0)
    hi = torch.where(lens2 > 0, ci2[(rp2[1:] - 1).clamp(min=0)].long(), 0)
    span = (hi - lo + 1).float()
    print(f"iter {it}: nnz {prev} -> {C.nvals}  products {int(ub.sum())}  kernels {kt}", flush=True)
    for l, h in zip(edges[:-1], edges[1:]):
        m = (ub >= l) & (ub < h)
        k = int(m.sum())
        if not k:
            continue
        u = ub[m].float(); d = lens2[m].float(); s = span[m]
        print(f"   ub [{l},{h}) rows {k:7d} prod {int(u.sum()):11d} dup(ub/distinct) mean {float((u / d.clamp(min=1)).mean()):8.2f}"
              f" max {float((u / d.clamp(min=1)).max()):8.1f}  span mean {float(s.mean()):9.0f}  span/ub mean {float((s / u.clamp(min=1)).mean()):8.2f}",
              flush=True)
    del rows_of
    if C.nvals == prev:
        break
