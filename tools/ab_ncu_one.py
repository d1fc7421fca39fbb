"""Scratch (not the bench contract): one configs[4] MxM for an ncu capture, package under argv[1]."""
import sys
sys.path.insert(0, sys.argv[1])
import torch, spgen
import paper_conf_ipps_orachevkkg21_b200 as sp
sp.Initialize(0)
r, c = spgen.rmat_pairs(22, 32, 0.4, 0.2, 0.2, seed=5, device="cuda")
n = 1 << 22
A = sp.Matrix.from_pairs(n, n, r, c)
del r, c
C = sp.mxm(A, A)
torch.cuda.synchronize()
