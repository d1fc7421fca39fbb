"""Scratch timing of A.A on a generated R-MAT (not the bench contract)."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import spgen
import paper_conf_ipps_orachevkkg21_b200 as sp

scale = int(sys.argv[1]) if len(sys.argv) > 1 else 20
ef = int(sys.argv[2]) if len(sys.argv) > 2 else 16
a, b, c = (float(x) for x in (sys.argv[3:6] if len(sys.argv) > 5 else (0.45, 0.22, 0.22)))
seed = int(sys.argv[6]) if len(sys.argv) > 6 else 1
sp.Initialize(0)
n = 1 << scale
t = time.time()
r, cc = spgen.rmat_pairs(scale, ef, a, b, c, seed=seed, device="cuda")
torch.cuda.synchronize(); print("gen", time.time() - t, flush=True)
t = time.time()
A = sp.Matrix.from_pairs(n, n, r, cc)
torch.cuda.synchronize(); print("build", time.time() - t, "nnz", A.nvals, flush=True)
rp, ci = A.device_tensors()
lens = rp[1:] - rp[:-1]
prods = int(lens[ci.long()].sum())
print("products", prods, flush=True)
rows_of = torch.repeat_interleave(torch.arange(n, device="cuda"), lens)
ub = torch.zeros(n, dtype=torch.int64, device="cuda").index_add_(0, rows_of, lens[ci.long()])
edges = [0, 1, 33, 65, 129, 257, 513, 2049, 8193, 1 << 62]
for lo, hi in zip(edges[:-1], edges[1:]):
    m = (ub >= lo) & (ub < hi)
    print(f"ub [{lo},{hi}) rows {int(m.sum()):9d} products {int(ub[m].sum())/prods*100:6.2f}%", flush=True)
del rows_of
st = torch.cuda.current_stream()
for i in range(int(os.environ.get("ITERS", "5"))):
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(st)
    C = sp.mxm(A, A)
    e1.record(st); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    print(f"mxm {ms:.2f} ms  nnzC {C.nvals}  {prods/ms/1e6:.2f} GProducts/s  peak {sp.memory_stats()[1]/1e9:.2f} GB", flush=True)
    del C
