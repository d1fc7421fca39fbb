"""Step-time variance probe: MxM into a reused C, with pool stats per step."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, spgen
import paper_conf_ipps_orachevkkg21_b200 as sp
sp.Initialize(0)
n = 1 << 22
r, c = spgen.rmat_pairs(22, 32, 0.4, 0.2, 0.2, seed=5, device="cuda")
A = sp.Matrix.from_pairs(n, n, r, c); del r, c
C = sp.Matrix.new(n, n)
flush = torch.empty(64 << 20, dtype=torch.int32, device="cuda")
for i in range(int(os.environ.get("N", "8"))):
    if os.environ.get("FLUSH"): flush.zero_()
    torch.cuda.synchronize(); t = time.perf_counter()
    if os.environ.get("NEWC"):
        C = sp.mxm(A, A)
    else:
        sp.MxM(C, A, A)
    torch.cuda.synchronize(); dt = time.perf_counter() - t
    res, used = sp.pool_stats()
    q = os.popen("nvidia-smi --query-gpu=clocks.sm,power.draw,temperature.gpu,clocks_event_reasons.active --format=csv,noheader").read().strip()
    print(f"[{q}] step {i}: {dt*1e3:.1f} ms  pool reserved {res/1e9:.1f} GB used {used/1e9:.1f} GB  torch reserved {torch.cuda.memory_reserved()/1e9:.1f} GB", flush=True)
