"""Benchmark of the SPbLA B200 hot path: Boolean SpGEMM C = A.A (BASELINE.json).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl b200|reference]

One step = one full MxM (upper-bound pass, binning, all bin kernels,
compaction) on the workload resident in HBM; at N > 1 (torchrun, one rank
per GPU) a step also all-gathers the row-partitioned B over NCCL first.
Prints ONE JSON line (rank 0).  Inputs are seeded synthetic R-MAT graphs
(DESIGN.md §3); A (0.5 GB at the default size) is larger than L2 and a 256 MB
buffer is also written between timed steps.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import spgen  # noqa: E402

METRIC = "Boolean SpGEMM A·A ms & GProducts/s, HBM GB/s vs peak, peak mem @1/2/4/8 B200"
UNIT = "GProducts/s"

# BASELINE.json configs; R-MAT (a, b, c) and the reading behind each choice
# are in DESIGN.md §3.
WORKLOADS = {
    "rmat22_ef32": dict(config="configs[4]", scale=22, ef=32, abc=(0.40, 0.20, 0.20), seed=5),
    "rmat20_ef16": dict(config="configs[1]", scale=20, ef=16, abc=(0.45, 0.22, 0.22), seed=1),
    "uniform4096": dict(config="configs[0]", scale=12, ef=8, abc=None, seed=1),
}
DEFAULT_WORKLOAD = "rmat22_ef32"
# the other BASELINE.json rows (own metric lines, not the headline): configs[2]
# EWiseAdd + Kronecker, configs[3] transitive closure
AUX_WORKLOADS = ("ewise_kron", "closure18")
FLUSH_BYTES = 256 << 20


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def gen_pairs(wl, device):
    n = 1 << wl["scale"]
    if wl["abc"] is None:
        r, c = spgen.uniform_pairs(n, n, wl["ef"], wl["seed"], device=device)
    else:
        r, c = spgen.rmat_pairs(wl["scale"], wl["ef"], *wl["abc"], seed=wl["seed"], device=device)
    return n, r, c


def row_products(rowptr, colidx, n):
    """Per-row product count sum_{k in A[i]} |B[k]| (B = A), planning only."""
    lens = rowptr[1:] - rowptr[:-1]
    rows = torch.repeat_interleave(torch.arange(n, device=rowptr.device), lens)
    ub = torch.zeros(n, dtype=torch.int64, device=rowptr.device)
    ub.index_add_(0, rows, lens[colidx.long()])
    return ub, rows


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled during the timed
    region, in-process through NVML (a background thread, 100 ms period):
    spawning nvidia-smi in a loop stalls CUDA calls of the measured process
    for tens to hundreds of ms.  Started before the warm-up; only samples in
    window() are kept (all samples if the window is not set)."""

    NAMES = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
             "hw_power_brake_slowdown": 0x80, "sw_power_cap": 0x4}
    t0 = t1 = None

    def __init__(self, gpu_index, period=0.1):
        import threading
        self.samples = []
        self.stop_ev = threading.Event()
        self.thread = None
        if os.environ.get("BENCH_NO_CLOCKS"):
            return
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nvml = pynvml
            # NVML indexes physical GPUs; map through CUDA_VISIBLE_DEVICES
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            idx = int(vis.split(",")[gpu_index]) if vis and vis.split(",")[gpu_index].isdigit() else gpu_index
            self.h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            return

        def run():
            while not self.stop_ev.is_set():
                try:
                    mhz = self.nvml.nvmlDeviceGetClockInfo(self.h, self.nvml.NVML_CLOCK_SM)
                    rs = self.nvml.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                    self.samples.append((time.time(), mhz, rs))
                except Exception:
                    pass
                self.stop_ev.wait(period)
        self.thread = threading.Thread(target=run, daemon=True)
        self.thread.start()

    def window(self, t0, t1):
        self.t0, self.t1 = t0, t1

    def stop(self):
        if self.thread is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["clock sampling unavailable"]}
        self.stop_ev.set()
        self.thread.join(timeout=2)
        use = self.samples
        if self.t0 is not None:
            win = [x for x in self.samples if self.t0 - 0.15 <= x[0] <= self.t1 + 0.15]
            use = win or self.samples
        reasons = set()
        for _, _, rs in use:
            for nm, bit in self.NAMES.items():
                if rs & bit:
                    reasons.add(nm)
        sm = [x[1] for x in use]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": self.max_mhz,
                "reasons": sorted(reasons), "samples": len(sm), "source": "NVML in-process, 100 ms"}


# ---------------------------------------------------------------------------
def cpu_oracle_sample(rp_host, ci_host, ub_host, target_products, threads=None):
    """Time the CPU oracle (as it stands: ``oracle.mxm_rows``) on a bounded
    sample of the workload, on every host core: 4 contiguous row chunks per
    thread spread evenly over the rows (oracle/parallel.py; ctypes releases
    the GIL).  Returns (products, seconds, rows, threads, nnz)."""
    import numpy as np
    import oracle
    from oracle import parallel as opar
    threads = threads or opar.host_cores()
    n = len(rp_host) - 1
    A = oracle.Csr(n, n, rp_host, ci_host)
    nch = 4 * threads
    per = target_products / nch
    cum = np.cumsum(ub_host.astype(np.float64))
    total = float(cum[-1]) if n else 0.0
    chunks = []
    for i in range(nch):  # chunk i starts at the row holding product (i + 0.5) / nch of the total
        r0 = int(np.searchsorted(cum, total * (i + 0.5) / nch))
        r1 = int(np.searchsorted(cum, cum[min(r0, n - 1)] + per)) + 1
        chunks.append((min(r0, n), min(max(r1, r0 + 1), n)))
    prods = sum(int(ub_host[a:b].sum()) for a, b in chunks)
    rows = sum(b - a for a, b in chunks)
    t = time.perf_counter()
    nnz = sum(opar.mxm_rows_chunked(A, A, chunks, lambda r0, r1, R: R.nvals, threads=threads))
    dt = time.perf_counter() - t
    return prods, dt, rows, threads, nnz


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, bounded sample per step."""
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if rank != 0:
        return
    import numpy as np
    wl = WORKLOADS[args.workload]
    dev = "cuda" if torch.cuda.is_available() else "cpu"
    n, r, c = gen_pairs(wl, dev)
    # setup only (untimed): sorted duplicate-free CSR with plain torch ops
    key = torch.unique(r.long() * n + c.long())
    rows = key // n
    ci = (key % n).to(torch.int32)
    rp = torch.zeros(n + 1, dtype=torch.int64, device=key.device)
    rp[1:] = torch.cumsum(torch.bincount(rows, minlength=n), 0)
    del r, c, key, rows
    ub, _ = row_products(rp, ci, n)
    rp_h = rp.cpu().numpy().astype(np.uint64)
    ci_h = ci.cpu().numpy().astype(np.uint32)
    ub = ub.cpu().numpy()
    target = float(os.environ.get("REF_SAMPLE_PRODUCTS", "2e8"))
    times, prods = [], 0
    for i in range(args.warmup + args.steps):
        p, dt, nrows, thr, _ = cpu_oracle_sample(rp_h, ci_h, ub, target)
        if i >= args.warmup:
            times.append(dt)
            prods = p
    ms = 1e3 * sum(times) / len(times)
    value = prods / (ms * 1e-3) / 1e9
    sample = (f"{4 * thr} contiguous row chunks spread over {args.workload} ({nrows} rows, {prods} products); "
              f"the unchanged std::set Gustavson oracle on {thr} threads")
    line = {"impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": args.workload, "baseline_config": wl["config"]},
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": thr, "kind": "oracle", "sample": sample},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)



# ---------------------------------------------------------------------------
AUX_GROUPS = ("mxm_ub", "warp_bins", "H0", "H1", "H2", "H3", "H4", "H5", "H6", "dense", "dense_ovf", "compact")


def aux_timer(sp, steps, warmup):
    """Device timing of a host-launched op (CUDA events on the library
    stream, 256 MB L2 flush before each step); returns (timed, state) where
    timed(fn) -> median ms and state collects launches and step lists."""
    stream = torch.cuda.current_stream()
    flush = torch.empty(FLUSH_BYTES // 4, dtype=torch.int32, device="cuda")
    state = {"launches": 0, "step_ms": []}

    def timed(fn):
        # timed steps without the per-kernel event records (a host-launched
        # loop of ~100 small launches per step would carry their cost); one
        # extra step afterwards records the kernel breakdown
        for i in range(warmup):
            fn()
        torch.cuda.synchronize()
        sp.set_kernel_timing(False)
        sp.reset_launch_count()
        ms = []
        for _ in range(steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            e1.synchronize()
            ms.append(e0.elapsed_time(e1))
        state["launches"] += sp.launch_count()
        sp.set_kernel_timing(True)
        fn()  # (the kernel breakdown step: kernel_timing() reads its records, per step)
        torch.cuda.synchronize()
        log(f"[aux] step ms: {[round(x, 2) for x in ms]}")
        state["step_ms"].append([round(x, 3) for x in ms])
        # median: these host-launched ops can see rare host stalls; the full
        # list is reported next to it
        return statistics.median(ms)
    return timed, state


def aux_ewise_kron(sp, steps, warmup, peak_gbs):
    """configs[2]: EWiseAdd of two 2^20-row matrices and Kronecker of a
    2^10-vertex graph with a 64-state RSM adjacency."""
    timed, state = aux_timer(sp, steps, warmup)
    n = 1 << 20
    r1, c1 = spgen.rmat_pairs(20, 16, 0.45, 0.22, 0.22, seed=1, device="cuda")
    r2, c2 = spgen.uniform_pairs(n, n, 8, seed=2, device="cuda")
    A = sp.Matrix.from_pairs(n, n, r1, c1)
    B = sp.Matrix.from_pairs(n, n, r2, c2)
    del r1, c1, r2, c2
    E = sp.Matrix.new(n, n)
    ms_e = timed(lambda: sp.Matrix_EWiseAdd(E, A, B))
    ke = {k: sp.kernel_timing(k) for k in ("ewise_split", "ewise_merge")}
    sp.set_kernel_timing(False)
    # algorithmic bytes: both inputs read once (colidx + rowptr), output written once
    alg_e = 4 * (A.nvals + B.nvals) + 16 * (n + 1) + 4 * E.nvals + 8 * (n + 1)
    rg, cg = spgen.rmat_pairs(10, 16, 0.45, 0.22, 0.22, seed=3, device="cuda")
    rr, cr = spgen.rsm_pairs(64, 1, 2, seed=4, device="cuda")
    G = sp.Matrix.from_pairs(1024, 1024, rg, cg)
    R = sp.Matrix.from_pairs(64, 64, rr, cr)
    K = sp.Matrix.new(1024 * 64, 1024 * 64)
    ms_k = timed(lambda: sp.Kronecker(K, G, R))
    kk = sp.kernel_timing("kron")
    sp.set_kernel_timing(False)
    alg_k = 4 * K.nvals + 8 * (K.nrows + 1)  # output-write bound (inputs are KB)
    per_e = ke["ewise_split"][0] + ke["ewise_merge"][0]  # (one breakdown step)
    out = {"ms": ms_e + ms_k, "unit": "ms",
           "ewise": {"ms": ms_e, "kernel_ms": per_e, "nnz_A": A.nvals, "nnz_B": B.nvals, "nnz_C": E.nvals,
                     "alg_bytes": alg_e, "GB/s": alg_e / (per_e * 1e-3) / 1e9,
                     "frac": alg_e / (per_e * 1e-3) / 1e9 / peak_gbs,
                     "kernel_ms_per_step": {k: v[0] for k, v in ke.items()}},
           "kron": {"ms": ms_k, "kernel_ms": kk[0], "nnz_K": K.nvals, "rows_K": K.nrows,
                    "alg_bytes": alg_k, "GB/s": alg_k / (kk[0] * 1e-3) / 1e9,
                    "frac": alg_k / (kk[0] * 1e-3) / 1e9 / peak_gbs},
           "gpu_launches": state["launches"], "step_ms": state["step_ms"]}
    for M in (A, B, E, G, R, K):
        M.free()
    return out


def aux_closure(sp, steps, warmup):
    """configs[3]: transitive closure C += C.C to the fixed point of the
    2^18-vertex edge-labelled DAG (label-0 + label-1 union)."""
    timed, state = aux_timer(sp, steps, warmup)
    n = 1 << 18
    (a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9, device="cuda")
    L0 = sp.Matrix.from_pairs(n, n, a0, b0)
    L1 = sp.Matrix.from_pairs(n, n, a1, b1)
    U = sp.ewise_add(L0, L1)
    st = {}

    def step():
        C = U.duplicate()
        st["it"] = sp.TransitiveClosure(C)
        st["nnz"] = C.nvals
        C.free()
    ms_c = timed(step)
    kt = {k: sp.kernel_timing(k)[0] for k in AUX_GROUPS}  # (one breakdown step)
    sp.set_kernel_timing(False)
    out = {"ms": ms_c, "unit": "ms", "vertices": n, "nnz_in": U.nvals, "nnz_closure": st["nnz"],
           "iterations": st["it"], "ms_per_iteration": ms_c / st["it"], "kernel_ms_per_step": kt,
           "kernel_ms_total": sum(kt.values()), "gpu_launches": state["launches"], "step_ms": state["step_ms"]}
    # the paper's incremental use: an index (the
    # closure of the graph without its last 1 % of label-1 edges) receives
    # those edges as an update
    k = (a1.numel() * 99) // 100
    G = sp.ewise_add(L0, sp.Matrix.from_pairs(n, n, a1[:k], b1[:k]))
    D = sp.Matrix.from_pairs(n, n, a1[k:], b1[k:])
    C0, _ = sp.closure(G)
    inc = {}

    def step_inc():
        C = C0.duplicate()
        inc["it"] = sp.TransitiveClosureIncremental(C, D)
        inc["nnz"] = C.nvals
        C.free()
    ms_i = timed(step_inc)
    sp.set_kernel_timing(False)
    out["incremental"] = {"ms": ms_i, "what": "closure(index + update) by spbla_TransitiveClosureIncremental; "
                                              "index = closure of the graph minus the last 1 % of label-1 edges",
                          "nnz_index": C0.nvals, "nnz_update": D.nvals, "nnz_result": inc["nnz"],
                          "steps": inc["it"], "step_ms": state["step_ms"][-1]}
    assert inc["nnz"] == st["nnz"], "incremental closure disagrees with the full closure"
    for M in (C0, G, D, L0, L1, U):
        M.free()
    return out


def run_aux(args):
    """--workload ewise_kron | closure18: the configs[2] / configs[3] rows on
    their own JSON line (they are also embedded in the default line under
    "aux").  1 GPU (replicas-only at N > 1)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import paper_conf_ipps_orachevkkg21_b200 as sp
    torch.cuda.set_device(0)
    sp.Initialize(0)
    peak_gbs, peak_src = load_peaks()
    steps, warmup = args.steps, max(args.warmup, 3)
    clocks = ClockSampler(0)
    if args.workload == "ewise_kron":
        r = aux_ewise_kron(sp, steps, warmup, peak_gbs)
        line = {"metric": "configs[2] EWiseAdd (2^20 rows) + Kronecker (2^10 x 64-state RSM): ms, GB/s vs HBM peak",
                "value": r["ms"], "config": {"workload": "ewise_kron", "baseline_config": "configs[2]",
                                             "l2": "256 MB write between timed steps"},
                "ewise": r["ewise"], "kron": r["kron"], "peak": peak_gbs, "peak_source": peak_src}
    else:
        r = aux_closure(sp, steps, warmup)
        line = {"metric": "configs[3] transitive closure C += C.C to fixed point (2^18-vertex labelled DAG): ms",
                "value": r["ms"], "config": {"workload": "closure18", "baseline_config": "configs[3]",
                                             "vertices": r["vertices"], "nnz_in": r["nnz_in"],
                                             "nnz_closure": r["nnz_closure"], "iterations": r["iterations"],
                                             "l2": "256 MB write between timed steps"},
                "ms_per_iteration": r["ms_per_iteration"], "kernel_ms_per_step": r["kernel_ms_per_step"],
                "incremental": r["incremental"]}
    line.update({"unit": "ms", "higher_is_better": False, "n_gpus": 1, "steps": steps, "warmup": warmup,
                 "dtype": "u32", "data": "synthetic (DESIGN.md §3)", "clocks": clocks.stop(),
                 "gpu_launches": r["gpu_launches"], "step_ms": r["step_ms"],
                 "value_is": "median of the timed steps (each step list in step_ms)"})
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--workload", default=DEFAULT_WORKLOAD, choices=sorted(WORKLOADS) + list(AUX_WORKLOADS))
    ap.add_argument("--impl", default="b200", choices=["b200", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-aux", action="store_true", help="skip the configs[2]/[3] rows in the default line")
    args = ap.parse_args()
    if args.workload in AUX_WORKLOADS:
        return run_aux(args)
    if args.impl == "reference":
        return run_reference(args)
    args.warmup = max(args.warmup, 3)

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(local)
    import torch.distributed as dist
    if world > 1:
        # NCCL over NVLink; SPBLA_DIST_BACKEND=gloo runs several ranks on one GPU (testing only)
        backend = os.environ.get("SPBLA_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
        else:
            dist.init_process_group(backend)
    import paper_conf_ipps_orachevkkg21_b200 as sp
    from paper_conf_ipps_orachevkkg21_b200 import dist as spdist
    sp.Initialize(local)
    stream = torch.cuda.current_stream()
    wl = WORKLOADS[args.workload]

    # ---- setup (untimed): generate, build, plan --------------------------------
    t0 = time.time()
    n, r, c = gen_pairs(wl, "cuda")
    Afull = sp.Matrix.from_pairs(n, n, r, c)
    del r, c
    rp_full, ci_full = Afull.device_tensors()
    ub_full, _ = row_products(rp_full, ci_full, n)
    if world > 1:
        bounds = spdist.product_balanced_bounds(ub_full, world)
    else:
        bounds = [0, n]
    r0, r1 = bounds[rank], bounds[rank + 1]
    if world > 1:
        A = sp.submatrix(Afull, r0, 0, r1 - r0, n)  # this rank's rows of A (and of B = A)
        del rp_full, ci_full
        Afull.free()
        ops = spdist.CudaOps(sp)
    else:
        A = Afull
    ub = ub_full[r0:r1]
    products_local = int(ub.sum())
    products = spdist.allreduce_int(products_local) if world > 1 else products_local
    nnzA = A.nvals
    log(f"[rank {rank}] setup {time.time() - t0:.1f}s: n={n} rows[{r0},{r1}) nnzA={nnzA} "
        f"products(total)={products}")

    C = sp.Matrix.new(r1 - r0, n)

    def step():
        if world > 1:
            return spdist.distributed_mxm(ops, A, A, n, n, C_local=C)
        sp.MxM(C, A, A)
        return C

    flush = torch.empty(FLUSH_BYTES // 4, dtype=torch.int32, device="cuda")
    clocks = ClockSampler(local)  # started before the warm-up: its start-up stays out of the timed steps
    ktime = not os.environ.get("BENCH_NO_KTIME")
    def timed_step():
        # the same body for the warm-up and the timed steps (L2 flush, events)
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step()
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    for i in range(args.warmup):
        if ktime and i == args.warmup - 1:
            sp.set_kernel_timing(True)  # event pool warmed up in the last warm-up step
        timed_step()
    torch.cuda.synchronize()
    nnzC_local = C.nvals

    # ---- timed region ------------------------------------------------------------
    sp.reset_peak_memory()
    sp.reset_launch_count()
    if ktime:
        sp.set_kernel_timing(True)  # (clears the warm-up records)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    t_begin = time.time()
    step_ms = [timed_step() for _ in range(args.steps)]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks.window(t_begin, time.time())
    clk = clocks.stop()
    log(f"[rank {rank}] step ms: {[round(x, 2) for x in step_ms]}")
    launches = sp.launch_count()
    ktimes = {k: sp.kernel_timing(k) for k in
              ("mxm_ub", "warp_bins", "H0", "H1", "H2", "H3", "H4", "H5", "H6", "dense", "dense_ovf", "compact")}
    sp.set_kernel_timing(False)
    peak_mem = sp.memory_stats()[1]
    pool_reserved = sp.pool_stats()[0]  # (device memory the pools hold, incl. the size-class cache)
    red_dev = "cpu" if world > 1 and dist.get_backend() == "gloo" else "cuda"
    tot = torch.tensor([sum(step_ms), peak_mem, nnzC_local, launches], dtype=torch.float64, device=red_dev)
    if world > 1:
        mx = tot.clone()
        dist.all_reduce(mx, op=dist.ReduceOp.MAX)
        sm = tot.clone()
        dist.all_reduce(sm, op=dist.ReduceOp.SUM)
        total_ms, peak_mem_max = float(mx[0]), float(mx[1])
        nnzC, launches_all = int(sm[2]), int(sm[3])
    else:
        total_ms, peak_mem_max, nnzC, launches_all = float(tot[0]), float(tot[1]), int(tot[2]), int(tot[3])
    ms = total_ms / args.steps
    value = products / (ms * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (rank-local, reported by rank 0) ---
    # algorithmic bytes per launch of each timed kernel group;
    # the dominant group is the one with the largest time in the step
    thr = sp.engine_thresholds()
    peak_gbs, peak_src = load_peaks()
    roof = None
    groups = ("mxm_ub", "warp_bins", "H0", "H1", "H2", "H3", "H4", "H5", "H6", "dense", "compact")
    if any(ktimes[k][1] for k in groups):
        rp_a, ci_a = A.device_tensors()
        crp, _ = C.device_tensors()
        lens_a = (rp_a[1:] - rp_a[:-1])
        outs = (crp[1:] - crp[:-1])
        nnz_out = int(crp[-1])
        bins = {"warp_bins": (0, thr[3]), "dense": (thr[10], 1 << 62)}
        bins.update({f"H{i}": (thr[3 + i], thr[4 + i]) for i in range(0, 7)})
        alg = {}
        for k, (lo, hi) in bins.items():
            sel = (ub > lo) & (ub <= hi)
            # 4 B per gathered product, 16 B per segment descriptor, 4 B per
            # output column written to scratch, 44 B per row (work record + count)
            alg[k] = 4 * int(ub[sel].sum()) + 16 * int(lens_a[sel].sum()) + 4 * int(outs[sel].sum()) + 44 * int(sel.sum())
        # upper-bound pass: 44 B per A entry (colidx, B row-offset pair, B span,
        # descriptor write) + 28 B per row, span table 32 B per B row
        alg["mxm_ub"] = 44 * nnzA + 28 * A.nrows + 32 * n
        # compaction: every output column read once and written once
        alg["compact"] = 8 * nnz_out
        per = {}
        for k in groups:
            ms_k, n_k = ktimes[k]
            if n_k:
                lm = ms_k / n_k
                per[k] = {"alg_bytes": alg[k], "launch_ms": lm, "GB/s": alg[k] / (lm * 1e-3) / 1e9,
                          "frac": alg[k] / (lm * 1e-3) / 1e9 / peak_gbs}
        dom = max(per, key=lambda k: ktimes[k][0])
        traffic = None
        tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
        if os.path.exists(tp):
            with open(tp) as f:
                tj = json.load(f)
            traffic = tj.get(args.workload, {}).get(dom)
        roof = {"bound": "hbm", "kernel": dom, "achieved": per[dom]["GB/s"], "peak": peak_gbs, "unit": "GB/s",
                "frac": per[dom]["frac"], "traffic": traffic, "alg_bytes_per_launch": per[dom]["alg_bytes"],
                "launch_ms": per[dom]["launch_ms"], "peak_source": peak_src,
                "kernel_ms_per_step": {k: v[0] / max(1, args.steps) for k, v in ktimes.items()},
                "per_kernel": {k: {"GB/s": round(v["GB/s"], 1), "frac": round(v["frac"], 4),
                                   "alg_bytes": v["alg_bytes"]} for k, v in per.items()}}

    # ---- e2e through the C ABI with host buffers --------------------------------
    e2e = None
    if not args.no_e2e:
        # (the device-timed result is no longer needed: its storage goes back
        # to the pools, so the e2e steps run with the same memory headroom)
        c_rows = C.nrows
        C.free()
        rp_h = torch.empty(A.nrows + 1, dtype=torch.int64).pin_memory()
        ci_h = torch.empty(max(nnzA, 1), dtype=torch.int32).pin_memory()
        A.export_csr(rp_h, ci_h[:nnzA])
        crp_h = torch.empty(c_rows + 1, dtype=torch.int64).pin_memory()
        cci_h = torch.empty(max(nnzC_local, 1), dtype=torch.int32).pin_memory()
        Ae = sp.Matrix.new(A.nrows, n)
        Ce = sp.Matrix.new(c_rows, n)
        e2e_steps = min(args.steps, 3)
        e2e_ms = []
        h2d = (A.nrows + 1) * 8 + nnzA * 4
        d2h = (c_rows + 1) * 8 + nnzC_local * 4
        for i in range(e2e_steps + 2):  # (two untimed steps: the pools' blocks reach their steady state)
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            t = time.perf_counter()
            Ae.import_csr(rp_h, ci_h[:nnzA])
            if world > 1:
                spdist.distributed_mxm(ops, Ae, Ae, n, n, C_local=Ce)
            else:
                sp.MxM(Ce, Ae, Ae)
            Ce.export_csr(crp_h, cci_h[:nnzC_local])
            torch.cuda.synchronize()
            if i >= 2:
                e2e_ms.append(1e3 * (time.perf_counter() - t))
        et = torch.tensor([sum(e2e_ms) / len(e2e_ms)], dtype=torch.float64, device=red_dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
        e2e = {"value": products / (float(et) * 1e-3) / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": d2h, "ms_per_step": float(et), "steps": e2e_steps,
               "path": "ImportCSR(pinned host) -> MxM -> ExportCSR(pinned host)"}
        Ae.free()
        Ce.free()

    # ---- CPU oracle baseline (rank 0, N = 1) --------------------------------------
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rp_h, ci_h = A.to_csr()
        p, dt, nr_s, thr, _ = cpu_oracle_sample(rp_h, ci_h, ub.cpu().numpy(),
                                                float(os.environ.get("CPU_SAMPLE_PRODUCTS", "2e8")))
        cpu = {"value": p / dt / 1e9, "unit": UNIT, "cores": thr, "kind": "oracle",
               "sample": f"{4 * thr} contiguous row chunks spread over {args.workload} ({nr_s} rows, {p} products); "
                         f"{dt:.1f}s wall of the unchanged std::set Gustavson oracle on {thr} threads"}

    # ---- the other BASELINE rows (configs[2], configs[3]), 1 GPU ----------------
    aux = None
    if world == 1 and not args.no_aux:
        C.free()
        A.free()
        torch.cuda.empty_cache()
        aux_steps, aux_warm = max(args.steps, 9), 5
        aux = {"configs[2] ewise_kron": aux_ewise_kron(sp, aux_steps, aux_warm, peak_gbs),
               "configs[3] closure18": aux_closure(sp, aux_steps, aux_warm),
               "note": "device-timed medians (CUDA events on the library stream, 256 MB L2 flush per step); "
                       "step lists in step_ms"}

    if rank == 0:
        a_, b_, c_ = wl["abc"] if wl["abc"] else (None, None, None)
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (seeded R-MAT, DESIGN.md §3)",
            "config": {"workload": args.workload, "baseline_config": wl["config"], "rows": n,
                       "edge_factor": wl["ef"], "rmat_abc": wl["abc"], "nnz_A": int(nnzA) if world == 1 else None,
                       "products": products, "nnz_C": nnzC, "parallelism": f"rows{world}",
                       "l2": "A larger than L2 (126 MB) and a 256 MB write between timed steps",
                       "peak_mem_gb": peak_mem_max / 1e9},
            "peak_mem_gb": peak_mem_max / 1e9,
            "pool_reserved_gb_rank0": pool_reserved / 1e9,
            "gpu_launches": launches_all,
            "clocks": clk,
            "roofline": roof,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "aux": aux,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
