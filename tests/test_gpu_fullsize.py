"""BASELINE.json configs at full size, in the launch configuration bench.py
times: the CUDA result is checked on sampled rows against the oracle computed
row by row (heaviest rows and a representative of every bin included), and
for all rows by properties that hold at any size (CSR invariants on the
device, nnz and row counts)."""
import collections

import numpy as np
import pytest
import torch

import oracle
import spgen
from helpers import assert_same, gpu_lib

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    return gpu_lib()


def host_csr(M):
    rp, ci = M.to_csr()
    return oracle.Csr(M.nrows, M.ncols, rp, ci)


def check_rows(C, A, rows, Cin=None):
    """C's rows `rows` equal the oracle's (C_in +) A.A rows, bit for bit."""
    Ah = host_csr(A)
    want = oracle.mxm_rows(Ah, Ah, rows, host_csr(Cin) if Cin is not None else None)
    rp, ci = C.device_tensors()
    rows_t = torch.as_tensor(rows.astype(np.int64), device="cuda")
    b, e = rp[rows_t].cpu().numpy(), rp[rows_t + 1].cpu().numpy()
    ci_h = ci.cpu().numpy().astype(np.uint32) if C.nvals < (1 << 31) else None
    for t, r in enumerate(rows):
        got = (ci_h[b[t]:e[t]] if ci_h is not None else ci[int(b[t]):int(e[t])].cpu().numpy().astype(np.uint32))
        exp = want.colidx[int(want.rowptr[t]):int(want.rowptr[t + 1])]
        assert np.array_equal(got, exp), f"row {r}: {len(got)} vs {len(exp)} entries"


def sample_rows(ub, n, k=300, seed=0):
    rng = np.random.default_rng(seed)
    ub_h = ub.cpu().numpy()
    heavy = np.argsort(ub_h)[-20:]
    edges = [0, 1, 33, 65, 129, 257, 513, 1025, 2049, 4097, 8193, 20481, 40961, 1 << 62]
    per_bin = []
    for lo, hi in zip(edges[:-1], edges[1:]):
        idx = np.nonzero((ub_h >= lo) & (ub_h < hi))[0]
        if len(idx):
            per_bin.append(rng.choice(idx, min(10, len(idx)), replace=False))
    rnd = rng.integers(0, n, k)
    return np.unique(np.concatenate([heavy, rnd, *per_bin, [0, n - 1]])).astype(np.uint32)


def ub_of(A):
    rp, ci = A.device_tensors()
    lens = rp[1:] - rp[:-1]
    rows = torch.repeat_interleave(torch.arange(A.nrows, device="cuda"), lens)
    return torch.zeros(A.nrows, dtype=torch.int64, device="cuda").index_add_(0, rows, lens[ci.long()])


def validate_on_device(sp, M):
    rp, ci = M.device_tensors()
    sp.Matrix.wrap(M.nrows, M.ncols, rp, ci, hints=sp.HINT_VALIDATE).free()  # raises on violation


@pytest.mark.parametrize("wl", ["rmat20_ef16", "rmat22_ef32"])
def test_mxm_full_size_sampled(sp, wl):
    import bench
    cfg = bench.WORKLOADS[wl]
    n, r, c = bench.gen_pairs(cfg, "cuda")
    A = sp.Matrix.from_pairs(n, n, r, c)
    del r, c
    ub = ub_of(A)
    C = sp.mxm(A, A)
    validate_on_device(sp, C)
    assert C.nvals <= int(ub.sum())
    rows = sample_rows(ub, n)
    check_rows(C, A, rows)
    C.free()
    if wl == "rmat20_ef16":  # accumulate in the same configuration
        Cacc = A.duplicate()
        sp.MxM(Cacc, A, A, accumulate=True)
        validate_on_device(sp, Cacc)
        check_rows(Cacc, A, rows[:120], Cin=A)


def test_ewise_kron_config2_full(sp):
    n = 1 << 20
    r1, c1 = spgen.rmat_pairs(20, 16, 0.45, 0.22, 0.22, seed=1)
    r2, c2 = spgen.uniform_pairs(n, n, 8, seed=2)
    A = sp.Matrix.from_pairs(n, n, r1.cuda(), c1.cuda())
    B = sp.Matrix.from_pairs(n, n, r2.cuda(), c2.cuda())
    E = sp.ewise_add(A, B)
    OA = oracle.build(n, n, r1.numpy(), c1.numpy())
    OB = oracle.build(n, n, r2.numpy(), c2.numpy())
    assert_same(A, OA, "A")
    assert_same(E, oracle.ewise_add(OA, OB), "A+B full")
    rg, cg = spgen.rmat_pairs(10, 16, 0.45, 0.22, 0.22, seed=3)
    rr, cr = spgen.rsm_pairs(64, 1, 2, seed=4)
    G = sp.Matrix.from_pairs(1024, 1024, rg.cuda(), cg.cuda())
    R = sp.Matrix.from_pairs(64, 64, rr.cuda(), cr.cuda())
    K = sp.kronecker(G, R)
    assert_same(K, oracle.kronecker(oracle.build(1024, 1024, rg.numpy(), cg.numpy()),
                                    oracle.build(64, 64, rr.numpy(), cr.numpy())), "G(x)R full")


def test_closure_config3_full_sampled(sp):
    """configs[3]: closure of a 2^18-vertex edge-labelled DAG; sampled rows
    against BFS reachability (paths of length >= 1)."""
    n = 1 << 18
    (a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9)
    L0 = sp.Matrix.from_pairs(n, n, a0.cuda(), b0.cuda())
    L1 = sp.Matrix.from_pairs(n, n, a1.cuda(), b1.cuda())
    U = sp.ewise_add(L0, L1)
    C, it = sp.closure(U)
    validate_on_device(sp, C)
    assert 2 <= it <= 40
    adj = collections.defaultdict(list)
    for x, y in zip(np.concatenate([a0.numpy(), a1.numpy()]).tolist(),
                    np.concatenate([b0.numpy(), b1.numpy()]).tolist()):
        adj[x].append(y)
    rp, ci = C.to_csr()
    rng = np.random.default_rng(1)
    for s in list(rng.integers(0, n, 150)) + [n - 1, 0]:
        seen, st = set(), list(adj[int(s)])
        while st:
            v = st.pop()
            if v in seen:
                continue
            seen.add(v)
            st.extend(adj[v])
        got = ci[int(rp[s]):int(rp[s + 1])]
        assert np.array_equal(got, np.array(sorted(seen), dtype=np.uint32)), f"source {s}"
