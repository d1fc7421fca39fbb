"""BASELINE.json configs at FULL size, in the launch configuration bench.py
times, compared bit for bit over EVERY row:

* configs[1] / configs[4] (A.A on R-MAT 2^20 / 2^22): A built by the CUDA
  Matrix_Build against the unchanged oracle's build (row blocks on all host
  cores), then C = A.A against the unchanged oracle's ``mxm_rows`` over row
  chunks on all host cores (``oracle/parallel.py``: ctypes releases the GIL,
  so a thread pool is truly parallel).  Every rowptr entry and every column
  of C is compared.  configs[1] also checks C += A.A (accumulate) the same way.
* configs[3] (closure of the 2^18-vertex labelled DAG): the whole closure
  CSR against reachability computed by an independent dynamic program over
  the DAG (edges point to smaller ids, so vertices in increasing order see
  their successors' closures complete), and the exact iteration count of the
  C += C.C loop from the same DP's longest shortest-path length D: after k
  evaluations C holds the paths of length 1..2^k, and the loop stops at the
  first evaluation that adds nothing, k* = ceil(log2 D) + 1 (R9).
* configs[2] (EWiseAdd 2^20 + Kronecker 2^10 (x) 64): whole CSR vs the oracle.
"""
import threading

import numpy as np
import pytest
import torch

import oracle
import spgen
from oracle import parallel as par
from helpers import assert_same, dag_reach_and_depth, gpu_lib

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    return gpu_lib()


def validate_on_device(sp, M):
    rp, ci = M.device_tensors()
    sp.Matrix.wrap(M.nrows, M.ncols, rp, ci, hints=sp.HINT_VALIDATE).free()  # raises on violation


def compare_csr_chunked(C, want_rows, chunks):
    """Every row of device matrix C against want_rows(r0, r1) -> oracle Csr of
    rows [r0, r1), chunk by chunk on all host cores.  Returns nnz checked."""
    rp_d, ci_d = C.device_tensors()
    rp = rp_d.cpu().numpy().view(np.uint64)
    assert rp[0] == 0 and int(rp[-1]) == C.nvals
    errs, lk = [], threading.Lock()
    checked = [0]

    def one(r0, r1):
        R = want_rows(r0, r1)
        b, e = int(rp[r0]), int(rp[r1])
        msg = None
        if not np.array_equal(R.rowptr + np.uint64(b), rp[r0:r1 + 1]):
            bad = np.nonzero(R.rowptr + np.uint64(b) != rp[r0:r1 + 1])[0][0]
            msg = f"rowptr differs first at row {r0 + bad}"
        else:
            got = ci_d[b:e].cpu().numpy().view(np.uint32)
            if not np.array_equal(got, R.colidx):
                bad = np.nonzero(got != R.colidx)[0][0]
                row = r0 + int(np.searchsorted(R.rowptr, bad, side="right")) - 1
                msg = f"colidx differs first at position {b + bad} (row {row})"
        with lk:
            checked[0] += R.nvals
            if msg:
                errs.append(msg)

    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(max_workers=par.host_cores()) as ex:
        list(ex.map(lambda ch: one(*ch), chunks))
    assert not errs, f"{len(errs)} chunks differ: {errs[:3]}"
    assert checked[0] == C.nvals
    return checked[0]


def mxm_chunks(Ah, Bh):
    w = par.row_products(Ah, Bh)
    return par.chunk_bounds(w, max(float(w.sum()) / (par.host_cores() * 24), 1e6))


@pytest.mark.parametrize("wl", ["rmat20_ef16", "rmat22_ef32"])
def test_mxm_full_size_exact(sp, wl):
    import bench
    cfg = bench.WORKLOADS[wl]
    n, r, c = bench.gen_pairs(cfg, "cuda")  # seeded generator (bit-identical on CPU and GPU)
    A = sp.Matrix.from_pairs(n, n, r, c)
    Ah = par.build_chunked(n, n, r.cpu().numpy(), c.cpu().numpy())
    del r, c
    torch.cuda.empty_cache()
    compare_csr_chunked(A, lambda r0, r1: oracle.Csr(
        r1 - r0, n, Ah.rowptr[r0:r1 + 1] - Ah.rowptr[r0], Ah.colidx[int(Ah.rowptr[r0]):int(Ah.rowptr[r1])]),
        par.chunk_bounds(np.diff(Ah.rowptr.astype(np.int64)), 4e6))
    C = sp.mxm(A, A)
    validate_on_device(sp, C)
    chunks = mxm_chunks(Ah, Ah)
    nnz = compare_csr_chunked(C, lambda r0, r1: oracle.mxm_rows(Ah, Ah, np.arange(r0, r1, dtype=np.uint32)),
                              chunks)
    print(f"{wl}: nnz(A) {Ah.nvals}, nnz(A.A) {nnz}: every row bit-exact vs the oracle")
    C.free()
    if wl == "rmat20_ef16":  # C += A.A (accumulate, C = A) in the same configuration
        Cacc = A.duplicate()
        sp.MxM(Cacc, A, A, accumulate=True)
        validate_on_device(sp, Cacc)
        compare_csr_chunked(Cacc, lambda r0, r1: oracle.mxm_rows(Ah, Ah, np.arange(r0, r1, dtype=np.uint32), Ah),
                            chunks)
        Cacc.free()
    A.free()


def test_ewise_kron_config2_full(sp):
    n = 1 << 20
    r1, c1 = spgen.rmat_pairs(20, 16, 0.45, 0.22, 0.22, seed=1)
    r2, c2 = spgen.uniform_pairs(n, n, 8, seed=2)
    A = sp.Matrix.from_pairs(n, n, r1.cuda(), c1.cuda())
    B = sp.Matrix.from_pairs(n, n, r2.cuda(), c2.cuda())
    E = sp.ewise_add(A, B)
    OA = par.build_chunked(n, n, r1.numpy(), c1.numpy())
    OB = par.build_chunked(n, n, r2.numpy(), c2.numpy())
    assert_same(A, OA, "A")
    assert_same(B, OB, "B")
    assert_same(E, oracle.ewise_add(OA, OB), "A+B full")
    rg, cg = spgen.rmat_pairs(10, 16, 0.45, 0.22, 0.22, seed=3)
    rr, cr = spgen.rsm_pairs(64, 1, 2, seed=4)
    G = sp.Matrix.from_pairs(1024, 1024, rg.cuda(), cg.cuda())
    R = sp.Matrix.from_pairs(64, 64, rr.cuda(), cr.cuda())
    K = sp.kronecker(G, R)
    assert_same(K, oracle.kronecker(oracle.build(1024, 1024, rg.numpy(), cg.numpy()),
                                    oracle.build(64, 64, rr.numpy(), cr.numpy())), "G(x)R full")


def test_closure_config3_full_exact(sp):
    """configs[3]: the whole closure CSR of the 2^18-vertex edge-labelled DAG
    and the exact number of C += C.C evaluations."""
    n = 1 << 18
    (a0, b0), (a1, b1) = spgen.labeled_dag(n, 0.25, seed=9)
    L0 = sp.Matrix.from_pairs(n, n, a0.cuda(), b0.cuda())
    L1 = sp.Matrix.from_pairs(n, n, a1.cuda(), b1.cuda())
    U = sp.ewise_add(L0, L1)
    C, it = sp.closure(U)
    validate_on_device(sp, C)
    want, D = dag_reach_and_depth(n, np.concatenate([a0.numpy(), a1.numpy()]),
                                  np.concatenate([b0.numpy(), b1.numpy()]))
    assert_same(C, want, "closure(configs[3]) vs DAG reachability")
    k_star = int(np.ceil(np.log2(D))) + 1 if D > 1 else 1
    assert it == k_star, f"iterations {it}, expected ceil(log2 {D}) + 1 = {k_star}"
    print(f"closure: nnz {C.nvals}, D = {D}, {it} evaluations")
