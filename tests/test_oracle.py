"""Pins for the CPU oracle (runs without a GPU).

Each test checks the oracle against something other than itself: hand-worked
golden fixtures, dense Boolean brute force (explicit loops or numpy integer
matmul thresholded, n <= 64), algebraic laws, scipy.sparse, and BFS
reachability.  A dropped term, a wrong index or a transposed operand in
oracle/spbla_oracle.cpp fails at least one of them.
"""
import collections

import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
import spgen
from golden_io import load


def G(m):
    nr, nc, r, c = m
    return oracle.build(nr, nc, r, c)


def rand_dense(rng, m, n, density):
    d = rng.random((m, n)) < density
    return d


def dense_mm(a, b):
    return (a.astype(np.int64) @ b.astype(np.int64)) > 0


# ----------------------------------------------------------------- golden

def test_golden_mxm():
    mats, _ = load("mxm_3x4x3.txt")
    A, B = G(mats["A"]), G(mats["B"])
    assert oracle.mxm(A, B) == G(mats["C"])
    assert oracle.mxm(A, B, G(mats["Cin"])) == G(mats["Cacc"])


def test_golden_kronecker():
    mats, _ = load("kron_2x2_2x3.txt")
    K = oracle.kronecker(G(mats["A"]), G(mats["B"]))
    assert K == G(mats["K"])
    assert K.nvals == 9


@pytest.mark.parametrize("name", ["closure_chain4.txt", "closure_cycle3.txt"])
def test_golden_closure(name):
    mats, sc = load(name)
    C, it = oracle.closure(G(mats["A"]))
    assert C == G(mats["C"])
    assert it == sc["iterations"]


def test_golden_misc():
    mats, _ = load("misc_ops.txt")
    A = G(mats["A"])
    assert oracle.transpose(A) == G(mats["T"])
    assert oracle.reduce_to_column(A) == G(mats["V"])
    assert oracle.submatrix(A, 1, 1, 2, 3) == G(mats["S"])
    assert oracle.ewise_add(A, G(mats["A2"])) == G(mats["E"])


# ----------------------------------------------------------------- build

def test_build_sorted_dedup():
    rng = np.random.default_rng(1)
    r = rng.integers(0, 50, 3000)
    c = rng.integers(0, 70, 3000)
    M = oracle.build(50, 70, r, c)
    want = sorted(set(zip(r.tolist(), c.tolist())))
    got = list(zip(*[x.tolist() for x in M.pairs()]))
    assert got == want
    assert M.rowptr[0] == 0 and M.rowptr[-1] == len(want)


def test_build_out_of_range():
    with pytest.raises(IndexError):
        oracle.build(4, 4, [0, 4], [0, 0])
    with pytest.raises(IndexError):
        oracle.build(4, 4, [0], [7])


def test_build_empty():
    M = oracle.build(5, 3, [], [])
    assert M.nvals == 0 and list(M.rowptr) == [0] * 6


# ----------------------------------------------------------------- mxm

def explicit_mm(a, b):
    """Triple loop, straight from l.210-211: C[i][j] = OR_k A[i][k] AND B[k][j]."""
    m, k = a.shape
    n = b.shape[1]
    c = np.zeros((m, n), dtype=bool)
    for i in range(m):
        for j in range(n):
            acc = False
            for t in range(k):
                acc = acc or (bool(a[i, t]) and bool(b[t, j]))
            c[i, j] = acc
    return c


def test_mxm_explicit_loops_tiny():
    rng = np.random.default_rng(7)
    for (m, k, n) in [(1, 1, 1), (3, 5, 2), (7, 4, 9), (12, 12, 12)]:
        for dens in (0.0, 0.2, 0.6, 1.0):
            a = rand_dense(rng, m, k, dens)
            b = rand_dense(rng, k, n, dens)
            C = oracle.mxm(oracle.from_dense(a), oracle.from_dense(b))
            assert np.array_equal(C.to_dense(), explicit_mm(a, b))


@pytest.mark.parametrize("seed", range(6))
def test_mxm_dense_bruteforce(seed):
    rng = np.random.default_rng(100 + seed)
    m, k, n = rng.integers(1, 65, 3)
    dens = [0.01, 0.05, 0.15, 0.4][seed % 4]
    a = rand_dense(rng, m, k, dens)
    b = rand_dense(rng, k, n, dens)
    a[rng.integers(0, m)] = False           # an empty row
    b[:, rng.integers(0, n)] = False        # an empty column
    C = oracle.mxm(oracle.from_dense(a), oracle.from_dense(b))
    assert np.array_equal(C.to_dense(), dense_mm(a, b))
    c0 = rand_dense(rng, m, n, dens)
    Cacc = oracle.mxm(oracle.from_dense(a), oracle.from_dense(b), oracle.from_dense(c0))
    assert np.array_equal(Cacc.to_dense(), c0 | dense_mm(a, b))


def test_mxm_identity_zero_laws():
    rng = np.random.default_rng(3)
    a = rand_dense(rng, 40, 30, 0.1)
    A = oracle.from_dense(a)
    I30 = oracle.from_dense(np.eye(30, dtype=bool))
    I40 = oracle.from_dense(np.eye(40, dtype=bool))
    Z = oracle.from_dense(np.zeros((30, 17), dtype=bool))
    assert oracle.mxm(A, I30) == A
    assert oracle.mxm(I40, A) == A
    assert oracle.mxm(A, Z).nvals == 0
    assert oracle.mxm(A, Z, A if False else None).nvals == 0
    # accumulate into itself with a zero product is the identity
    Zs = oracle.from_dense(np.zeros((30, 30), dtype=bool))
    assert oracle.mxm(A, Zs, A) == A


def test_mxm_associative():
    rng = np.random.default_rng(4)
    a = oracle.from_dense(rand_dense(rng, 50, 40, 0.05))
    b = oracle.from_dense(rand_dense(rng, 40, 60, 0.05))
    c = oracle.from_dense(rand_dense(rng, 60, 30, 0.05))
    assert oracle.mxm(oracle.mxm(a, b), c) == oracle.mxm(a, oracle.mxm(b, c))


def to_scipy(M):
    return sp.csr_matrix((np.ones(M.nvals, dtype=np.int64), M.colidx.astype(np.int64),
                          M.rowptr.astype(np.int64)), shape=(M.nrows, M.ncols))


def from_scipy_bool(S):
    S = S.tocsr()
    S.sum_duplicates()
    S.eliminate_zeros()
    S.sort_indices()
    return oracle.Csr(S.shape[0], S.shape[1], S.indptr, S.indices)


def test_mxm_scipy_config1():
    """BASELINE configs[0]: 4096 x 4096 uniform, 8 draws/row, A.A."""
    r, c = spgen.uniform_pairs(4096, 4096, 8, seed=1)
    A = oracle.build(4096, 4096, r.numpy(), c.numpy())
    C = oracle.mxm(A, A)
    S = to_scipy(A)
    assert C == from_scipy_bool(S @ S)


def test_mxm_scipy_rmat():
    r, c = spgen.rmat_pairs(11, 8, 0.45, 0.22, 0.22, seed=2)
    A = oracle.build(2048, 2048, r.numpy(), c.numpy())
    C = oracle.mxm(A, A, A)
    S = to_scipy(A)
    assert C == from_scipy_bool(S @ S + S)


def test_mxm_rows_matches_full():
    r, c = spgen.rmat_pairs(10, 8, 0.45, 0.22, 0.22, seed=3)
    A = oracle.build(1024, 1024, r.numpy(), c.numpy())
    full = oracle.mxm(A, A).to_dense()
    rows = np.array([0, 5, 1023, 17, 17, 512], dtype=np.uint32)
    part = oracle.mxm_rows(A, A, rows).to_dense()
    assert np.array_equal(part, full[rows.astype(np.int64)])
    acc = oracle.mxm_rows(A, A, rows, A).to_dense()
    assert np.array_equal(acc, full[rows.astype(np.int64)] | A.to_dense()[rows.astype(np.int64)])


# ----------------------------------------------------------------- ewise add

def test_ewise_add_dense_and_laws():
    rng = np.random.default_rng(5)
    for (m, n, d) in [(1, 1, 0.5), (30, 64, 0.1), (64, 5, 0.5), (20, 20, 0.0)]:
        a = rand_dense(rng, m, n, d)
        b = rand_dense(rng, m, n, d)
        A, B = oracle.from_dense(a), oracle.from_dense(b)
        E = oracle.ewise_add(A, B)
        assert np.array_equal(E.to_dense(), a | b)
        assert oracle.ewise_add(B, A) == E
        assert oracle.ewise_add(A, A) == A
        assert oracle.ewise_add(A, oracle.from_dense(np.zeros((m, n), bool))) == A


def test_ewise_add_scipy():
    r1, c1 = spgen.rmat_pairs(12, 8, 0.45, 0.22, 0.22, seed=5)
    r2, c2 = spgen.uniform_pairs(4096, 4096, 8, seed=6)
    A = oracle.build(4096, 4096, r1.numpy(), c1.numpy())
    B = oracle.build(4096, 4096, r2.numpy(), c2.numpy())
    assert oracle.ewise_add(A, B) == from_scipy_bool(to_scipy(A) + to_scipy(B))


# ----------------------------------------------------------------- kronecker

def test_kronecker_dense():
    rng = np.random.default_rng(6)
    for (ma, na, mb, nb, d) in [(1, 1, 1, 1, 1.0), (5, 7, 3, 4, 0.3), (8, 8, 8, 8, 0.2),
                                 (6, 2, 1, 9, 0.5), (4, 4, 4, 4, 0.0)]:
        a = rand_dense(rng, ma, na, d)
        b = rand_dense(rng, mb, nb, d)
        K = oracle.kronecker(oracle.from_dense(a), oracle.from_dense(b))
        assert np.array_equal(K.to_dense(), np.kron(a.astype(int), b.astype(int)) > 0)


def test_kronecker_nnz_law():
    rg, cg = spgen.rmat_pairs(8, 8, 0.45, 0.22, 0.22, seed=7)
    G_ = oracle.build(256, 256, rg.numpy(), cg.numpy())
    rr, cr = spgen.rsm_pairs(16, 1, 2, seed=8)
    R = oracle.build(16, 16, rr.numpy(), cr.numpy())
    K = oracle.kronecker(G_, R)
    assert K.nvals == G_.nvals * R.nvals
    assert K.nrows == 256 * 16 and K.ncols == 256 * 16
    assert oracle.kronecker(R, G_).nvals == G_.nvals * R.nvals
    S = sp.kron(to_scipy(G_), to_scipy(R), format="csr")
    assert K == from_scipy_bool(S)


# ----------------------------------------------------------------- transpose / reduce / submatrix

def test_transpose_dense_and_product_law():
    rng = np.random.default_rng(9)
    a = rand_dense(rng, 33, 47, 0.1)
    b = rand_dense(rng, 47, 21, 0.1)
    A, B = oracle.from_dense(a), oracle.from_dense(b)
    assert np.array_equal(oracle.transpose(A).to_dense(), a.T)
    assert oracle.transpose(oracle.transpose(A)) == A
    lhs = oracle.transpose(oracle.mxm(A, B))
    rhs = oracle.mxm(oracle.transpose(B), oracle.transpose(A))
    assert lhs == rhs


def test_reduce_dense():
    rng = np.random.default_rng(10)
    a = rand_dense(rng, 64, 20, 0.03)
    V = oracle.reduce_to_column(oracle.from_dense(a))
    assert V.ncols == 1
    assert np.array_equal(V.to_dense()[:, 0], a.any(axis=1))


def test_submatrix_dense():
    rng = np.random.default_rng(11)
    a = rand_dense(rng, 40, 50, 0.2)
    A = oracle.from_dense(a)
    for (i0, j0, nr, nc) in [(0, 0, 40, 50), (3, 7, 10, 20), (39, 49, 1, 1), (5, 5, 0, 3), (0, 10, 40, 0)]:
        S = oracle.submatrix(A, i0, j0, nr, nc)
        assert np.array_equal(S.to_dense(), a[i0:i0 + nr, j0:j0 + nc])


# ----------------------------------------------------------------- closure

def bfs_reach(n, rows, cols):
    adj = collections.defaultdict(list)
    for i, j in zip(rows.tolist(), cols.tolist()):
        adj[i].append(j)
    out = np.zeros((n, n), dtype=bool)
    for s in range(n):
        seen = set()
        dq = collections.deque(adj[s])
        while dq:
            v = dq.popleft()
            if v in seen:
                continue
            seen.add(v)
            dq.extend(adj[v])
        for v in seen:
            out[s, v] = True
    return out


@pytest.mark.parametrize("seed", range(4))
def test_closure_bfs(seed):
    rng = np.random.default_rng(200 + seed)
    n = int(rng.integers(2, 64))
    a = rand_dense(rng, n, n, [0.02, 0.05, 0.1, 0.3][seed])
    A = oracle.from_dense(a)
    C, it = oracle.closure(A)
    r, c = np.nonzero(a)
    assert np.array_equal(C.to_dense(), bfs_reach(n, r, c))
    assert it >= 1


def test_closure_labeled_dag_bfs():
    (r0, c0), (r1, c1) = spgen.labeled_dag(600, 0.25, seed=9)
    r = np.concatenate([r0.numpy(), r1.numpy()])
    c = np.concatenate([c0.numpy(), c1.numpy()])
    A = oracle.build(600, 600, r, c)
    C, it = oracle.closure(A)
    assert np.array_equal(C.to_dense(), bfs_reach(600, r, c))
    # squaring doubles path length per iteration: depth d needs ~log2(d)+1 rounds
    assert 2 <= it <= 12


# ----------------------------------------------------------------- generators

def test_generator_hash_matches_python_ints():
    ctr = torch.arange(0, 5000, dtype=torch.int64) * 7919 + 3
    h = spgen.hash64(5, 3, ctr)
    for i in range(0, 5000, 37):
        assert (int(h[i]) & ((1 << 64) - 1)) == spgen.hash64_int(5, 3, int(ctr[i]))


def test_generator_deterministic_and_in_range():
    r1, c1 = spgen.rmat_pairs(10, 4, 0.45, 0.22, 0.22, seed=11)
    r2, c2 = spgen.rmat_pairs(10, 4, 0.45, 0.22, 0.22, seed=11)
    assert torch.equal(r1, r2) and torch.equal(c1, c2)
    assert int(r1.min()) >= 0 and int(r1.max()) < 1024 and int(c1.max()) < 1024
    # scramble is a bijection
    v = torch.arange(1 << 12, dtype=torch.int64)
    assert torch.unique(spgen.scramble(v, 12, 3)).numel() == 1 << 12
    # power-law: max out-degree far above the mean
    deg = torch.bincount(r1.long(), minlength=1024)
    assert deg.max() > 4 * deg.float().mean()


def test_parallel_driver_matches_serial_oracle():
    """oracle/parallel.py only chunks rows: its results equal the serial oracle."""
    import threading
    from oracle import parallel as par
    n = 1 << 12
    r, c = spgen.rmat_pairs(12, 8, 0.45, 0.22, 0.22, seed=7)
    A = oracle.build(n, n, r.numpy(), c.numpy())
    assert par.build_chunked(n, n, r.numpy(), c.numpy(), block_rows=300, threads=4) == A
    want = oracle.mxm(A, A, A)
    w = par.row_products(A, A)
    ch = par.chunk_bounds(w, float(w.sum()) / 13)
    assert ch[0][0] == 0 and ch[-1][1] == n and all(a[1] == b[0] for a, b in zip(ch[:-1], ch[1:]))
    got = {}
    lk = threading.Lock()

    def keep(r0, r1, R):
        with lk:
            got[r0] = R
    par.mxm_rows_chunked(A, A, ch, keep, c=A, threads=4)
    rp = [np.zeros(1, np.uint64)]
    base = np.uint64(0)
    for r0, _ in ch:
        rp.append(got[r0].rowptr[1:] + base)
        base += np.uint64(got[r0].nvals)
    assert np.array_equal(np.concatenate(rp), want.rowptr)
    assert np.array_equal(np.concatenate([got[r0].colidx for r0, _ in ch]), want.colidx)


@pytest.mark.parametrize("n,p,seed", [(1500, 0.25, 9), (3000, 0.6, 2)])
def test_dag_dp_matches_oracle_closure(n, p, seed):
    """The full-size closure check's independent DAG dynamic program agrees
    with the oracle's C += C.C loop, including the iteration count
    ceil(log2 D) + 1 (R9)."""
    from helpers import dag_reach_and_depth
    (a0, b0), (a1, b1) = spgen.labeled_dag(n, p, seed=seed)
    src = np.concatenate([a0.numpy(), a1.numpy()])
    dst = np.concatenate([b0.numpy(), b1.numpy()])
    want, it = oracle.closure(oracle.build(n, n, src, dst))
    got, D = dag_reach_and_depth(n, src, dst)
    assert got == want
    assert it == int(np.ceil(np.log2(D))) + 1
