"""Randomised shape sweep of the CUDA path against the oracle (bit-exact
CSR): seeded cases with extreme shapes and densities -- one column, one row,
empty rows, dense rows, 2^31-wide column spaces, skewed row lengths -- for
MxM (plain, accumulate, aliased), EWiseAdd, Kronecker, Transpose, Reduce and
SubMatrix.  Complements the structured tests in test_gpu_parity.py."""
import numpy as np
import pytest

import oracle
from helpers import assert_same, both_from_pairs, gpu_lib

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    return gpu_lib()


def rand_pairs(rng, m, n, kind):
    if m == 0 or n == 0:
        return np.zeros(0, np.uint32), np.zeros(0, np.uint32)
    if kind == "uniform":
        nv = int(rng.integers(0, 4 * m + 1))
        r = rng.integers(0, m, nv)
    elif kind == "skewed":  # a few heavy rows, many empty ones
        nv = int(rng.integers(1, 40 * m + 1))
        r = np.minimum(rng.zipf(1.6, nv) - 1, m - 1)
    else:  # "dense": some fully dense rows
        rows = rng.choice(m, size=max(1, m // 8), replace=False)
        r = np.repeat(rows, min(n, 3000))
        nv = len(r)
    if kind == "dense":
        c = np.concatenate([rng.permutation(min(n, 3000)) for _ in range(len(r) // min(n, 3000))]) if nv else r
        c = (c.astype(np.int64) * max(1, n // 3000)) % n
    else:
        c = rng.integers(0, n, nv)
    return r.astype(np.uint32), c.astype(np.uint32)


CASES = [(s, kind) for s in range(12) for kind in ("uniform", "skewed", "dense")]


@pytest.mark.parametrize("seed,kind", CASES)
def test_random_mxm_ewise(sp, seed, kind):
    rng = np.random.default_rng(1000 + seed)
    dims = [1, 2, 31, 33, 257, 1000, 4096]
    m, k = (int(rng.choice(dims)) for _ in range(2))
    n = int(rng.choice(dims + [1 << 20, (1 << 31) + 7]))
    A, OA = both_from_pairs(sp, m, k, *rand_pairs(rng, m, k, kind))
    B, OB = both_from_pairs(sp, k, n, *rand_pairs(rng, k, n, kind))
    assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), f"A.B {m}x{k}x{n} {kind}")
    C, OC = both_from_pairs(sp, m, n, *rand_pairs(rng, m, n, "uniform"))
    sp.MxM(C, A, B, accumulate=True)
    assert_same(C, oracle.mxm(OA, OB, OC), "C += A.B")
    D, OD = both_from_pairs(sp, m, n, *rand_pairs(rng, m, n, kind))
    assert_same(sp.ewise_add(C, D), oracle.ewise_add(oracle.mxm(OA, OB, OC), OD), "C + D")
    assert_same(sp.transpose(A), oracle.transpose(OA), "A^T")
    assert_same(sp.reduce_to_column(A), oracle.reduce_to_column(OA), "reduce")
    if m > 1 and k > 1:
        i0, j0 = int(rng.integers(0, m)), int(rng.integers(0, k))
        nr, nc = int(rng.integers(0, m - i0 + 1)), int(rng.integers(0, k - j0 + 1))
        assert_same(sp.submatrix(A, i0, j0, nr, nc), oracle.submatrix(OA, i0, j0, nr, nc), "sub")
    if m == k:  # aliased closure step D += D.D
        E = A.duplicate()
        sp.MxM(E, E, E, accumulate=True, closure_step=True)
        assert_same(E, oracle.mxm(OA, OA, OA), "E += E.E")


@pytest.mark.parametrize("seed", range(6))
def test_random_kronecker(sp, seed):
    rng = np.random.default_rng(2000 + seed)
    ma, na, mb, nb = (int(rng.choice([1, 3, 17, 64, 200])) for _ in range(4))
    A, OA = both_from_pairs(sp, ma, na, *rand_pairs(rng, ma, na, "uniform"))
    B, OB = both_from_pairs(sp, mb, nb, *rand_pairs(rng, mb, nb, "skewed"))
    assert_same(sp.kronecker(A, B), oracle.kronecker(OA, OB), f"kron {ma}x{na} (x) {mb}x{nb}")


@pytest.mark.parametrize("seed", range(6))
def test_random_mxm_in_place_compaction(sp, seed):
    """The same random shapes with the engine's in-place compaction (the mode
    the library falls back to when memory is short) -- bit-exact."""
    rng = np.random.default_rng(3000 + seed)
    kind = ("uniform", "skewed", "dense")[seed % 3]
    dims = [1, 33, 257, 1000, 4096]
    m, k = (int(rng.choice(dims)) for _ in range(2))
    n = int(rng.choice(dims + [1 << 20]))
    A, OA = both_from_pairs(sp, m, k, *rand_pairs(rng, m, k, kind))
    B, OB = both_from_pairs(sp, k, n, *rand_pairs(rng, k, n, kind))
    sp.set_out_of_place_compaction(False)
    try:
        assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), f"A.B {m}x{k}x{n} {kind} in place")
        C, OC = both_from_pairs(sp, m, n, *rand_pairs(rng, m, n, "uniform"))
        sp.MxM(C, A, B, accumulate=True)
        assert_same(C, oracle.mxm(OA, OB, OC), "C += A.B in place")
    finally:
        sp.set_out_of_place_compaction(True)
