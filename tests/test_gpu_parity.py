"""CUDA path vs oracle, element by element (bit-exact CSR: identical rowptr and
colidx), on the same seeded inputs.  Sizes span several tiles / bins and a
ragged tail; edge cases: empty matrices and rows, single rows, rectangular
shapes, heavy rows (hash and bitmap bins, multi-window bitmap), aliasing."""
import numpy as np
import pytest

import oracle
import spgen
from golden_io import load
from helpers import assert_same, both_from_pairs, csr_is_valid, gpu_lib

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    return gpu_lib()


# ------------------------------------------------------------------ Build

@pytest.mark.parametrize("shape,nv,seed", [((1, 1), 1, 0), ((7, 5), 40, 1), ((1000, 3000), 20000, 2),
                                           ((50000, 70), 300000, 3), ((3, 100000), 60000, 4)])
def test_build_random(sp, shape, nv, seed):
    r, c = spgen.random_pairs(shape[0], shape[1], nv, seed)
    M, O = both_from_pairs(sp, shape[0], shape[1], r, c)
    assert_same(M, O, "build")


def test_build_heavy_rows(sp):
    # rows with 20k and 9k raw entries (bitmap / hash bins) plus light rows
    rng = np.random.default_rng(5)
    r = np.concatenate([np.zeros(20000), np.full(9000, 3), rng.integers(0, 64, 5000)]).astype(np.uint32)
    c = rng.integers(0, 1 << 21, len(r)).astype(np.uint32)
    M, O = both_from_pairs(sp, 64, 1 << 21, r, c)
    assert_same(M, O, "build heavy")


@pytest.mark.parametrize("nrows,per_row,ncols,dup_every", [(1 << 20, 4, 1 << 20, 16), (1 << 12, 3000, 1 << 22, 5),
                                                            (1 << 16, 40, 1 << 16, 1)])
def test_build_inplace_compaction(sp, nrows, per_row, ncols, dup_every):
    """Row-engine compaction regimes: a few duplicates per many rows leave a
    small capacity slack (in-place ordered compaction over ~500-1500 tiles of
    8192 entries; short rows take the unstaged row search, long rows the
    smem-staged one); dup_every=1 gives a large slack (out-of-place path)."""
    rng = np.random.default_rng(nrows + per_row)
    r = np.repeat(np.arange(nrows, dtype=np.uint32), per_row)
    c = rng.integers(0, ncols, len(r)).astype(np.uint32)
    c2 = c.reshape(nrows, per_row)
    dup_rows = np.arange(0, nrows, dup_every)
    c2[dup_rows, 1] = c2[dup_rows, 0]  # one forced duplicate in every dup_every-th row
    if dup_every == 1:
        c2[:, per_row // 2:] = c2[:, :per_row - per_row // 2]
    perm = rng.permutation(len(r))
    M, O = both_from_pairs(sp, nrows, ncols, r[perm], c[perm])
    assert_same(M, O, "build in-place compaction")


@pytest.mark.parametrize("oop", [False, True], ids=["in_place", "out_of_place"])
def test_compaction_modes(sp, oop):
    """spbla_SetOutOfPlaceCompaction: the engine's final move into CSR in place
    (tiles ordered by their overlaps) and into a new exact buffer give the
    same CSR (Build with a small slack over many tiles, A.A, C += A.A)."""
    sp.set_out_of_place_compaction(oop)
    try:
        rng = np.random.default_rng(9)
        nrows, per_row = 1 << 18, 6
        r = np.repeat(np.arange(nrows, dtype=np.uint32), per_row)
        c = rng.integers(0, 1 << 20, len(r)).astype(np.uint32)
        M, O = both_from_pairs(sp, nrows, 1 << 20, r[::-1].copy(), c)
        assert_same(M, O, "build")
        rr, cc = spgen.rmat_pairs(12, 16, 0.45, 0.22, 0.22, seed=11)
        A, OA = both_from_pairs(sp, 4096, 4096, rr, cc)
        assert_same(sp.mxm(A, A), oracle.mxm(OA, OA), "A.A")
        r2, c2 = spgen.uniform_pairs(4096, 4096, 3, seed=22)
        C, OC = both_from_pairs(sp, 4096, 4096, r2, c2)
        sp.MxM(C, A, A, accumulate=True)
        assert_same(C, oracle.mxm(OA, OA, OC), "C += A.A")
    finally:
        sp.set_out_of_place_compaction(True)


def test_build_empty_and_errors(sp):
    M = sp.Matrix.new(10, 10)
    M.build(np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    assert M.nvals == 0
    rp, _ = M.to_csr()
    assert np.all(rp == 0)
    with pytest.raises(sp.SpblaError, match="INDEX_OUT_OF_BOUNDS"):
        M.build(np.array([0, 10], np.uint32), np.array([0, 0], np.uint32))


def test_build_presorted_hint(sp):
    r, c = spgen.random_pairs(500, 500, 4000, 6)
    O = oracle.build(500, 500, r.numpy(), c.numpy())
    pr, pc = O.pairs()
    M = sp.Matrix.new(500, 500)
    M.build(pr, pc, sp.HINT_SORTED | sp.HINT_NO_DUPLICATES | sp.HINT_VALIDATE)
    assert_same(M, O, "presorted")


def test_extract_pairs_roundtrip(sp):
    r, c = spgen.rmat_pairs(12, 4, 0.45, 0.22, 0.22, seed=7)
    M, O = both_from_pairs(sp, 4096, 4096, r, c)
    hr, hc = M.extract_pairs()
    orr, occ = O.pairs()
    assert np.array_equal(hr, orr) and np.array_equal(hc, occ)
    dr, dc = M.extract_pairs(device=True)
    assert np.array_equal(dr.cpu().numpy().astype(np.uint32), orr)
    assert np.array_equal(dc.cpu().numpy().astype(np.uint32), occ)


def test_import_export_wrap(sp):
    import torch
    r, c = spgen.uniform_pairs(300, 400, 5, seed=8)
    M, O = both_from_pairs(sp, 300, 400, r, c)
    rp = torch.empty(301, dtype=torch.int64, device="cuda")
    ci = torch.empty(M.nvals, dtype=torch.int32, device="cuda")
    M.export_csr(rp, ci)
    W = sp.Matrix.wrap(300, 400, rp, ci, hints=sp.HINT_VALIDATE)
    I = sp.Matrix.from_csr(300, 400, O.rowptr, O.colidx, sp.HINT_VALIDATE)
    assert_same(W, O, "wrap")
    assert_same(I, O, "import")
    D = W.duplicate()
    assert_same(D, O, "dup")
    bad = O.colidx.copy()
    if len(bad) > 1:
        bad[1], bad[0] = bad[0], bad[1]
    with pytest.raises(sp.SpblaError):
        sp.Matrix.from_csr(300, 400, O.rowptr, bad[::-1].copy(), sp.HINT_VALIDATE)


# ------------------------------------------------------------------ MxM

def test_mxm_golden(sp):
    mats, _ = load("mxm_3x4x3.txt")
    A, _ = both_from_pairs(sp, *mats["A"])
    B, _ = both_from_pairs(sp, *mats["B"])
    C = sp.mxm(A, B)
    assert_same(C, oracle.build(*mats["C"]), "golden C")
    Cin, _ = both_from_pairs(sp, *mats["Cin"])
    sp.MxM(Cin, A, B, accumulate=True)
    assert_same(Cin, oracle.build(*mats["Cacc"]), "golden Cacc")


def test_mxm_config1(sp):
    """BASELINE configs[0] at full size: 4096 x 4096 uniform, 8 draws/row."""
    r, c = spgen.uniform_pairs(4096, 4096, 8, seed=1)
    A, OA = both_from_pairs(sp, 4096, 4096, r, c)
    assert_same(sp.mxm(A, A), oracle.mxm(OA, OA), "config1 A.A")


@pytest.mark.parametrize("scale,ef,params,seed", [(12, 16, (0.45, 0.22, 0.22), 11), (13, 8, (0.57, 0.19, 0.19), 12),
                                                  (11, 32, (0.40, 0.20, 0.20), 13)])
def test_mxm_rmat(sp, scale, ef, params, seed):
    n = 1 << scale
    r, c = spgen.rmat_pairs(scale, ef, *params, seed=seed)
    A, OA = both_from_pairs(sp, n, n, r, c)
    assert_same(sp.mxm(A, A), oracle.mxm(OA, OA), "rmat A.A")


def test_mxm_rectangular_and_empty(sp):
    for (m, k, n, nv1, nv2, seed) in [(1, 1, 1, 1, 1, 0), (37, 1000, 3, 200, 900, 1), (2000, 17, 5000, 9000, 40, 2),
                                      (100, 100, 100, 0, 500, 3), (100, 100, 100, 500, 0, 4), (0, 5, 5, 0, 3, 5)]:
        r1, c1 = spgen.random_pairs(max(m, 1), k, nv1, seed)
        r2, c2 = spgen.random_pairs(k, n, nv2, seed + 100)
        if m == 0:
            r1, c1 = r1[:0], c1[:0]
        A, OA = both_from_pairs(sp, m, k, r1, c1)
        B, OB = both_from_pairs(sp, k, n, r2, c2)
        assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), f"rect {m}x{k}x{n}")


def test_mxm_accumulate_and_alias(sp):
    r, c = spgen.rmat_pairs(12, 8, 0.45, 0.22, 0.22, seed=21)
    A, OA = both_from_pairs(sp, 4096, 4096, r, c)
    r2, c2 = spgen.uniform_pairs(4096, 4096, 3, seed=22)
    C, OC = both_from_pairs(sp, 4096, 4096, r2, c2)
    sp.MxM(C, A, A, accumulate=True)
    assert_same(C, oracle.mxm(OA, OA, OC), "C += A.A")
    D = A.duplicate()
    sp.MxM(D, D, D, accumulate=True)  # D += D.D, all aliased
    assert_same(D, oracle.mxm(OA, OA, OA), "D += D.D")


def test_mxm_heavy_rows_multiwindow(sp):
    """Rows with ub > 8192 over 3*2^20 columns: bitmap bin with 3 windows;
    rows with 513..8192 products: hash bin."""
    ncols = 3 << 20
    rng = np.random.default_rng(31)
    k = 600
    rb = np.repeat(np.arange(k), 400).astype(np.uint32)           # B: 600 rows x ~400 entries
    cb = rng.integers(0, ncols, len(rb)).astype(np.uint32)
    ra = np.concatenate([np.zeros(60), np.ones(5), np.full(2, 2), rng.integers(3, 200, 3000)]).astype(np.uint32)
    ca = rng.integers(0, k, len(ra)).astype(np.uint32)
    A, OA = both_from_pairs(sp, 200, k, ra, ca)
    B, OB = both_from_pairs(sp, k, ncols, rb, cb)
    assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), "heavy")


@pytest.mark.parametrize("ncols,label", [(1 << 18, "narrow span: small bitmap fallback"),
                                         (1 << 22, "wide span: large bitmap fallback")])
def test_mxm_duplicate_heavy_fallback(sp, ncols, label):
    """Hash-bin rows whose products are ~50 copies of ~50 columns (closure-like):
    buckets overflow with duplicates, the rows fall back to a bitmap kernel
    chosen by span (2^18 columns: the 256-thread small-window kernel; 2^22: the
    1.5 Mi-window one).  Mixed with ordinary rows in the same launch."""
    rng = np.random.default_rng(77)
    hub_cols = np.sort(rng.choice(ncols, 50, replace=False)).astype(np.uint32)
    nb_hub = 64
    # B: 64 hub rows sharing the same 50 columns, 400 ordinary rows of 8 random columns
    rb = np.concatenate([np.repeat(np.arange(nb_hub), 50), np.repeat(np.arange(nb_hub, nb_hub + 400), 8)])
    cb = np.concatenate([np.tile(hub_cols, nb_hub), rng.integers(0, ncols, 400 * 8)])
    # A: rows 0..299 take 30..60 hub rows (1500..3000 products, 50 distinct);
    # rows 300..599 take 100 ordinary rows (800 products, mostly distinct)
    ra, ca = [], []
    for i in range(300):
        k = rng.choice(nb_hub, rng.integers(30, 61), replace=False)
        ra += [i] * len(k); ca += list(k)
    for i in range(300, 600):
        k = rng.choice(np.arange(nb_hub, nb_hub + 400), 100, replace=False)
        ra += [i] * len(k); ca += list(k)
    A, OA = both_from_pairs(sp, 600, nb_hub + 400, np.array(ra, np.uint32), np.array(ca, np.uint32))
    B, OB = both_from_pairs(sp, nb_hub + 400, ncols, rb.astype(np.uint32), cb.astype(np.uint32))
    assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), label)


# ------------------------------------------------------------------ EWiseAdd

@pytest.mark.parametrize("seed", range(3))
def test_ewise_add(sp, seed):
    n = 1 << 13
    r1, c1 = spgen.rmat_pairs(13, 8, 0.45, 0.22, 0.22, seed=40 + seed)
    r2, c2 = spgen.uniform_pairs(n, n, 4 + seed, seed=50 + seed)
    A, OA = both_from_pairs(sp, n, n, r1, c1)
    B, OB = both_from_pairs(sp, n, n, r2, c2)
    assert_same(sp.ewise_add(A, B), oracle.ewise_add(OA, OB), "A+B")
    assert_same(sp.ewise_add(B, A), oracle.ewise_add(OA, OB), "B+A")
    assert_same(sp.ewise_add(A, A), OA, "A+A")


def test_ewise_add_edge_cases(sp):
    mats, _ = load("misc_ops.txt")
    A, OA = both_from_pairs(sp, *mats["A"])
    A2, OA2 = both_from_pairs(sp, *mats["A2"])
    assert_same(sp.ewise_add(A, A2), oracle.build(*mats["E"]), "golden E")
    Z = sp.Matrix.new(3, 4)
    assert_same(sp.ewise_add(A, Z), OA, "A+0")
    assert_same(sp.ewise_add(Z, Z), oracle.build(3, 4, [], []), "0+0")
    # many empty rows, one long row, ragged tail across merge-path tiles
    rng = np.random.default_rng(3)
    r1 = np.concatenate([np.full(5000, 7), rng.integers(0, 100000, 3000)]).astype(np.uint32)
    c1 = rng.integers(0, 9000, len(r1)).astype(np.uint32)
    r2 = np.concatenate([np.full(4000, 7), np.full(10, 99999)]).astype(np.uint32)
    c2 = rng.integers(0, 9000, len(r2)).astype(np.uint32)
    X, OX = both_from_pairs(sp, 100000, 9000, r1, c1)
    Y, OY = both_from_pairs(sp, 100000, 9000, r2, c2)
    assert_same(sp.ewise_add(X, Y), oracle.ewise_add(OX, OY), "ragged")
    sp.Matrix_EWiseAdd(X, X, Y)  # M += N
    assert_same(X, oracle.ewise_add(OX, OY), "M += N")


@pytest.mark.parametrize("kind", ["one_per_row", "long_row_dups", "empty_gaps", "rows_512", "rows_1024"])
def test_ewise_add_tile_structure(sp, kind):
    """Merge-path tiles (4096 merged items) whose rows are: more than the
    1024 staged per tile (one item per row), one row spanning many tiles with
    duplicates at every tile boundary, thousands of empty rows between rows,
    and about 512 or 1024 rows per tile (around the staging limit)."""
    rng = np.random.default_rng(11)
    if kind == "one_per_row":
        n, ncols = 30000, 64
        ra = np.arange(n); ca = rng.integers(0, 4, n)
        rb = np.arange(0, n, 2); cb = rng.integers(0, 4, len(rb))
    elif kind == "long_row_dups":
        n, ncols = 16, 120000
        ra = np.concatenate([np.full(60000, 3), [0, 15]]); ca = np.concatenate([np.arange(0, 120000, 2), [5, 6]])
        rb = np.concatenate([np.full(40000, 3), [0, 1]]); cb = np.concatenate([np.arange(0, 120000, 3), [5, 7]])
    elif kind == "empty_gaps":
        n, ncols = 400000, 5000
        rows = rng.choice(n, 300, replace=False)
        ra = np.repeat(rows, 40); ca = rng.integers(0, ncols, len(ra))
        rb = np.repeat(rows[::2], 25); cb = rng.integers(0, ncols, len(rb))
    else:  # 4096 / (na + nb) rows per tile
        na, nb = (6, 2) if kind == "rows_512" else (3, 1)
        n, ncols = 12000, 20
        ra = np.repeat(np.arange(n), na); ca = rng.integers(0, ncols, len(ra))
        rb = np.repeat(np.arange(n), nb); cb = rng.integers(0, ncols, len(rb))
    A, OA = both_from_pairs(sp, n, ncols, ra.astype(np.uint32), ca.astype(np.uint32))
    B, OB = both_from_pairs(sp, n, ncols, rb.astype(np.uint32), cb.astype(np.uint32))
    want = oracle.ewise_add(OA, OB)
    assert_same(sp.ewise_add(A, B), want, kind + " A+B")
    assert_same(sp.ewise_add(B, A), want, kind + " B+A")
    assert_same(sp.ewise_add(A, A), OA, kind + " A+A")


# ------------------------------------------------------------------ Kronecker

def test_kronecker(sp):
    mats, _ = load("kron_2x2_2x3.txt")
    A, _ = both_from_pairs(sp, *mats["A"])
    B, _ = both_from_pairs(sp, *mats["B"])
    assert_same(sp.kronecker(A, B), oracle.build(*mats["K"]), "golden K")
    # configs[2] shape, reduced graph: 2^8-row graph (x) 64-state RSM
    rg, cg = spgen.rmat_pairs(8, 8, 0.45, 0.22, 0.22, seed=60)
    G, OG = both_from_pairs(sp, 256, 256, rg, cg)
    rr, cr = spgen.rsm_pairs(64, 1, 2, seed=61)
    R, OR = both_from_pairs(sp, 64, 64, rr, cr)
    assert_same(sp.kronecker(G, R), oracle.kronecker(OG, OR), "G(x)R")
    assert_same(sp.kronecker(R, G), oracle.kronecker(OR, OG), "R(x)G")
    Z = sp.Matrix.new(3, 5)
    K = sp.kronecker(G, Z)
    assert K.nvals == 0 and K.shape == (256 * 3, 256 * 5)


@pytest.mark.parametrize("mb,nb,nvb", [(64, 64, 20), (2048, 100, 8192), (2049, 50, 3000), (4096, 4096, 16384)])
def test_kronecker_b_sizes(sp, mb, nb, nvb):
    """Both Kronecker kernels: B staged in shared memory (<= 2048 rows and
    <= 8192 entries; B with empty rows, B at both limits) and the general
    kernel (B over either limit); A with empty rows."""
    ra, ca = spgen.random_pairs(40, 30, 90, seed=mb)
    A, OA = both_from_pairs(sp, 40, 30, ra, ca)
    rb, cb = spgen.random_pairs(mb, nb, nvb, seed=nb)
    B, OB = both_from_pairs(sp, mb, nb, rb, cb)
    assert_same(sp.kronecker(A, B), oracle.kronecker(OA, OB), f"A(x)B {mb}x{nb}")
    assert_same(sp.kronecker(B, A), oracle.kronecker(OB, OA), f"B(x)A {mb}x{nb}")


# ------------------------------------------------------------------ transpose / reduce / submatrix

def test_misc_golden(sp):
    mats, _ = load("misc_ops.txt")
    A, _ = both_from_pairs(sp, *mats["A"])
    assert_same(sp.transpose(A), oracle.build(*mats["T"]), "T")
    assert_same(sp.reduce_to_column(A), oracle.build(*mats["V"]), "V")
    assert_same(sp.submatrix(A, 1, 1, 2, 3), oracle.build(*mats["S"]), "S")


def test_transpose_reduce_submatrix(sp):
    r, c = spgen.rmat_pairs(13, 8, 0.57, 0.19, 0.19, seed=70)
    A, OA = both_from_pairs(sp, 8192, 8192, r, c)
    assert_same(sp.transpose(A), oracle.transpose(OA), "transpose")
    assert_same(sp.reduce_to_column(A), oracle.reduce_to_column(OA), "reduce")
    for (i0, j0, nr, nc) in [(0, 0, 8192, 8192), (100, 2000, 3000, 50), (8191, 8191, 1, 1), (5, 5, 0, 9)]:
        assert_same(sp.submatrix(A, i0, j0, nr, nc), oracle.submatrix(OA, i0, j0, nr, nc), f"sub {i0},{j0}")
    r2, c2 = spgen.random_pairs(300, 70000, 5000, seed=71)
    B, OB = both_from_pairs(sp, 300, 70000, r2, c2)
    assert_same(sp.transpose(B), oracle.transpose(OB), "transpose rect")
    with pytest.raises(sp.SpblaError, match="INDEX_OUT_OF_BOUNDS"):
        sp.submatrix(A, 8000, 0, 500, 10)


# ------------------------------------------------------------------ closure

@pytest.mark.parametrize("name", ["closure_chain4.txt", "closure_cycle3.txt"])
def test_closure_golden(sp, name):
    mats, sc = load(name)
    A, _ = both_from_pairs(sp, *mats["A"])
    C, it = sp.closure(A)
    assert_same(C, oracle.build(*mats["C"]), name)
    assert it == sc["iterations"]


def test_closure_labeled_dag(sp):
    """configs[3] shape at 2^12 vertices: union of the two labels, closure."""
    n = 1 << 12
    (r0, c0), (r1, c1) = spgen.labeled_dag(n, 0.25, seed=80)
    L0, O0 = both_from_pairs(sp, n, n, r0, c0)
    L1, O1 = both_from_pairs(sp, n, n, r1, c1)
    U = sp.ewise_add(L0, L1)
    OU = oracle.ewise_add(O0, O1)
    assert_same(U, OU, "union")
    C, it = sp.closure(U)
    OC, oit = oracle.closure(OU)
    assert_same(C, OC, "closure")
    assert it == oit


def test_mxm_closure_step_hint_dup_rows(sp):
    """SPBLA_HINT_CLOSURE_STEP routes rows with products > 4x their length
    (duplicate-heavy) to the bitmap kernel: C += C.C on a partly closed DAG
    (hash-bin-sized dup-heavy rows), bit-exact vs the oracle, with and
    without the hint."""
    n = 1 << 14
    (r0, c0), (r1, c1) = spgen.labeled_dag(n, 0.6, seed=83)
    r = np.concatenate([r0.numpy(), r1.numpy()])
    c = np.concatenate([c0.numpy(), c1.numpy()])
    C, OC = both_from_pairs(sp, n, n, r, c)
    for step in range(5):
        want = oracle.mxm(OC, OC, OC)
        D = C.duplicate()
        sp.MxM(C, C, C, accumulate=True, closure_step=True)
        sp.MxM(D, D, D, accumulate=True)
        assert_same(C, want, f"C += C.C with the hint, step {step}")
        assert_same(D, want, f"C += C.C without the hint, step {step}")
        OC = want


def test_closure_rmat_small(sp):
    r, c = spgen.rmat_pairs(9, 2, 0.45, 0.22, 0.22, seed=81)
    A, OA = both_from_pairs(sp, 512, 512, r, c)
    C, it = sp.closure(A)
    OC, oit = oracle.closure(OA)
    assert_same(C, OC, "closure rmat")
    assert it == oit


# ------------------------------------------------------------------ generators on device

def test_generator_cpu_gpu_identical():
    import torch
    r1, c1 = spgen.rmat_pairs(14, 4, 0.45, 0.22, 0.22, seed=3)
    r2, c2 = spgen.rmat_pairs(14, 4, 0.45, 0.22, 0.22, seed=3, device="cuda")
    assert torch.equal(r1, r2.cpu()) and torch.equal(c1, c2.cpu())
    (a, b), (x, y) = spgen.labeled_dag(5000, 0.25, seed=4)
    (a2, b2), (x2, y2) = spgen.labeled_dag(5000, 0.25, seed=4, device="cuda")
    assert torch.equal(b, b2.cpu()) and torch.equal(y, y2.cpu())


def test_mxm_heavy_rows_wide_span_partition(sp):
    """Heavy rows (> 40960 products, the dense bin) over ncols = 2^26: 43
    bitmap windows, handled by the partition-by-window mode (two gathers and
    one slice pass per row instead of one gather per window); also a
    small-span heavy row and a wide heavy row with duplicate columns."""
    ncols = 1 << 26
    rng = np.random.default_rng(37)
    k = 300
    rb = np.repeat(np.arange(k), 500).astype(np.uint32)                     # B: 300 rows x ~500 entries
    cb = rng.integers(0, ncols, len(rb)).astype(np.uint32)
    cb[: 500 * 10] = rng.integers(0, 5000, 500 * 10).astype(np.uint32)      # rows 0..9: narrow columns
    ra = np.concatenate([np.repeat(np.arange(4), 150),                       # 4 heavy wide rows (~75K products)
                         np.full(10, 4),                                     # narrow-span heavy-ish row
                         rng.integers(5, 40, 400)]).astype(np.uint32)
    ca = np.concatenate([rng.integers(10, k, 600), np.arange(10),
                         rng.integers(0, k, 400)]).astype(np.uint32)
    # B rows 100..109 are copies of row 100 and row 0 uses all of them:
    # duplicate columns across its segments
    cb.reshape(k, 500)[101:110] = cb.reshape(k, 500)[100]
    ca[:10] = np.arange(100, 110)
    A, OA = both_from_pairs(sp, 40, k, ra, ca)
    B, OB = both_from_pairs(sp, k, ncols, rb, cb)
    assert_same(sp.mxm(A, B), oracle.mxm(OA, OB), "heavy rows over 2^26 columns")


@pytest.mark.parametrize("n,p,extra,seed", [(1 << 11, 0.25, 300, 90), (1 << 13, 0.1, 2000, 91), (700, 0.5, 0, 92)])
def test_incremental_closure(sp, n, p, extra, seed):
    """spbla_TransitiveClosureIncremental: C = closure(G), then new edges D
    (some inside C already); C becomes closure(G + D) -- the oracle's closure
    of the union -- and D inside C leaves C unchanged with 0 steps."""
    (r0, c0), (r1, c1) = spgen.labeled_dag(n, p, seed=seed)
    rg = np.concatenate([r0.numpy(), r1.numpy()])
    cg = np.concatenate([c0.numpy(), c1.numpy()])
    G, OG = both_from_pairs(sp, n, n, rg, cg)
    C, _ = sp.closure(G)
    OC, _ = oracle.closure(OG)
    assert_same(C, OC, "closure(G)")
    rng = np.random.default_rng(seed)
    rd = rng.integers(1, n, extra).astype(np.uint32)
    cd = (rng.integers(0, 1 << 30, extra) % np.maximum(rd, 1)).astype(np.uint32)  # DAG edges v -> u < v
    rd = np.concatenate([rd, rg[:50]]).astype(np.uint32)  # plus edges C already has
    cd = np.concatenate([cd, cg[:50]]).astype(np.uint32)
    D, OD = both_from_pairs(sp, n, n, rd, cd)
    it = sp.TransitiveClosureIncremental(C, D)
    want, _ = oracle.closure(oracle.ewise_add(OG, OD))
    assert_same(C, want, "closure(G + D) incrementally")
    assert (it == 0) == (extra == 0)
    # D inside C: nothing changes
    E, _ = both_from_pairs(sp, n, n, rg[:100], cg[:100])
    assert sp.TransitiveClosureIncremental(C, E) == 0
    assert_same(C, want, "unchanged by edges already present")
