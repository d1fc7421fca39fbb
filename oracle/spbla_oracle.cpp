// SPbLA CPU ORACLE — test infrastructure only.
//
// Plain, slow, obviously-correct C++ definitions of every operation on the
// hot path, used ONLY by tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference leg.  It shares no code with the CUDA path
// (paper_conf_ipps_orachevkkg21_b200/csrc) and neither side includes the other.
//
// Semiring (§II "Libraries Design", l.210-211): values {1,0},
// '+' = logical or, 'x' = logical and, 0 the identity of '+'.
// Storage (§III-A "cuBool", l.253-257): value-free CSR, a row-offset
// array and a column-index array; a stored (i,j) pair means M[i][j] = 1.
// Operations (§II bullet list, l.228-239).
//
// Every result row is a std::set<uint32_t>, so output rows are sorted and
// duplicate-free by construction (reading R2).
//
// Parity pins (tests/test_oracle.py): dense brute force n<=64, identity/zero
// laws, nnz(A(x)B)=nnz(A)nnz(B), associativity, closure == BFS reachability,
// scipy.sparse products, hand-worked golden fixtures under tests/golden/.

#include <cstdint>
#include <cstring>
#include <set>
#include <vector>
#include <algorithm>
#include <iterator>

extern "C" {

struct OCsr {
    uint32_t nrows, ncols;
    std::vector<uint64_t> rowptr;
    std::vector<uint32_t> colidx;
};

typedef std::vector<std::set<uint32_t>> Rows;

static OCsr* to_csr(uint32_t nrows, uint32_t ncols, const Rows& rows) {
    OCsr* r = new OCsr;
    r->nrows = nrows;
    r->ncols = ncols;
    r->rowptr.assign((size_t)nrows + 1, 0);
    for (uint32_t i = 0; i < nrows; ++i) r->rowptr[i + 1] = r->rowptr[i] + rows[i].size();
    r->colidx.reserve(r->rowptr[nrows]);
    for (uint32_t i = 0; i < nrows; ++i)
        for (uint32_t j : rows[i]) r->colidx.push_back(j);
    return r;
}

void ocsr_free(OCsr* m) { delete m; }
uint64_t ocsr_nvals(const OCsr* m) { return m->colidx.size(); }
uint32_t ocsr_nrows(const OCsr* m) { return m->nrows; }
uint32_t ocsr_ncols(const OCsr* m) { return m->ncols; }
void ocsr_copy(const OCsr* m, uint64_t* rowptr, uint32_t* colidx) {
    std::memcpy(rowptr, m->rowptr.data(), m->rowptr.size() * sizeof(uint64_t));
    if (!m->colidx.empty()) std::memcpy(colidx, m->colidx.data(), m->colidx.size() * sizeof(uint32_t));
}

// Fill matrix with values {(i,j)_k}_k: M[i][j] = 1 for each
// listed pair, duplicates collapse (or-semiring).  status=1 on an index out
// of range.
OCsr* oracle_build(uint32_t nrows, uint32_t ncols, const uint32_t* r, const uint32_t* c,
                   uint64_t n, int* status) {
    *status = 0;
    Rows rows(nrows);
    for (uint64_t k = 0; k < n; ++k) {
        if (r[k] >= nrows || c[k] >= ncols) { *status = 1; return nullptr; }
        rows[r[k]].insert(c[k]);
    }
    return to_csr(nrows, ncols, rows);
}

// Matrix-matrix multiplication C += M x N, row-wise
// Gustavson: C[i] = (accumulate ? C[i] : {}) U  U_{k in A[i]} B[k].
// (A[i] x B)[j] = OR_k A[i][k] AND B[k][j]; the set union is exactly that OR.
OCsr* oracle_mxm(uint32_t m, uint32_t k, uint32_t n,
                 const uint64_t* arp, const uint32_t* aci,
                 const uint64_t* brp, const uint32_t* bci,
                 const uint64_t* crp, const uint32_t* cci) {
    (void)k;
    Rows rows(m);
    for (uint32_t i = 0; i < m; ++i) {
        std::set<uint32_t>& s = rows[i];
        if (crp)
            for (uint64_t q = crp[i]; q < crp[i + 1]; ++q) s.insert(cci[q]);
        for (uint64_t p = arp[i]; p < arp[i + 1]; ++p) {
            uint32_t kk = aci[p];
            for (uint64_t q = brp[kk]; q < brp[kk + 1]; ++q) s.insert(bci[q]);
        }
    }
    return to_csr(m, n, rows);
}

// Same definition evaluated only on the listed rows of A (sampled parity at
// full sizes).  Result has nsample rows, row t = (A x B)[rows[t]].
OCsr* oracle_mxm_rows(uint32_t n,
                      const uint64_t* arp, const uint32_t* aci,
                      const uint64_t* brp, const uint32_t* bci,
                      const uint64_t* crp, const uint32_t* cci,
                      const uint32_t* sample, uint32_t nsample) {
    Rows rows(nsample);
    for (uint32_t t = 0; t < nsample; ++t) {
        uint32_t i = sample[t];
        std::set<uint32_t>& s = rows[t];
        if (crp)
            for (uint64_t q = crp[i]; q < crp[i + 1]; ++q) s.insert(cci[q]);
        for (uint64_t p = arp[i]; p < arp[i + 1]; ++p) {
            uint32_t kk = aci[p];
            for (uint64_t q = brp[kk]; q < brp[kk + 1]; ++q) s.insert(bci[q]);
        }
    }
    return to_csr(nsample, n, rows);
}

// Element-wise addition M += N: per row the sorted merge
// (std::set_union) of two sorted duplicate-free rows.
OCsr* oracle_ewise_add(uint32_t m, uint32_t n,
                       const uint64_t* arp, const uint32_t* aci,
                       const uint64_t* brp, const uint32_t* bci) {
    Rows rows(m);
    for (uint32_t i = 0; i < m; ++i) {
        std::vector<uint32_t> u;
        std::set_union(aci + arp[i], aci + arp[i + 1], bci + brp[i], bci + brp[i + 1],
                       std::back_inserter(u));
        rows[i].insert(u.begin(), u.end());
    }
    return to_csr(m, n, rows);
}

// Kronecker product K = M (x) N, the textbook definition:
// K[ia*mB + ib][ja*nB + jb] = A[ia][ja] AND B[ib][jb].
OCsr* oracle_kronecker(uint32_t ma, uint32_t na, const uint64_t* arp, const uint32_t* aci,
                       uint32_t mb, uint32_t nb, const uint64_t* brp, const uint32_t* bci) {
    uint64_t m = (uint64_t)ma * mb, n = (uint64_t)na * nb;
    Rows rows(m);
    for (uint32_t ia = 0; ia < ma; ++ia)
        for (uint32_t ib = 0; ib < mb; ++ib)
            for (uint64_t p = arp[ia]; p < arp[ia + 1]; ++p)
                for (uint64_t q = brp[ib]; q < brp[ib + 1]; ++q)
                    rows[(uint64_t)ia * mb + ib].insert((uint32_t)((uint64_t)aci[p] * nb + bci[q]));
    return to_csr((uint32_t)m, (uint32_t)n, rows);
}

// Transpose M = N^T: T[j][i] = M[i][j].
OCsr* oracle_transpose(uint32_t m, uint32_t n, const uint64_t* rp, const uint32_t* ci) {
    Rows rows(n);
    for (uint32_t i = 0; i < m; ++i)
        for (uint64_t p = rp[i]; p < rp[i + 1]; ++p) rows[ci[p]].insert(i);
    return to_csr(n, m, rows);
}

// Matrix to vector reduce V = reduceToColumn(M):
// V[i] = OR_j M[i][j], stored as an m x 1 matrix.
OCsr* oracle_reduce(uint32_t m, uint32_t n, const uint64_t* rp, const uint32_t* ci) {
    (void)n; (void)ci;
    Rows rows(m);
    for (uint32_t i = 0; i < m; ++i)
        if (rp[i + 1] > rp[i]) rows[i].insert(0);
    return to_csr(m, 1, rows);
}

// Sub-matrix extraction M = N[i..i+nr, j..j+nc].
OCsr* oracle_submatrix(uint32_t m, uint32_t n, const uint64_t* rp, const uint32_t* ci,
                       uint32_t i0, uint32_t j0, uint32_t nr, uint32_t nc) {
    (void)m; (void)n;
    Rows rows(nr);
    for (uint32_t i = 0; i < nr; ++i)
        for (uint64_t p = rp[i0 + i]; p < rp[i0 + i + 1]; ++p)
            if (ci[p] >= j0 && ci[p] - j0 < nc) rows[i].insert(ci[p] - j0);
    return to_csr(nr, nc, rows);
}

// Transitive closure by the loop C += C x C until nnz(C) stops changing
// (§I: RPQ/CFPQ index creation reduces to incremental transitive
// closure; BASELINE north_star "closure loop C += C.C").  *iters = number of
// C += C x C evaluations, including the last one that confirms the fixed point.
OCsr* oracle_closure(uint32_t n, const uint64_t* rp, const uint32_t* ci, int* iters) {
    Rows c(n);
    for (uint32_t i = 0; i < n; ++i)
        for (uint64_t p = rp[i]; p < rp[i + 1]; ++p) c[i].insert(ci[p]);
    uint64_t nnz = 0;
    for (auto& s : c) nnz += s.size();
    *iters = 0;
    for (;;) {
        Rows next(c);
        for (uint32_t i = 0; i < n; ++i)
            for (uint32_t k : c[i])
                for (uint32_t j : c[k]) next[i].insert(j);
        ++*iters;
        uint64_t nnz2 = 0;
        for (auto& s : next) nnz2 += s.size();
        c.swap(next);
        if (nnz2 == nnz) break;
        nnz = nnz2;
    }
    return to_csr(n, n, c);
}

}  // extern "C"
