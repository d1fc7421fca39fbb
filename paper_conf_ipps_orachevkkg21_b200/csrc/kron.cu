// Kronecker product K = A (x) B: pure index arithmetic.
//   rowptrK[ia*mB + ib] = rpA[ia] * nnz(B) + |A[ia]| * rpB[ib]   (closed form,
//                          no scan: rows before (ia,ib) are all of A's rows
//                          < ia times nnz(B), plus |A[ia]| * B's rows < ib)
//   K row (ia,ib), item e:  ja = A[ia][e / |B[ib]|], jb = B[ib][e % |B[ib]|],
//                          col = ja * nB + jb — ascending in e, so rows come
//                          out sorted and duplicate-free with no sort.
// HBM-write bound: 4 nnz(K) + 8 (mA mB + 1) bytes written, reads are tiny.
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

// Eight lanes per K row (four rows per warp in flight: rows average tens of
// items, so a warp per row would idle most lanes behind its dependent
// row-offset loads).  The row offset comes from the closed form (lane 0 of
// the group also stores it, so one launch writes both arrays); lane l walks
// items e = l, l+8, ... keeping (e / lb, e % lb) incrementally.
constexpr unsigned kKG = 8;
__global__ void kron_kernel(CsrView A, CsrView B, uint64_t nnzB, off_t64* __restrict__ rp, idx_t* __restrict__ out) {
    const uint64_t n = uint64_t(A.nrows) * B.nrows;
    const unsigned gl = threadIdx.x & (kKG - 1);
    const uint64_t ng = uint64_t(gridDim.x) * (blockDim.x / kKG);
    const uint64_t r0 = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) / kKG;
    if (r0 == 0 && gl == 0) rp[n] = A.rowptr[A.nrows] * nnzB;
    for (uint64_t r = r0; r < n; r += ng) {
        const idx_t ia = idx_t(r / B.nrows), ib = idx_t(r - uint64_t(ia) * B.nrows);
        const off_t64 sa = A.rowptr[ia], sb = B.rowptr[ib];
        const uint32_t la = uint32_t(A.rowptr[ia + 1] - sa), lb = uint32_t(B.rowptr[ib + 1] - sb);
        const uint64_t base = sa * nnzB + uint64_t(la) * sb;
        if (gl == 0) rp[r] = base;
        const uint64_t cnt = uint64_t(la) * lb;
        if (cnt == 0) continue;
        idx_t* o = out + base;
        const uint32_t da = kKG / lb, db = kKG % lb;
        uint32_t ai = gl / lb, bi = gl % lb;
        for (uint64_t e = gl; e < cnt; e += kKG) {
            o[e] = A.colidx[sa + ai] * B.ncols + B.colidx[sb + bi];
            ai += da;
            bi += db;
            if (bi >= lb) {
                bi -= lb;
                ++ai;
            }
        }
    }
}

}  // namespace

void kronecker(Matrix* K, const Matrix* A, const Matrix* B) {
    const uint64_t m = uint64_t(A->nrows) * B->nrows, n = uint64_t(A->ncols) * B->ncols;
    if (m > 0xFFFFFFFEull || n > 0xFFFFFFFEull)
        SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "Kronecker: product shape exceeds 32-bit indices");
    if (K->nrows != m || K->ncols != n) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "Kronecker: K has the wrong shape");
    if (!K->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Kronecker: output is a non-owning view");
    const uint64_t nnz = A->nnz * B->nnz;
    DevBuf<off_t64> rp(m + 1, kMat);
    DevBuf<idx_t> ci(nnz, kMat);
    const int nsm = ctx().num_sms;
    const int t = ktime_begin("kron", ctx().stream);
    const unsigned g = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(m * kKG, 256), uint64_t(nsm) * 8));
    kron_kernel<<<g, 256, 0, ctx().stream>>>(view(A), view(B), B->nnz, rp.p, ci.p);
    ktime_end(t);
    count_launch();
    check_launch("kron_kernel");
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(K, rp.detach(), rc, ci.detach(), cc, nnz);
}

}  // namespace spbla
