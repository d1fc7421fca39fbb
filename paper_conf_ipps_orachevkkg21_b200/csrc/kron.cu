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

__global__ void kron_rowptr_kernel(CsrView A, CsrView B, uint64_t nnzB, off_t64* __restrict__ rp) {
    const uint64_t n = uint64_t(A.nrows) * B.nrows;
    for (uint64_t r = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; r <= n;
         r += uint64_t(gridDim.x) * blockDim.x) {
        if (r == n) {
            rp[r] = A.rowptr[A.nrows] * nnzB;
            continue;
        }
        const idx_t ia = idx_t(r / B.nrows), ib = idx_t(r - uint64_t(ia) * B.nrows);
        const uint64_t la = A.rowptr[ia + 1] - A.rowptr[ia];
        rp[r] = A.rowptr[ia] * nnzB + la * B.rowptr[ib];
    }
}

// One warp per K row; the row's la*lb items are spread over the 32 lanes.
__global__ void kron_cols_kernel(CsrView A, CsrView B, const off_t64* __restrict__ rp,
                                 idx_t* __restrict__ out) {
    const uint64_t n = uint64_t(A.nrows) * B.nrows;
    const unsigned lane = lane_id();
    const uint64_t nw = uint64_t(gridDim.x) * (blockDim.x >> 5);
    for (uint64_t r = (blockIdx.x * uint64_t(blockDim.x) + threadIdx.x) >> 5; r < n; r += nw) {
        const idx_t ia = idx_t(r / B.nrows), ib = idx_t(r - uint64_t(ia) * B.nrows);
        const off_t64 sa = A.rowptr[ia], sb = B.rowptr[ib];
        const uint32_t lb = uint32_t(B.rowptr[ib + 1] - sb);
        const uint64_t cnt = uint64_t(A.rowptr[ia + 1] - sa) * lb;
        idx_t* o = out + rp[r];
        for (uint64_t e = lane; e < cnt; e += 32) {
            const uint64_t a = e / lb, b = e - a * lb;
            o[e] = A.colidx[sa + a] * B.ncols + B.colidx[sb + b];
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
    unsigned g1 = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(m + 1, 256), uint64_t(nsm) * 16));
    const int t = ktime_begin("kron", ctx().stream);
    kron_rowptr_kernel<<<g1, 256, 0, ctx().stream>>>(view(A), view(B), B->nnz, rp.p);
    count_launch();
    check_launch("kron_rowptr_kernel");
    if (nnz) {
        unsigned g2 = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(ceil_div(m * 32, 256), uint64_t(nsm) * 32));
        kron_cols_kernel<<<g2, 256, 0, ctx().stream>>>(view(A), view(B), rp.p, ci.p);
        count_launch();
        check_launch("kron_cols_kernel");
    }
    ktime_end(t);
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(K, rp.detach(), rc, ci.detach(), cc, nnz);
}

}  // namespace spbla
