// Transpose, sub-matrix extraction (l.234) and
// matrix-to-vector reduce (l.235).
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

unsigned grid_for(uint64_t work, int threads, int per_sm = 16) {
    uint64_t g = ceil_div(work, threads);
    uint64_t cap = uint64_t(ctx().num_sms) * per_sm;
    return (unsigned)std::max<uint64_t>(1, std::min(g, cap));
}

__global__ void col_hist_kernel(const idx_t* __restrict__ ci, uint64_t nnz, unsigned long long* __restrict__ cnt) {
    for (uint64_t p = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; p < nnz; p += uint64_t(gridDim.x) * blockDim.x)
        atomicAdd(&cnt[ci[p]], 1ull);
}

// warp per source row: entry (i, j) goes to bucket j
__global__ void transpose_scatter_kernel(CsrView M, unsigned long long* __restrict__ cursor, idx_t* __restrict__ lst) {
    const unsigned lane = lane_id();
    const size_t nw = size_t(gridDim.x) * (blockDim.x >> 5);
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < M.nrows; r += nw) {
        const off_t64 b = M.rowptr[r], e = M.rowptr[r + 1];
        for (off_t64 p = b + lane; p < e; p += 32) {
            unsigned long long pos = atomicAdd(&cursor[M.colidx[p]], 1ull);
            lst[pos] = idx_t(r);
        }
    }
}

__global__ void reduce_flags_kernel(const off_t64* __restrict__ rp, idx_t n, uint32_t* __restrict__ f) {
    for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i < n; i += size_t(gridDim.x) * blockDim.x)
        f[i] = rp[i + 1] > rp[i] ? 1u : 0u;
}

__device__ __forceinline__ uint64_t lb64(const idx_t* p, uint64_t lo, uint64_t hi, uint64_t key) {
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (uint64_t(p[mid]) < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void sub_count_kernel(CsrView M, idx_t i0, idx_t j0, idx_t nr, idx_t nc, uint32_t* __restrict__ cnt,
                                 uint64_t* __restrict__ beg) {
    for (size_t r = blockIdx.x * size_t(blockDim.x) + threadIdx.x; r < nr; r += size_t(gridDim.x) * blockDim.x) {
        const off_t64 b = M.rowptr[i0 + r], e = M.rowptr[i0 + r + 1];
        const uint64_t s = lb64(M.colidx, b, e, j0);
        const uint64_t t = lb64(M.colidx, s, e, uint64_t(j0) + nc);
        cnt[r] = uint32_t(t - s);
        beg[r] = s;
    }
}

__global__ void sub_copy_kernel(const idx_t* __restrict__ ci, const uint64_t* __restrict__ beg,
                                const off_t64* __restrict__ rp, idx_t nr, idx_t j0, idx_t* __restrict__ out) {
    const unsigned lane = lane_id();
    const size_t nw = size_t(gridDim.x) * (blockDim.x >> 5);
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < nr; r += nw) {
        const off_t64 o = rp[r], n = rp[r + 1] - o;
        const idx_t* s = ci + beg[r];
        for (uint64_t t = lane; t < n; t += 32) out[o + t] = s[t] - j0;
    }
}

// Set difference per row, D = C \ P (the semi-naive closure's new entries,
// DESIGN.md §4.2): warp per row, every C entry binary-searched in P's row,
// kept entries placed by ballot.  WRITE = false counts, true writes.
template <bool WRITE>
__global__ void row_diff_kernel(CsrView C, CsrView P, uint32_t* __restrict__ cnt, const off_t64* __restrict__ rp,
                                idx_t* __restrict__ out) {
    const unsigned lane = lane_id();
    const size_t nw = size_t(gridDim.x) * (blockDim.x >> 5);
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < C.nrows; r += nw) {
        const off_t64 b = C.rowptr[r], e = C.rowptr[r + 1];
        const off_t64 pb = P.rowptr[r], pe = P.rowptr[r + 1];
        uint64_t o = WRITE ? rp[r] : 0;
        for (off_t64 q0 = b; q0 < e; q0 += 32) {
            const off_t64 q = q0 + lane;
            bool keep = false;
            idx_t c = 0;
            if (q < e) {
                c = C.colidx[q];
                const uint64_t at = lb64(P.colidx, pb, pe, c);
                keep = at == pe || P.colidx[at] != c;
            }
            const uint32_t bal = __ballot_sync(0xffffffffu, keep);
            if (WRITE && keep) out[o + __popc(bal & ((1u << lane) - 1u))] = c;
            o += __popc(bal);
        }
        if (!WRITE && lane == 0) cnt[r] = uint32_t(o);
    }
}

}  // namespace

void row_difference(Matrix* D, const Matrix* C, const Matrix* P) {
    if (C->nrows != P->nrows || C->ncols != P->ncols || D->nrows != C->nrows || D->ncols != C->ncols)
        SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "difference: shapes differ");
    const idx_t m = C->nrows;
    if (m == 0 || C->nnz == 0) {
        matrix_set_empty(D);
        return;
    }
    DevBuf<uint32_t> cnt(m);
    DevBuf<off_t64> rp(size_t(m) + 1, kMat);
    const unsigned g = grid_for(uint64_t(m) * 32, 256);
    row_diff_kernel<false><<<g, 256, 0, ctx().stream>>>(view(C), view(P), cnt.p, nullptr, nullptr);
    count_launch();
    check_launch("row_diff_kernel");
    exclusive_scan_u32(cnt.p, rp.p, m);
    uint64_t nnz;
    read_words(rp.p + m, &nnz, 1);
    DevBuf<idx_t> ci(nnz, kMat);
    if (nnz) {
        row_diff_kernel<true><<<g, 256, 0, ctx().stream>>>(view(C), view(P), nullptr, rp.p, ci.p);
        count_launch();
        check_launch("row_diff_kernel");
    }
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(D, rp.detach(), rc, ci.detach(), cc, nnz);
}

void transpose(Matrix* T, const Matrix* M) {
    if (T->nrows != M->ncols || T->ncols != M->nrows) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "Transpose: T must be n x m");
    if (!T->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Transpose: output is a non-owning view");
    const idx_t nt = M->ncols;
    if (M->nnz == 0 || nt == 0) {
        matrix_set_empty(T);
        return;
    }
    cudaStream_t st = ctx().stream;
    DevBuf<uint64_t> cnt(size_t(nt) + 1), bkt(size_t(nt) + 1), cursor(size_t(nt) + 1);
    memset_async(cnt.p, 0, cnt.n * 8);
    col_hist_kernel<<<grid_for(M->nnz, 256), 256, 0, st>>>(M->colidx, M->nnz, (unsigned long long*)cnt.p);
    count_launch();
    check_launch("col_hist_kernel");
    exclusive_scan_u64(cnt.p, bkt.p, nt);
    copy_async(cursor.p, bkt.p, cursor.n * 8, cudaMemcpyDeviceToDevice);
    DevBuf<idx_t> lst(M->nnz);
    transpose_scatter_kernel<<<grid_for(uint64_t(M->nrows) * 32, 256), 256, 0, st>>>(
        view(M), (unsigned long long*)cursor.p, lst.p);
    count_launch();
    check_launch("transpose_scatter_kernel");
    cursor.release();
    SegSource src{};
    src.kind = 1;
    src.lrp = bkt.p;
    src.lst = lst.p;
    Matrix tmp;
    tmp.nrows = nt;
    tmp.ncols = M->nrows;
    row_engine(src, nt, M->nrows, cnt.p, nullptr, &tmp);
    matrix_replace(T, tmp.rowptr, tmp.rowptr_cap, tmp.colidx, tmp.colidx_cap, tmp.nnz);
}

void reduce_to_column(Matrix* V, const Matrix* M) {
    if (V->nrows != M->nrows || V->ncols != 1) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "Reduce: V must be m x 1");
    if (!V->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Reduce: output is a non-owning view");
    const idx_t m = M->nrows;
    if (m == 0 || M->nnz == 0) {
        matrix_set_empty(V);
        return;
    }
    DevBuf<uint32_t> f(m);
    DevBuf<off_t64> rp(size_t(m) + 1, kMat);
    reduce_flags_kernel<<<grid_for(m, 256), 256, 0, ctx().stream>>>(M->rowptr, m, f.p);
    count_launch();
    check_launch("reduce_flags_kernel");
    exclusive_scan_u32(f.p, rp.p, m);
    uint64_t nnz;
    read_words(rp.p + m, &nnz, 1);
    DevBuf<idx_t> ci(nnz, kMat);
    memset_async(ci.p, 0, nnz * sizeof(idx_t));  // the single column index 0
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(V, rp.detach(), rc, ci.detach(), cc, nnz);
}

void submatrix(Matrix* R, const Matrix* M, idx_t i0, idx_t j0, idx_t nr, idx_t nc) {
    if (uint64_t(i0) + nr > M->nrows || uint64_t(j0) + nc > M->ncols)
        SPBLA_THROW(SPBLA_STATUS_INDEX_OUT_OF_BOUNDS, "ExtractSubMatrix: window leaves the matrix");
    if (R->nrows != nr || R->ncols != nc) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "ExtractSubMatrix: R has the wrong shape");
    if (!R->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "ExtractSubMatrix: output is a non-owning view");
    if (nr == 0 || nc == 0 || M->nnz == 0) {
        matrix_set_empty(R);
        return;
    }
    DevBuf<uint32_t> cnt(nr);
    DevBuf<uint64_t> beg(nr);
    DevBuf<off_t64> rp(size_t(nr) + 1, kMat);
    sub_count_kernel<<<grid_for(nr, 256), 256, 0, ctx().stream>>>(view(M), i0, j0, nr, nc, cnt.p, beg.p);
    count_launch();
    check_launch("sub_count_kernel");
    exclusive_scan_u32(cnt.p, rp.p, nr);
    uint64_t nnz;
    read_words(rp.p + nr, &nnz, 1);
    DevBuf<idx_t> ci(nnz, kMat);
    if (nnz) {
        sub_copy_kernel<<<grid_for(uint64_t(nr) * 32, 256), 256, 0, ctx().stream>>>(M->colidx, beg.p, rp.p, nr, j0, ci.p);
        count_launch();
        check_launch("sub_copy_kernel");
    }
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(R, rp.detach(), rc, ci.detach(), cc, nnz);
}

}  // namespace spbla
