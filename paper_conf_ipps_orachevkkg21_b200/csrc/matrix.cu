// Matrix life cycle (§II l.229-232): New / Free / Build (fill with
// pairs) / ExtractPairs (read pairs), plus CSR import/export, zero-copy
// wrapping and row-block assembly for the row-partitioned multi-GPU path.
//
// Build = row histogram + in-house scan + bucket scatter + the row engine's
// per-row sort/dedup (rowsort.cu).  With SORTED|NO_DUPLICATES hints it is a
// histogram + scan + copy.
#include "common.cuh"

#include <algorithm>
#include <vector>

namespace spbla {

namespace {

unsigned grid_for(uint64_t work, int threads, int per_sm = 16) {
    uint64_t g = ceil_div(work, threads);
    uint64_t cap = uint64_t(ctx().num_sms) * per_sm;
    return (unsigned)std::max<uint64_t>(1, std::min(g, cap));
}

__global__ void pair_hist_kernel(const idx_t* __restrict__ r, const idx_t* __restrict__ c, uint64_t n,
                                 idx_t nrows, idx_t ncols, unsigned long long* __restrict__ cnt,
                                 unsigned long long* __restrict__ flag) {
    for (uint64_t e = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; e < n;
         e += uint64_t(gridDim.x) * blockDim.x) {
        idx_t i = r[e], j = c[e];
        if (i >= nrows || j >= ncols) {
            *flag = 1ull;
            continue;
        }
        atomicAdd(&cnt[i], 1ull);
    }
}

__global__ void pair_scatter_kernel(const idx_t* __restrict__ r, const idx_t* __restrict__ c, uint64_t n,
                                    unsigned long long* __restrict__ cursor, idx_t* __restrict__ lst) {
    for (uint64_t e = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; e < n;
         e += uint64_t(gridDim.x) * blockDim.x) {
        unsigned long long pos = atomicAdd(&cursor[r[e]], 1ull);
        lst[pos] = c[e];
    }
}

__global__ void expand_rows_kernel(const off_t64* __restrict__ rowptr, idx_t nrows, idx_t* __restrict__ rows) {
    const unsigned lane = lane_id();
    const size_t nw = size_t(gridDim.x) * (blockDim.x >> 5);
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < nrows; r += nw) {
        const off_t64 b = rowptr[r], e = rowptr[r + 1];
        for (off_t64 p = b + lane; p < e; p += 32) rows[p] = idx_t(r);
    }
}

// CSR invariant check: rowptr[0] == 0, non-decreasing, rowptr[n] == nnz,
// columns < ncols and strictly increasing inside each row.
__global__ void validate_kernel(const off_t64* __restrict__ rowptr, const idx_t* __restrict__ colidx,
                                idx_t nrows, idx_t ncols, uint64_t nnz, unsigned long long* flag) {
    const unsigned lane = lane_id();
    const size_t nw = size_t(gridDim.x) * (blockDim.x >> 5);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
        if (rowptr[0] != 0 || rowptr[nrows] != nnz) *flag = 1ull;
    }
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < nrows; r += nw) {
        const off_t64 b = rowptr[r], e = rowptr[r + 1];
        if (e < b || e > nnz) {
            if (lane == 0) *flag = 1ull;
            continue;
        }
        for (off_t64 p = b + lane; p < e; p += 32) {
            idx_t c = colidx[p];
            if (c >= ncols || (p > b && colidx[p - 1] >= c)) *flag = 1ull;
        }
    }
}

__global__ void shift_rowptr_kernel(const off_t64* __restrict__ in, idx_t n, off_t64 add,
                                    off_t64* __restrict__ out) {
    for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i < n; i += size_t(gridDim.x) * blockDim.x)
        out[i] = in[i] + add;
}

__global__ void set_word_kernel(off_t64* p, off_t64 v) { *p = v; }

// One row block pushed to up to kMaxPeerDst destinations at once (the
// all-gather over peer memory): every element is loaded once
// and stored to each destination -- on an NVSwitch box the destinations are
// the other GPUs' gathered buffers, mapped into this process (CUDA IPC), so
// the stores travel over NVLink.  Warps store contiguous 128-B runs.
constexpr uint32_t kMaxPeerDst = 8;
struct PeerDst {
    off_t64* rp[kMaxPeerDst];
    idx_t* ci[kMaxPeerDst];
};
__global__ void export_multi_kernel(const off_t64* __restrict__ rp, idx_t nrows, const idx_t* __restrict__ ci,
                                    uint64_t nnz, off_t64 add, PeerDst d, uint32_t ndst) {
    const size_t stride = size_t(gridDim.x) * blockDim.x;
    for (size_t i = blockIdx.x * size_t(blockDim.x) + threadIdx.x; i <= nrows; i += stride) {
        const off_t64 v = rp[i] + add;
        for (uint32_t k = 0; k < ndst; ++k) d.rp[k][i] = v;
    }
    for (size_t j = blockIdx.x * size_t(blockDim.x) + threadIdx.x; j < nnz; j += stride) {
        const idx_t c = ci[j];
        for (uint32_t k = 0; k < ndst; ++k) d.ci[k][j] = c;
    }
}

}  // namespace

void validate_csr(const off_t64* rowptr, const idx_t* colidx, idx_t nrows, idx_t ncols, uint64_t nnz) {
    DevBuf<uint64_t> flag(1);
    memset_async(flag.p, 0, 8);
    validate_kernel<<<grid_for(uint64_t(nrows) * 32, 256), 256, 0, ctx().stream>>>(
        rowptr, colidx, nrows, ncols, nnz, (unsigned long long*)flag.p);
    count_launch();
    check_launch("validate_kernel");
    uint64_t h;
    read_words(flag.p, &h, 1);
    if (h) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "CSR arrays violate the invariants");
}

void matrix_build(Matrix* m, const idx_t* rows, const idx_t* cols, uint64_t n, uint32_t hints) {
    if (!m->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Build: matrix is a non-owning view");
    if (n && (!rows || !cols)) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Build: null pair arrays");
    cudaStream_t st = ctx().stream;
    DevBuf<idx_t> hr, hc;
    if (n && (hints & SPBLA_HINT_HOST_MEMORY)) {
        hr.alloc(n);
        hc.alloc(n);
        copy_async(hr.p, rows, n * sizeof(idx_t), cudaMemcpyHostToDevice);
        copy_async(hc.p, cols, n * sizeof(idx_t), cudaMemcpyHostToDevice);
        rows = hr.p;
        cols = hc.p;
    }
    const idx_t nr = m->nrows;
    DevBuf<uint64_t> cnt(size_t(nr) + 1);
    DevBuf<uint64_t> bkt(size_t(nr) + 2);  // [0..nr] offsets, [nr+1] error flag
    memset_async(cnt.p, 0, cnt.n * 8);
    memset_async(bkt.p, 0, bkt.n * 8);
    if (n) {
        pair_hist_kernel<<<grid_for(n, 256), 256, 0, st>>>(rows, cols, n, nr, m->ncols,
                                                         (unsigned long long*)cnt.p,
                                                         (unsigned long long*)(bkt.p + nr + 1));
        count_launch();
        check_launch("pair_hist_kernel");
    }
    exclusive_scan_u64(cnt.p, bkt.p, nr);
    uint64_t h[2];
    read_words(bkt.p + nr, h, 2);
    if (h[1]) SPBLA_THROW(SPBLA_STATUS_INDEX_OUT_OF_BOUNDS, "Build: pair outside the matrix");
    const bool presorted = (hints & SPBLA_HINT_SORTED) && (hints & SPBLA_HINT_NO_DUPLICATES);
    if (presorted || n == 0) {
        DevBuf<off_t64> rp(size_t(nr) + 1, kMat);
        copy_async(rp.p, bkt.p, rp.n * 8, cudaMemcpyDeviceToDevice);
        DevBuf<idx_t> ci(n, kMat);
        copy_async(ci.p, cols, n * sizeof(idx_t), cudaMemcpyDeviceToDevice);
        if (hints & SPBLA_HINT_VALIDATE) validate_csr(rp.p, ci.p, nr, m->ncols, n);
        size_t rc = rp.n, cc = ci.n;
        matrix_replace(m, rp.detach(), rc, ci.detach(), cc, n);
        return;
    }
    DevBuf<uint64_t> cursor(size_t(nr) + 1);
    copy_async(cursor.p, bkt.p, cursor.n * 8, cudaMemcpyDeviceToDevice);
    DevBuf<idx_t> lst(n);
    pair_scatter_kernel<<<grid_for(n, 256), 256, 0, st>>>(rows, cols, n, (unsigned long long*)cursor.p, lst.p);
    count_launch();
    check_launch("pair_scatter_kernel");
    cursor.release();
    hr.release();
    hc.release();
    SegSource src{};
    src.kind = 1;
    src.lrp = bkt.p;
    src.lst = lst.p;
    Matrix tmp;
    tmp.nrows = nr;
    tmp.ncols = m->ncols;
    row_engine(src, nr, m->ncols, cnt.p, nullptr, &tmp);
    matrix_replace(m, tmp.rowptr, tmp.rowptr_cap, tmp.colidx, tmp.colidx_cap, tmp.nnz);
}

void matrix_extract_pairs(const Matrix* m, idx_t* rows, idx_t* cols, uint32_t hints) {
    const uint64_t n = m->nnz;
    if (n == 0) return;
    const bool host = hints & SPBLA_HINT_HOST_MEMORY;
    DevBuf<idx_t> dr;
    idx_t* r = rows;
    if (host) {
        dr.alloc(n);
        r = dr.p;
    }
    expand_rows_kernel<<<grid_for(uint64_t(m->nrows) * 32, 256), 256, 0, ctx().stream>>>(m->rowptr, m->nrows, r);
    count_launch();
    check_launch("expand_rows_kernel");
    if (host) {
        copy_async(rows, r, n * sizeof(idx_t), cudaMemcpyDeviceToHost);
        copy_async(cols, m->colidx, n * sizeof(idx_t), cudaMemcpyDeviceToHost);
        CUDA_CHECK(cudaStreamSynchronize(ctx().stream));
    } else {
        copy_async(cols, m->colidx, n * sizeof(idx_t), cudaMemcpyDeviceToDevice);
    }
}

void matrix_export(const Matrix* m, off_t64* rowptr, idx_t* colidx, uint32_t hints) {
    const bool host = hints & SPBLA_HINT_HOST_MEMORY;
    cudaMemcpyKind k = host ? cudaMemcpyDeviceToHost : cudaMemcpyDeviceToDevice;
    if (rowptr) copy_async(rowptr, m->rowptr, (size_t(m->nrows) + 1) * 8, k);
    if (colidx) copy_async(colidx, m->colidx, m->nnz * sizeof(idx_t), k);
    if (host) CUDA_CHECK(cudaStreamSynchronize(ctx().stream));
}

void matrix_import(Matrix* m, const off_t64* rowptr, const idx_t* colidx, uint64_t nnz, uint32_t hints) {
    if (!m->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Import: matrix is a non-owning view");
    const bool host = hints & SPBLA_HINT_HOST_MEMORY;
    cudaMemcpyKind k = host ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
    DevBuf<off_t64> rp(size_t(m->nrows) + 1, kMat);
    DevBuf<idx_t> ci(nnz, kMat);
    copy_async(rp.p, rowptr, rp.n * 8, k);
    if (nnz) copy_async(ci.p, colidx, nnz * sizeof(idx_t), k);
    if (hints & SPBLA_HINT_VALIDATE) validate_csr(rp.p, ci.p, m->nrows, m->ncols, nnz);
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(m, rp.detach(), rc, ci.detach(), cc, nnz);
}

void matrix_duplicate(const Matrix* m, Matrix* d) {
    d->nrows = m->nrows;
    d->ncols = m->ncols;
    matrix_import(d, m->rowptr, m->colidx, m->nnz, 0);
}

// Export m as one row block of a larger matrix: rowptr_out[i] = rowptr[i] +
// offset for i in [0, nrows] (nrows + 1 entries), colidx_out = colidx (device
// arrays, stream-ordered, no synchronisation).  The all-gather of a
// row-partitioned matrix writes every shard straight into its slice of the
// gathered buffers with this.
void matrix_export_block(const Matrix* m, off_t64* rowptr_out, idx_t* colidx_out, off_t64 offset) {
    shift_rowptr_kernel<<<grid_for(uint64_t(m->nrows) + 1, 256), 256, 0, ctx().stream>>>(m->rowptr, m->nrows + 1,
                                                                                       offset, rowptr_out);
    count_launch();
    check_launch("shift_rowptr_kernel");
    if (m->nnz) copy_async(colidx_out, m->colidx, m->nnz * sizeof(idx_t), cudaMemcpyDeviceToDevice);
}

// matrix_export_block to ndst destination pairs in one pass (loads once,
// stores ndst times); ndst > kMaxPeerDst is split into launches.
void matrix_export_block_multi(const Matrix* m, off_t64* const* rowptr_out, idx_t* const* colidx_out, uint32_t ndst,
                               off_t64 offset) {
    for (uint32_t k0 = 0; k0 < ndst; k0 += kMaxPeerDst) {
        PeerDst d{};
        const uint32_t nd = std::min<uint32_t>(kMaxPeerDst, ndst - k0);
        for (uint32_t k = 0; k < nd; ++k) {
            d.rp[k] = rowptr_out[k0 + k];
            d.ci[k] = colidx_out[k0 + k];
        }
        const uint64_t work = std::max<uint64_t>(uint64_t(m->nrows) + 1, m->nnz);
        export_multi_kernel<<<grid_for(work, 256), 256, 0, ctx().stream>>>(m->rowptr, m->nrows, m->colidx, m->nnz,
                                                                          offset, d, nd);
        count_launch();
        check_launch("export_multi_kernel");
    }
}

void matrix_assemble(Matrix* m, uint32_t nblocks, const idx_t* nrows, const off_t64* const* rowptr,
                     const idx_t* const* colidx, const uint64_t* nnz) {
    if (!m->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "Assemble: matrix is a non-owning view");
    uint64_t tot_rows = 0, tot_nnz = 0;
    for (uint32_t b = 0; b < nblocks; ++b) {
        tot_rows += nrows[b];
        tot_nnz += nnz[b];
    }
    if (tot_rows != m->nrows) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "Assemble: row blocks do not sum to nrows");
    DevBuf<off_t64> rp(size_t(m->nrows) + 1, kMat);
    DevBuf<idx_t> ci(tot_nnz, kMat);
    uint64_t rbase = 0, nbase = 0;
    for (uint32_t b = 0; b < nblocks; ++b) {
        if (nrows[b]) {
            shift_rowptr_kernel<<<grid_for(nrows[b], 256), 256, 0, ctx().stream>>>(rowptr[b], nrows[b], nbase,
                                                                                  rp.p + rbase);
            count_launch();
            check_launch("shift_rowptr_kernel");
        }
        if (nnz[b]) copy_async(ci.p + nbase, colidx[b], nnz[b] * sizeof(idx_t), cudaMemcpyDeviceToDevice);
        rbase += nrows[b];
        nbase += nnz[b];
    }
    set_word_kernel<<<1, 1, 0, ctx().stream>>>(rp.p + m->nrows, tot_nnz);
    count_launch();
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(m, rp.detach(), rc, ci.detach(), cc, tot_nnz);
}

}  // namespace spbla
