// Element-wise addition C = A + B (§III-A l.266-269: "GPU
// Merge Path algorithm with dynamic work balancing and two pass processing").
//
// The two CSR matrices are treated as two sorted sequences of (row, col)
// keys; their merge (ties: A first) is the row-major concatenation of the
// per-row merges, and row r starts at merged position p(r) = rpA[r] + rpB[r].
// Merge path cuts the merged sequence into equal tiles of kTile items, so
// every thread gets exactly kItems merged items whatever the row-length
// skew.  A B item is a duplicate iff the A item just before it in its row
// has the same column (rows are sorted and duplicate-free).  Output position
// of a kept item at merged position d is d - (#duplicates before d), and
// rowptrC[r] = p(r) - (#duplicates before p(r)).
//   pass 1: duplicates per tile  -> in-house scan -> nnz(C)
//   pass 2: same merge, block scan of per-thread duplicates, write colidx and
//           the row offsets of rows starting inside the thread's range.
// HBM bytes (algorithmic): 2 x 4(nnzA + nnzB) read + 4 nnz(C) + 8(m+1) written.
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

constexpr int kThreads = 128;
constexpr int kItems = 16;
constexpr int kTile = kThreads * kItems;

struct MergeIn {
    idx_t nrows;
    const off_t64* __restrict__ rpa;
    const idx_t* __restrict__ ca;
    const off_t64* __restrict__ rpb;
    const idx_t* __restrict__ cb;
    uint64_t L;
};

__device__ __forceinline__ uint64_t P(const MergeIn& m, idx_t r) { return m.rpa[r] + m.rpb[r]; }

// first row r in [lo, hi] with P(r) >= d (hi if none)
__device__ __forceinline__ idx_t rows_lower_bound(const MergeIn& m, idx_t lo, idx_t hi, uint64_t d) {
    while (lo < hi) {
        idx_t mid = lo + (hi - lo) / 2;
        if (P(m, mid) < d) lo = mid + 1; else hi = mid;
    }
    return lo;
}
// first row r in [lo, hi] with P(r) > d
__device__ __forceinline__ idx_t rows_upper_bound(const MergeIn& m, idx_t lo, idx_t hi, uint64_t d) {
    while (lo < hi) {
        idx_t mid = lo + (hi - lo) / 2;
        if (P(m, mid) <= d) lo = mid + 1; else hi = mid;
    }
    return lo;
}

struct Cursor {
    idx_t r;        // current row
    uint64_t a, b;  // global positions in A / B colidx
    uint64_t ea, eb, sa;  // row end in A, end in B, row start in A
};

// Position the cursor at merged position d < L (row search within [rlo, rhi]).
__device__ __forceinline__ Cursor locate(const MergeIn& m, uint64_t d, idx_t rlo, idx_t rhi) {
    Cursor c;
    c.r = rows_upper_bound(m, rlo, rhi, d) - 1;  // largest r with P(r) <= d
    const uint64_t sa = m.rpa[c.r], sb = m.rpb[c.r];
    const uint64_t la = m.rpa[c.r + 1] - sa, lb = m.rpb[c.r + 1] - sb;
    const uint64_t q = d - (sa + sb);
    uint64_t lo = q > lb ? q - lb : 0, hi = q < la ? q : la;
    while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        if (m.ca[sa + mid] <= m.cb[sb + q - 1 - mid]) lo = mid + 1; else hi = mid;
    }
    c.a = sa + lo;
    c.b = sb + (q - lo);
    c.sa = sa;
    c.ea = sa + la;
    c.eb = sb + lb;
    return c;
}

// Take the next merged item; returns its column and whether it duplicates
// the previous A item of the same row.
__device__ __forceinline__ idx_t take(const MergeIn& m, Cursor& c, bool& dup) {
    while (c.a == c.ea && c.b == c.eb) {  // row exhausted: advance (skips empty rows)
        ++c.r;
        c.sa = c.ea;
        c.ea = m.rpa[c.r + 1];
        c.eb = m.rpb[c.r + 1];
    }
    if (c.a < c.ea && (c.b == c.eb || m.ca[c.a] <= m.cb[c.b])) {
        dup = false;
        return m.ca[c.a++];
    }
    idx_t v = m.cb[c.b++];
    dup = (c.a > c.sa) && (m.ca[c.a - 1] == v);
    return v;
}

__device__ __forceinline__ void tile_rows(const MergeIn& m, uint64_t d0, uint64_t d1, idx_t* sr) {
    if (threadIdx.x == 0) {
        // one row before the first row starting at or after d0, so that empty
        // rows starting exactly at d0 are inside [sr0, sr1]
        idx_t lo = rows_lower_bound(m, 0, m.nrows, d0);
        sr[0] = lo > 0 ? lo - 1 : 0;
        sr[1] = rows_upper_bound(m, sr[0], m.nrows, d1);
    }
    __syncthreads();
}

__global__ void __launch_bounds__(kThreads) merge_count_kernel(MergeIn m, uint64_t* __restrict__ tile_dups) {
    __shared__ idx_t sr[2];
    __shared__ uint32_t swarp[kThreads / 32];
    const uint64_t d0 = uint64_t(blockIdx.x) * kTile;
    const uint64_t d1 = min(d0 + kTile, m.L);
    tile_rows(m, d0, d1, sr);
    const uint64_t db = d0 + uint64_t(threadIdx.x) * kItems;
    uint32_t dups = 0;
    if (db < d1) {
        Cursor c = locate(m, db, sr[0], sr[1]);
        const uint64_t de = min(db + kItems, d1);
        for (uint64_t d = db; d < de; ++d) {
            bool dup;
            take(m, c, dup);
            dups += dup;
        }
    }
    dups = warp_sum(dups);
    if (lane_id() == 0) swarp[threadIdx.x >> 5] = dups;
    __syncthreads();
    if (threadIdx.x == 0) {
        uint64_t s = 0;
        for (int w = 0; w < kThreads / 32; ++w) s += swarp[w];
        tile_dups[blockIdx.x] = s;
    }
}

__global__ void __launch_bounds__(kThreads)
merge_write_kernel(MergeIn m, const uint64_t* __restrict__ tile_base, idx_t* __restrict__ out,
                   off_t64* __restrict__ rowptr) {
    __shared__ idx_t sr[2];
    __shared__ uint64_t shs[33];
    const uint64_t d0 = uint64_t(blockIdx.x) * kTile;
    const uint64_t d1 = min(d0 + kTile, m.L);
    tile_rows(m, d0, d1, sr);
    const uint64_t db = d0 + uint64_t(threadIdx.x) * kItems;
    const uint64_t de = min(db + kItems, d1);
    // pass A: this thread's duplicate count (re-merge; cheap, data in L1)
    uint64_t mydups = 0;
    Cursor c0;
    if (db < d1) {
        c0 = locate(m, db, sr[0], sr[1]);
        Cursor c = c0;
        for (uint64_t d = db; d < de; ++d) {
            bool dup;
            take(m, c, dup);
            mydups += dup;
        }
    }
    uint64_t tot;
    uint64_t before = tile_base[blockIdx.x] + block_exclusive_scan<uint64_t>(mydups, shs, &tot);
    if (db >= d1) return;
    // rows whose merged start lies in [db, de) (including empty rows)
    idx_t nr = rows_lower_bound(m, sr[0], sr[1], db);
    Cursor c = c0;
    for (uint64_t d = db; d < de; ++d) {
        while (nr < m.nrows && P(m, nr) == d) rowptr[nr++] = d - before;
        bool dup;
        idx_t v = take(m, c, dup);
        if (dup) ++before;
        else out[d - before] = v;
    }
    if (de == m.L) {  // trailing empty rows and rowptr[nrows]
        while (nr <= m.nrows && P(m, nr) == m.L) rowptr[nr++] = m.L - before;
    }
}

}  // namespace

void ewise_add(Matrix* C, const Matrix* A, const Matrix* B) {
    if (A->nrows != B->nrows || A->ncols != B->ncols || C->nrows != A->nrows || C->ncols != A->ncols)
        SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "EWiseAdd: shapes differ");
    if (!C->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "EWiseAdd: output is a non-owning view");
    MergeIn m{A->nrows, A->rowptr, A->colidx, B->rowptr, B->colidx, A->nnz + B->nnz};
    if (m.L == 0 || A->nrows == 0) {
        matrix_set_empty(C);
        return;
    }
    const uint64_t ntiles = ceil_div(m.L, kTile);
    DevBuf<uint64_t> tdup(ntiles);
    DevBuf<uint64_t> tbase(ntiles + 1);
    merge_count_kernel<<<(unsigned)ntiles, kThreads, 0, ctx().stream>>>(m, tdup.p);
    count_launch();
    check_launch("merge_count_kernel");
    exclusive_scan_u64(tdup.p, tbase.p, ntiles);
    uint64_t h;
    read_words(tbase.p + ntiles, &h, 1);
    const uint64_t nnz = m.L - h;
    DevBuf<off_t64> rp(size_t(A->nrows) + 1, kMat);
    DevBuf<idx_t> ci(nnz, kMat);
    merge_write_kernel<<<(unsigned)ntiles, kThreads, 0, ctx().stream>>>(m, tbase.p, ci.p, rp.p);
    count_launch();
    check_launch("merge_write_kernel");
    size_t rc = rp.n, cc = ci.n;
    matrix_replace(C, rp.detach(), rc, ci.detach(), cc, nnz);
}

}  // namespace spbla
