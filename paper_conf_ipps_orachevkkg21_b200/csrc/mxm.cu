// Boolean SpGEMM C (+)= A x B (§III-A l.259-264) and the
// transitive-closure loop C += C x C (§I l.117/126).
//
// Step 1 (this file): the upper-bound product count per row,
//   ub[i] = |C[i]| (accumulate) + sum_{k in A[i]} |B[k]|,
// one 8-lane group per row (A rows average 8..32 entries in the configs),
// coalesced colidx loads, two B row-offset loads per entry.
// Step 2: the row engine (rowsort.cu) bins rows by ub and runs the
// warp-bitonic / block-hash / block-bitmap kernels.
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

constexpr int kGroup = 8;

// Per-B-row info, one 16-B record: binfo[k] = (start, length, first column,
// last column) (rows are sorted; (0xFFFFFFFF, 0) as span of an empty row).
// The upper-bound pass then reads one aligned sector per A entry instead of
// the row-offset pair and two scattered colidx sectors.  32-bit starts need
// nnz(B) < 2^32; larger B keeps 64-bit offsets (binfo = null).
__global__ void row_info_kernel(CsrView B, uint4* __restrict__ binfo) {
    for (size_t k = blockIdx.x * size_t(blockDim.x) + threadIdx.x; k < B.nrows; k += size_t(gridDim.x) * blockDim.x) {
        const off_t64 x = B.rowptr[k], y = B.rowptr[k + 1];
        binfo[k] = y > x ? make_uint4(uint32_t(x), uint32_t(y - x), B.colidx[x], B.colidx[y - 1])
                         : make_uint4(uint32_t(x), 0u, 0xFFFFFFFFu, 0u);
    }
}
__global__ void row_span_kernel(CsrView B, uint2* __restrict__ bspan) {
    for (size_t k = blockIdx.x * size_t(blockDim.x) + threadIdx.x; k < B.nrows; k += size_t(gridDim.x) * blockDim.x) {
        const off_t64 x = B.rowptr[k], y = B.rowptr[k + 1];
        bspan[k] = y > x ? make_uint2(B.colidx[x], B.colidx[y - 1]) : make_uint2(0xFFFFFFFFu, 0u);
    }
}

#ifndef SPBLA_UB_MINB
#define SPBLA_UB_MINB 1
#endif
template <bool INFO>
__global__ void __launch_bounds__(256, SPBLA_UB_MINB) mxm_ub_kernel(CsrView A, const off_t64* __restrict__ brp, const idx_t* __restrict__ bci,
                              const uint2* __restrict__ bspan, const uint4* __restrict__ binfo,
                              const off_t64* __restrict__ crp,
                              const idx_t* __restrict__ cci, uint64_t* __restrict__ ub, uint2* __restrict__ range,
                              uint4* __restrict__ desc, uint32_t* __restrict__ nseg, uint32_t dup_ratio) {
    const unsigned lane = threadIdx.x & 31, g = lane & (kGroup - 1);
    const unsigned gshift = lane & ~(kGroup - 1);  // first lane of this row's group
    const size_t ngroups = (size_t(gridDim.x) * blockDim.x) / kGroup;
    // warp-uniform loop: every lane of a warp runs the same trip count.  The
    // row offsets of the group's next row are loaded one iteration ahead
    // (the loop is a chain of dependent loads: offsets, colidx, B records)
    size_t rb = (blockIdx.x * size_t(blockDim.x) + (threadIdx.x & ~31u)) / kGroup;
    off_t64 bn = 0, en = 0;
    if (rb + lane / kGroup < A.nrows) {
        bn = A.rowptr[rb + lane / kGroup];
        en = A.rowptr[rb + lane / kGroup + 1];
    }
    for (; rb < A.nrows; rb += ngroups) {
        const size_t r = rb + lane / kGroup;
        const bool valid = r < A.nrows;
        uint64_t s = 0;
        const off_t64 b = valid ? bn : 0, e = valid ? en : 0;
        if (r + ngroups < A.nrows) {
            bn = A.rowptr[r + ngroups];
            en = A.rowptr[r + ngroups + 1];
        }
        uint32_t cn = 0, cl = 0;  // running non-empty count / product prefix of the row
        uint32_t lcr = 0;         // |C[r]| (accumulate)
        idx_t lo = 0xFFFFFFFFu, hi = 0;
        uint4* drow = nullptr;
        if (valid) {
            drow = desc + (b + r);  // room for the C[r] segment in front
            if (crp) {
                const off_t64 cb = crp[r];
                const uint32_t lc = uint32_t(crp[r + 1] - cb);
                if (lc) {
                    if (g == 0) {
                        const uint64_t ptr = reinterpret_cast<uint64_t>(cci + cb);
                        drow[0] = make_uint4(uint32_t(ptr), uint32_t(ptr >> 32), lc, lc);
                        s = lc;
                        lo = cci[cb];
                        hi = cci[cb + lc - 1];
                    }
                    cn = 1;
                    cl = lc;
                    lcr = lc;
                }
            }
        }
        // kR entries per lane per trip (entry b + 8*(kR*it + j) + g): all kR
        // colidx loads, then all kR B-row records, are in flight together
        constexpr int kR = 4;
        const uint32_t trips =
            __reduce_max_sync(0xffffffffu, valid ? uint32_t((e - b + kGroup * kR - 1) / (kGroup * kR)) : 0u);
        for (uint32_t it = 0; it < trips; ++it) {
            idx_t kk[kR];
#pragma unroll
            for (int j = 0; j < kR; ++j) {
                const off_t64 p = b + (uint64_t(it) * kR + j) * kGroup + g;
                kk[j] = (valid && p < e) ? A.colidx[p] : 0xFFFFFFFFu;
            }
            uint32_t len[kR];
            uint64_t ptr[kR];
#pragma unroll
            for (int j = 0; j < kR; ++j) {
                len[j] = 0;
                ptr[j] = 0;
                if (kk[j] != 0xFFFFFFFFu) {
                    const idx_t k = kk[j];
                    if (INFO) {
                        const uint4 bi = binfo[k];  // span (0xFFFFFFFF, 0) when empty: neutral
                        len[j] = bi.y;
                        ptr[j] = reinterpret_cast<uint64_t>(bci + bi.x);
                        lo = min(lo, bi.z);
                        hi = max(hi, bi.w);
                    } else {
                        const off_t64 x = brp[k], y = brp[k + 1];
                        const uint2 sp = bspan[k];  // (0xFFFFFFFF, 0) when empty: neutral
                        len[j] = uint32_t(y - x);
                        ptr[j] = reinterpret_cast<uint64_t>(bci + x);
                        lo = min(lo, sp.x);
                        hi = max(hi, sp.y);
                    }
                }
            }
#pragma unroll
            for (int j = 0; j < kR; ++j) {
                s += len[j];
                // compacted position and inclusive length prefix inside the group
                const uint32_t m = (__ballot_sync(0xffffffffu, len[j] > 0) >> gshift) & 0xFFu;
                uint32_t inc = len[j];
#pragma unroll
                for (int d = 1; d < kGroup; d <<= 1) {
                    const uint32_t t = __shfl_up_sync(0xffffffffu, inc, d, kGroup);
                    if (g >= unsigned(d)) inc += t;
                }
                if (len[j])
                    drow[cn + __popc(m & ((1u << g) - 1u))] =
                        make_uint4(uint32_t(ptr[j]), uint32_t(ptr[j] >> 32), len[j], cl + inc);
                cn += __popc(m);
                cl += __shfl_sync(0xffffffffu, inc, kGroup - 1, kGroup);
            }
        }
        // row totals and column span (segments are sorted: first / last
        // entries), the span used by the hash and bitmap bins of the engine
#pragma unroll
        for (int d = kGroup / 2; d > 0; d >>= 1) {
            s += __shfl_xor_sync(0xffffffffu, s, d, kGroup);
            lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, d, kGroup));
            hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, d, kGroup));
        }
        if (valid && g == 0) {
            // dup_ratio (closure steps): products far above the row's current
            // length mean mostly repeated columns (C[k] largely inside C[r])
            const bool dup = dup_ratio && s > kRangeMinUb && s > uint64_t(dup_ratio) * lcr;
            // (a row whose only products are its accumulate input: a copy)
            const bool copy = crp && cn == 1 && s == lcr;
            ub[r] = s | (dup ? kUbDupFlag : 0) | (copy ? kUbCopyFlag : 0);
            nseg[r] = cn;
            if (s > kRangeMinUb) range[r] = make_uint2(lo, hi);
        }
    }
}

}  // namespace

static void mxm_impl(Matrix* C, const Matrix* A, const Matrix* B, bool accumulate, uint32_t dup_ratio) {
    if (A->ncols != B->nrows || C->nrows != A->nrows || C->ncols != B->ncols)
        SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "MxM: shapes do not conform");
    if (!C->owned) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "MxM: output matrix is a non-owning view");
    const idx_t m = A->nrows;
    // C = A x B does not read C: give its storage back to the pool before the
    // engine allocates scratch and the result (lowers the peak by nnz(C_old))
    if (!accumulate && C != A && C != B) matrix_release(C);
    if (m == 0) {
        matrix_set_empty(C);
        return;
    }
    trace_mark("mxm start");
    DevBuf<uint64_t> ub(m);
    DevBuf<uint2> range(m);
    DevBuf<uint4> desc(A->nnz + m);  // per row: C[r] (accumulate) + non-empty B rows
    DevBuf<uint32_t> nseg(m);
    const unsigned grid = (unsigned)std::min<uint64_t>(ceil_div(uint64_t(m) * kGroup, 256),
                                                       uint64_t(ctx().num_sms) * 16);
    const off_t64* crp = accumulate ? C->rowptr : nullptr;
    const bool info = B->nnz < (uint64_t(1) << 32);
    DevBuf<uint4> binfo(info ? B->nrows : 0);
    DevBuf<uint2> bspan(info ? 0 : B->nrows);
    int tk = ktime_begin("mxm_ub", ctx().stream);
    if (B->nrows) {
        const unsigned gs = (unsigned)std::min<uint64_t>(ceil_div(B->nrows, 256), uint64_t(ctx().num_sms) * 16);
        if (info) row_info_kernel<<<gs, 256, 0, ctx().stream>>>(view(B), binfo.p);
        else row_span_kernel<<<gs, 256, 0, ctx().stream>>>(view(B), bspan.p);
        count_launch();
    }
    if (info)
        mxm_ub_kernel<true><<<grid, 256, 0, ctx().stream>>>(view(A), B->rowptr, B->colidx, nullptr, binfo.p, crp,
                                                            accumulate ? C->colidx : nullptr, ub.p, range.p, desc.p,
                                                            nseg.p, dup_ratio);
    else
        mxm_ub_kernel<false><<<grid, 256, 0, ctx().stream>>>(view(A), B->rowptr, B->colidx, bspan.p, nullptr, crp,
                                                             accumulate ? C->colidx : nullptr, ub.p, range.p, desc.p,
                                                             nseg.p, dup_ratio);
    ktime_end(tk);
    count_launch();
    check_launch("mxm_ub_kernel");
    SegSource src{};
    src.kind = 0;
    src.dbase = A->rowptr;
    src.nseg = nseg.p;
    src.desc = desc.p;
    // the engine writes fresh storage and only then installs it into C, so
    // C may alias A and/or B
    Matrix tmp;
    tmp.nrows = m;
    tmp.ncols = B->ncols;
    row_engine(src, m, B->ncols, ub.p, range.p, &tmp);
    matrix_replace(C, tmp.rowptr, tmp.rowptr_cap, tmp.colidx, tmp.colidx_cap, tmp.nnz);
    tmp.rowptr = nullptr;
    tmp.colidx = nullptr;
    trace_mark("mxm done");
}

void mxm(Matrix* C, const Matrix* A, const Matrix* B, bool accumulate, uint32_t dup_ratio) {
    try {
        mxm_impl(C, A, B, accumulate, accumulate ? dup_ratio : 0u);
    } catch (...) {
        // a non-accumulating MxM may have released C already: leave it a
        // valid empty matrix rather than a dangling one
        if (C->rowptr == nullptr) {
            try {
                matrix_set_empty(C);
            } catch (...) {
            }
        }
        throw;
    }
}

constexpr uint32_t kClosureDupRatio = 4;

void matrix_duplicate(const Matrix* m, Matrix* d);
void row_difference(Matrix* D, const Matrix* C, const Matrix* P);

namespace {
struct OwnedMatrix {  // a library-internal matrix released on scope exit
    Matrix m;
    OwnedMatrix(idx_t r, idx_t c) {
        m.nrows = r;
        m.ncols = c;
    }
    ~OwnedMatrix() {
        try {
            matrix_release(&m);
        } catch (...) {
        }
    }
};
void swap_storage(Matrix* a, Matrix* b) { std::swap(*a, *b); }
}  // namespace

// Transitive closure C += C x C to the fixed point (§I l.113-117,
// l.126; R9).  Squaring step k: C_{k+1} = C_k + C_k C_k.  With
// Delta_k = C_k \ C_{k-1} the same iterate is C_k + Delta_k C_k + C_k Delta_k
// (C_{k-1} C_{k-1} is inside C_k already), the semi-naive step: two products
// with the small Delta instead of one with C.  The loop switches to it when
// the last step added less than 1/kSemiNaiveDiv of the entries (|Delta| is
// known from the nnz read-backs), typically the final confirming step; the
// iterates and the iteration count are those of the plain loop.
#ifndef SPBLA_SEMI_DIV  // (overridable for a sweep)
#define SPBLA_SEMI_DIV 8
#endif
constexpr uint64_t kSemiNaiveDiv = SPBLA_SEMI_DIV;

// The loop after the first step: prev = C_{k-1}, C = C_k, with
// C_{k-1} C_{k-1} inside C_k; plain squaring or the semi-naive step
// (R11) by the share of new entries; returns the steps evaluated.
static int closure_steps(Matrix* C, OwnedMatrix& prev) {
    const idx_t n = C->nrows;
    int it = 0;
    while (C->nnz != prev.m.nnz) {  // C only grows: equal nnz <=> fixed point
        const uint64_t added = C->nnz - prev.m.nnz;
        if (added * kSemiNaiveDiv < C->nnz) {
            OwnedMatrix delta(n, n);
            row_difference(&delta.m, C, &prev.m);
            OwnedMatrix next(n, n);
            matrix_duplicate(C, &next.m);
            mxm(&next.m, &delta.m, C, true, kClosureDupRatio);  // C + Delta C
            mxm(&next.m, C, &delta.m, true, kClosureDupRatio);  // ... + C Delta
            swap_storage(&prev.m, C);                           // prev = C_k
            swap_storage(C, &next.m);                           // C = C_{k+1} (next holds the old prev)
        } else {
            matrix_release(&prev.m);
            prev.m.nrows = prev.m.ncols = n;
            matrix_duplicate(C, &prev.m);
            mxm(C, C, C, true, kClosureDupRatio);
        }
        ++it;
    }
    return it;
}

int transitive_closure(Matrix* C) {
    if (C->nrows != C->ncols) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "closure: matrix must be square");
    const idx_t n = C->nrows;
    OwnedMatrix prev(n, n);  // C_{k-1}
    matrix_duplicate(C, &prev.m);
    // closure steps: rows whose products exceed kClosureDupRatio x their
    // current length are routed to the bitmap kernel
    mxm(C, C, C, true, kClosureDupRatio);
    return 1 + closure_steps(C, prev);
}

// Incremental closure (§I l.117, l.126: CFPQ/RPQ index updates add
// edges to an already closed relation): C is transitively closed, D holds
// new edges; C becomes the closure of C + D.  With C_{-1} = C (closed: C C is
// inside C) and C_0 = C + D, the loop above applies from the start; its first
// step is semi-naive with Delta_0 = D \ C (the new entries only).  Returns the
// closure steps evaluated, the confirming one included (0 when D adds
// nothing).
void ewise_add(Matrix* C, const Matrix* A, const Matrix* B);

int transitive_closure_incremental(Matrix* C, const Matrix* D) {
    if (C->nrows != C->ncols) SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "closure: matrix must be square");
    if (D->nrows != C->nrows || D->ncols != C->ncols)
        SPBLA_THROW(SPBLA_STATUS_DIM_MISMATCH, "incremental closure: D must have C's shape");
    const idx_t n = C->nrows;
    OwnedMatrix prev(n, n);
    matrix_duplicate(C, &prev.m);
    ewise_add(C, C, D);  // C_0 = C + D
    return closure_steps(C, prev);
}

}  // namespace spbla
