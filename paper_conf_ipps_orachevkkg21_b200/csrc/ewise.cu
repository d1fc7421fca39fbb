// Element-wise addition C = A + B (§III-A l.266-269: "GPU
// Merge Path algorithm with dynamic work balancing and two pass processing").
//
// The two CSR matrices are two sorted sequences of (row, col) keys; their
// merge (ties: A first) is the row-major concatenation of the per-row merges,
// and row r starts at merged position P(r) = rpA[r] + rpB[r].  Merge path cuts
// the merged sequence into equal tiles of kTile items, so every block gets
// exactly kTile merged items whatever the row-length skew.  A B item is a
// duplicate iff the merged item just before it is the A item with the same
// key (rows are sorted and duplicate-free).
//
// B200 design: ONE pass over the inputs instead of the paper's two.
//   ewise_split_kernel : per row, the merge-path split (A count) of every
//                        tile boundary inside the row, and for every tile the
//                        first row whose merged start lies in it.
//   ewise_merge_kernel : per tile (ticket order): coalesced staging of the
//                        tile's A and B ranges as 64-bit (row, col) keys in
//                        shared memory, merge path per thread in smem, block
//                        scan of duplicates, decoupled look-back over the
//                        tiles' kept counts for the output base, coalesced
//                        writes of colidx through smem, and the row offsets
//                        of the rows starting in the tile.
// HBM bytes: 4(nnzA + nnzB) + 16(m+1) read, 4 nnz(C) + 8(m+1) written.
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

#ifndef SPBLA_EW_THREADS  // (overridable for a sweep)
#define SPBLA_EW_THREADS 512
#endif
constexpr int kThreads = SPBLA_EW_THREADS;
constexpr int kMinBlocks = 1536 / kThreads;  // 1536 threads per SM at ~30 KB smem per 2048 items
constexpr int kItems = 8;
constexpr uint32_t kTile = kThreads * kItems;  // merged items per tile (4096 at 512 threads)
// padded smem indices: threads own kItems consecutive positions, so a plain
// layout puts the lanes of a warp kItems words apart (8- to 16-way bank
// conflicts); one pad word per 16 (keys, 64-bit) / 32 (marks, output) words
// spreads them over all banks
__device__ __forceinline__ uint32_t KI(uint32_t p) { return p + (p >> 4); }
__device__ __forceinline__ uint32_t OI(uint32_t p) { return p + (p >> 5); }
constexpr uint32_t kKeyWords = kTile + kTile / 16, kOutWords = kTile + kTile / 32 + 1;
constexpr size_t kMergeSmem = size_t(kKeyWords) * 8 + size_t(kOutWords) * 4 + (kTile + 1) * 2;
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagPre = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

struct MergeIn {
    idx_t nrows;
    const off_t64* __restrict__ rpa;
    const idx_t* __restrict__ ca;
    const off_t64* __restrict__ rpb;
    const idx_t* __restrict__ cb;
    uint64_t L;  // nnzA + nnzB
};

__device__ __forceinline__ uint64_t P(const MergeIn& m, idx_t r) { return m.rpa[r] + m.rpb[r]; }

// Per row r: for every tile boundary d = t*kTile in [P(r), P(r+1)) (non-empty
// rows only), tile_row[t] = r and tile_a[t] = the A position of the
// merge-path split of the row's first q = d - P(r) merged items (ties: A
// first); for every tile t with P(r-1) < t*kTile <= P(r), tile_rlo[t] = r
// (the first row whose merged start is in tile t or later).  The sentinel
// tile_row / tile_a[ntiles] is written by row nrows.  tile_prev[t]: the key
// of the A item just before the split if it lies in the same row.
__global__ void ewise_split_kernel(MergeIn m, uint64_t ntiles, uint32_t* __restrict__ tile_row,
                                   uint64_t* __restrict__ tile_a, uint32_t* __restrict__ tile_rlo,
                                   uint64_t* __restrict__ tile_prev) {
    for (size_t r = blockIdx.x * size_t(blockDim.x) + threadIdx.x; r <= m.nrows; r += size_t(gridDim.x) * blockDim.x) {
        const uint64_t p = P(m, idx_t(r));
        const uint64_t pprev = r ? P(m, idx_t(r - 1)) : 0;
        for (uint64_t t = r ? pprev / kTile + 1 : 0; t * kTile <= p && t <= ntiles; ++t) tile_rlo[t] = uint32_t(r);
        if (r == m.nrows) {
            tile_row[ntiles] = m.nrows;
            tile_a[ntiles] = m.rpa[m.nrows];
            continue;
        }
        const uint64_t sa = m.rpa[r], sb = m.rpb[r];
        const uint64_t la = m.rpa[r + 1] - sa, lb = m.rpb[r + 1] - sb;
        for (uint64_t t = (p + kTile - 1) / kTile; t * kTile < p + la + lb; ++t) {
            const uint64_t q = t * kTile - p;
            uint64_t lo = q > lb ? q - lb : 0, hi = q < la ? q : la;
            while (lo < hi) {
                const uint64_t mid = (lo + hi) >> 1;
                if (m.ca[sa + mid] <= m.cb[sb + q - 1 - mid]) lo = mid + 1; else hi = mid;
            }
            tile_row[t] = uint32_t(r);
            tile_a[t] = sa + lo;
            // the A item just before the split as a key: only an item of the
            // same row can equal a B key of tile t
            tile_prev[t] = lo > 0 ? ((uint64_t(r) << 32) | m.ca[sa + lo - 1]) : ~0ull;
        }
    }
}

__device__ __forceinline__ void st_relaxed(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_relaxed(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__global__ void __launch_bounds__(kThreads, kMinBlocks)
ewise_merge_kernel(MergeIn m, uint64_t ntiles, const uint32_t* __restrict__ tile_row,
                   const uint64_t* __restrict__ tile_a, const uint32_t* __restrict__ tile_rlo,
                   const uint64_t* __restrict__ tile_prev, uint64_t* status, uint32_t* ticket,
                   idx_t* __restrict__ out, off_t64* __restrict__ rowptr) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint64_t* s_key = reinterpret_cast<uint64_t*>(smem_raw);    // [kTile] A keys [0, na), B keys [na, len)
    uint32_t* s_out = reinterpret_cast<uint32_t*>(s_key + kKeyWords);  // kept columns in output order (OI)
    uint16_t* s_dpre = reinterpret_cast<uint16_t*>(s_out + kOutWords);  // [kTile+1] duplicates before each position
    __shared__ uint64_t sh[33];
    __shared__ uint32_t s_t;
    __shared__ uint64_t s_base;
    uint32_t* s_mark = s_out;  // row marks (scratch until the output is staged)
#pragma unroll
    for (int k = 0; k < kItems; ++k) s_mark[OI(threadIdx.x * kItems + k)] = 0u;
    if (threadIdx.x == 0) s_t = atomicAdd(ticket, 1u);  // ticket order: the look-back never waits on a later block
    __syncthreads();
    const uint64_t t = s_t;
    const uint64_t d0 = t * kTile, d1 = min(d0 + kTile, m.L);
    const uint32_t len = uint32_t(d1 - d0);
    const uint64_t a0 = tile_a[t], a1 = tile_a[t + 1];
    const uint64_t b0 = d0 - a0, b1 = d1 - a1;
    const uint32_t na = uint32_t(a1 - a0), nb = uint32_t(b1 - b0);
    const uint32_t r0 = tile_row[t], r1 = min(tile_row[t + 1], m.nrows - 1);
    const uint64_t prevA = tile_prev[t];
    // 1. stage the columns (coalesced) and, in the same round trip, mark the
    //    first tile position of every row segment (0 = no mark; B marks are
    //    offset by nrows + 1 so that no A row carries into the B part); a
    //    max-scan then gives every position its row, ORed into the key
    {
        idx_t cv[kItems];  // all loads in flight before the first smem store
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const uint32_t pos = k * kThreads + threadIdx.x;
            cv[k] = pos < na ? m.ca[a0 + pos] : (pos < len ? m.cb[b0 + (pos - na)] : 0u);
        }
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const uint32_t pos = k * kThreads + threadIdx.x;
            if (pos < len) s_key[KI(pos)] = cv[k];
        }
    }
    const uint32_t boff = m.nrows + 1;
#pragma unroll 1
    for (uint32_t r = r0 + threadIdx.x; r <= r1; r += kThreads) {
        const uint64_t ra = max(m.rpa[r], a0), rae = min(m.rpa[r + 1], a1);
        const uint64_t rb = max(m.rpb[r], b0), rbe = min(m.rpb[r + 1], b1);
        if (ra < rae) s_mark[OI(uint32_t(ra - a0))] = r + 1;
        if (rb < rbe) s_mark[OI(na + uint32_t(rb - b0))] = boff + r + 1;
    }
    __syncthreads();
    {
        uint32_t v[kItems], run = 0;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            run = max(run, s_mark[OI(threadIdx.x * kItems + k)]);
            v[k] = run;
        }
        // block exclusive max-scan of the thread maxima
        uint32_t inc = run;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, inc, d);
            if (int(lane_id()) >= d) inc = max(inc, y);
        }
        __shared__ uint32_t s_wmax[kThreads / 32];
        if (lane_id() == 31) s_wmax[threadIdx.x >> 5] = inc;
        __syncthreads();
        uint32_t carry = 0;
        for (unsigned w = 0; w < (threadIdx.x >> 5); ++w) carry = max(carry, s_wmax[w]);
        const uint32_t ex = max(carry, __shfl_up_sync(0xffffffffu, inc, 1) * (lane_id() > 0));
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const uint32_t pos = threadIdx.x * kItems + k;
            if (pos < len) {
                uint32_t rr = max(ex, v[k]) - 1;
                if (pos >= na) rr -= boff;
                s_key[KI(pos)] |= uint64_t(rr) << 32;
            }
        }
    }
    __syncthreads();
    // 2. merge path per thread over the smem keys, kItems items each
    const uint32_t k0 = min(uint32_t(threadIdx.x) * kItems, len), k1 = min(k0 + kItems, len);
    uint32_t lo = k0 > nb ? k0 - nb : 0, hi = min(k0, na);
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_key[KI(mid)] <= s_key[KI(na + k0 - 1 - mid)]) lo = mid + 1; else hi = mid;
    }
    uint32_t ai = lo, bi = k0 - lo;
    idx_t col[kItems];
    uint32_t dmask = 0, ndup = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        col[k] = 0;
        if (k0 + k < k1) {
            const bool takeA = ai < na && (bi == nb || s_key[KI(ai)] <= s_key[KI(na + bi)]);
            if (takeA) {
                col[k] = idx_t(s_key[KI(ai++)]);
            } else {
                const uint64_t kb = s_key[KI(na + bi++)];
                const uint64_t pa = ai > 0 ? s_key[KI(ai - 1)] : prevA;
                col[k] = idx_t(kb);
                if (pa == kb) {
                    dmask |= 1u << k;
                    ++ndup;
                }
            }
        }
    }
    // 3. duplicates before every tile position; the tile's kept count
    uint64_t tdup;
    const uint32_t dex = uint32_t(block_exclusive_scan<uint64_t>(ndup, sh, &tdup));
    {
        uint32_t run = dex;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            if (k0 + k < k1) s_dpre[k0 + k] = uint16_t(run);
            run += (dmask >> k) & 1u;
        }
        if (k1 == len && k0 < k1) s_dpre[len] = uint16_t(run);
    }
    const uint64_t kept = len - tdup;
    // 4. decoupled look-back over the tiles' kept counts, one warp reading a
    //    window of 32 predecessors per round trip (a serial one-tile-per-load
    //    look-back falls behind the tiles in flight and serialises the grid)
    if (threadIdx.x < 32) {
        const unsigned lane = lane_id();
        uint64_t prefix = 0;
        if (t == 0) {
            if (lane == 0) st_relaxed(&status[0], kFlagPre | kept);
        } else {
            if (lane == 0) st_relaxed(&status[t], kFlagAgg | kept);
            for (long j = long(t) - 1;; j -= 32) {
                const long idx = j - long(lane);  // lane 0 = the nearest predecessor
                uint64_t s = idx >= 0 ? ld_relaxed(&status[idx]) : kFlagPre;
                while (__any_sync(0xffffffffu, (s >> 62) == 0))
                    if ((s >> 62) == 0) s = ld_relaxed(&status[idx]);
                const uint32_t pre = __ballot_sync(0xffffffffu, (s >> 62) == 2);
                const int first = pre ? __ffs(pre) - 1 : 31;
                prefix += warp_sum(int(lane) <= first ? (s & kValMask) : 0ull);
                if (pre) break;
            }
            if (lane == 0) st_relaxed(&status[t], kFlagPre | (prefix + kept));
        }
        if (lane == 0) s_base = prefix;
    }
    // 5. kept columns to smem in output order, then coalesced stores
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
        const uint32_t pos = k0 + k;
        if (pos < k1 && !((dmask >> k) & 1u)) s_out[OI(pos - s_dpre[pos])] = col[k];
    }
    __syncthreads();
    const uint64_t base = s_base;
    for (uint32_t i = threadIdx.x; i < kept; i += kThreads) out[base + i] = s_out[OI(i)];
    // 6. row offsets of the rows starting in [d0, d1); the last tile also
    //    writes the rows starting at L (trailing empty rows, rowptr[nrows])
    const uint32_t rlo = tile_rlo[t], rhi = (t + 1 == ntiles) ? m.nrows + 1 : tile_rlo[t + 1];
    for (uint32_t r = rlo + threadIdx.x; r < rhi; r += kThreads) {
        const uint32_t p = uint32_t(P(m, r) - d0);
        rowptr[r] = base + p - s_dpre[p];
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
    const int nsm = ctx().num_sms;
    // tile_row[ntiles+1] | tile_rlo[ntiles+1] (u32), tile_a[ntiles+1] | tile_prev[ntiles+1],
    // status[ntiles] + ticket
    DevBuf<uint32_t> trow(2 * (ntiles + 1));
    DevBuf<uint64_t> ta(2 * (ntiles + 1));
    DevBuf<uint64_t> status(ntiles + 1);
    memset_async(status.p, 0, status.n * sizeof(uint64_t));
    // the result: colidx capacity nnzA + nnzB (>= nnz(C)); the exact nnz is
    // read back, and a result with more than 1/8 of that capacity unused is
    // moved into an exact-size buffer
    DevBuf<off_t64> rp(size_t(A->nrows) + 1, kMat);
    DevBuf<idx_t> ci(m.L, kMat);
    int t = ktime_begin("ewise_split", ctx().stream);
    const unsigned g1 = (unsigned)std::min<uint64_t>(ceil_div(uint64_t(A->nrows) + 1, 256), uint64_t(nsm) * 8);
    ewise_split_kernel<<<g1, 256, 0, ctx().stream>>>(m, ntiles, trow.p, ta.p, trow.p + ntiles + 1, ta.p + ntiles + 1);
    ktime_end(t);
    count_launch();
    check_launch("ewise_split_kernel");
    static int attr_dev = -1;
    if (attr_dev != ctx().device) {
        CUDA_CHECK(cudaFuncSetAttribute(ewise_merge_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kMergeSmem)));
        attr_dev = ctx().device;
    }
    t = ktime_begin("ewise_merge", ctx().stream);
    ewise_merge_kernel<<<(unsigned)ntiles, kThreads, kMergeSmem, ctx().stream>>>(
        m, ntiles, trow.p, ta.p, trow.p + ntiles + 1, ta.p + ntiles + 1, status.p,
        reinterpret_cast<uint32_t*>(status.p + ntiles),
        ci.p, rp.p);
    ktime_end(t);
    count_launch();
    check_launch("ewise_merge_kernel");
    uint64_t nnz;
    read_words(rp.p + A->nrows, &nnz, 1);
    size_t rc = rp.n, cc = ci.n;
    if (m.L - nnz > m.L / 8) {
        // many shared entries (e.g. A + A): keep an exact-size colidx instead
        // of holding nnzA + nnzB words for the matrix's lifetime
        DevBuf<idx_t> exact(nnz, kMat);
        if (nnz) copy_async(exact.p, ci.p, nnz * sizeof(idx_t), cudaMemcpyDeviceToDevice);
        cc = exact.n;
        matrix_replace(C, rp.detach(), rc, exact.detach(), cc, nnz);
        return;
    }
    matrix_replace(C, rp.detach(), rc, ci.detach(), cc, nnz);
}

}  // namespace spbla
