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
#define SPBLA_EW_THREADS 256
#endif
#ifndef SPBLA_EW_ITEMS
#define SPBLA_EW_ITEMS 16
#endif
constexpr int kThreads = SPBLA_EW_THREADS;
constexpr int kItems = SPBLA_EW_ITEMS;  // merged items per thread (<= 32: one dup-mask word)
constexpr uint32_t kTile = kThreads * kItems;  // merged items per tile (4096)
#ifndef SPBLA_EW_ROWS
#define SPBLA_EW_ROWS 1024
#endif
constexpr uint32_t kRowStage = SPBLA_EW_ROWS;  // rows of a tile staged in smem (else read from global)
static_assert(kItems <= 32, "dup mask");
// padded smem index: threads own kItems consecutive positions, so a plain
// layout puts the lanes of a warp kItems words apart; one pad word per 32
// spreads them over the banks
__device__ __forceinline__ uint32_t OI(uint32_t p) { return p + (p >> 5); }
constexpr uint32_t kColWords = kTile + kTile / 32 + 1;
constexpr size_t kMergeSmem = size_t(kTile + 4 + kColWords) * 4 + size_t(2 * (kRowStage + 1)) * 2;
static_assert(kTile <= 65535, "16-bit local row offsets");
static_assert(2 * kThreads <= kTile, "duplicate scan words alias the staged columns");
#ifndef SPBLA_EW_LB
#define SPBLA_EW_LB 1
#endif
#ifndef SPBLA_EW_UNROLL
#define SPBLA_EW_UNROLL 1
#endif
constexpr int kLB = SPBLA_EW_LB;  // look-back statuses per lane per round trip
constexpr int kUnroll = SPBLA_EW_UNROLL;  // merge-loop copies
constexpr int kChunks = (kTile / 4 + 4 + kThreads - 1) / kThreads;  // 16-B staging chunks per thread
#ifndef SPBLA_EW_MINB
#define SPBLA_EW_MINB (1536 / SPBLA_EW_THREADS)  // 40 registers at 256 threads (8 blocks spill)
#endif
constexpr int kMinBlocks = SPBLA_EW_MINB;
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

// local offset of a row boundary v (global A or B position) in the tile's
// range [x0, x0 + n)
__device__ __forceinline__ uint32_t tile_seg(uint64_t v, uint64_t x0, uint32_t n) {
    return v <= x0 ? 0u : uint32_t(min(v - x0, uint64_t(n)));
}

// Step 2 of the merge kernel: the calling thread's kItems merged positions
// [k0, k1) into s_m; returns the duplicate mask (bit k: position k0 + k is a
// B item equal to the A item before it).  STAGED: the tile rows' local
// segment starts are in s_ra / s_rb, else they are read from global.
template <bool STAGED>
__device__ __forceinline__ uint32_t merge_thread(const MergeIn& m, const uint32_t* s_col, uint32_t* s_m,
                                                 const uint16_t* s_ra, const uint16_t* s_rb, uint32_t r0,
                                                 uint32_t nr, uint32_t na, uint32_t nb, uint32_t len,
                                                 uint64_t a0, uint64_t b0, uint64_t prev) {
    const uint32_t k0 = min(uint32_t(threadIdx.x) * kItems, len), k1 = min(k0 + kItems, len);
    if (k0 >= k1) return 0u;
    auto SA = [&](uint32_t i) -> uint32_t { return STAGED ? uint32_t(s_ra[i]) : tile_seg(m.rpa[r0 + i], a0, na); };
    auto SB = [&](uint32_t i) -> uint32_t { return STAGED ? uint32_t(s_rb[i]) : tile_seg(m.rpb[r0 + i], b0, nb); };
    // last tile row i in [lo, nr - 1] whose local merged start is <= p
    auto find_row = [&](uint32_t lo, uint32_t p) -> uint32_t {
        uint32_t hi = nr - 1;
        while (lo < hi) {
            const uint32_t mid = (lo + hi + 1) >> 1;
            if (SA(mid) + SB(mid) <= p) lo = mid; else hi = mid - 1;
        }
        return lo;
    };
    uint32_t i = find_row(0, k0);
    const uint32_t as = SA(i), bs = SB(i);
    uint32_t aend = SA(i + 1), bend = SB(i + 1);
    // merge-path split of local position k0 inside row i
    uint32_t lo = max(as, k0 > bend ? k0 - bend : 0u), hi = min(aend, k0 - bs);
    while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (s_col[mid] <= s_col[na + k0 - 1 - mid]) lo = mid + 1; else hi = mid;
    }
    uint32_t ai = lo, bi = k0 - lo;
    uint32_t nxt = aend + bend;
    // A duplicate B item directly follows its equal A item in the merge
    // (ties take A; rows are sorted and duplicate-free), so it is exactly an
    // item equal to the previous merged item of its row.  `last`: that item
    // (the row's last A item before k0 suffices: a B item before k0 is
    // smaller than every later B item); ~0 is no column (ncols < 2^32).
    uint32_t last = ai > as ? s_col[ai - 1] : (i == 0 ? uint32_t(prev) : ~0u);
    uint32_t va = s_col[ai], vb = s_col[na + bi];
    uint32_t dmask = 0;
#pragma unroll kUnroll
    for (uint32_t k = 0; k < k1 - k0; ++k) {
        const uint32_t pos = k0 + k;
        if (__builtin_expect(pos == nxt, 0)) {  // next non-empty row
            ++i;
            if (SA(i + 1) + SB(i + 1) <= pos) i = find_row(i + 1, pos);
            aend = SA(i + 1);
            bend = SB(i + 1);
            nxt = aend + bend;
            last = ~0u;
        }
        const bool takeA = ai < aend && (bi == bend || va <= vb);
        const uint32_t c = takeA ? va : vb;
        dmask |= uint32_t(c == last) << k;
        last = c;
        ai += takeA;
        bi += !takeA;
        const uint32_t nv = s_col[takeA ? ai : na + bi];
        va = takeA ? nv : va;
        vb = takeA ? vb : nv;
        s_m[OI(pos)] = c;
    }
    return dmask;
}

// One tile of kTile merged items per block (ticket order).  The tile's A
// range [a0, a1) and B range [b0, b1) (from the split kernel) are staged as
// columns; every thread then merges kItems consecutive merged positions
// sequentially, row by row: rows are the tile's per-row segments of A and B
// (local offsets staged in smem), the thread's first row and its merge-path
// split inside that row come from two binary searches, and a row change
// only moves the segment ends (the local merged start of row i is the sum
// of its A and B starts).  A B item is a duplicate iff it equals the last A
// item taken in its row (ties take A first; for the tile's first row the A
// item before the tile is tile_prev).  The merged columns go to smem at
// their merged positions; a tile with duplicates (block-uniform test) then
// closes the gaps in smem.  Kept counts: warp scans + one smem round; the
// tile's output base: decoupled look-back by warp 0; 16-B coalesced stores.
__global__ void __launch_bounds__(kThreads, kMinBlocks)
ewise_merge_kernel(MergeIn m, uint64_t ntiles, const uint32_t* __restrict__ tile_row,
                   const uint64_t* __restrict__ tile_a, const uint32_t* __restrict__ tile_rlo,
                   const uint64_t* __restrict__ tile_prev, uint64_t* status, uint32_t* ticket,
                   idx_t* __restrict__ out, off_t64* __restrict__ rowptr) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint32_t* s_col = reinterpret_cast<uint32_t*>(smem_raw);  // A cols [0, na), B cols [na, len) (+1 pad)
    uint32_t* s_m = s_col + (kTile + 4);                         // merged columns at [OI(pos)]
    uint16_t* s_ra = reinterpret_cast<uint16_t*>(s_m + kColWords);  // local A start of tile row i
    uint16_t* s_rb = s_ra + (kRowStage + 1);                         // local B start of tile row i
    uint32_t* s_tdup = s_col;            // (after the merge) duplicates before each thread
    uint32_t* s_dmask = s_col + kThreads;  // (after the merge) each thread's duplicate mask
    __shared__ uint32_t s_wdup[kThreads / 32];
    __shared__ uint32_t s_t;
    __shared__ uint64_t s_base;
    if (threadIdx.x == 0) s_t = atomicAdd(ticket, 1u);  // ticket order: the look-back never waits on a later block
    __syncthreads();
    const uint64_t t = s_t;
    const uint64_t d0 = t * kTile, d1 = min(d0 + kTile, m.L);
    const uint32_t len = uint32_t(d1 - d0);
    const uint64_t a0 = tile_a[t], a1 = tile_a[t + 1];
    const uint64_t b0 = d0 - a0, b1 = d1 - a1;
    const uint32_t na = uint32_t(a1 - a0), nb = uint32_t(b1 - b0);
    const uint32_t r0 = tile_row[t], r1 = min(tile_row[t + 1], m.nrows - 1);
    const uint32_t nr = r1 - r0 + 1;  // tile rows r0..r1; row nr's start is the tile end
    const uint64_t prev = tile_prev[t];
    uint32_t dmask;
    // 1. stage the columns as aligned 16-B chunks (A's chunks, then B's;
    //    all loads in flight before the first smem store) and the rows'
    //    local segment starts, clamped to the tile
    {
        const uintptr_t pa = reinterpret_cast<uintptr_t>(m.ca + a0), pb = reinterpret_cast<uintptr_t>(m.cb + b0);
        const uint4* ga = reinterpret_cast<const uint4*>(pa & ~uintptr_t(15));
        const uint4* gb = reinterpret_cast<const uint4*>(pb & ~uintptr_t(15));
        const uint32_t offa = uint32_t(pa & 15) >> 2, offb = uint32_t(pb & 15) >> 2;
        const uint32_t nca = na ? (offa + na + 3) >> 2 : 0u, ncb = nb ? (offb + nb + 3) >> 2 : 0u;
        uint4 cv[kChunks];
#pragma unroll
        for (int j = 0; j < kChunks; ++j) {
            const uint32_t c = j * kThreads + threadIdx.x;
            cv[j] = c < nca ? ga[c] : (c < nca + ncb ? gb[c - nca] : make_uint4(0, 0, 0, 0));
        }
#pragma unroll
        for (int j = 0; j < kChunks; ++j) {
            const uint32_t c = j * kThreads + threadIdx.x;
            if (c < nca + ncb) {
                const bool isa = c < nca;
                // smem position of the chunk's first word and the valid range
                const int32_t e = isa ? int32_t(4 * c) - int32_t(offa) : int32_t(na + 4 * (c - nca)) - int32_t(offb);
                const int32_t lo = isa ? 0 : int32_t(na), hi = isa ? int32_t(na) : int32_t(len);
                const uint32_t w[4] = {cv[j].x, cv[j].y, cv[j].z, cv[j].w};
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (e + q >= lo && e + q < hi) s_col[e + q] = w[q];
            }
        }
    }
    if (nr <= kRowStage) {
        for (uint32_t i = threadIdx.x; i <= nr; i += kThreads) {
            s_ra[i] = uint16_t(tile_seg(m.rpa[r0 + i], a0, na));
            s_rb[i] = uint16_t(tile_seg(m.rpb[r0 + i], b0, nb));
        }
        __syncthreads();
        dmask = merge_thread<true>(m, s_col, s_m, s_ra, s_rb, r0, nr, na, nb, len, a0, b0, prev);
    } else {  // (many empty or single-item rows: row starts read from global)
        __syncthreads();
        dmask = merge_thread<false>(m, s_col, s_m, s_ra, s_rb, r0, nr, na, nb, len, a0, b0, prev);
    }
    const uint32_t k0 = min(uint32_t(threadIdx.x) * kItems, len), k1 = min(k0 + kItems, len);
    // 3. duplicates before this thread (warp scan + one smem round); the
    //    tile's kept count
    const uint32_t ndup = __popc(dmask);
    uint32_t inc = ndup;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, d);
        if (int(lane_id()) >= d) inc += y;
    }
    if (lane_id() == 31) s_wdup[threadIdx.x >> 5] = inc;
    __syncthreads();
    uint32_t dex = inc - ndup, tdup = 0;
#pragma unroll
    for (int w = 0; w < kThreads / 32; ++w) {
        const uint32_t x = s_wdup[w];
        dex += w < int(threadIdx.x >> 5) ? x : 0u;
        tdup += x;
    }
    const uint64_t kept = len - tdup;
    if (tdup) {  // block-uniform: close the duplicates' gaps (kept items move left)
        s_tdup[threadIdx.x] = dex;
        s_dmask[threadIdx.x] = dmask;
        uint32_t v[kItems];
#pragma unroll
        for (int k = 0; k < kItems; ++k) v[k] = k0 + k < k1 ? s_m[OI(k0 + k)] : 0u;
        __syncthreads();
        uint32_t run = dex;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
            const uint32_t pos = k0 + k;
            if (pos < k1) {
                if ((dmask >> k) & 1u) ++run;
                else s_m[OI(pos - run)] = v[k];
            }
        }
    }
    // 4. decoupled look-back over the tiles' kept counts, one warp reading a
    //    window of 32 x kLB predecessors per round trip (lane l holds the
    //    l-th group of kLB, nearest first)
#ifdef SPBLA_EW_FAKE_LB  // timing experiment only: no look-back (wrong offsets)
    if (threadIdx.x == 0) s_base = d0;
    if (false) {
#else
    if (threadIdx.x < 32) {
#endif
        const unsigned lane = lane_id();
        uint64_t prefix = 0;
        if (t == 0) {
            if (lane == 0) st_relaxed(&status[0], kFlagPre | kept);
        } else {
            if (lane == 0) st_relaxed(&status[t], kFlagAgg | kept);
            for (long j = long(t) - 1;; j -= 32 * kLB) {
                uint64_t v[kLB];
#pragma unroll
                for (int q = 0; q < kLB; ++q) {
                    const long idx = j - long(lane) * kLB - q;
                    v[q] = idx >= 0 ? ld_relaxed(&status[idx]) : kFlagPre;
                }
                for (;;) {
                    bool wait = false;
#pragma unroll
                    for (int q = 0; q < kLB; ++q) wait |= (v[q] >> 62) == 0;
                    if (!__any_sync(0xffffffffu, wait)) break;
                    __nanosleep(32);
#pragma unroll
                    for (int q = 0; q < kLB; ++q)
                        if ((v[q] >> 62) == 0) v[q] = ld_relaxed(&status[j - long(lane) * kLB - q]);
                }
                // the lane's sum up to and including its first inclusive prefix
                int fq = kLB;
#pragma unroll
                for (int q = kLB - 1; q >= 0; --q)
                    if ((v[q] >> 62) == 2) fq = q;
                uint64_t lsum = 0;
#pragma unroll
                for (int q = 0; q < kLB; ++q) lsum += q <= fq ? (v[q] & kValMask) : 0ull;
                const uint32_t pre = __ballot_sync(0xffffffffu, fq < kLB);
                const int first = pre ? __ffs(pre) - 1 : 31;
                prefix += warp_sum(int(lane) <= first ? lsum : 0ull);
                if (pre) break;
            }
            if (lane == 0) st_relaxed(&status[t], kFlagPre | (prefix + kept));
        }
        if (lane == 0) s_base = prefix;
    }
    // the row offsets' inputs load while warp 0 looks back
    const uint32_t rlo = tile_rlo[t], rhi = (t + 1 == ntiles) ? m.nrows + 1 : tile_rlo[t + 1];
    const uint32_t rme = rlo + threadIdx.x;
    const uint32_t pme = rme < rhi ? uint32_t(P(m, rme) - d0) : 0u;
    __syncthreads();
    const uint64_t base = s_base;
    {
        // 16-B stores: a head of h words brings base + h to a 16-B boundary
        const uint32_t h = min(uint32_t((4 - (base & 3)) & 3), uint32_t(kept));
        if (threadIdx.x < h) out[base + threadIdx.x] = s_m[OI(threadIdx.x)];
        const uint32_t nv = (uint32_t(kept) - h) >> 2;
        uint4* o4 = reinterpret_cast<uint4*>(out + base + h);
        for (uint32_t v = threadIdx.x; v < nv; v += kThreads) {
            const uint32_t i = h + 4 * v;
            o4[v] = make_uint4(s_m[OI(i)], s_m[OI(i + 1)], s_m[OI(i + 2)], s_m[OI(i + 3)]);
        }
        for (uint32_t i = h + 4 * nv + threadIdx.x; i < kept; i += kThreads) out[base + i] = s_m[OI(i)];
    }
    // 5. row offsets of the rows starting in [d0, d1); the last tile also
    //    writes the rows starting at L (trailing empty rows, rowptr[nrows])
    for (uint32_t r = rme; r < rhi; r += kThreads) {
        const uint32_t p = r == rme ? pme : uint32_t(P(m, r) - d0);
        uint32_t dpre = tdup;
        if (p < len) {
            dpre = 0;
            if (tdup) {
                const uint32_t th = p / kItems, j = p % kItems;
                dpre = s_tdup[th] + __popc(s_dmask[th] & ((1u << j) - 1u));
            }
        }
        rowptr[r] = base + p - dpre;
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
