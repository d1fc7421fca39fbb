// Row engine: per output row, the sorted duplicate-free union of a list of
// column segments, written as CSR.  This is the Gustavson row step of
// Boolean SpGEMM (§III-A l.259-264: nsparse-style row-wise SpGEMM;
// for the Boolean semiring the symbolic phase IS the numeric phase, so there
// is no value array), and the per-row sort+dedup that Build and Transpose
// need.  DESIGN.md §4.2 describes the binning and each kernel's roofline.
//
// Pipeline (all on the device; two host read-backs for allocation sizes):
//   1. bin_count   : cap[r] = min(ub[r], ncols), bin[r] by ub, bin histogram
//   2. scan(cap)   : scratch offsets (in-house decoupled look-back scan)
//   3. bin_scatter : row lists per bin
//   4. per-bin kernels, forked over 4 streams:
//        warp bitonic (ub <= 32*E, E = 1..16): flattened gather into smem,
//            register bitonic sort, shuffle dedup
//        block hash (ub <= 2048 / 8192): if the row's column span fits the
//            table as a bitmap -> smem bitmap (atomicOr); else an
//            ORDER-PRESERVING smem hash (home slot monotone in the column,
//            linear probing without wrap-around) whose clusters are the
//            only unsorted runs -> per-cluster insertion sort -> the table
//            is sorted; rows whose probes run long go to the bitmap bin
//        block bitmap (heavier rows): smem bitmap over the row's column
//            span in windows of <= 2^20 bits, atomicOr inserts
//      every block kernel gathers products "flattened": 32 segment
//      descriptors per warp, lanes spread over their concatenation (shuffle
//      binary search), 4 independent loads in flight per lane; emission is
//      warp-chunked ballot/popc so stores are coalesced and in order.
//   5. scan(counts): CSR row offsets
//   6. compact     : scratch -> colidx
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

constexpr unsigned FULL = 0xffffffffu;
constexpr int kNumBins = 9;
enum { BIN_EMPTY = 0, BIN_W1 = 1, BIN_W2, BIN_W4, BIN_W8, BIN_W16, BIN_HASH_S = 6, BIN_HASH_L = 7, BIN_DENSE = 8 };
constexpr uint64_t kWarpMaxUb = kRangeMinUb;
constexpr uint64_t kHashSMaxUb = 2048;     // table <= 4096 slots
constexpr uint64_t kHashLMaxUb = 8192;     // table <= 16384 slots
constexpr int kHashSThreads = 256;
constexpr int kHashLThreads = 512;
constexpr uint32_t kSlack = 128;           // overflow slots past T (no wrap-around)
constexpr uint32_t kMaxProbe = 96;
constexpr int kDenseThreads = 1024;
constexpr uint32_t kDenseMaxBits = 1u << 20;  // 128 KB smem bitmap window
constexpr int kUnroll = 4;
constexpr uint32_t kHashSBatch = 1024;
constexpr uint32_t kHashLBatch = 640;
constexpr uint32_t kDenseBatch = 4096;

__device__ __forceinline__ int bin_of(uint64_t ub) {
    if (ub == 0) return BIN_EMPTY;
    if (ub <= 32) return BIN_W1;
    if (ub <= 64) return BIN_W2;
    if (ub <= 128) return BIN_W4;
    if (ub <= 256) return BIN_W8;
    if (ub <= kWarpMaxUb) return BIN_W16;
    if (ub <= kHashSMaxUb) return BIN_HASH_S;
    if (ub <= kHashLMaxUb) return BIN_HASH_L;
    return BIN_DENSE;
}

// ---- segment access --------------------------------------------------------
__device__ __forceinline__ uint32_t num_segs(const SegSource& s, idx_t r) {
    if (s.kind == 1) return 1;
    return uint32_t(s.arp[r + 1] - s.arp[r]) + (s.crp ? 1u : 0u);
}

__device__ __forceinline__ const idx_t* get_seg(const SegSource& s, idx_t r, uint32_t j, uint32_t& len) {
    if (s.kind == 1) {
        off_t64 b = s.lrp[r];
        len = uint32_t(s.lrp[r + 1] - b);
        return s.lst + b;
    }
    if (s.crp) {
        if (j == 0) {
            off_t64 b = s.crp[r];
            len = uint32_t(s.crp[r + 1] - b);
            return s.cci + b;
        }
        --j;
    }
    idx_t k = s.aci[s.arp[r] + j];
    off_t64 b = s.brp[k];
    len = uint32_t(s.brp[k + 1] - b);
    return s.bci + b;
}

// Flattened warp gather: every lane holds one segment (p, len); the warp
// walks the concatenation of the 32 segments with all lanes busy and
// kUnroll independent loads in flight per lane, calling f(q, c) for the
// element c at concatenated position q.  Returns the total length.
template <typename F>
__device__ __forceinline__ uint32_t warp_flat(const idx_t* p, uint32_t len, F&& f) {
    const unsigned lane = lane_id();
    const uint32_t inc = warp_inclusive_scan(len);
    const uint32_t tot = __shfl_sync(FULL, inc, 31);
    const uint32_t exc = inc - len;
    const unsigned long long pp = (unsigned long long)p;
    for (uint32_t q0 = 0; q0 < tot; q0 += 32 * kUnroll) {
        idx_t v[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
            const uint32_t q = q0 + u * 32 + lane;
            uint32_t pos = 0;  // number of lanes whose inclusive end <= q
#pragma unroll
            for (int st = 16; st > 0; st >>= 1) {
                uint32_t t = __shfl_sync(FULL, inc, pos + st - 1);
                if (t <= q) pos += st;
            }
            const uint32_t sl = pos > 31 ? 31 : pos;
            const idx_t* ps = (const idx_t*)__shfl_sync(FULL, pp, sl);
            const uint32_t es = __shfl_sync(FULL, exc, sl);
            v[u] = q < tot ? __ldg(ps + (q - es)) : kEmpty;
        }
#pragma unroll
        for (int u = 0; u < kUnroll; ++u)
            if (v[u] != kEmpty) f(q0 + u * 32 + lane, v[u]);
    }
    return tot;
}

// Block-flattened gather of all products of row r:
// segment descriptors (pointer, inclusive end) are staged in smem in batches
// of `batch`; a block scan gives the concatenated positions; then every
// thread takes products q = tid, tid + THREADS, ... (consecutive lanes ->
// consecutive addresses), finds its segment by binary search in smem and
// keeps kFlatUnroll independent loads in flight.  All warps get equal work
// whatever the segment-length skew.
constexpr int kFlatUnroll = 8;
template <int THREADS, typename F>
__device__ __forceinline__ void block_flat(const SegSource& s, idx_t r, const idx_t** sd_ptr, uint32_t* sd_end,
                                           uint32_t batch, uint64_t* s_scan, F&& f) {
    const uint32_t nseg = num_segs(s, r);
    for (uint32_t s0 = 0; s0 < nseg; s0 += batch) {
        const uint32_t n = min(batch, nseg - s0);
        const uint32_t per = (n + THREADS - 1) / THREADS;
        const uint32_t b = threadIdx.x * per, e = min(b + per, n);
        uint64_t sum = 0;
        for (uint32_t i = b; i < e; ++i) {
            uint32_t len;
            sd_ptr[i] = get_seg(s, r, s0 + i, len);
            sd_end[i] = len;  // temporarily the length
            sum += len;
        }
        uint64_t tot;
        uint64_t run = block_exclusive_scan<uint64_t>(sum, s_scan, &tot);
        for (uint32_t i = b; i < e; ++i) {
            run += sd_end[i];
            sd_end[i] = uint32_t(run);
        }
        __syncthreads();
        const uint32_t total = uint32_t(tot);
        for (uint32_t q0 = threadIdx.x; q0 < total; q0 += THREADS * kFlatUnroll) {
            idx_t v[kFlatUnroll];
#pragma unroll
            for (int u = 0; u < kFlatUnroll; ++u) {
                const uint32_t q = q0 + u * THREADS;
                v[u] = kEmpty;
                if (q < total) {
                    uint32_t lo = 0, hi = n - 1;  // first segment whose end > q
                    while (lo < hi) {
                        const uint32_t mid = (lo + hi) >> 1;
                        if (sd_end[mid] <= q) lo = mid + 1; else hi = mid;
                    }
                    const uint32_t st = lo ? sd_end[lo - 1] : 0u;
                    v[u] = __ldg(sd_ptr[lo] + (q - st));
                }
            }
#pragma unroll
            for (int u = 0; u < kFlatUnroll; ++u)
                if (v[u] != kEmpty) f(v[u]);
        }
        __syncthreads();  // smem descriptors are reused by the next batch
    }
}

// Ordered, coalesced emission of the set bits of bm[0..nwords) as columns
// base_col + 32*i + b.  Warp w owns a contiguous run of words; one block scan
// of the per-warp counts.  Returns the count (all threads).
__device__ __forceinline__ uint32_t emit_bitmap(const uint32_t* bm, uint32_t nwords, uint64_t base_col,
                                                idx_t* __restrict__ out, uint32_t* s_w) {
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const uint32_t chunk = ((nwords + nw - 1) / nw + 31) & ~31u;
    const uint32_t b = wib * chunk, e = min(b + chunk, nwords);
    uint32_t cnt = 0;
    for (uint32_t i = b + lane; i < e; i += 32) cnt += __popc(bm[i]);
    cnt = warp_sum(cnt);
    if (lane == 0) s_w[wib] = cnt;
    __syncthreads();
    if (wib == 0) {
        uint32_t v = lane < nw ? s_w[lane] : 0u;
        uint32_t inc = warp_inclusive_scan(v);
        if (lane < nw) s_w[lane] = inc - v;
        if (lane == nw - 1) s_w[32] = inc;
    }
    __syncthreads();
    uint32_t pos = s_w[wib];
    for (uint32_t i0 = b; i0 < e; i0 += 32) {
        const uint32_t i = i0 + lane;
        uint32_t word = i < e ? bm[i] : 0u;
        const uint32_t c = __popc(word);
        const uint32_t inc = warp_inclusive_scan(c);
        uint32_t o = pos + inc - c;
        while (word) {
            const int bit = __ffs(word) - 1;
            word &= word - 1;
            out[o++] = idx_t(base_col + (uint64_t(i) << 5) + bit);
        }
        pos += __shfl_sync(FULL, inc, 31);
    }
    const uint32_t total = s_w[32];
    __syncthreads();
    return total;
}

// Ordered, coalesced emission of an order-preserving hash table: clusters
// (maximal runs of occupied slots) are ordered relative to each other, so an
// element at slot i goes to  (#occupied slots before its cluster start cs)
// + (its rank inside the cluster)  — no in-smem sort, no extra barrier.
__device__ __forceinline__ uint32_t emit_table_ranked(const idx_t* tab, uint32_t nslots, idx_t* __restrict__ out,
                                                      uint32_t* s_w) {
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const uint32_t chunk = ((nslots + nw - 1) / nw + 31) & ~31u;
    const uint32_t b = wib * chunk, e = min(b + chunk, nslots);
    uint32_t cnt = 0;
    for (uint32_t i0 = b; i0 < e; i0 += 32) {
        const uint32_t i = i0 + lane;
        cnt += __popc(__ballot_sync(FULL, i < e && tab[i] != kEmpty));
    }
    if (lane == 0) s_w[wib] = cnt;
    __syncthreads();
    if (wib == 0) {
        uint32_t v = lane < nw ? s_w[lane] : 0u;
        uint32_t inc = warp_inclusive_scan(v);
        if (lane < nw) s_w[lane] = inc - v;
        if (lane == nw - 1) s_w[32] = inc;
    }
    __syncthreads();
    uint32_t pos = s_w[wib];
    const uint32_t lt = (1u << lane) - 1u;
    for (uint32_t i0 = b; i0 < e; i0 += 32) {
        const uint32_t i = i0 + lane;
        const idx_t v = i < e ? tab[i] : kEmpty;
        const uint32_t m = __ballot_sync(FULL, v != kEmpty);
        if (v != kEmpty) {
            uint32_t cs = i;
            while (cs > 0 && tab[cs - 1] != kEmpty) --cs;
            uint32_t rank = 0;
            for (uint32_t j = cs; j < nslots; ++j) {
                const idx_t w = tab[j];
                if (w == kEmpty) break;
                rank += (w < v);
            }
            out[pos + __popc(m & lt) - (i - cs) + rank] = v;
        }
        pos += __popc(m);
    }
    const uint32_t total = s_w[32];
    __syncthreads();
    return total;
}

// ---- 1. binning ------------------------------------------------------------
__global__ void bin_count_kernel(const uint64_t* __restrict__ ub, idx_t nrows, idx_t ncols,
                                 uint64_t* __restrict__ cap, uint8_t* __restrict__ bin,
                                 uint32_t* __restrict__ counts, uint32_t* __restrict__ hist) {
    __shared__ uint32_t sh[kNumBins];
    if (threadIdx.x < kNumBins) sh[threadIdx.x] = 0;
    __syncthreads();
    for (size_t r = blockIdx.x * size_t(blockDim.x) + threadIdx.x; r < nrows;
         r += size_t(gridDim.x) * blockDim.x) {
        uint64_t u = ub[r];
        cap[r] = u < ncols ? u : uint64_t(ncols);
        int b = bin_of(u);
        bin[r] = uint8_t(b);
        if (b == BIN_EMPTY) counts[r] = 0;
        atomicAdd(&sh[b], 1u);
    }
    __syncthreads();
    if (threadIdx.x < kNumBins && sh[threadIdx.x]) atomicAdd(&hist[threadIdx.x], sh[threadIdx.x]);
}

// hist[0..9) -> binoff[0..10) (tiny)
__global__ void bin_offsets_kernel(const uint32_t* hist, uint32_t* binoff, uint32_t* cursor) {
    if (threadIdx.x == 0) {
        uint32_t s = 0;
        for (int b = 0; b < kNumBins; ++b) {
            binoff[b] = s;
            cursor[b] = s;
            s += hist[b];
        }
        binoff[kNumBins] = s;
    }
}

__global__ void bin_scatter_kernel(const uint8_t* __restrict__ bin, idx_t nrows,
                                   uint32_t* __restrict__ cursor, idx_t* __restrict__ rows) {
    __shared__ uint32_t sh_cnt[kNumBins], sh_base[kNumBins];
    const size_t stride = size_t(gridDim.x) * blockDim.x;
    for (size_t r0 = blockIdx.x * size_t(blockDim.x); r0 < nrows; r0 += stride) {
        if (threadIdx.x < kNumBins) sh_cnt[threadIdx.x] = 0;
        __syncthreads();
        size_t r = r0 + threadIdx.x;
        int b = -1;
        uint32_t local = 0;
        if (r < nrows) {
            b = bin[r];
            if (b != BIN_EMPTY) local = atomicAdd(&sh_cnt[b], 1u);
        }
        __syncthreads();
        if (threadIdx.x < kNumBins && sh_cnt[threadIdx.x])
            sh_base[threadIdx.x] = atomicAdd(&cursor[threadIdx.x], sh_cnt[threadIdx.x]);
        __syncthreads();
        if (b > 0) rows[sh_base[b] + local] = idx_t(r);
        __syncthreads();
    }
}

// ---- 4a. warp bitonic bins -------------------------------------------------
template <int E>
__device__ __forceinline__ void warp_bitonic_sort(idx_t (&x)[E]) {
    const unsigned lane = lane_id();
    constexpr int N = 32 * E;
#pragma unroll
    for (int k = 2; k <= N; k <<= 1) {
#pragma unroll
        for (int j = k >> 1; j > 0; j >>= 1) {
            if (j < E) {
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    if ((e & j) == 0) {
                        int i = int(lane) * E + e;
                        bool asc = (i & k) == 0;
                        idx_t a = x[e], b = x[e | j];
                        bool sw = asc ? (a > b) : (a < b);
                        x[e] = sw ? b : a;
                        x[e | j] = sw ? a : b;
                    }
                }
            } else {
                const int lj = j / E;
#pragma unroll
                for (int e = 0; e < E; ++e) {
                    int i = int(lane) * E + e;
                    idx_t o = __shfl_xor_sync(FULL, x[e], lj);
                    bool lower = (i & j) == 0;
                    bool asc = (i & k) == 0;
                    x[e] = (lower == asc) ? min(x[e], o) : max(x[e], o);
                }
            }
        }
    }
}

template <int E>
__global__ void __launch_bounds__(256)
warp_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ binoff,
                int bin, idx_t* __restrict__ scratch, const uint64_t* __restrict__ soff,
                uint32_t* __restrict__ counts) {
    __shared__ idx_t sbuf[8][32 * E];
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5;
    idx_t* buf = sbuf[wib];
    const uint32_t lo = binoff[bin], hi = binoff[bin + 1];
    const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
    for (uint32_t t = lo + blockIdx.x * (blockDim.x >> 5) + wib; t < hi; t += nwarps) {
        const idx_t r = rows[t];
        const uint32_t nseg = num_segs(src, r);
        uint32_t n = 0;
        for (uint32_t base = 0; base < nseg; base += 32) {
            const uint32_t j = base + lane;
            uint32_t len = 0;
            const idx_t* p = nullptr;
            if (j < nseg) p = get_seg(src, r, j, len);
            n += warp_flat(p, len, [&](uint32_t q, idx_t c) { buf[n + q] = c; });
        }
        __syncwarp();
        idx_t x[E];
#pragma unroll
        for (int e = 0; e < E; ++e) {
            uint32_t i = lane * E + e;
            x[e] = i < n ? buf[i] : kEmpty;
        }
        __syncwarp();
        warp_bitonic_sort<E>(x);
        idx_t prev_last = __shfl_up_sync(FULL, x[E - 1], 1);
        uint32_t keep = 0;
        bool uniq[E];
#pragma unroll
        for (int e = 0; e < E; ++e) {
            idx_t pv = e == 0 ? prev_last : x[e - 1];
            bool first = (e == 0 && lane == 0);
            uniq[e] = x[e] != kEmpty && (first || x[e] != pv);
            keep += uniq[e];
        }
        uint32_t inc = warp_inclusive_scan(keep);
        uint32_t o = inc - keep;
        idx_t* out = scratch + soff[r];
#pragma unroll
        for (int e = 0; e < E; ++e)
            if (uniq[e]) out[o++] = x[e];
        if (lane == 31) counts[r] = inc;
    }
}

// ---- 4b. block hash / small-span bitmap bins -------------------------------
__device__ __forceinline__ uint32_t next_pow2(uint32_t v) {
    return v <= 1 ? 1u : 1u << (32 - __clz(v - 1));
}

// dynamic smem: table[TMAX + kSlack] | sd_ptr[BATCH] | sd_end[BATCH]
template <int THREADS, uint32_t TMAX, uint32_t BATCH>
__global__ void __launch_bounds__(THREADS)
hash_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ bounds,
                const uint64_t* __restrict__ ub, const uint2* __restrict__ range, idx_t ncols,
                idx_t* __restrict__ scratch, const uint64_t* __restrict__ soff, uint32_t* __restrict__ counts,
                uint32_t* __restrict__ work, idx_t* __restrict__ ovf_rows, uint32_t* __restrict__ ovf_cnt) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const idx_t** sd_ptr = reinterpret_cast<const idx_t**>(smem_raw);
    uint32_t* sd_end = reinterpret_cast<uint32_t*>(smem_raw + BATCH * sizeof(void*));
    idx_t* tab = reinterpret_cast<idx_t*>(smem_raw + BATCH * (sizeof(void*) + sizeof(uint32_t)));
    __shared__ uint64_t s_scan[33];
    __shared__ uint32_t s_w[33];
    __shared__ uint32_t s_item, s_flag;
    const uint32_t lo_i = bounds[0], hi_i = bounds[1];
    for (;;) {
        if (threadIdx.x == 0) {
            s_item = lo_i + atomicAdd(work, 1u);
            s_flag = 0;
        }
        __syncthreads();
        const uint32_t item = s_item;
        if (item >= hi_i) break;
        const idx_t r = rows[item];
        const uint32_t u = uint32_t(ub[r]);
        uint32_t clo = 0, chi = ncols - 1;
        if (range) {
            uint2 rg = range[r];
            clo = rg.x;
            chi = rg.y;
        }
        const uint64_t span = uint64_t(chi) - clo + 1;
        const uint32_t T = min(next_pow2(2 * u), TMAX);
        const uint64_t words = (span + 31) >> 5;
        const bool bitmap = words <= T;
        const uint32_t nslots = bitmap ? uint32_t(words) : T + kSlack;
        const idx_t fill = bitmap ? 0u : kEmpty;
        for (uint32_t i = threadIdx.x; i < nslots; i += THREADS) tab[i] = fill;
        __syncthreads();
        if (bitmap) {
            block_flat<THREADS>(src, r, sd_ptr, sd_end, BATCH, s_scan, [&](idx_t c) {
                const uint32_t d = c - clo;
                atomicOr(&tab[d >> 5], 1u << (d & 31));
            });
            const uint32_t n = emit_bitmap(tab, nslots, clo, scratch + soff[r], s_w);
            if (threadIdx.x == 0) counts[r] = n;
            continue;  // emit_bitmap ends with a barrier
        }
        // order-preserving home slot: floor((c - clo) * T / span) via a
        // 32.32 fixed-point scale; monotone in c and < T
        const uint64_t scale = (uint64_t(T) << 32) / span;
        block_flat<THREADS>(src, r, sd_ptr, sd_end, BATCH, s_scan, [&](idx_t c) {
            uint32_t h = uint32_t((uint64_t(c - clo) * scale) >> 32);
            for (uint32_t probe = 0;; ++probe) {
                const idx_t cur = tab[h];
                if (cur == c) break;
                if (cur == kEmpty) {
                    const idx_t old = atomicCAS(&tab[h], kEmpty, c);
                    if (old == kEmpty || old == c) break;
                }
                if (++h >= nslots || probe >= kMaxProbe) {
                    s_flag = 1;  // long cluster: hand the row to the bitmap bin
                    break;
                }
            }
        });
        // block_flat ends with a barrier
        if (s_flag) {
            if (threadIdx.x == 0) ovf_rows[atomicAdd(ovf_cnt + 1, 1u)] = r;
            __syncthreads();  // everyone has read s_flag / s_item before reuse
            continue;
        }
        const uint32_t n = emit_table_ranked(tab, nslots, scratch + soff[r], s_w);
        if (threadIdx.x == 0) counts[r] = n;
    }
}

// ---- 4c. block bitmap bin ----------------------------------------------------
// dynamic smem: bitmap[kDenseMaxBits/32] | sd_ptr[kDenseBatch] | sd_end[kDenseBatch]
__global__ void __launch_bounds__(kDenseThreads)
dense_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ bounds,
                 const uint2* __restrict__ range, idx_t ncols, idx_t* __restrict__ scratch,
                 const uint64_t* __restrict__ soff, uint32_t* __restrict__ counts, uint32_t* __restrict__ work) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const idx_t** sd_ptr = reinterpret_cast<const idx_t**>(smem_raw);
    uint32_t* sd_end = reinterpret_cast<uint32_t*>(smem_raw + kDenseBatch * sizeof(void*));
    uint32_t* bm = reinterpret_cast<uint32_t*>(smem_raw + kDenseBatch * (sizeof(void*) + sizeof(uint32_t)));
    __shared__ uint64_t s_scan[33];
    __shared__ uint32_t s_w[33];
    __shared__ uint32_t s_item;
    for (;;) {
        if (threadIdx.x == 0) s_item = bounds[0] + atomicAdd(work, 1u);
        __syncthreads();
        const uint32_t item = s_item;
        if (item >= bounds[1]) break;
        const idx_t r = rows[item];
        uint32_t clo = 0, chi = ncols - 1;
        if (range) {
            uint2 rg = range[r];
            clo = rg.x;
            chi = rg.y;
        }
        const uint64_t span = uint64_t(chi) - clo + 1;
        const uint32_t nwin = uint32_t((span + kDenseMaxBits - 1) / kDenseMaxBits);
        idx_t* out = scratch + soff[r];
        uint32_t written = 0;
        for (uint32_t w = 0; w < nwin; ++w) {
            const uint64_t wlo = uint64_t(clo) + uint64_t(w) * kDenseMaxBits;
            const uint64_t whi = min(wlo + kDenseMaxBits, uint64_t(chi) + 1);
            const uint32_t nwords = uint32_t((whi - wlo + 31) >> 5);
            for (uint32_t i = threadIdx.x; i < nwords; i += blockDim.x) bm[i] = 0;
            __syncthreads();
            block_flat<kDenseThreads>(src, r, sd_ptr, sd_end, kDenseBatch, s_scan, [&](idx_t c) {
                if (c >= wlo && c < whi) {
                    const uint32_t d = uint32_t(c - wlo);
                    atomicOr(&bm[d >> 5], 1u << (d & 31));
                }
            });
            written += emit_bitmap(bm, nwords, wlo, out + written, s_w);
        }
        if (threadIdx.x == 0) counts[r] = written;
    }
}

// ---- 6. compaction -------------------------------------------------------------
__global__ void compact_kernel(const idx_t* __restrict__ scratch, const uint64_t* __restrict__ soff,
                               const uint64_t* __restrict__ rowptr, idx_t nrows,
                               idx_t* __restrict__ colidx) {
    const unsigned lane = lane_id();
    const size_t nwarps = size_t(gridDim.x) * (blockDim.x >> 5);
    for (size_t r = (blockIdx.x * size_t(blockDim.x) + threadIdx.x) >> 5; r < nrows; r += nwarps) {
        const uint64_t b = rowptr[r], n = rowptr[r + 1] - b;
        const idx_t* s = scratch + soff[r];
        idx_t* d = colidx + b;
        for (uint64_t t = lane; t < n; t += 32) d[t] = s[t];
    }
}

}  // namespace

// ------------------------------------------------------------------------------
struct AuxStreams {
    cudaStream_t s[3] = {nullptr, nullptr, nullptr};
    cudaEvent_t fork = nullptr, join[3] = {nullptr, nullptr, nullptr};
    int device = -1;
};
static AuxStreams g_aux;

constexpr size_t kSegBytes = sizeof(void*) + sizeof(uint32_t);
constexpr size_t kHashSSmem = (2 * kHashSMaxUb + kSlack) * sizeof(idx_t) + kHashSBatch * kSegBytes;
constexpr size_t kHashLSmem = (2 * kHashLMaxUb + kSlack) * sizeof(idx_t) + kHashLBatch * kSegBytes;
constexpr size_t kDenseSmem = kDenseMaxBits / 8 + kDenseBatch * kSegBytes;
#define HASH_S hash_bin_kernel<kHashSThreads, 2 * kHashSMaxUb, kHashSBatch>
#define HASH_L hash_bin_kernel<kHashLThreads, 2 * kHashLMaxUb, kHashLBatch>

static void ensure_aux() {
    if (g_aux.device == ctx().device) return;
    for (int i = 0; i < 3; ++i) {
        CUDA_CHECK(cudaStreamCreateWithFlags(&g_aux.s[i], cudaStreamNonBlocking));
        CUDA_CHECK(cudaEventCreateWithFlags(&g_aux.join[i], cudaEventDisableTiming));
    }
    CUDA_CHECK(cudaEventCreateWithFlags(&g_aux.fork, cudaEventDisableTiming));
    CUDA_CHECK(cudaFuncSetAttribute(HASH_S, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kHashSSmem)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH_L, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kHashLSmem)));
    CUDA_CHECK(cudaFuncSetAttribute(dense_bin_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kDenseSmem)));
    g_aux.device = ctx().device;
}

void row_engine(const SegSource& src, idx_t nrows, idx_t ncols, const uint64_t* ub, const uint2* range,
                Matrix* out) {
    cudaStream_t st = ctx().stream;
    const int nsm = ctx().num_sms;
    if (nrows == 0 || ncols == 0) {
        matrix_set_empty(out);
        return;
    }
    ensure_aux();
    // 1. bins
    DevBuf<uint64_t> cap(size_t(nrows) + 1);
    DevBuf<uint64_t> soff(size_t(nrows) + 1);
    DevBuf<uint8_t> bin(nrows);
    DevBuf<uint32_t> counts(nrows);
    // meta: hist[9] binoff[10] cursor[9] work[4] ovf[2]
    DevBuf<uint32_t> meta(64);
    uint32_t* hist = meta.p;
    uint32_t* binoff = meta.p + 10;
    uint32_t* cursor = meta.p + 21;
    uint32_t* work = meta.p + 31;
    uint32_t* ovf = meta.p + 36;  // ovf[0] = 0 (list start), ovf[1] = count
    memset_async(meta.p, 0, meta.n * sizeof(uint32_t));
    const unsigned gb = (unsigned)std::min<uint64_t>(ceil_div(nrows, 256), uint64_t(nsm) * 8);
    bin_count_kernel<<<gb, 256, 0, st>>>(ub, nrows, ncols, cap.p, bin.p, counts.p, hist);
    count_launch();
    check_launch("bin_count_kernel");
    exclusive_scan_u64(cap.p, soff.p, nrows);
    bin_offsets_kernel<<<1, 32, 0, st>>>(hist, binoff, cursor);
    count_launch();
    DevBuf<idx_t> rows(nrows);
    bin_scatter_kernel<<<gb, 256, 0, st>>>(bin.p, nrows, cursor, rows.p);
    count_launch();
    check_launch("bin_scatter_kernel");
    uint64_t h[2];
    read_words(soff.p + nrows, h, 1);
    const uint64_t scratch_total = h[0];
    cap.release();
    bin.release();
    DevBuf<idx_t> scratch(scratch_total);
    DevBuf<idx_t> ovf_rows(nrows);

    // 4. per-bin kernels on forked streams
    CUDA_CHECK(cudaEventRecord(g_aux.fork, st));
    for (int i = 0; i < 3; ++i) CUDA_CHECK(cudaStreamWaitEvent(g_aux.s[i], g_aux.fork, 0));
    const unsigned gw = nsm * 8;  // 256-thread blocks, grid-stride over bin rows
    {
        cudaStream_t s3 = g_aux.s[2];  // heaviest first
        dense_bin_kernel<<<nsm, kDenseThreads, kDenseSmem, s3>>>(
            src, rows.p, binoff + BIN_DENSE, range, ncols, scratch.p, soff.p, counts.p, work);
        count_launch();
        check_launch("dense_bin_kernel");
        cudaStream_t s2 = g_aux.s[1];
        HASH_L<<<nsm * 3, kHashLThreads, kHashLSmem, s2>>>(
            src, rows.p, binoff + BIN_HASH_L, ub, range, ncols, scratch.p, soff.p, counts.p, work + 1,
            ovf_rows.p, ovf);
        HASH_S<<<nsm * 7, kHashSThreads, kHashSSmem, s2>>>(
            src, rows.p, binoff + BIN_HASH_S, ub, range, ncols, scratch.p, soff.p, counts.p, work + 2,
            ovf_rows.p, ovf);
        // rows whose hash probes ran long: bitmap path
        dense_bin_kernel<<<nsm, kDenseThreads, kDenseSmem, s2>>>(
            src, ovf_rows.p, ovf, range, ncols, scratch.p, soff.p, counts.p, work + 3);
        count_launch(3);
        check_launch("hash_bin_kernel");
        cudaStream_t s1 = g_aux.s[0];
        warp_bin_kernel<16><<<gw, 256, 0, s1>>>(src, rows.p, binoff, BIN_W16, scratch.p, soff.p, counts.p);
        warp_bin_kernel<8><<<gw, 256, 0, s1>>>(src, rows.p, binoff, BIN_W8, scratch.p, soff.p, counts.p);
        warp_bin_kernel<4><<<gw, 256, 0, st>>>(src, rows.p, binoff, BIN_W4, scratch.p, soff.p, counts.p);
        warp_bin_kernel<2><<<gw, 256, 0, st>>>(src, rows.p, binoff, BIN_W2, scratch.p, soff.p, counts.p);
        warp_bin_kernel<1><<<gw, 256, 0, st>>>(src, rows.p, binoff, BIN_W1, scratch.p, soff.p, counts.p);
        count_launch(5);
        check_launch("warp_bin_kernel");
    }
    for (int i = 0; i < 3; ++i) {
        CUDA_CHECK(cudaEventRecord(g_aux.join[i], g_aux.s[i]));
        CUDA_CHECK(cudaStreamWaitEvent(st, g_aux.join[i], 0));
    }
    // 5. row offsets
    DevBuf<off_t64> rowptr(size_t(nrows) + 1);
    exclusive_scan_u32(counts.p, rowptr.p, nrows);
    read_words(rowptr.p + nrows, h, 1);
    const uint64_t nnz = h[0];
    DevBuf<idx_t> colidx(nnz);
    if (nnz) {
        const unsigned gc = (unsigned)std::min<uint64_t>(ceil_div(uint64_t(nrows) * 32, 256), uint64_t(nsm) * 16);
        compact_kernel<<<gc, 256, 0, st>>>(scratch.p, soff.p, rowptr.p, nrows, colidx.p);
        count_launch();
        check_launch("compact_kernel");
    }
    size_t rcap = rowptr.n, ccap = colidx.n;
    matrix_replace(out, rowptr.detach(), rcap, colidx.detach(), ccap, nnz);
}

}  // namespace spbla
