// Row engine: per output row, the sorted duplicate-free union of a list of
// sorted column segments, written as CSR.  This is the Gustavson row step of
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
//        warp bitonic (ub <= 32*E, E = 1..16): gather into smem, register
//            bitonic sort, ballot/shuffle dedup
//        block hash (ub <= kHashMaxUb): smem linear-probe hash, in-place
//            compaction, smem bitonic sort
//        block bitmap (heavier rows): smem bitmap per column window,
//            atomicOr inserts, popc/scan emission — sorted by construction
//   5. scan(counts): CSR row offsets
//   6. compact     : scratch -> colidx
#include "common.cuh"

#include <algorithm>

namespace spbla {

namespace {

constexpr int kNumBins = 8;
enum { BIN_EMPTY = 0, BIN_W1 = 1, BIN_W2, BIN_W4, BIN_W8, BIN_W16, BIN_HASH = 6, BIN_DENSE = 7 };
constexpr uint64_t kHashMaxUb = 8192;      // table <= 16384 slots (64 KB smem)
constexpr int kHashThreads = 512;
constexpr int kDenseThreads = 1024;
constexpr uint32_t kDenseMaxBits = 1u << 20; // 128 KB smem bitmap window

__device__ __forceinline__ int bin_of(uint64_t ub) {
    if (ub == 0) return BIN_EMPTY;
    if (ub <= 32) return BIN_W1;
    if (ub <= 64) return BIN_W2;
    if (ub <= 128) return BIN_W4;
    if (ub <= 256) return BIN_W8;
    if (ub <= 512) return BIN_W16;
    if (ub <= kHashMaxUb) return BIN_HASH;
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

// hist[0..8) -> binoff[0..9) (tiny)
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
// Gather all segments of row r into the warp's smem buffer; returns the count.
__device__ __forceinline__ uint32_t warp_gather(const SegSource& s, idx_t r, idx_t* buf) {
    const unsigned lane = lane_id();
    const uint32_t nseg = num_segs(s, r);
    uint32_t pos = 0;
    for (uint32_t base = 0; base < nseg; base += 32) {
        uint32_t j = base + lane;
        uint32_t len = 0;
        const idx_t* p = nullptr;
        if (j < nseg) p = get_seg(s, r, j, len);
        uint32_t inc = warp_inclusive_scan(len);
        uint32_t off = pos + inc - len;
        uint32_t tot = __shfl_sync(0xffffffffu, inc, 31);
        uint32_t nj = min(32u, nseg - base);
        for (uint32_t q = 0; q < nj; ++q) {
            const idx_t* pq = (const idx_t*)__shfl_sync(0xffffffffu, (unsigned long long)p, q);
            uint32_t lq = __shfl_sync(0xffffffffu, len, q);
            uint32_t oq = __shfl_sync(0xffffffffu, off, q);
            for (uint32_t t = lane; t < lq; t += 32) buf[oq + t] = __ldg(pq + t);
        }
        pos += tot;
    }
    return pos;
}

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
                    idx_t o = __shfl_xor_sync(0xffffffffu, x[e], lj);
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
        uint32_t n = warp_gather(src, r, buf);
        __syncwarp();
        idx_t x[E];
#pragma unroll
        for (int e = 0; e < E; ++e) {
            uint32_t i = lane * E + e;
            x[e] = i < n ? buf[i] : kEmpty;
        }
        __syncwarp();
        warp_bitonic_sort<E>(x);
        idx_t prev_last = __shfl_up_sync(0xffffffffu, x[E - 1], 1);
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

// ---- 4b. block hash bin ----------------------------------------------------
__device__ __forceinline__ uint32_t next_pow2(uint32_t v) {
    return v <= 1 ? 1u : 1u << (32 - __clz(v - 1));
}

__global__ void __launch_bounds__(kHashThreads)
hash_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ binoff,
                const uint64_t* __restrict__ ub, idx_t* __restrict__ scratch,
                const uint64_t* __restrict__ soff, uint32_t* __restrict__ counts,
                uint32_t* __restrict__ work) {
    extern __shared__ idx_t tab[];
    __shared__ uint64_t shs[33];
    __shared__ uint32_t s_item;
    const uint32_t lo = binoff[BIN_HASH], hi = binoff[BIN_HASH + 1];
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5, nw = blockDim.x >> 5;
    for (;;) {
        if (threadIdx.x == 0) s_item = lo + atomicAdd(work, 1u);
        __syncthreads();
        const uint32_t item = s_item;
        if (item >= hi) break;
        const idx_t r = rows[item];
        const uint32_t T = next_pow2(uint32_t(2 * ub[r]));  // <= 16384
        const uint32_t mask = T - 1;
        const int shift = 32 - (31 - __clz(T));
        for (uint32_t i = threadIdx.x; i < T; i += blockDim.x) tab[i] = kEmpty;
        __syncthreads();
        // insert: warp per segment
        const uint32_t nseg = num_segs(src, r);
        for (uint32_t j = wib; j < nseg; j += nw) {
            uint32_t len;
            const idx_t* p = get_seg(src, r, j, len);
            for (uint32_t t = lane; t < len; t += 32) {
                idx_t c = __ldg(p + t);
                uint32_t h = (c * 2654435761u) >> shift;
                if (T == 1) h = 0;
                for (;;) {
                    idx_t cur = tab[h];
                    if (cur == c) break;
                    if (cur == kEmpty) {
                        idx_t old = atomicCAS(&tab[h], kEmpty, c);
                        if (old == kEmpty || old == c) break;
                    }
                    h = (h + 1) & mask;
                }
            }
        }
        __syncthreads();
        // in-place compaction: each thread owns T/blockDim consecutive slots
        const uint32_t per = T >= blockDim.x ? T / blockDim.x : 1u;
        const uint32_t beg = threadIdx.x * per;
        idx_t v[32];
        uint64_t cnt = 0;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
            v[i] = kEmpty;
            if (uint32_t(i) < per && beg + i < T) v[i] = tab[beg + i];
            cnt += (v[i] != kEmpty);
        }
        uint64_t total;
        uint64_t ex = block_exclusive_scan<uint64_t>(cnt, shs, &total);  // has syncs
        uint32_t o = uint32_t(ex);
#pragma unroll
        for (int i = 0; i < 32; ++i)
            if (v[i] != kEmpty) tab[o++] = v[i];
        const uint32_t n = uint32_t(total);
        const uint32_t N = next_pow2(n);
        for (uint32_t i = n + threadIdx.x; i < N; i += blockDim.x) tab[i] = kEmpty;
        __syncthreads();
        // bitonic sort of tab[0..N)
        for (uint32_t k = 2; k <= N; k <<= 1) {
            for (uint32_t j = k >> 1; j > 0; j >>= 1) {
                for (uint32_t i = threadIdx.x; i < N / 2; i += blockDim.x) {
                    uint32_t a = 2 * j * (i / j) + (i % j);
                    uint32_t b = a + j;
                    bool asc = (a & k) == 0;
                    idx_t x = tab[a], y = tab[b];
                    if ((x > y) == asc) { tab[a] = y; tab[b] = x; }
                }
                __syncthreads();
            }
        }
        idx_t* out = scratch + soff[r];
        for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) out[i] = tab[i];
        if (threadIdx.x == 0) counts[r] = n;
        __syncthreads();
    }
}

// ---- 4c. block bitmap bin ----------------------------------------------------
__device__ __forceinline__ uint32_t lower_bound_u32(const idx_t* p, uint32_t len, idx_t key) {
    uint32_t lo = 0, hi = len;
    while (lo < hi) {
        uint32_t mid = (lo + hi) >> 1;
        if (__ldg(p + mid) < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

__global__ void __launch_bounds__(kDenseThreads)
dense_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ binoff,
                 idx_t ncols, uint32_t wbits, idx_t* __restrict__ scratch,
                 const uint64_t* __restrict__ soff, uint32_t* __restrict__ counts,
                 uint32_t* __restrict__ work) {
    extern __shared__ uint32_t bm[];
    __shared__ uint64_t shs[33];
    __shared__ uint32_t s_item;
    const uint32_t lo = binoff[BIN_DENSE], hi = binoff[BIN_DENSE + 1];
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5, nw = blockDim.x >> 5;
    const uint32_t wwords = wbits >> 5;
    const uint32_t nwin = uint32_t((uint64_t(ncols) + wbits - 1) / wbits);
    for (;;) {
        if (threadIdx.x == 0) s_item = lo + atomicAdd(work, 1u);
        __syncthreads();
        const uint32_t item = s_item;
        if (item >= hi) break;
        const idx_t r = rows[item];
        const uint32_t nseg = num_segs(src, r);
        idx_t* out = scratch + soff[r];
        uint64_t written = 0;
        for (uint32_t w = 0; w < nwin; ++w) {
            const uint64_t wlo = uint64_t(w) * wbits;
            const uint64_t whi = wlo + wbits;
            for (uint32_t i = threadIdx.x; i < wwords; i += blockDim.x) bm[i] = 0;
            __syncthreads();
            for (uint32_t j = wib; j < nseg; j += nw) {
                uint32_t len;
                const idx_t* p = get_seg(src, r, j, len);
                uint32_t b = 0, e = len;
                if (nwin > 1 && !src.sorted) {
                    // unsorted bucket: filter every element by window
                    for (uint32_t t = lane; t < len; t += 32) {
                        idx_t cc = __ldg(p + t);
                        if (cc >= wlo && cc < whi) {
                            uint32_t c = uint32_t(cc - wlo);
                            atomicOr(&bm[c >> 5], 1u << (c & 31));
                        }
                    }
                    continue;
                }
                if (nwin > 1) {
                    if (lane == 0) {
                        b = lower_bound_u32(p, len, idx_t(wlo));
                        e = whi >= ncols ? len : lower_bound_u32(p, len, idx_t(whi));
                    }
                    b = __shfl_sync(0xffffffffu, b, 0);
                    e = __shfl_sync(0xffffffffu, e, 0);
                }
                for (uint32_t t = b + lane; t < e; t += 32) {
                    uint32_t c = uint32_t(__ldg(p + t) - wlo);
                    atomicOr(&bm[c >> 5], 1u << (c & 31));
                }
            }
            __syncthreads();
            // emission: thread owns a contiguous run of words
            const uint32_t per = (wwords + blockDim.x - 1) / blockDim.x;
            const uint32_t beg = threadIdx.x * per;
            const uint32_t end = min(beg + per, wwords);
            uint64_t cnt = 0;
            for (uint32_t i = beg; i < end; ++i) cnt += __popc(bm[i]);
            uint64_t total;
            uint64_t ex = block_exclusive_scan<uint64_t>(cnt, shs, &total);
            idx_t* o = out + written + ex;
            for (uint32_t i = beg; i < end; ++i) {
                uint32_t word = bm[i];
                while (word) {
                    int bit = __ffs(word) - 1;
                    word &= word - 1;
                    *o++ = idx_t(wlo + (uint64_t(i) << 5) + bit);
                }
            }
            written += total;
            __syncthreads();
        }
        if (threadIdx.x == 0) counts[r] = uint32_t(written);
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

static void ensure_aux() {
    if (g_aux.device == ctx().device) return;
    for (int i = 0; i < 3; ++i) {
        CUDA_CHECK(cudaStreamCreateWithFlags(&g_aux.s[i], cudaStreamNonBlocking));
        CUDA_CHECK(cudaEventCreateWithFlags(&g_aux.join[i], cudaEventDisableTiming));
    }
    CUDA_CHECK(cudaEventCreateWithFlags(&g_aux.fork, cudaEventDisableTiming));
    static bool attr_done = false;
    if (!attr_done) {
        CUDA_CHECK(cudaFuncSetAttribute(hash_bin_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        int(2 * kHashMaxUb * sizeof(idx_t))));
        CUDA_CHECK(cudaFuncSetAttribute(dense_bin_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                        int(kDenseMaxBits / 8)));
        attr_done = true;
    }
    g_aux.device = ctx().device;
}

void row_engine(const SegSource& src, idx_t nrows, idx_t ncols, const uint64_t* ub, Matrix* out) {
    cudaStream_t st = ctx().stream;
    const int nsm = ctx().num_sms;
    if (nrows == 0) {
        matrix_set_empty(out);
        return;
    }
    ensure_aux();
    // 1. bins
    DevBuf<uint64_t> cap(size_t(nrows) + 1);  // reused later for soff (scan in place is not allowed)
    DevBuf<uint64_t> soff(size_t(nrows) + 1);
    DevBuf<uint8_t> bin(nrows);
    DevBuf<uint32_t> counts(nrows);
    DevBuf<uint32_t> meta(64);  // hist[8] binoff[9] cursor[8] work[2]
    uint32_t* hist = meta.p;
    uint32_t* binoff = meta.p + 8;
    uint32_t* cursor = meta.p + 17;
    uint32_t* work = meta.p + 25;
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

    // 4. per-bin kernels on forked streams
    CUDA_CHECK(cudaEventRecord(g_aux.fork, st));
    for (int i = 0; i < 3; ++i) CUDA_CHECK(cudaStreamWaitEvent(g_aux.s[i], g_aux.fork, 0));
    const unsigned gw = nsm * 8;  // 256-thread blocks, grid-stride over bin rows
    {
        cudaStream_t s3 = g_aux.s[2];  // heaviest first: dense bin
        uint32_t wbits = kDenseMaxBits;
        uint64_t ncr = (uint64_t(ncols) + 31) & ~uint64_t(31);
        if (ncr < wbits) wbits = uint32_t(ncr);
        dense_bin_kernel<<<nsm, kDenseThreads, wbits / 8, s3>>>(src, rows.p, binoff, ncols, wbits,
                                                                scratch.p, soff.p, counts.p, work);
        count_launch();
        check_launch("dense_bin_kernel");
        cudaStream_t s2 = g_aux.s[1];
        hash_bin_kernel<<<nsm * 3, kHashThreads, 2 * kHashMaxUb * sizeof(idx_t), s2>>>(
            src, rows.p, binoff, ub, scratch.p, soff.p, counts.p, work + 1);
        count_launch();
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
