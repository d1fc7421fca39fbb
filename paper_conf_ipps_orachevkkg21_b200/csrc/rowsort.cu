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
//   3. bin_scatter : row lists per bin and the 40-B work records of the
//                    hash-bin rows
//   4. per-bin kernels (heaviest first, persistent grids):
//        dense (ub > 40960): one-level smem bitmap over 1.5 Mi-column
//            windows (non-returning atomics, word-walk emission), one
//            1024-thread block per row; a span of more than three windows
//            is partitioned by window first (two gathers)
//        dense_ovf: the same kernel with 256 Ki-column windows and a
//            two-level bitmap for rows the producer flagged duplicate-heavy
//            (closure steps) and for hash-bin rows that fell back
//        hash H6..H0 (ub <= 40960 .. 512): bucketed order-preserving hash in
//            smem (bucket = floor((c - lo) / W), 16 slots of 16-bit offsets,
//            one atomicAdd per insert), 16x2 SIMD Batcher sort per bucket
//            pair, warp-cooperative emission; a smem span bitmap when the
//            span is small
//        warp W8..W1 (ub <= 256): one warp per row, register bitonic sort
//   5. scan(counts): CSR row offsets
//   6. compact     : move from capacity offsets to CSR offsets -- a tile copy
//                    into a new exact buffer when memory allows, else in
//                    place (tiles ordered by their overlaps)
#include "common.cuh"

#include <algorithm>
#include <cstdlib>

namespace spbla {

namespace {

constexpr unsigned FULL = 0xffffffffu;

#ifdef SPBLA_PROBE
// Debug-only phase timing (built into a separate .so by tools/probe.sh):
// block 0, thread 0 prints per-phase nanoseconds for its first rows.
__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__shared__ unsigned long long s_probe_ext[12];
#define PROBE_DECL uint32_t probe_rows = 0;
#define PROBE(i) do { if (threadIdx.x == 0) s_probe_ext[i] = gtimer(); } while (0)
#define PROBE_PRINT(tag, u, ns)                                                                      \
    do {                                                                                           \
        if (blockIdx.x == 0 && threadIdx.x == 0 && probe_rows++ < 24)                              \
            printf("%s u=%u nseg=%u meta=%llu fill=%llu stage=%llu prod=%llu ovf=%llu cnt=%llu emit=%llu\n", tag, \
                   u, ns, s_probe_ext[1] - s_probe_ext[0], s_probe_ext[2] - s_probe_ext[1],                \
                   s_probe_ext[3] - s_probe_ext[2], s_probe_ext[4] - s_probe_ext[3],                   \
                   s_probe_ext[5] - s_probe_ext[4], s_probe_ext[6] - s_probe_ext[5],                   \
                   s_probe_ext[7] - s_probe_ext[6]);                                                  \
    } while (0)
#else
#define PROBE_DECL
#define PROBE(i) do {} while (0)
#define PROBE_PRINT(tag, u, ns) do {} while (0)
#endif
constexpr int kNumBins = 15;
enum {
    BIN_EMPTY = 0, BIN_W1 = 1, BIN_W2, BIN_W4, BIN_W8, BIN_H0,
    BIN_H1 = 6, BIN_H2, BIN_H3, BIN_H4, BIN_H5, BIN_H6, BIN_DENSE = 12,
    BIN_DUP = 13,  // rows flagged duplicate-heavy (kUbDupFlag): straight to the small bitmap kernel
    BIN_COPY = 14  // rows flagged copy-only (kUbCopyFlag): their single segment is the output
};
constexpr uint64_t kWarpMaxUb = kRangeMinUb;   // 256
// hash bins: ub limits (each sized so its tables fit the residency below)
#ifndef SPBLA_HB  // hash-bin ub limits (overridable for a sweep)
#define SPBLA_HB 512, 1024, 2048, 4096, 8192, 20480, 40960
#endif
constexpr uint64_t kHB[7] = {SPBLA_HB};
constexpr uint64_t kH0 = kHB[0], kH1 = kHB[1], kH2 = kHB[2], kH3 = kHB[3], kH4 = kHB[4], kH5 = kHB[5], kH6 = kHB[6];
#ifndef SPBLA_EARLY_STOP_MAX  // early stop in the hash bins of at most this many threads (sweeps)
#define SPBLA_EARLY_STOP_MAX 128
#endif
#ifndef SPBLA_PART_MIN  // partition-by-window above this many windows (overridable for a sweep)
#define SPBLA_PART_MIN 3
#endif
constexpr uint32_t kDenseBits = 3u << 19;      // bitmap window: 1.5 Mi columns, 192 KB of smem
constexpr int kUnroll = 4;                     // warp_flat (warp bins)

__device__ __forceinline__ int bin_of(uint64_t ub) {
    if (ub == 0) return BIN_EMPTY;
    if (ub <= 32 && 32 <= kWarpMaxUb) return BIN_W1;
    if (ub <= 64 && 64 <= kWarpMaxUb) return BIN_W2;
    if (ub <= 128 && 128 <= kWarpMaxUb) return BIN_W4;
    if (ub <= kWarpMaxUb) return BIN_W8;
    if (ub <= kH0) return BIN_H0;
    if (ub <= kH1) return BIN_H1;
    if (ub <= kH2) return BIN_H2;
    if (ub <= kH3) return BIN_H3;
    if (ub <= kH4) return BIN_H4;
    if (ub <= kH5) return BIN_H5;
    if (ub <= kH6) return BIN_H6;
    return BIN_DENSE;
}

// ---- segment access --------------------------------------------------------
__device__ __forceinline__ uint32_t num_segs(const SegSource& s, idx_t r) {
    if (s.kind == 1) return 1;
    return s.nseg[r];
}

__device__ __forceinline__ const idx_t* get_seg(const SegSource& s, idx_t r, uint32_t j, uint32_t& len) {
    if (s.kind == 1) {
        off_t64 b = s.lrp[r];
        len = uint32_t(s.lrp[r + 1] - b);
        return s.lst + b;
    }
    const uint4 d = s.desc[s.dbase[r] + r + j];
    len = d.z;
    return reinterpret_cast<const idx_t*>((uint64_t(d.y) << 32) | d.x);
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

// ---- block gather ----------------------------------------------------------
// Stage segments [s0, s0+n) of row r: sd_ptr[k] points at the segment minus
// its start offset in the batch's concatenation (so product q of segment k
// is sd_ptr[k][q]), sd_end[k] is its exclusive end.  Descriptor mode: a
// plain copy of the precomputed descriptors (non-empty, prefix ends).
// sd_first (nullable): sd_first[j] = the segment holding product j << kFirstShift,
// written by that segment (each multiple of 2^kFirstShift lies in exactly one
// non-empty segment); replaces the binary search of the gather.
// Returns the number of products in the batch; ends with a barrier.
#ifndef SPBLA_FIRST_SHIFT  // (overridable for a sweep)
#define SPBLA_FIRST_SHIFT 6
#endif
constexpr uint32_t kFirstShift = SPBLA_FIRST_SHIFT;
// descriptor-mode segment base of row r: its descriptors are desc[seg_base + j]
__device__ __forceinline__ uint64_t seg_base(const SegSource& s, idx_t r) {
    return s.kind == 1 ? 0 : s.dbase[r] + r;
}
// stage one descriptor as entry i of the batch whose concatenation starts at base
// (nf: entries of sd_first; a batch with more products than nf << kFirstShift
// leaves the table partial and the gather binary-searches instead)
__device__ __forceinline__ void stage_one(const uint4& e, uint32_t i, uint32_t base, const idx_t** sd_ptr,
                                          uint32_t* sd_end, uint32_t* sd_first, uint32_t nf = 0xFFFFFFFFu) {
    const idx_t* p = reinterpret_cast<const idx_t*>((uint64_t(e.y) << 32) | e.x);
    const uint32_t end = e.w - base, start = end - e.z;
    sd_ptr[i] = p - start;
    sd_end[i] = end;
    if (sd_first) {
#pragma unroll 1
        for (uint32_t j = (start + (1u << kFirstShift) - 1) >> kFirstShift; (j << kFirstShift) < end && j < nf; ++j)
            sd_first[j] = i;
    }
}
// KINDT >= 0: the segment-source kind as a compile-time constant
template <int THREADS, int KINDT = -1>
__device__ __forceinline__ uint32_t stage_segments(const SegSource& s, idx_t r, uint64_t sbase, uint32_t s0,
                                                   uint32_t n, const idx_t** sd_ptr, uint32_t* sd_end,
                                                   uint32_t* sd_first, uint32_t nf = 0xFFFFFFFFu) {
    if ((KINDT >= 0 ? KINDT : s.kind) == 1) {  // one segment
        if (threadIdx.x == 0) {
            const off_t64 b = s.lrp[r];
            sd_ptr[0] = s.lst + b;
            sd_end[0] = uint32_t(s.lrp[r + 1] - b);
        }
        __syncthreads();
        return sd_end[0];
    }
    const uint4* d = s.desc + (sbase + s0);
    const uint32_t base = s0 ? s.desc[sbase + s0 - 1].w : 0u;
#pragma unroll 1
    for (uint32_t i = threadIdx.x; i < n; i += THREADS) stage_one(d[i], i, base, sd_ptr, sd_end, sd_first, nf);
    __syncthreads();
    return d[n - 1].w - base;
}

// Call f(c) for every product of row r.  Thread t takes U consecutive
// products q0 = (t + i*THREADS)*U .. q0+U-1 of the concatenated segments:
// the segment holding q0 comes from the sd_first table plus a short linear
// advance (binary search when there is no table), then a linear advance
// inside the run (segments average tens of products, so a run rarely
// crosses more than one boundary); the U loads are issued before any
// insert.  A warp covers 32*U consecutive products, i.e. a few sectors of
// each B row.  Ends with a barrier.  abort (optional): a shared flag; once it
// is set every thread skips the rest of its products (the caller discards
// the row).
// prestaged: the first batch is already staged (and visible to all threads).
template <int THREADS, int U, int KINDT = -1, typename F>
__device__ __forceinline__ void block_products(const SegSource& s, idx_t r, uint64_t sbase, uint32_t nseg,
                                               const idx_t** sd_ptr, uint32_t* sd_end, uint32_t* sd_first,
                                               uint32_t batch, bool prestaged, F&& f,
                                               const volatile uint32_t* abort = nullptr, uint32_t nf = 0xFFFFFFFFu) {
    for (uint32_t s0 = 0; s0 < nseg; s0 += batch) {
        const uint32_t ns = min(batch, nseg - s0);
        const uint32_t total = (s0 == 0 && prestaged)
                                   ? sd_end[ns - 1]
                                   : stage_segments<THREADS, KINDT>(s, r, sbase, s0, ns, sd_ptr, sd_end, sd_first, nf);
        // (a partial lookup table: binary search)
        const uint32_t* sdf = (sd_first && uint64_t(total) <= (uint64_t(nf) << kFirstShift)) ? sd_first : nullptr;
#ifdef SPBLA_PROBE
        if (threadIdx.x == 0 && s0 == 0) s_probe_ext[3] = gtimer();  // stage done
#endif
        for (uint32_t q0 = threadIdx.x * U; q0 < total; q0 += THREADS * U) {
            // a row already bound for the fallback stops gathering (per
            // thread: no barrier inside this loop)
            // (a volatile shared load -- LDS -- : the flag is set concurrently,
            // by atomicExch, from inserting threads; a cuda::atomic_ref load
            // compiled to a generic strong load)
            if (abort) {
                uint32_t fl;
                asm volatile("ld.volatile.shared.u32 %0, [%1];"
                             : "=r"(fl)
                             : "r"(uint32_t(__cvta_generic_to_shared(const_cast<uint32_t*>(abort)))));
                if (fl) break;
            }
            uint32_t k;
            if ((KINDT >= 0 ? KINDT : s.kind) == 1) {
                k = 0;
            } else if (sdf) {
                k = sdf[q0 >> kFirstShift];
                while (sd_end[k] <= q0) ++k;
            } else {
                uint32_t lo = 0, hi = ns - 1;  // first segment whose end exceeds q0
                while (lo < hi) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if (sd_end[mid] <= q0) lo = mid + 1; else hi = mid;
                }
                k = lo;
            }
            uint32_t end = sd_end[k];
            const idx_t* p = sd_ptr[k];
            idx_t v[U];
            // consecutive products cross at most one boundary (segments are
            // non-empty), so each step is a single predicated advance
            if (q0 + U <= total) {
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const uint32_t q = q0 + u;
                    if (u > 0 && q >= end) {
                        ++k;
                        end = sd_end[k];
                        p = sd_ptr[k];
                    }
                    v[u] = __ldg(p + q);
                }
#pragma unroll
                for (int u = 0; u < U; ++u) f(v[u]);
            } else {  // ragged tail of the row: rolled (keeps the kernel small)
#pragma unroll 1
                for (uint32_t q = q0; q < total; ++q) {
                    if (q > q0 && q >= end) {
                        ++k;
                        end = sd_end[k];
                        p = sd_ptr[k];
                    }
                    f(__ldg(p + q));
                }
            }
        }
        __syncthreads();  // descriptors are reused by the next batch
    }
}

// Block scan of per-warp counts held in s_w[0..NW); s_w[w] becomes the
// warp's output base, s_w[32] the total.
template <int NW>
__device__ __forceinline__ void scan_warp_counts(uint32_t* s_w) {
    const unsigned lane = lane_id();
    if (NW == 1) {  // one warp: no scan (and no speculative reads of s_w[lane])
        if (threadIdx.x == 0) {
            s_w[32] = s_w[0];
            s_w[0] = 0u;
        }
        __syncthreads();
        return;
    }
    if ((threadIdx.x >> 5) == 0) {
        const uint32_t v = lane < NW ? s_w[lane] : 0u;
        const uint32_t inc = warp_inclusive_scan(v);
        if (lane < NW) s_w[lane] = inc - v;
        if (lane == NW - 1) s_w[32] = inc;
    }
    __syncthreads();
}

// Ordered emission of the set bits of bm[0..nwords) as base_col + 32 i + b,
// warp w owning words [w*chunk, (w+1)*chunk).  Returns the count.
template <int NW>
__device__ __forceinline__ uint32_t emit_bitmap(const uint32_t* bm, uint32_t nwords, uint64_t base_col,
                                                idx_t* __restrict__ out, uint32_t* s_w) {
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5;
    const uint32_t chunk = ((nwords + NW - 1) / NW + 31) & ~31u;
    const uint32_t b = wib * chunk, e = min(b + chunk, nwords);
    uint32_t cnt = 0;
    for (uint32_t i = b + lane; i < e; i += 32) cnt += __popc(bm[i]);
    cnt = warp_sum(cnt);
    if (lane == 0) s_w[wib] = cnt;
    __syncthreads();
    scan_warp_counts<NW>(s_w);
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

__device__ __forceinline__ void fill_words(uint32_t* p, uint32_t n, uint32_t v, int threads) {
    // p is 16-byte aligned; vector stores for the bulk
    uint4* p4 = reinterpret_cast<uint4*>(p);
    const uint4 v4 = make_uint4(v, v, v, v);
#pragma unroll 1
    for (uint32_t i = threadIdx.x; i < n / 4; i += threads) p4[i] = v4;
#pragma unroll 1
    for (uint32_t i = (n & ~3u) + threadIdx.x; i < n; i += threads) p[i] = v;
}

// ---- 4b. block hash / span-bitmap bins --------------------------------------
// Bucketed ORDER-PRESERVING hash: bucket b = floor((c - lo) / W) is monotone
// in c, so buckets are mutually ordered.  A bucket has 16 slots of 16-bit
// offsets c - lo - b*W (W <= 65535; 0xFFFF marks an empty slot) and a fill
// counter: an insert is one smem atomicAdd on the counter and one 16-bit
// store - no probing, no CAS, no lane divergence; duplicates are dropped at
// emission.  nb = ub/8 buckets (mean load <= 8, 4.5 bytes of smem per
// product); a product arriving at a full bucket (p ~ 0.4%) is appended to a
// small overflow list.  The table is slot-major: slot s of bucket b at
// tab16[s*MAXB + b], so one 32-bit word holds slot s of the bucket pair
// (2m, 2m+1) - exactly one 16x2 SIMD register of the pair's sort.
//
// Emission: thread t owns bucket pairs t, t+T, t+2T, ... (KP of them).
//  pass A: per pair, 16 conflict-free LDS.32 give x[s] = (slot s of 2m+1,
//          slot s of 2m); a 16-input Batcher network (63 comparators) on
//          VIMNMX.U16x2 sorts both buckets, the sorted slots are written
//          back, the distinct values are counted (n_valid minus adjacent
//          equal pairs, via max(x_i, x_{i-1}+1) - x_i summed in 32-bit
//          arithmetic).  A bucket that overflowed is listed instead;
//  overflow: one warp per listed bucket gathers its 16 slots and its list
//          entries (ballot over the list), bitonic-sorts <= 32 values across
//          lanes, dedups, writes the first 16 back to the slots and parks the
//          rest in a pool;
//  multi-scan: a block scan of the KP per-thread pair counts at once gives
//          every pair its output offset (pair order = (round, thread) order);
//  pass B: stream each sorted pair to out[offset], skipping adjacent
//          duplicates (predicated stores, no sort).  Adjacent lanes write
//          adjacent pairs, so a warp's stores cover a ~2 KB window.
__device__ __forceinline__ void cswap2(uint32_t& a, uint32_t& b) {
    const uint32_t x = __vminu2(a, b), y = __vmaxu2(a, b);
    a = x;
    b = y;
}
__device__ __forceinline__ void sort16x2(uint32_t (&v)[16]) {  // Batcher odd-even merge sort, 63 comparators
    cswap2(v[0], v[1]); cswap2(v[2], v[3]); cswap2(v[0], v[2]); cswap2(v[1], v[3]); cswap2(v[1], v[2]);
    cswap2(v[4], v[5]); cswap2(v[6], v[7]); cswap2(v[4], v[6]); cswap2(v[5], v[7]); cswap2(v[5], v[6]);
    cswap2(v[0], v[4]); cswap2(v[2], v[6]); cswap2(v[2], v[4]); cswap2(v[1], v[5]); cswap2(v[3], v[7]);
    cswap2(v[3], v[5]); cswap2(v[1], v[2]); cswap2(v[3], v[4]); cswap2(v[5], v[6]);
    cswap2(v[8], v[9]); cswap2(v[10], v[11]); cswap2(v[8], v[10]); cswap2(v[9], v[11]); cswap2(v[9], v[10]);
    cswap2(v[12], v[13]); cswap2(v[14], v[15]); cswap2(v[12], v[14]); cswap2(v[13], v[15]); cswap2(v[13], v[14]);
    cswap2(v[8], v[12]); cswap2(v[10], v[14]); cswap2(v[10], v[12]); cswap2(v[9], v[13]); cswap2(v[11], v[15]);
    cswap2(v[11], v[13]); cswap2(v[9], v[10]); cswap2(v[11], v[12]); cswap2(v[13], v[14]);
    cswap2(v[0], v[8]); cswap2(v[4], v[12]); cswap2(v[4], v[8]); cswap2(v[2], v[10]); cswap2(v[6], v[14]);
    cswap2(v[6], v[10]); cswap2(v[2], v[4]); cswap2(v[6], v[8]); cswap2(v[10], v[12]); cswap2(v[1], v[9]);
    cswap2(v[5], v[13]); cswap2(v[5], v[9]); cswap2(v[3], v[11]); cswap2(v[7], v[15]); cswap2(v[7], v[11]);
    cswap2(v[3], v[5]); cswap2(v[7], v[9]); cswap2(v[11], v[13]); cswap2(v[1], v[2]); cswap2(v[3], v[4]);
    cswap2(v[5], v[6]); cswap2(v[7], v[8]); cswap2(v[9], v[10]); cswap2(v[11], v[12]); cswap2(v[13], v[14]);
}
__device__ __forceinline__ uint32_t vadd2(uint32_t a, uint32_t b) {  // per-16-bit-lane add (wrapping)
    uint32_t r;
    asm("add.u16x2 %0, %1, %2;" : "=r"(r) : "r"(a), "r"(b));
    return r;
}
// *p = v if q (predicated store: no branch / reconvergence around it)
__device__ __forceinline__ void st_if(idx_t* p, uint32_t v, bool q) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q st.global.u32 [%0], %1;\n\t}" ::"l"(p), "r"(v),
                 "r"(uint32_t(q))
                 : "memory");
}
constexpr uint32_t kOvfFlag = 0x80000000u;
constexpr uint32_t kSlots = 16;

template <int E>
__device__ __forceinline__ void warp_bitonic_sort(idx_t (&x)[E]);

// A hash-bin row that cannot use its table goes to a bitmap kernel: rows whose
// span fits two small windows to list 0 (items [ovf_cnt[0] = 0, ovf_cnt[1])),
// the others to list 1 (items [ovf_cnt[2] = nrows, ovf_cnt[3]), ovf_cnt[3]
// starting at nrows): each pair is the bounds of one bitmap kernel launch.
constexpr uint32_t kSmallSpan = 2u << 18;
__device__ __forceinline__ void push_fallback(idx_t r, uint32_t span_m1, idx_t* ovf_rows, uint32_t* ovf_cnt) {
    if (span_m1 < kSmallSpan) ovf_rows[atomicAdd(ovf_cnt + 1, 1u)] = r;
    else ovf_rows[atomicAdd(ovf_cnt + 3, 1u)] = r;
}

// Per-row work record of the hash bins (written by bin_scatter_kernel while
// binning): one 40-B load gives everything the row needs.
struct RowRec {
    uint32_t r, u, clo, chi;  // row, upper bound, column span [clo, chi]
    uint64_t out, seg;        // scratch offset, descriptor base (kind 0)
    uint32_t nseg, pad;
};
// A row's plan, computed once by thread 0 (one row ahead) and read by all
// threads from shared memory: mode, bucket count, width and exact reciprocal.
enum : uint32_t { kPlanHash = 0, kPlanBitmap = 1, kPlanWide = 2, kPlanEnd = 3 };
// mean bucket load: nb = ub / kLoadDiv buckets of 16 slots
#ifndef SPBLA_LOAD_DIV
#define SPBLA_LOAD_DIV 8
#endif
constexpr uint32_t kLoadDiv = SPBLA_LOAD_DIV;
struct RowPlan {
    RowRec rec;
    uint32_t mode, nb, W, l, M, nw;
};
template <uint32_t MAXB>
__device__ __forceinline__ RowPlan make_plan(const RowRec& x) {
    RowPlan P;
    P.rec = x;
    const uint64_t span = uint64_t(x.chi) - x.clo + 1;
    // nb buckets of width W <= 65535 (16-bit offsets); too wide a span for the
    // table goes to the bitmap bin.  nb is even (buckets are sorted in pairs).
    const uint64_t nbw = (span + 65534) / 65535;
    const uint32_t nb =
        (uint32_t(min(max(max(uint64_t((x.u + kLoadDiv - 1) / kLoadDiv), nbw), uint64_t(1)), uint64_t(MAXB))) + 1) & ~1u;
    const uint64_t words = (span + 31) >> 5;
    P.nb = nb;
    P.nw = uint32_t(min(words, uint64_t(0xFFFFFFFFu)));
    P.W = P.l = P.M = 0;
    if (words <= 9ull * nb) {  // the span bitmap is no larger than the table
        P.mode = kPlanBitmap;
    } else if (nbw > MAXB) {  // span too wide for 16-bit offsets in this table
        P.mode = kPlanWide;
    } else {
        // bucket width W (> 288 here: smaller spans took the bitmap) and an exact
        // 32-bit reciprocal: d < nb*W < 2^29, M = ceil(2^(32+l) / W) with
        // 2^(l+3) >= W gives floor(d / W) = umulhi(d, M) >> l (M < 2^30)
        P.mode = kPlanHash;
        P.W = uint32_t((span + nb - 1) / nb);
        P.l = (32 - __clz(P.W - 1)) - 3;
        P.M = uint32_t(((uint64_t(1) << (32 + P.l)) + P.W - 1) / P.W);
    }
    return P;
}

// Pair stride of the slot-major table: MPP = 2 (mod 32), so slot s of pair m
// sits in bank 2s + m (mod 32): the per-thread pass A (lanes = consecutive
// pairs, one slot) and the warp-cooperative pass B (lanes = 4 slots x 8
// consecutive pairs) are both conflict-free.
__host__ __device__ constexpr uint32_t pair_stride(uint32_t mp) { return ((mp + 29) / 32) * 32 + 2; }
__host__ __device__ constexpr uint32_t first_entries(uint64_t maxub) { return uint32_t((maxub >> kFirstShift) + 1); }

// Rows flow through a 3-stage software pipeline (one block, rows claimed
// from an atomic counter): while row i runs, thread 0 holds the claim of row
// i+2, loads row i+1's record at row start and publishes its plan after the
// gather; after pass A every thread issues the loads of row i+1's first
// descriptor batch and stages it at the end of row i.  A row therefore starts
// with its metadata and descriptors already in shared memory: no global
// round trip and no staging barrier before its gather.
//
// dynamic smem: tabw[16*MPP] | bcnt[MAXB] | sd_ptr[BATCH] | sd_end[BATCH] | sd_first[NF] |
//               ovl[OVCAP] | pool[OVCAP] u16 | obl[OBCAP] | obcnt[OBCAP] | poff[MAXB/2]
// (the per-warp overflow buffers wbuf[THREADS] alias the segment descriptors,
// which are dead once the products are inserted: BATCH * 3 >= THREADS)
template <int THREADS, uint32_t MAXB, uint32_t OVCAP, uint32_t OBCAP, uint32_t BATCH, int MINB, int FLATU, bool DEDUP_B,
          int KIND>
__global__ void __launch_bounds__(THREADS, MINB)
hash_bin_kernel(SegSource src, const RowRec* __restrict__ recs, const uint32_t* __restrict__ bounds,
                idx_t* __restrict__ scratch, uint32_t* __restrict__ counts,
                uint32_t* __restrict__ work, idx_t* __restrict__ ovf_rows, uint32_t* __restrict__ ovf_cnt) {
    constexpr int NW = THREADS / 32;
    constexpr uint32_t MP = MAXB / 2;                      // bucket pairs
    constexpr uint32_t MPP = pair_stride(MP);              // padded pair stride of the table
    constexpr uint32_t TABW = 16 * MPP;                    // table words
    constexpr uint32_t KP = (MP + THREADS - 1) / THREADS;  // pairs per thread
    constexpr uint32_t NF = first_entries(uint64_t(MAXB) * 8);
    constexpr int PF = (BATCH + THREADS - 1) / THREADS;    // prefetched descriptors per thread
    extern __shared__ __align__(16) unsigned char smem_raw[];
    uint32_t* tabw = reinterpret_cast<uint32_t*>(smem_raw);  // word s*MPP + m = slot s of pair m
    uint16_t* tab16 = reinterpret_cast<uint16_t*>(smem_raw);
    uint32_t* bmw = tabw;  // bitmap-mode view: TABW + MAXB words
    uint32_t* bcnt = tabw + TABW;
    const idx_t** sd_ptr = reinterpret_cast<const idx_t**>(bcnt + MAXB);
    uint32_t* sd_end = reinterpret_cast<uint32_t*>(sd_ptr + BATCH);
    uint32_t* sd_first = sd_end + BATCH;
    idx_t* ovl = sd_first + NF;
    uint16_t* pool = reinterpret_cast<uint16_t*>(ovl + OVCAP);
    uint32_t* obl = reinterpret_cast<uint32_t*>(pool + OVCAP);
    uint32_t* obcnt = obl + OBCAP;
    uint32_t* poff = obcnt + OBCAP;  // [MP] output offset of each bucket pair
    uint32_t* wbuf = reinterpret_cast<uint32_t*>(sd_ptr);
    static_assert(BATCH * 3 >= THREADS && OVCAP % 2 == 0 && MAXB % 2 == 0 && MP % 32 == 0, "hash bin layout");
    __shared__ uint32_t s_w[33];
    __shared__ uint32_t s_wt[KP][NW];
    // s_flag / s_novf are written (and s_flag read) during the gather, which
    // starts without a barrier: thread 0 clears them for the next row just
    // before the barrier that ends the current row, after their last reads
    // (the fallback decision, behind the pass-A / overflow barriers)
    __shared__ uint32_t s_flag, s_novf, s_nob, s_pool;
    // early stop of the gather once the row is bound for the fallback: the
    // small bins, where duplicate-heavy closure rows overflow
    constexpr bool kEarlyStop = THREADS <= SPBLA_EARLY_STOP_MAX;
    __shared__ RowPlan s_plan[2];
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5;
    const uint32_t lt = (1u << lane) - 1u;
    const uint32_t lo_i = bounds[0], hi_i = bounds[1];
    src.kind = KIND;  // compile-time segment source: the helpers' kind branches fold away
    const bool pre = KIND == 0;  // descriptor mode: first batches are prefetched
    RowPlan end_plan;
    end_plan.mode = kPlanEnd;
    // descriptor prefetch of a row's first batch: issue (loads in flight) ...
    uint4 pfd[PF];
    auto pf_issue = [&](const RowPlan& N) {
        if (!pre || N.mode == kPlanEnd) return;
        const uint32_t n = min(N.rec.nseg, BATCH);
#pragma unroll
        for (int k = 0; k < PF; ++k) {
            const uint32_t i = threadIdx.x + k * THREADS;
            if (i < n) pfd[k] = src.desc[N.rec.seg + i];
        }
    };
    // ... and commit (staged into the descriptor arrays; visible after the next barrier)
    auto pf_commit = [&](const RowPlan& N) {
        if (!pre || N.mode == kPlanEnd) return;
        const uint32_t n = min(N.rec.nseg, BATCH);
#pragma unroll
        for (int k = 0; k < PF; ++k) {
            const uint32_t i = threadIdx.x + k * THREADS;
            if (i < n) stage_one(pfd[k], i, 0u, sd_ptr, sd_end, sd_first);
        }
    };
    // ... and, once the descriptors have arrived, a bulk-async L2 prefetch of
    // the B rows they point at (cp.async.bulk.prefetch: one instruction per
    // segment), issued before pass B so the next row's
    // gather finds its first batch in L2
    auto pf_l2 = [&](const RowPlan& N) {
        if (!pre || N.mode == kPlanEnd) return;
        const uint32_t n = min(N.rec.nseg, BATCH);
#pragma unroll
        for (int k = 0; k < PF; ++k) {
            const uint32_t i = threadIdx.x + k * THREADS;
            if (i < n) {
                const uint64_t a = (uint64_t(pfd[k].y) << 32) | pfd[k].x;
                // (16-B aligned inside the segment's allocation: rounded
                // down at both ends, a tail of < 16 B is not prefetched)
                const uint64_t a0 = a & ~uint64_t(15), a1 = (a + 4ull * pfd[k].z) & ~uint64_t(15);
                if (a1 > a0)
                    asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(a0), "r"(uint32_t(a1 - a0))
                                 : "memory");
            }
        }
    };
    // the table is kept clean between rows (all slots 0xFFFF, counters 0):
    // every row restores what it dirtied before the end-of-row barrier
#pragma unroll 1
    for (uint32_t i = threadIdx.x; i < TABW; i += THREADS) tabw[i] = 0xFFFFFFFFu;
#pragma unroll 1
    for (uint32_t i = threadIdx.x; i < MAXB; i += THREADS) bcnt[i] = 0u;
    if (threadIdx.x == 0) {
        s_flag = 0;
        s_novf = 0;
    }
    // prologue: claim rows 0 and 1, plan row 0, stage its first batch
    // the pipeline thread is the last one: it has the least pass-A work
    constexpr unsigned PT = THREADS - 1;
    uint32_t nxt1 = 0, nxt2 = 0;  // (thread PT) claimed items of rows i+1 and i+2
    if (threadIdx.x == PT) {
        const uint32_t i0 = lo_i + atomicAdd(work, 1u);
        nxt1 = lo_i + atomicAdd(work, 1u);
        s_plan[0] = i0 < hi_i ? make_plan<MAXB>(recs[i0]) : end_plan;
    }
    __syncthreads();
    {
        const RowPlan P0 = s_plan[0];
        pf_issue(P0);
        pf_commit(P0);
    }
    __syncthreads();
    PROBE_DECL
#pragma unroll 1
    for (uint32_t it = 0;; ++it) {
        const RowPlan P = s_plan[it & 1];
        if (P.mode == kPlanEnd) break;
        RowRec nx;
        bool have_nx = false;
        if (threadIdx.x == PT) {
            nxt2 = lo_i + atomicAdd(work, 1u);
            have_nx = nxt1 < hi_i;
            if (have_nx) nx = recs[nxt1];
        }
        if (threadIdx.x == 0) {  // (used only behind this row's insert barrier)
            s_nob = 0;
            s_pool = 0;
        }
        // the next row's gather starts right after this row's last barrier
        auto clear_row_flags = [&]() {
            if (threadIdx.x == 0) {
                s_flag = 0;
                s_novf = 0;
            }
        };
        // thread PT: plan of row i+1 into s_plan (visible after the next barrier)
        auto publish_next = [&]() {
            if (threadIdx.x == PT) {
                s_plan[(it + 1) & 1] = have_nx ? make_plan<MAXB>(nx) : end_plan;
                nxt1 = nxt2;
            }
        };
        PROBE(0);
        const idx_t r = P.rec.r;
        const uint32_t clo = P.rec.clo;
        const uint32_t nb = P.nb, np = nb / 2;
        idx_t* out = scratch + P.rec.out;
        if (P.mode == kPlanBitmap) {
            const uint32_t nw = P.nw;
#pragma unroll 1
            for (uint32_t i = threadIdx.x; i < nw; i += THREADS) bmw[i] = 0u;
            __syncthreads();
            block_products<THREADS, FLATU>(src, r, P.rec.seg, P.rec.nseg, sd_ptr, sd_end, sd_first, BATCH, pre,
                                           [&](idx_t c) {
                                               const uint32_t d = c - clo;
                                               atomicOr(&bmw[d >> 5], 1u << (d & 31));
                                           });
            publish_next();
            const uint32_t n = emit_bitmap<NW>(bmw, nw, clo, out, s_w);  // (barriers inside)
            if (threadIdx.x == 0) counts[r] = n;
#pragma unroll 1
            for (uint32_t i = threadIdx.x; i < nw; i += THREADS) bmw[i] = i < TABW ? 0xFFFFFFFFu : 0u;
            const RowPlan N = s_plan[(it + 1) & 1];
            pf_issue(N);
            clear_row_flags();
            pf_commit(N);
            __syncthreads();
            continue;
        }
        PROBE(1);
        if (P.mode == kPlanWide) {
            if (threadIdx.x == 0) push_fallback(r, P.rec.chi - P.rec.clo, ovf_rows, ovf_cnt);
            publish_next();
            __syncthreads();
            const RowPlan N = s_plan[(it + 1) & 1];
            pf_issue(N);
            clear_row_flags();
            pf_commit(N);
            __syncthreads();
            continue;
        }
        const uint32_t W = P.W, l = P.l, M = P.M;
        PROBE(2);
        block_products<THREADS, FLATU>(src, r, P.rec.seg, P.rec.nseg, sd_ptr, sd_end, sd_first, BATCH, pre,
                                       [&](idx_t c) {
            const uint32_t d = c - clo;
            const uint32_t b = __umulhi(d, M) >> l;
            const uint32_t slot = atomicAdd(&bcnt[b], 1u);
            if (slot < kSlots) {
                tab16[slot * (2 * MPP) + b] = uint16_t(d - b * W);
            } else {
                const uint32_t i = atomicAdd(&s_novf, 1u);
                if (i < OVCAP) ovl[i] = c; else atomicExch(&s_flag, 1u);  // (polled concurrently: atomic)
            }
        }, kEarlyStop ? &s_flag : nullptr);
        PROBE(4);
        bool fallback = s_flag != 0;  // overflow list full: the row goes to the bitmap bin
        if (!fallback) {
            // ---- pass A: sort each owned bucket pair in 16x2 SIMD ----------------
            // Every bucket leaves pass A sorted (duplicates adjacent, empty
            // 0xFFFF slots last; DEDUP_B = false: duplicates already replaced by
            // 0xFFFF and re-sorted here, the better choice for the small
            // bins); bcnt[b] becomes the bucket's distinct count,
            // or kOvfFlag | list index (the overflow pass then leaves the first
            // 16 distinct values in its slots)
#pragma unroll 1
            for (uint32_t m = threadIdx.x; m < np; m += THREADS) {
                const uint2 nn = reinterpret_cast<const uint2*>(bcnt)[m];
                uint32_t keep = 0xFFFFFFFFu;  // lanes of an overflowed bucket are masked out of the sort
                uint2 res;
                if (nn.x > kSlots) {
                    const uint32_t j = atomicAdd(&s_nob, 1u);
                    if (j < OBCAP) obl[j] = 2 * m; else s_flag = 1;
                    res.x = kOvfFlag | j;
                    keep &= 0xFFFF0000u;
                }
                if (nn.y > kSlots) {
                    const uint32_t j = atomicAdd(&s_nob, 1u);
                    if (j < OBCAP) obl[j] = 2 * m + 1; else s_flag = 1;
                    res.y = kOvfFlag | j;
                    keep &= 0x0000FFFFu;
                }
                uint32_t x[16];
#pragma unroll
                for (int sl = 0; sl < 16; ++sl) x[sl] = tabw[sl * MPP + m] | ~keep;
                sort16x2(x);
                // adjacent equal pairs: max(x_i, x_{i-1}+1) - x_i is 1 iff x_i == x_{i-1}
                // (an empty 0xFFFF predecessor wraps to 0 and counts nothing); the
                // per-half differences are >= 0, so a plain 32-bit sum keeps them apart
                uint32_t dsum = 0;
#pragma unroll
                for (int k2 = 1; k2 < 16; ++k2) dsum += __vmaxu2(x[k2], vadd2(x[k2 - 1], 0x00010001u)) - x[k2];
                if (!DEDUP_B) {
                    // drop the duplicates here: mark them empty (0xFFFF, the maximum),
                    // then h bubble passes (adjacent compare-swaps) move the h holes
                    // of a bucket behind its values; h = the warp's largest
                    // per-bucket duplicate count (usually 0 or 1)
                    const uint32_t h = __reduce_max_sync(__activemask(), max(dsum & 0xFFFFu, dsum >> 16));
                    if (h) {
                        uint32_t prev = x[0];
#pragma unroll
                        for (int k2 = 1; k2 < 16; ++k2) {
                            const uint32_t cur = x[k2];
                            x[k2] = cur | __vcmpeq2(cur, prev);
                            prev = cur;
                        }
#pragma unroll 1
                        for (uint32_t ps = 0; ps < h; ++ps) {
#pragma unroll
                            for (int k2 = 0; k2 < 15; ++k2) cswap2(x[k2], x[k2 + 1]);
                        }
                    }
                }
                if (nn.x <= kSlots) res.x = nn.x - (dsum & 0xFFFFu);
                if (nn.y <= kSlots) res.y = nn.y - (dsum >> 16);
                reinterpret_cast<uint2*>(bcnt)[m] = res;
                // an overflowed bucket keeps its raw slots for the overflow pass
#pragma unroll
                for (int sl = 0; sl < 16; ++sl) tabw[sl * MPP + m] = (x[sl] & keep) | (tabw[sl * MPP + m] & ~keep);
            }
            publish_next();  // (after PT's pass-A share, which is the smallest)
            __syncthreads();
            fallback = s_flag != 0;
        } else {
            publish_next();
            __syncthreads();  // (the published plan of row i+1 becomes visible)
        }
        const RowPlan N = s_plan[(it + 1) & 1];
        pf_issue(N);  // row i+1's first descriptor batch: loads in flight through the rest of the row
        const uint32_t nob = s_nob;
        if (!fallback && nob) {
            // ---- overflow buckets: one warp each, <= 32 values sorted across lanes
            const uint32_t novf = s_novf;
            uint32_t* wb = wbuf + wib * 32;
            for (uint32_t j = wib; j < nob; j += NW) {
                const uint32_t b = obl[j];
                const idx_t base = clo + b * W;
                uint32_t filled = kSlots;
                for (uint32_t i0 = 0; i0 < novf; i0 += 32) {
                    const uint32_t i = i0 + lane;
                    const idx_t cv = i < novf ? ovl[i] : kEmpty;
                    const bool match = cv != kEmpty && (__umulhi(cv - clo, M) >> l) == b;
                    const uint32_t mm = __ballot_sync(FULL, match);
                    const uint32_t rank = filled + __popc(mm & lt);
                    if (match && rank < 32) wb[rank] = cv;
                    filled += __popc(mm);
                }
                __syncwarp();
                if (filled > 32) {  // warp-uniform
                    if (lane == 0) s_flag = 1;
                    continue;
                }
                idx_t xv[1];
                xv[0] = lane < kSlots ? base + tab16[lane * (2 * MPP) + b] : (lane < filled ? wb[lane] : kEmpty);
                __syncwarp();
                warp_bitonic_sort<1>(xv);
                const idx_t prev = __shfl_up_sync(FULL, xv[0], 1);
                const bool uniq = xv[0] != kEmpty && (lane == 0 || xv[0] != prev);
                const uint32_t um = __ballot_sync(FULL, uniq);
                const uint32_t mcnt = __popc(um), rank = __popc(um & lt);
                // the first 16 distinct values go back to the bucket's slots
                // (0xFFFF-padded), the rest to the pool (extras <= list entries)
                const uint32_t extras = mcnt > kSlots ? mcnt - kSlots : 0u;
                uint32_t off = 0;
                if (lane == 0 && extras) off = atomicAdd(&s_pool, extras);
                off = __shfl_sync(FULL, off, 0);
                if (uniq) {
                    const uint16_t o = uint16_t(xv[0] - base);
                    if (rank < kSlots) tab16[rank * (2 * MPP) + b] = o; else pool[off + rank - kSlots] = o;
                }
                if (lane < kSlots && lane >= mcnt) tab16[lane * (2 * MPP) + b] = 0xFFFFu;
                if (lane == 0) obcnt[j] = (mcnt << 16) | off;
            }
            __syncthreads();
            fallback = s_flag != 0;
        }
        if (fallback) {
            if (threadIdx.x == 0) push_fallback(r, P.rec.chi - P.rec.clo, ovf_rows, ovf_cnt);
        } else {
            PROBE(5);
            // ---- multi-scan: output offset of every owned pair (one barrier) -----
            auto bucket_count = [&](uint32_t x) { return (x & kOvfFlag) ? obcnt[x & ~kOvfFlag] >> 16 : x; };
            uint32_t cpair[KP], inc[KP];
#pragma unroll
            for (uint32_t i = 0; i < KP; ++i) {
                const uint32_t m = threadIdx.x + i * THREADS;
                cpair[i] = 0;
                if (m < np) {
                    const uint2 nn = reinterpret_cast<const uint2*>(bcnt)[m];
                    cpair[i] = bucket_count(nn.x) + bucket_count(nn.y);
                }
                inc[i] = warp_inclusive_scan(cpair[i]);
                if (lane == 31) s_wt[i][wib] = inc[i];
            }
            __syncthreads();
            // every warp scans the (round, warp) totals itself
            uint32_t carry = 0;
#pragma unroll
            for (uint32_t i = 0; i < KP; ++i) {
                const uint32_t v = lane < NW ? s_wt[i][lane] : 0u;
                const uint32_t vi = warp_inclusive_scan(v);
                const uint32_t wpre = __shfl_sync(FULL, vi - v, wib);  // (all lanes: not inside the branch)
                const uint32_t m = threadIdx.x + i * THREADS;
                if (m < np) poff[m] = carry + wpre + inc[i] - cpair[i];
                carry += __shfl_sync(FULL, vi, 31);
            }
            if (threadIdx.x == 0) counts[r] = carry;
            __syncwarp();
#ifndef SPBLA_NO_L2PF
            pf_l2(N);  // (the descriptors were loaded before the overflow pass and the multi-scan)
#endif
            PROBE(6);
            // ---- pass B: warp-cooperative emission of the warp's own pairs --------
            // (pairs 32w + i*THREADS + j were sorted and scanned by this warp's
            // lanes: no barrier needed).  Lane = (pair m0 + lane/16, slot lane%16):
            // one word holds slot s of both buckets of the pair; the buckets are
            // compacted, so slot s of bucket 2m goes to out[poff[m] + s] and of
            // bucket 2m+1 to out[poff[m] + count(2m) + s].  Each store writes two
            // runs of <= 16 consecutive columns.  The lane also restores its word.
            // lane = (pair g of 8, slots 4t .. 4t+3): 4 lanes per pair, each
            // reading four table words (banks 8t + 2k + g: conflict-free with
            // MPP = 2 mod 32) and storing up to 8 values.  A word holds slot s
            // of both buckets of the pair, so the dedup runs in 16x2 SIMD: a
            // slot is kept if valid and not equal to the previous slot (the
            // previous lane's last word for k = 0); its output position is the
            // number of kept slots before it (packed per-bucket counts,
            // exclusive scan over the pair's 4 lanes)
            const uint32_t t8 = lane & 3u, g4 = lane >> 2;
#pragma unroll 1
            for (uint32_t i = 0; i < KP; ++i) {
                const uint32_t mb = i * THREADS + wib * 32;
                if (mb >= np) break;
                const uint32_t jn = min(32u, np - mb);
#pragma unroll 1
                for (uint32_t j = 0; j < jn; j += 8) {
                    // past the row's last pair (np <= m < mb + 32 <= MP: MP and mb
                    // are multiples of 32) a lane group works on a pair this row
                    // never touched: its words are empty and its counters zero,
                    // so it emits nothing and rewrites clean values that no
                    // other lane reads (no aliasing of a live pair)
                    const uint32_t m = mb + j + g4;
                    uint32_t* wp = tabw + (4 * t8) * MPP + m;
                    uint32_t wv[4];
#pragma unroll
                    for (int k = 0; k < 4; ++k) wv[k] = wp[k * MPP];
#pragma unroll
                    for (int k = 0; k < 4; ++k) wp[k * MPP] = 0xFFFFFFFFu;
                    uint32_t inc[4], ex;
                    if (DEDUP_B) {
                        uint32_t prevw = __shfl_up_sync(FULL, wv[3], 1, 4);
                        if (t8 == 0) prevw = 0xFFFFFFFFu;
                        uint32_t keep[4], cnt = 0;
#pragma unroll
                        for (int k = 0; k < 4; ++k)
                            keep[k] = __vcmpne2(wv[k], 0xFFFFFFFFu) & ~__vcmpeq2(wv[k], k ? wv[k - 1] : prevw);
#pragma unroll
                        for (int k = 0; k < 4; ++k) {
                            inc[k] = cnt;  // kept slots of this lane before slot k (packed)
                            cnt += keep[k] & 0x00010001u;
                            wv[k] |= ~keep[k];  // dropped slots read as empty below
                        }
                        uint32_t sc = cnt;  // inclusive scan of the packed counts over the 4 lanes
                        uint32_t y = __shfl_up_sync(FULL, sc, 1, 4);
                        if (t8 >= 1) sc += y;
                        y = __shfl_up_sync(FULL, sc, 2, 4);
                        if (t8 >= 2) sc += y;
                        ex = sc - cnt;
                    } else {  // buckets already compacted: slot s goes to position s
#pragma unroll
                        for (int k = 0; k < 4; ++k) inc[k] = uint32_t(k) * 0x00010001u;
                        ex = 4 * t8 * 0x00010001u;
                    }
                    // (for a pair past np: zero counters, a stale offset, and every
                    // store predicated off)
                    const uint2 nn = reinterpret_cast<const uint2*>(bcnt)[m];
                    const uint32_t pm = poff[m];
                    const uint32_t c0 = (nn.x & kOvfFlag) ? obcnt[nn.x & ~kOvfFlag] >> 16 : nn.x;
                    const uint32_t base0 = clo + m * (2 * W), base1 = base0 + W;
                    idx_t* o0 = out + (pm + (ex & 0xFFFFu));
                    idx_t* o1 = out + (pm + c0 + (ex >> 16));
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        st_if(o0 + (inc[k] & 0xFFFFu), base0 + (wv[k] & 0xFFFFu), (wv[k] & 0xFFFFu) != 0xFFFFu);
#pragma unroll
                    for (int k = 0; k < 4; ++k)
                        st_if(o1 + (inc[k] >> 16), base1 + (wv[k] >> 16), (wv[k] >> 16) != 0xFFFFu);
                    __syncwarp();  // the group's lanes have read the pair's counters
                    if (t8 == 0) {
                        if ((nn.x | nn.y) & kOvfFlag) {  // overflowed bucket: its sorted extras follow the slots
                            if (nn.x & kOvfFlag) {
                                const uint32_t e = obcnt[nn.x & ~kOvfFlag], mc = e >> 16, off = e & 0xFFFFu;
                                for (uint32_t q = kSlots; q < mc; ++q) out[pm + q] = base0 + pool[off + q - kSlots];
                            }
                            if (nn.y & kOvfFlag) {
                                const uint32_t e = obcnt[nn.y & ~kOvfFlag], mc = e >> 16, off = e & 0xFFFFu;
                                for (uint32_t q = kSlots; q < mc; ++q) out[pm + c0 + q] = base1 + pool[off + q - kSlots];
                            }
                        }
                        reinterpret_cast<uint2*>(bcnt)[m] = make_uint2(0u, 0u);
                    }
                }
            }
            clear_row_flags();
            pf_commit(N);
            __syncthreads();
            PROBE(7);
            PROBE_PRINT("hash", P.rec.u, P.rec.nseg);
            continue;
        }
        // ---- fallback: restore the pairs this row dirtied (each thread its own) --
        __syncthreads();  // (every thread is past its reads of the row's flags)
        // (pass A touched only owned pairs; inserts and the overflow pass
        // touched pairs < np, all of which have an owner)
#pragma unroll 1
        for (uint32_t m = threadIdx.x; m < np; m += THREADS) {
#pragma unroll
            for (int sl = 0; sl < 16; ++sl) tabw[sl * MPP + m] = 0xFFFFFFFFu;
            reinterpret_cast<uint2*>(bcnt)[m] = make_uint2(0u, 0u);
        }
        clear_row_flags();
        pf_commit(N);
        __syncthreads();
    }
}

// ---- 4c. block bitmap bin ----------------------------------------------------
// dynamic smem: sd_ptr[BATCH] | sd_end[BATCH] | bm[BITS/32] | top[BITS/1024]
// Two configs:
// * 256 threads x 256 Ki-bit windows, 6 blocks per SM (TOPLVL: hash-bin rows
//   that fell back - e.g. duplicate-heavy closure rows - and whose span fits
//   two windows): two levels, top bit t set <=> bm word t may be non-zero;
//   emission walks the top level, so clearing and emitting cost O(words
//   touched + BITS/1024) -- those rows are sparse in their window.
// * 1024 threads x 1.5 Mi-bit windows, one block per SM (the dense bin: rows
//   with > 40960 products, at least ~1 product per 40 columns of the span):
//   one level -- the products set bits with non-returning atomics and the
//   emission walks the window's words directly (a count pass and an emit
//   pass); the top-level words serve as the gather's segment lookup table
//   (sd_first) instead.
template <int THREADS, uint32_t BATCH, int FLATU, uint32_t BITS, bool FCOUNT, bool TOPLVL>
__global__ void __launch_bounds__(THREADS)
dense_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ bounds,
                 const uint2* __restrict__ range, idx_t ncols, idx_t* __restrict__ scratch,
                 const uint64_t* __restrict__ soff, const uint64_t* __restrict__ ub, uint32_t* __restrict__ counts,
                 uint32_t* __restrict__ work) {
    constexpr int NW = THREADS / 32;
    constexpr uint32_t kWords = BITS / 32, kTop = kWords / 32;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const idx_t** sd_ptr = reinterpret_cast<const idx_t**>(smem_raw);
    uint32_t* sd_end = reinterpret_cast<uint32_t*>(smem_raw + BATCH * sizeof(void*));
    uint32_t* bm = reinterpret_cast<uint32_t*>(smem_raw + BATCH * (sizeof(void*) + sizeof(uint32_t)));
    uint32_t* top = bm + kWords;
    uint32_t* sd_first = TOPLVL ? nullptr : top;  // (one level: the top words hold the segment lookup table)
    static_assert(!FCOUNT || TOPLVL, "the gather-time count needs the top level");
    __shared__ uint32_t s_w[33];
    const unsigned lane = lane_id(), wib = threadIdx.x >> 5;
    fill_words(bm, kWords + kTop, 0u, THREADS);  // kept clean between rows
    __syncthreads();
    // thread 0 claims a row one ahead and loads its row id during the
    // current row (the claim and the id load left the block idle at every
    // row start)
    __shared__ uint32_t s_item2[2];
    __shared__ idx_t s_r2[2];
    const uint32_t lo_b = bounds[0], hi_b = bounds[1];
    uint32_t c1 = 0;  // (thread 0) claimed item of the next row
    if (threadIdx.x == 0) {
        const uint32_t c0 = lo_b + atomicAdd(work, 1u);
        s_item2[0] = c0;
        if (c0 < hi_b) s_r2[0] = rows[c0];
        c1 = c0 < hi_b ? lo_b + atomicAdd(work, 1u) : hi_b;
    }
    __syncthreads();
#pragma unroll 1
    for (uint32_t it = 0;; ++it) {
        const uint32_t cur = it & 1u;
        const uint32_t item = s_item2[cur];
        if (item >= hi_b) break;
        const idx_t r = s_r2[cur];
        idx_t rn = 0;
        uint32_t c2 = hi_b;
        if (threadIdx.x == 0 && c1 < hi_b) {
            rn = rows[c1];
            c2 = lo_b + atomicAdd(work, 1u);
        }
        uint32_t clo = 0, chi = ncols - 1;
        if (range) {
            const uint2 rg = range[r];
            clo = rg.x;
            chi = rg.y;
        }
        const uint64_t span = uint64_t(chi) - clo + 1;
        const uint32_t nwin = uint32_t((span + BITS - 1) / BITS);
        idx_t* out = scratch + soff[r];
        uint32_t written = 0;
        // Partition mode (a span of more than three windows, e.g. a heavy row
        // over 2^26 columns): instead of one gather per window, count the
        // products per window (gather 1), scatter them by window into the
        // row's own output region (gather 2; its capacity holds every product
        // when ub <= ncols), then each window reads only its slice.  The
        // window-w emission writes below the start of slice w+1 (distinct <=
        // products), so it never overwrites an unread slice.  Two gathers
        // and a slice pass per row, whatever the number of windows.
        const uint64_t prods = ub[r] & kUbValue;
        const bool part = nwin > SPBLA_PART_MIN && prods <= soff[r + 1] - soff[r] && nwin < 2 * BATCH;
        uint32_t* wcur = bm;               // (partition mode, during the gathers) per-window cursors
        uint32_t* wbeg = bm + kWords / 2;  // ... and slice starts (nwin + 1 entries)
        uint32_t* slb = reinterpret_cast<uint32_t*>(sd_ptr);  // slice bounds while the windows run
        if (part) {
            for (uint32_t i = threadIdx.x; i < nwin; i += THREADS) wcur[i] = 0u;
            __syncthreads();
            block_products<THREADS, FLATU>(src, r, seg_base(src, r), num_segs(src, r), sd_ptr, sd_end, nullptr, BATCH,
                                           false, [&](idx_t c) { atomicAdd(&wcur[(c - clo) / BITS], 1u); });
            if (threadIdx.x == 0) {  // exclusive scan of < 2*BATCH window counts (rare rows: serial is fine)
                uint32_t acc = 0;
                for (uint32_t i = 0; i < nwin; ++i) {
                    const uint32_t v = wcur[i];
                    wbeg[i] = acc;
                    wcur[i] = acc;
                    acc += v;
                }
                wbeg[nwin] = acc;
            }
            __syncthreads();
            block_products<THREADS, FLATU>(src, r, seg_base(src, r), num_segs(src, r), sd_ptr, sd_end, nullptr, BATCH,
                                           false, [&](idx_t c) { out[atomicAdd(&wcur[(c - clo) / BITS], 1u)] = c; });
            // (the barrier ending the gather orders the scatter before the slice reads)
            for (uint32_t i = threadIdx.x; i <= nwin; i += THREADS) slb[i] = wbeg[i];  // descriptors are dead now
            __syncthreads();
            for (uint32_t i = threadIdx.x; i < kWords; i += THREADS) bm[i] = 0u;  // the counters lived in the bitmap
            __syncthreads();
        }
        for (uint32_t w = 0; w < nwin; ++w) {
            const uint64_t wlo = uint64_t(clo) + uint64_t(w) * BITS;
            const uint64_t whi = min(wlo + BITS, uint64_t(chi) + 1);
            const uint32_t sb = part ? slb[w] : 0u, se = part ? slb[w + 1] : 0u;  // this window's slice of out
            // the window's used top words are split evenly over the warps
            // (a fixed split left the warps outside the row's span idle)
            const uint32_t used = uint32_t((whi - wlo + 1023) >> 10);
            const uint32_t tcw = (used + NW - 1) / NW;
            const uint32_t tb = min(used, wib * tcw), te = min(used, tb + tcw);
            // FCOUNT: every newly set bit is counted for its owner warp during
            // the gather (s_w is clean before the gather's staging barrier),
            // so the emission needs one walk instead of two
            if (FCOUNT && threadIdx.x < NW) s_w[threadIdx.x] = 0u;
            auto set_bit = [&](idx_t c) {
                if (c >= wlo && c < whi) {
                    const uint32_t d = uint32_t(c - wlo);
                    const uint32_t bit = 1u << (d & 31);
                    if (TOPLVL) {
                        const uint32_t old = atomicOr(&bm[d >> 5], bit);
                        if (old == 0) atomicOr(&top[d >> 10], 1u << ((d >> 5) & 31));
                        if (FCOUNT && !(old & bit)) atomicAdd(&s_w[(d >> 10) / tcw], 1u);
                    } else {
                        atomicOr(&bm[d >> 5], bit);  // (result unused: no wait on the atomic)
                    }
                }
            };
            if (part) {  // this window's slice: coalesced reads of the scattered products
                if (FCOUNT) __syncthreads();  // (the s_w clear before any count)
                for (uint32_t i = sb + threadIdx.x; i < se; i += THREADS) set_bit(out[i]);
                __syncthreads();
            } else {
                block_products<THREADS, FLATU>(src, r, seg_base(src, r), num_segs(src, r), sd_ptr, sd_end, sd_first, BATCH,
                                               false, set_bit, nullptr, kTop);
            }
            if (!TOPLVL) {
                // one level: warp w owns the words [wb, we) of the window
                // (32 top-word spans); a count pass, a scan, an emit pass that
                // also clears the words
                const uint32_t nwd = uint32_t((whi - wlo + 31) >> 5);
                const uint32_t wb = min(nwd, tb * 32), we = min(nwd, te * 32);
                uint32_t cnt = 0;
                for (uint32_t i = wb + lane; i < we; i += 32) cnt += __popc(bm[i]);
                cnt = warp_sum(cnt);
                if (lane == 0) s_w[wib] = cnt;
                __syncthreads();
                scan_warp_counts<NW>(s_w);
                uint32_t pos = s_w[wib];
                for (uint32_t i0 = wb; i0 < we; i0 += 32) {
                    const uint32_t i = i0 + lane;
                    uint32_t word = i < we ? bm[i] : 0u;
                    if (!__any_sync(FULL, word != 0)) continue;  // warp-uniform
                    if (word) bm[i] = 0u;  // clean for the next row/window
                    const uint32_t c = __popc(word);
                    const uint32_t inc = warp_inclusive_scan(c);
                    uint32_t o = pos + inc - c;
                    const uint64_t colbase = wlo + (uint64_t(i) << 5);
                    while (word) {
                        const int bit = __ffs(word) - 1;
                        word &= word - 1;
                        out[written + o++] = idx_t(colbase + bit);
                    }
                    pos += __shfl_sync(FULL, inc, 31);
                }
            } else {
                // emission over the top level: warp w owns top words [tb, te),
                // read 32 at a time (one per lane); a ballot gives the non-zero
                // ones and the warp visits only those (rows of a few hundred
                // columns leave most top words empty: the per-word loop was the
                // kernel's largest instruction count)
                if (!FCOUNT) {  // (FCOUNT: the gather ended with a barrier after the counts)
                    uint32_t cnt = 0;
                    for (uint32_t t0 = tb; t0 < te; t0 += 32) {
                        const uint32_t tl = t0 + lane < te ? top[t0 + lane] : 0u;
                        for (uint32_t m = __ballot_sync(FULL, tl != 0); m; m &= m - 1) {  // warp-uniform
                            const uint32_t j = __ffs(m) - 1, t = t0 + j;
                            const uint32_t tw = __shfl_sync(FULL, tl, j);
                            const uint32_t word = (tw >> lane) & 1u ? bm[t * 32 + lane] : 0u;
                            cnt += __popc(word);
                        }
                    }
                    cnt = warp_sum(cnt);
                    if (lane == 0) s_w[wib] = cnt;
                    __syncthreads();
                }
                scan_warp_counts<NW>(s_w);
                uint32_t pos = s_w[wib];
                for (uint32_t t0 = tb; t0 < te; t0 += 32) {
                    const uint32_t tl = t0 + lane < te ? top[t0 + lane] : 0u;
                    for (uint32_t m = __ballot_sync(FULL, tl != 0); m; m &= m - 1) {
                        const uint32_t j = __ffs(m) - 1, t = t0 + j;
                        const uint32_t tw = __shfl_sync(FULL, tl, j);
                        uint32_t word = (tw >> lane) & 1u ? bm[t * 32 + lane] : 0u;
                        if ((tw >> lane) & 1u) bm[t * 32 + lane] = 0u;  // clean for the next row/window
                        const uint32_t c = __popc(word);
                        const uint32_t inc = warp_inclusive_scan(c);
                        uint32_t o = pos + inc - c;
                        const uint64_t colbase = wlo + (uint64_t(t * 32 + lane) << 5);
                        while (word) {
                            const int bit = __ffs(word) - 1;
                            word &= word - 1;
                            out[written + o++] = idx_t(colbase + bit);
                        }
                        pos += __shfl_sync(FULL, inc, 31);
                    }
                    if (tl) top[t0 + lane] = 0u;  // (each lane its own top word; tw came by shuffle)
                }
            }
            written += s_w[32];
            __syncthreads();
        }
        if (threadIdx.x == 0) {
            counts[r] = written;
            s_item2[cur ^ 1u] = c1;
            s_r2[cur ^ 1u] = rn;
            c1 = c2;
        }
        __syncthreads();
    }
}

// ---- 1. binning ------------------------------------------------------------
__global__ void bin_count_kernel(const uint64_t* __restrict__ ub, const uint2* __restrict__ range, idx_t nrows,
                                 idx_t ncols, uint64_t* __restrict__ cap, uint8_t* __restrict__ bin,
                                 uint32_t* __restrict__ counts, uint32_t* __restrict__ hist) {
    __shared__ uint32_t sh[kNumBins];
    if (threadIdx.x < kNumBins) sh[threadIdx.x] = 0;
    __syncthreads();
    for (size_t r = blockIdx.x * size_t(blockDim.x) + threadIdx.x; r < nrows;
         r += size_t(gridDim.x) * blockDim.x) {
        const uint64_t uf = ub[r], u = uf & kUbValue;
        cap[r] = u < ncols ? u : uint64_t(ncols);
        int b = bin_of(u);
        // a duplicate-heavy row (flagged by the producer) whose span fits two
        // small bitmap windows skips the hash bins: its duplicates would
        // overflow the 16-slot buckets and send it to the same bitmap kernel
        // after a wasted gather
        if (uf & kUbCopyFlag)  // (exact count: the copy kernel writes the row as it is)
            b = BIN_COPY;
        else if ((uf & kUbDupFlag) && u <= 256)  // (the warp bitonic bin is indifferent to duplicates)
            b = u <= 32 ? BIN_W1 : u <= 64 ? BIN_W2 : u <= 128 ? BIN_W4 : BIN_W8;
        else if ((uf & kUbDupFlag) && b >= BIN_H0 && b <= BIN_H6 && range && range[r].y - range[r].x < kSmallSpan)
            b = BIN_DUP;
        bin[r] = uint8_t(b);
        if (b == BIN_EMPTY) counts[r] = 0;
        if (b == BIN_COPY) counts[r] = uint32_t(u);
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

// The hash bins' 40-B work record of row r (row, ub, span, scratch offset,
// descriptor base, segment count).
__device__ __forceinline__ RowRec make_rec(const SegSource& src, idx_t r, const uint64_t* __restrict__ ub,
                                          const uint2* __restrict__ range, idx_t ncols,
                                          const uint64_t* __restrict__ soff) {
    RowRec x;
    x.r = r;
    x.u = uint32_t(min(ub[r] & kUbValue, uint64_t(0xFFFFFFFFu)));
    if (range) {
        const uint2 rg = range[r];
        x.clo = rg.x;
        x.chi = rg.y;
    } else {
        x.clo = 0;
        x.chi = ncols - 1;
    }
    x.out = soff[r];
    x.seg = seg_base(src, r);
    x.nseg = num_segs(src, r);
    x.pad = 0;
    return x;
}

// rows[] lists per bin; a hash-bin row's work record is written at its item
// position at the same time (recs indexed by item)
__global__ void bin_scatter_kernel(const uint8_t* __restrict__ bin, idx_t nrows,
                                   uint32_t* __restrict__ cursor, idx_t* __restrict__ rows, SegSource src,
                                   const uint64_t* __restrict__ ub, const uint2* __restrict__ range, idx_t ncols,
                                   const uint64_t* __restrict__ soff, RowRec* __restrict__ recs) {
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
        if (b > 0) {
            const uint32_t item = sh_base[b] + local;
            rows[item] = idx_t(r);
            if (b >= BIN_H0 && b <= BIN_H6) recs[item] = make_rec(src, idx_t(r), ub, range, ncols, soff);
        }
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

// ---- 4d. copy bin: rows whose only segment is the output (accumulate input
// of a row without products, e.g. most rows of C += C Delta): warp per row
__global__ void __launch_bounds__(256)
copy_bin_kernel(SegSource src, const idx_t* __restrict__ rows, const uint32_t* __restrict__ binoff,
                idx_t* __restrict__ scratch, const uint64_t* __restrict__ soff) {
    const unsigned lane = lane_id();
    const uint32_t lo = binoff[BIN_COPY], hi = binoff[BIN_COPY + 1];
    const uint32_t nwarps = gridDim.x * (blockDim.x >> 5);
    for (uint32_t t = lo + blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); t < hi; t += nwarps) {
        const idx_t r = rows[t];
        uint32_t len;
        const idx_t* p = get_seg(src, r, 0, len);
        idx_t* o = scratch + soff[r];
        for (uint32_t i = lane; i < len; i += 32) o[i] = p[i];
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

// In-place compaction: the rows sit in one buffer at their capacity offsets
// soff[r] >= rowptr[r]; move every row down to rowptr[r] without a second
// buffer.  Destination tiles of kCT elements are claimed in increasing order
// (atomic ticket).  A tile first loads its elements into registers and
// publishes "read done"; it may then overwrite [d0, d1) once every earlier
// tile that reads sources inside [d0, d1) has published.  Sources of
// destination d lie at d + slack(row(d)), slack = soff - rowptr nondecreasing,
// so those tiles are the ones in [t - 1 - slack(r0) / kCT, t).  Waits only
// point at lower tickets, held by running blocks that never wait before
// publishing, so the chain cannot deadlock.  Tiles with zero slack are
// already in place and only publish.
#ifndef SPBLA_CT_T  // threads, words per thread, blocks per SM (overridable for a sweep)
// (configs[4] sweep, round 2: 128x32x8 14.08 ms < 96x32x10 14.25 < 128x24x10
// 14.33 < 256x32x4 14.73 < 64x32x16 15.31 < 256x16x8 16.44 < 512x16x4 17.27)
#define SPBLA_CT_T 128
#define SPBLA_CT_I 32
#define SPBLA_CT_B 8
#endif
constexpr int kCThreads = SPBLA_CT_T, kCItems = SPBLA_CT_I, kCMinB = SPBLA_CT_B;
constexpr uint32_t kCT = kCThreads * kCItems;  // 4096 elements per tile
constexpr uint32_t kCStage = 1024;             // rows of a tile staged in smem

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// index of the row holding position d: largest r in [lo, hi] with rp[r] <= d
__device__ __forceinline__ uint32_t row_of(const uint64_t* rp, uint32_t lo, uint32_t hi, uint64_t d) {
    while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (rp[mid] <= d) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// tile_row[t] = row holding position t*kCT (t < ntiles), tile_row[ntiles] =
// nrows-1; src_lo[t] = source position of the tile's first element.
__global__ void tile_rows_kernel(const uint64_t* __restrict__ rowptr, const uint64_t* __restrict__ soff,
                                 idx_t nrows, uint64_t ntiles, uint32_t* __restrict__ tile_row,
                                 uint64_t* __restrict__ src_lo) {
    for (size_t r = blockIdx.x * size_t(blockDim.x) + threadIdx.x; r < nrows; r += size_t(gridDim.x) * blockDim.x) {
        const uint64_t b = rowptr[r], e = rowptr[r + 1];
        for (uint64_t t = (b + kCT - 1) / kCT; t * kCT < e; ++t) {
            tile_row[t] = uint32_t(r);
            src_lo[t] = t * kCT + (soff[r] - b);
        }
        if (r == nrows - 1) tile_row[ntiles] = uint32_t(r);
    }
}

// Tiles that tile t must wait for: the j < t whose sources overlap [d0, d1).
// src is strictly increasing in the destination, so tile j's sources lie in
// [src_lo[j], src_lo[j+1]).  Overlap needs src_lo[j+1] > d0 and
// src_lo[j] < d1: j in [J0 - 1, J1) with J0 the first tile whose src_lo
// exceeds d0 and J1 the first whose src_lo reaches d1 (usually 1-2 tiles).
__global__ void tile_deps_kernel(const uint64_t* __restrict__ src_lo, uint64_t ntiles, uint64_t nnz,
                                 uint2* __restrict__ wait_range) {
    for (size_t t = blockIdx.x * size_t(blockDim.x) + threadIdx.x; t < ntiles; t += size_t(gridDim.x) * blockDim.x) {
        const uint64_t d0 = t * kCT, d1 = min(d0 + kCT, nnz);
        // src_lo[j] <= j*kCT + slack(t) for j <= t: the answers lie within `back` tiles
        const uint64_t back = (src_lo[t] - d0) / kCT + 2;
        const uint64_t start = t > back ? t - back : 0;
        auto first_above = [&](uint64_t x, bool strict) {  // first j in [start, t] with src_lo[j] > x (>= x)
            uint64_t lo = start, hi = t;
            while (lo < hi) {
                const uint64_t mid = (lo + hi) >> 1;
                const uint64_t v = src_lo[mid];
                if (strict ? v <= x : v < x) lo = mid + 1; else hi = mid;
            }
            return lo;
        };
        const uint64_t j0 = first_above(d0, true);
        const uint64_t j1 = first_above(d1, false);
        wait_range[t] = make_uint2(uint32_t(j0 > 0 ? j0 - 1 : 0), uint32_t(min(j1, uint64_t(t))));
    }
}

// INPLACE = false: the same tile copy from the scratch buf into a separate
// exact-size buffer dst (no read/write ordering between tiles: a plain
// streaming copy)
template <bool INPLACE>
__global__ void __launch_bounds__(kCThreads, kCMinB)
compact_inplace_kernel(idx_t* buf, idx_t* dst, const uint64_t* __restrict__ soff, const uint64_t* __restrict__ rowptr,
                       const uint32_t* __restrict__ tile_row, const uint2* __restrict__ wait_range,
                       idx_t nrows, uint64_t nnz, uint32_t* flags, uint32_t* ticket) {
    // staged rows of the tile in tile-local coordinates: s_beg[i] = start of
    // row r0+i relative to d0 (clamped to 0), s_beg[nr] = kCT; s_src[i] =
    // source pointer of tile-local position 0 for that row (buf + d0 + slack)
    __shared__ int32_t s_beg[kCStage + 1];
    __shared__ const idx_t* s_src[kCStage];
    __shared__ uint32_t s_t, s_r0, s_r1;
    __shared__ uint2 s_w;
    const uint64_t ntiles = (nnz + kCT - 1) / kCT;
    for (;;) {
        if (threadIdx.x == 0) {
            const uint32_t t = atomicAdd(ticket, 1u);
            s_t = t;
            if (t < ntiles) {
                // rows holding d0 and (a bound on the row holding) d1-1
                s_r0 = tile_row[t];
                s_r1 = tile_row[t + 1];
                if (INPLACE) s_w = wait_range[t];
            }
        }
        __syncthreads();
        const uint32_t t = s_t;
        if (t >= ntiles) break;
        const uint64_t d0 = uint64_t(t) * kCT;
        const uint32_t n = uint32_t(min(uint64_t(kCT), nnz - d0));  // tile length
        const uint32_t r0 = s_r0, r1 = s_r1;
        const uint64_t slack1 = soff[r1] - rowptr[r1];
        if (INPLACE && slack1 == 0) {  // whole tile already in place (slack is nondecreasing)
            if (threadIdx.x == 0) st_release_u32(&flags[t], 1u);
            __syncthreads();
            continue;
        }
        const uint32_t nr = r1 - r0 + 1;
        const bool staged = nr <= kCStage;
        if (staged) {
            for (uint32_t i = threadIdx.x; i < nr; i += kCThreads) {
                const uint64_t rp = rowptr[r0 + i];
                s_beg[i] = rp <= d0 ? 0 : int32_t(min(rp - d0, uint64_t(kCT)));
                s_src[i] = buf + (d0 + (soff[r0 + i] - rp));
            }
            if (threadIdx.x == 0) s_beg[nr] = int32_t(kCT);
        }
        __syncthreads();
        // thread-owned 4-word chunks c = k*kCThreads + tid of the tile: the
        // destination is one aligned 16-B store; the chunk's 4 source words
        // (one row's run, shifted by that row's slack, any alignment) are 4
        // coalesced word loads.  The row check is per chunk, not per word.
        constexpr int kCChunks = kCItems / 4;
        idx_t v[kCItems];
        if (staged) {
            uint32_t ri = 0;
            int32_t nxt = s_beg[1];
            const idx_t* sp = s_src[0];
#pragma unroll
            for (int k = 0; k < kCChunks; ++k) {
                const int32_t e0 = 4 * (k * kCThreads + int32_t(threadIdx.x));
                if (e0 + 3 < nxt) {  // the whole chunk in the current row (rows average thousands of words)
                    // (a row whose shift is a multiple of 4 words: one 16-B
                    // load; two aligned loads and a word select for the
                    // others measured 1.5x slower)
                    if (uint32_t(e0 + 3) < n && (reinterpret_cast<uintptr_t>(sp + e0) & 15) == 0) {
                        const uint4 w = *reinterpret_cast<const uint4*>(sp + e0);
                        v[4 * k] = w.x;
                        v[4 * k + 1] = w.y;
                        v[4 * k + 2] = w.z;
                        v[4 * k + 3] = w.w;
                    } else
#pragma unroll
                    for (int j = 0; j < 4; ++j)
                        if (uint32_t(e0 + j) < n) v[4 * k + j] = sp[e0 + j];
                } else {
#pragma unroll
                    for (int j = 0; j < 4; ++j) {
                        const int32_t e = e0 + j;
                        if (e >= nxt) {  // next row(s): binary search over the staged starts
                            uint32_t lo = ri + 1, hi = nr - 1;  // last row with start <= e
                            while (lo < hi) {
                                const uint32_t mid = (lo + hi + 1) >> 1;
                                if (s_beg[mid] <= e) lo = mid; else hi = mid - 1;
                            }
                            ri = lo;
                            nxt = s_beg[ri + 1];
                            sp = s_src[ri];
                        }
                        if (uint32_t(e) < n) v[4 * k + j] = sp[e];
                    }
                }
            }
        } else {
#pragma unroll
            for (int k = 0; k < kCChunks; ++k)
#pragma unroll
                for (int j = 0; j < 4; ++j) {
                    const uint32_t e = 4 * (k * kCThreads + threadIdx.x) + j;
                    if (e < n) {
                        const uint64_t d = d0 + e;
                        const uint32_t r = row_of(rowptr, r0, r1, d);
                        v[4 * k + j] = buf[d + (soff[r] - rowptr[r])];
                    }
                }
        }
        if (INPLACE) {
            // publish "read done": the barrier orders every thread's loads before
            // thread 0's gpu-scope fence and release store
            __syncthreads();
            if (threadIdx.x == 0) {
                __threadfence();
                st_release_u32(&flags[t], 1u);
            }
            // wait for the earlier tiles that read sources inside [d0, d1)
            for (uint32_t j = s_w.x + threadIdx.x; j < s_w.y; j += kCThreads)
                while (ld_acquire_u32(&flags[j]) == 0) __nanosleep(64);
            __syncthreads();
        }
        // (out of place: each thread stores what it loaded, no barrier)
        idx_t* dp = (INPLACE ? buf : dst) + d0;  // 16-B aligned (kCT and the buffers are)
#pragma unroll
        for (int k = 0; k < kCChunks; ++k) {
            const uint32_t e0 = 4 * (k * kCThreads + threadIdx.x);
            if (e0 + 4 <= n) {
                *reinterpret_cast<uint4*>(dp + e0) = make_uint4(v[4 * k], v[4 * k + 1], v[4 * k + 2], v[4 * k + 3]);
            } else {
#pragma unroll
                for (int j = 0; j < 4; ++j)
                    if (e0 + j < n) dp[e0 + j] = v[4 * k + j];
            }
        }
        __syncthreads();  // s_beg / s_t reuse
    }
}

}  // namespace

// ------------------------------------------------------------------------------
constexpr size_t kSegBytes = sizeof(void*) + sizeof(uint32_t);
// hash bins: <threads, max buckets (= ub limit / 4), overflow slots, descriptor
// batch, blocks per SM, loads in flight>; smem per block is checked against
// the residency so each bin keeps its blocks/SM (register-limited at 40 regs)
constexpr uint32_t kDBatch = 1024;
constexpr size_t hash_smem(uint32_t threads, uint32_t batch, uint32_t buckets, uint32_t ovcap, uint32_t obcap) {
    return size_t(16) * pair_stride(buckets / 2) * sizeof(uint32_t) +          // table
           buckets * sizeof(uint32_t) + (buckets / 2) * sizeof(uint32_t) +     // counters, pair offsets
           batch * kSegBytes + first_entries(uint64_t(buckets) * 8) * sizeof(uint32_t) +
           ovcap * (sizeof(idx_t) + sizeof(uint16_t)) + obcap * 2 * sizeof(uint32_t);
}
#define HBIN_(NAME, T, UB, OVCAP, OBCAP, BATCH, PERSM, U, DB)                                       \
    constexpr int NAME##_T = T, NAME##_PERSM = PERSM, NAME##_U = U;                                \
    constexpr bool NAME##_DB = DB;                                                                 \
    constexpr uint32_t NAME##_B = uint32_t(UB / 8), NAME##_OVCAP = OVCAP, NAME##_OBCAP = OBCAP,     \
                       NAME##_BATCH = BATCH;                                                       \
    constexpr size_t NAME##_SMEM = hash_smem(T, BATCH, uint32_t(UB / 8), OVCAP, OBCAP);            \
    static_assert(PERSM * (NAME##_SMEM + 1024 + 512) <= 228 * 1024, #NAME " residency");         \
    static_assert(PERSM * T <= 2048, #NAME " threads");
// <threads, ub limit, overflow list, overflow buckets, descriptor batch, blocks/SM, loads per thread,
//  dedup in pass B (else re-sort in pass A)>
// (round-2 sweep on configs[4], tools/sweep_*.sh: 6 loads per thread for H1, H2, H6 -0.6 ms; 8 loads
//  or 5 for H3-H5, 1024 threads for H5 all slower)
// (expected per row at mean load 8 with 16 slots: list ~ub/1500, buckets ~ub/2000)
#define HBIN(NAME, ...) HBIN_(NAME, __VA_ARGS__)
#ifndef H0_CFG  // (overridable for tools/sweep.sh)
#define H0_CFG 32, kH0, 32, 16, 64, 32, 4, false
#endif
HBIN(H0, H0_CFG)
#ifndef H1_CFG  // (overridable for tools/sweep.sh)
#define H1_CFG 32, kH1, 32, 16, 32, 28, 6, false
#endif
HBIN(H1, H1_CFG)
#ifndef H2_CFG  // (overridable for tools/sweep.sh)
#define H2_CFG 64, kH2, 32, 16, 64, 18, 6, false
#endif
HBIN(H2, H2_CFG)
#ifndef H3_CFG  // (overridable for tools/sweep.sh)
#define H3_CFG 128, kH3, 64, 32, 128, 8, 6, false
#endif
HBIN(H3, H3_CFG)
#ifndef H4_CFG  // (overridable for tools/sweep.sh)
#define H4_CFG 256, kH4, 64, 32, 256, 5, 6, false
#endif
HBIN(H4, H4_CFG)
#ifndef H5_CFG  // (overridable for tools/sweep.sh)
#define H5_CFG 512, kH5, 128, 64, 256, 2, 6, false
#endif
HBIN(H5, H5_CFG)
#ifndef H6_CFG  // (overridable for tools/sweep.sh)
#define H6_CFG 1024, kH6, 192, 96, 384, 1, 6, false
#endif
HBIN(H6, H6_CFG)
#define HASHK(N, KIND) hash_bin_kernel<N##_T, N##_B, N##_OVCAP, N##_OBCAP, N##_BATCH, N##_PERSM, N##_U, N##_DB, KIND>
#define HASH0(KIND) HASHK(H0, KIND)
#define HASH1(KIND) HASHK(H1, KIND)
#define HASH2(KIND) HASHK(H2, KIND)
#define HASH3(KIND) HASHK(H3, KIND)
#define HASH4(KIND) HASHK(H4, KIND)
#define HASH5(KIND) HASHK(H5, KIND)
#define HASH6(KIND) HASHK(H6, KIND)
constexpr size_t kDSmem = kDBatch * kSegBytes + (kDenseBits / 32 + kDenseBits / 1024) * sizeof(uint32_t);
static_assert(kDSmem + 2048 <= 227 * 1024, "dense bin smem");
static_assert((kDenseBits / 1024) % 32 == 0, "dense bin: top words per warp");
#define DENSE dense_bin_kernel<1024, kDBatch, 8, kDenseBits, false, false>
constexpr uint32_t kSDenseBits = 1u << 18, kSDBatch = 192;
constexpr int kSDPerSM = 6;  // blocks per SM (the kernel is barrier/latency-bound: residency pays)
constexpr size_t kSDSmem = kSDBatch * kSegBytes + (kSDenseBits / 32 + kSDenseBits / 1024) * sizeof(uint32_t);
static_assert(kSDPerSM * (kSDSmem + 1024 + 512) <= 228 * 1024, "small dense bin residency");
#define SDENSE dense_bin_kernel<256, kSDBatch, 4, kSDenseBits, true, true>

static void ensure_attrs() {
    static int done_dev = -1;
    if (done_dev == ctx().device) return;
    CUDA_CHECK(cudaFuncSetAttribute(HASH0(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H0_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH0(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H0_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH1(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H1_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH1(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H1_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH2(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H2_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH2(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H2_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH3(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H3_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH3(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H3_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH4(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H4_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH4(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H4_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH5(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H5_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH5(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H5_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH6(0), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H6_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(HASH6(1), cudaFuncAttributeMaxDynamicSharedMemorySize, int(H6_SMEM)));
    CUDA_CHECK(cudaFuncSetAttribute(DENSE, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kDSmem)));
    CUDA_CHECK(cudaFuncSetAttribute(SDENSE, cudaFuncAttributeMaxDynamicSharedMemorySize, int(kSDSmem)));
    done_dev = ctx().device;
}

// out-of-place compaction allowed (spbla_SetCompactionMode; env SPBLA_INPLACE_COMPACT=1 turns it off)
static bool g_oop_compact = std::getenv("SPBLA_INPLACE_COMPACT") == nullptr;

void row_engine(const SegSource& src, idx_t nrows, idx_t ncols, const uint64_t* ub, const uint2* range,
                Matrix* out) {
    cudaStream_t st = ctx().stream;
    const int nsm = ctx().num_sms;
    if (nrows == 0 || ncols == 0) {
        matrix_set_empty(out);
        return;
    }
    ensure_attrs();
    trace_mark("engine start");
    // 1-3. bins
    DevBuf<uint64_t> cap(size_t(nrows) + 1);
    DevBuf<uint64_t> soff(size_t(nrows) + 1);
    DevBuf<uint8_t> bin(nrows);
    DevBuf<uint32_t> counts(nrows);
    // meta: hist[15] binoff[16] cursor[15] work[9] ovf[4] work2[1] work3[1]
    DevBuf<uint32_t> meta(64);
    uint32_t* hist = meta.p;
    uint32_t* binoff = meta.p + 15;
    uint32_t* cursor = meta.p + 31;
    uint32_t* work = meta.p + 46;
    uint32_t* ovf = meta.p + 55;  // fallback lists: [0, ovf[1]) and [nrows, ovf[3])
    uint32_t* work2 = meta.p + 59;
    uint32_t* work3 = meta.p + 60;
    memset_async(meta.p, 0, meta.n * sizeof(uint32_t));
    {
        const uint32_t lst1[2] = {nrows, nrows};
        copy_async(ovf + 2, lst1, sizeof(lst1), cudaMemcpyHostToDevice);
    }
    const unsigned gb = (unsigned)std::min<uint64_t>(ceil_div(nrows, 256), uint64_t(nsm) * 8);
    bin_count_kernel<<<gb, 256, 0, st>>>(ub, range, nrows, ncols, cap.p, bin.p, counts.p, hist);
    count_launch();
    check_launch("bin_count_kernel");
    exclusive_scan_u64(cap.p, soff.p, nrows);
    bin_offsets_kernel<<<1, 32, 0, st>>>(hist, binoff, cursor);
    count_launch();
    DevBuf<idx_t> rows(nrows);
    DevBuf<RowRec> recs(nrows);  // indexed by bin item (only hash-bin items are written)
    bin_scatter_kernel<<<gb, 256, 0, st>>>(bin.p, nrows, cursor, rows.p, src, ub, range, ncols, soff.p, recs.p);
    count_launch();
    check_launch("bin_scatter_kernel");
    // one synchronisation: the scratch size and the bin histogram (empty bins
    // are not launched; small ones get only as many blocks as rows)
    uint64_t h[2];
    uint32_t hcnt[kNumBins];
    read_words2(soff.p + nrows, h, 1, hist, hcnt, sizeof(hcnt));
    const uint64_t scratch_total = h[0];
    auto grid_for = [&](int b, uint32_t full) { return std::min<uint32_t>(full, hcnt[b]); };
    uint32_t hash_rows = 0;
    for (int b = BIN_H0; b <= BIN_H6; ++b) hash_rows += hcnt[b];
    cap.release();
    bin.release();
    trace_mark("binning");
    // the scratch is matrix storage: compacted in place it becomes colidx
    DevBuf<idx_t> scratch(scratch_total, kMat);
    DevBuf<idx_t> ovf_rows(2 * size_t(nrows));

    trace_mark("scratch alloc");

    // 4. per-bin kernels, heaviest first, back to back on the library stream
    //    (persistent grids sized to the SM count x residency; rows are handed
    //    out by an atomic work counter, so heavy rows balance dynamically)
    int t;
    t = ktime_begin("dense", st);
    if (hcnt[BIN_DENSE]) {
        DENSE<<<grid_for(BIN_DENSE, nsm), 1024, kDSmem, st>>>(src, rows.p, binoff + BIN_DENSE, range, ncols,
                                                              scratch.p, soff.p, ub, counts.p, work);
        count_launch();
    }
    ktime_end(t);
    if (hcnt[BIN_COPY]) {
        t = ktime_begin("warp_bins", st);
        copy_bin_kernel<<<std::min<uint32_t>(nsm * 8, (hcnt[BIN_COPY] + 7) / 8), 256, 0, st>>>(src, rows.p, binoff,
                                                                                           scratch.p, soff.p);
        count_launch();
        ktime_end(t);
        check_launch("copy_bin_kernel");
    }
    t = ktime_begin("dense_ovf", st);
    if (hcnt[BIN_DUP]) {  // duplicate-heavy rows flagged by the producer
        SDENSE<<<std::min<uint32_t>(nsm * kSDPerSM, hcnt[BIN_DUP]), 256, kSDSmem, st>>>(
            src, rows.p, binoff + BIN_DUP, range, ncols, scratch.p, soff.p, ub, counts.p, work3);
        count_launch();
    }
    ktime_end(t);
#define LAUNCH_HASH(K, NAME, BIN, W)                                                                   \
    t = ktime_begin(#NAME, st);                                                                          \
    if (hcnt[BIN]) {                                                                                     \
        const uint32_t g = grid_for(BIN, uint32_t(nsm * NAME##_PERSM));                                  \
        if (src.kind == 0)                                                                               \
            K(0)<<<g, NAME##_T, NAME##_SMEM, st>>>(src, recs.p, binoff + BIN, scratch.p, counts.p, work + W, \
                                                   ovf_rows.p, ovf);                                     \
        else                                                                                             \
            K(1)<<<g, NAME##_T, NAME##_SMEM, st>>>(src, recs.p, binoff + BIN, scratch.p, counts.p, work + W, \
                                                   ovf_rows.p, ovf);                                     \
        count_launch();                                                                                  \
    }                                                                                                    \
    ktime_end(t);
    LAUNCH_HASH(HASH6, H6, BIN_H6, 7)
    LAUNCH_HASH(HASH5, H5, BIN_H5, 1)
    LAUNCH_HASH(HASH4, H4, BIN_H4, 2)
    LAUNCH_HASH(HASH3, H3, BIN_H3, 3)
    LAUNCH_HASH(HASH2, H2, BIN_H2, 4)
    LAUNCH_HASH(HASH1, H1, BIN_H1, 5)
    LAUNCH_HASH(HASH0, H0, BIN_H0, 8)
#undef LAUNCH_HASH
    // rows whose hash probes ran long: bitmap path
    t = ktime_begin("dense_ovf", st);
    if (hash_rows) {  // (fallback rows come only from the hash bins)
        const uint32_t g = std::min<uint32_t>(nsm * kSDPerSM, hash_rows);
        SDENSE<<<g, 256, kSDSmem, st>>>(src, ovf_rows.p, ovf, range, ncols, scratch.p, soff.p, ub, counts.p, work2);
        DENSE<<<std::min<uint32_t>(nsm, hash_rows), 1024, kDSmem, st>>>(src, ovf_rows.p, ovf + 2, range, ncols,
                                                                        scratch.p, soff.p, ub, counts.p, work + 6);
        count_launch(2);
    }
    ktime_end(t);
    check_launch("block bins");
    const unsigned gw = nsm * 8;  // 256-thread blocks, grid-stride over bin rows
    t = ktime_begin("warp_bins", st);
#define LAUNCH_WARP(E, BIN)                                                                                \
    if (hcnt[BIN]) {                                                                                     \
        warp_bin_kernel<E><<<std::min<uint32_t>(gw, (hcnt[BIN] + 7) / 8), 256, 0, st>>>(src, rows.p, binoff, BIN, \
                                                                                        scratch.p, soff.p, counts.p); \
        count_launch();                                                                                  \
    }
    LAUNCH_WARP(8, BIN_W8)
    LAUNCH_WARP(4, BIN_W4)
    LAUNCH_WARP(2, BIN_W2)
    LAUNCH_WARP(1, BIN_W1)
#undef LAUNCH_WARP
    ktime_end(t);
    check_launch("warp_bin_kernel");
    trace_mark("bin kernels");
    // 5. row offsets
    DevBuf<off_t64> rowptr(size_t(nrows) + 1, kMat);
    exclusive_scan_u32(counts.p, rowptr.p, nrows);
    read_words(rowptr.p + nrows, h, 1);
    const uint64_t nnz = h[0];
    ovf_rows.release();
    counts.release();
    // 6. compaction: when the capacity slack is small, a tile copy -- into a
    //    separate exact-size buffer when the device has room for it (a plain
    //    streaming copy), else in place (tiles ordered by their read/write
    //    overlaps; the result keeps the scratch buffer, colidx_cap >= nnz);
    //    a large slack is copied row by row into an exact buffer
    const bool small_slack = scratch_total - nnz <= scratch_total / 8;
    DevBuf<idx_t> colidx;
    bool inplace = false;
    if (nnz && small_slack) {
        const uint64_t ntiles = ceil_div(nnz, kCT);
        inplace = !(g_oop_compact && dev_can_alloc(nnz * sizeof(idx_t), kMat));
        if (!inplace) colidx.alloc(nnz, kMat);
        // flags[ntiles] | ticket | tile_row[ntiles + 1]; src_lo[ntiles]; wait_range[ntiles]
        DevBuf<uint32_t> flags(2 * ntiles + 2);
        DevBuf<uint64_t> src_lo(ntiles);
        DevBuf<uint2> wait_range(inplace ? ntiles : 0);
        uint32_t* tile_row = flags.p + ntiles + 1;
        memset_async(flags.p, 0, (ntiles + 1) * sizeof(uint32_t));
        t = ktime_begin("compact", st);
        tile_rows_kernel<<<gb, 256, 0, st>>>(rowptr.p, soff.p, nrows, ntiles, tile_row, src_lo.p);
        if (inplace) {
            tile_deps_kernel<<<(unsigned)std::min<uint64_t>(ceil_div(ntiles, 256), uint64_t(nsm) * 8), 256, 0, st>>>(
                src_lo.p, ntiles, nnz, wait_range.p);
            compact_inplace_kernel<true><<<nsm * kCMinB * 2, kCThreads, 0, st>>>(
                scratch.p, nullptr, soff.p, rowptr.p, tile_row, wait_range.p, nrows, nnz, flags.p, flags.p + ntiles);
            count_launch(3);
        } else {
            compact_inplace_kernel<false><<<nsm * kCMinB * 2, kCThreads, 0, st>>>(
                scratch.p, colidx.p, soff.p, rowptr.p, tile_row, nullptr, nrows, nnz, flags.p, flags.p + ntiles);
            count_launch(2);
        }
        ktime_end(t);
        check_launch("compact_inplace_kernel");
    } else if (nnz) {
        colidx.alloc(nnz, kMat);
        const unsigned gc = (unsigned)std::min<uint64_t>(ceil_div(uint64_t(nrows) * 32, 256), uint64_t(nsm) * 16);
        t = ktime_begin("compact", st);
        compact_kernel<<<gc, 256, 0, st>>>(scratch.p, soff.p, rowptr.p, nrows, colidx.p);
        ktime_end(t);
        count_launch();
        check_launch("compact_kernel");
    }
    trace_mark("compact");
    size_t rcap = rowptr.n;
    if (nnz && inplace) {
        size_t ccap = scratch.n;
        matrix_replace(out, rowptr.detach(), rcap, scratch.detach(), ccap, nnz);
    } else {
        size_t ccap = colidx.n;
        matrix_replace(out, rowptr.detach(), rcap, colidx.detach(), ccap, nnz);
    }
}

void set_out_of_place_compaction(bool on) { g_oop_compact = on; }

void engine_thresholds(uint64_t* out, uint32_t* n) {
    // ub upper limits of bins W1, W2, W4, W8, H0..H6 (DENSE above)
    const uint64_t t[11] = {32, 64, 128, kWarpMaxUb, kH0, kH1, kH2, kH3, kH4, kH5, kH6};
    const uint32_t k = *n < 11 ? *n : 11;
    for (uint32_t i = 0; i < k; ++i) out[i] = t[i];
    *n = 11;
}

}  // namespace spbla
