// In-house single-pass exclusive prefix sum (decoupled look-back, Merrill &
// Garland 2016), CUB-free as the north star requires.  Used for every CSR
// row-offset array the hot path builds (MxM capacities and counts, Build
// buckets, EWiseAdd tile duplicates, Transpose, Reduce, SubMatrix).
//
// One pass: 8 B/elem read (u64 input) + 8 B/elem written; the look-back
// touches one status word per preceding tile until an inclusive prefix is
// found.
#include "common.cuh"

namespace spbla {

namespace {

constexpr int kScanThreads = 256;
constexpr int kScanItems = 16;
constexpr int kScanTile = kScanThreads * kScanItems;
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagPre = 2ull << 62;
constexpr uint64_t kValMask = (1ull << 62) - 1;

__device__ __forceinline__ void st_volatile(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ uint64_t ld_volatile(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

template <typename Tin>
__global__ void __launch_bounds__(kScanThreads)
scan_kernel(const Tin* __restrict__ in, uint64_t* __restrict__ out, size_t n,
            uint64_t* status, unsigned* tile_ctr) {
    __shared__ uint64_t sh[33];
    __shared__ unsigned s_tile;
    __shared__ uint64_t s_prefix;
    if (threadIdx.x == 0) s_tile = atomicAdd(tile_ctr, 1u);
    __syncthreads();
    const size_t tile = s_tile;
    const size_t base = tile * kScanTile + size_t(threadIdx.x) * kScanItems;
    uint64_t v[kScanItems];
    uint64_t sum = 0;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
        size_t idx = base + i;
        v[i] = idx < n ? uint64_t(in[idx]) : 0ull;
        sum += v[i];
    }
    uint64_t tot;
    uint64_t excl = block_exclusive_scan<uint64_t>(sum, sh, &tot);
    if (threadIdx.x == 0) {
        uint64_t prefix = 0;
        if (tile == 0) {
            st_volatile(&status[0], kFlagPre | tot);
        } else {
            st_volatile(&status[tile], kFlagAgg | tot);
            long t = long(tile) - 1;
            for (;;) {
                uint64_t s;
                do { s = ld_volatile(&status[t]); } while ((s >> 62) == 0);
                prefix += s & kValMask;
                if ((s >> 62) == 2) break;
                --t;
            }
            st_volatile(&status[tile], kFlagPre | (prefix + tot));
        }
        s_prefix = prefix;
    }
    __syncthreads();
    uint64_t run = s_prefix + excl;
#pragma unroll
    for (int i = 0; i < kScanItems; ++i) {
        size_t idx = base + i;
        if (idx <= n) out[idx] = run;
        run += v[i];
    }
}

template <typename Tin>
void scan_impl(const Tin* in, uint64_t* out, size_t n) {
    // n / tile + 1 tiles so that index n (the total) is always covered
    size_t ntiles = n / kScanTile + 1;
    DevBuf<uint64_t> status(ntiles + 1);
    memset_async(status.p, 0, status.n * sizeof(uint64_t));
    unsigned* ctr = reinterpret_cast<unsigned*>(status.p + ntiles);
    scan_kernel<Tin><<<(unsigned)ntiles, kScanThreads, 0, ctx().stream>>>(in, out, n, status.p, ctr);
    count_launch();
    check_launch("scan_kernel");
}

}  // namespace

void exclusive_scan_u32(const uint32_t* in, uint64_t* out, size_t n) { scan_impl<uint32_t>(in, out, n); }
void exclusive_scan_u64(const uint64_t* in, uint64_t* out, size_t n) { scan_impl<uint64_t>(in, out, n); }

}  // namespace spbla
