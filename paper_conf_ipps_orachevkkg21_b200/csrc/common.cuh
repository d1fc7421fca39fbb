// Internal shared definitions of the CUDA path (NOT shared with oracle/).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>
#include <string>
#include <stdexcept>

#include "../../include/spbla_b200.h"

namespace spbla {

typedef uint32_t idx_t;
typedef uint64_t off_t64;

constexpr int kNumSMs = 148;  // B200 (2 dies x 74)
constexpr idx_t kEmpty = 0xFFFFFFFFu;

// Error carried by exceptions inside the library; converted to spbla_Status at
// the C boundary (api.cu).
struct Error : std::runtime_error {
    spbla_Status status;
    Error(spbla_Status s, const std::string& m) : std::runtime_error(m), status(s) {}
};

void cuda_check(cudaError_t e, const char* what, const char* file, int line);
#define CUDA_CHECK(x) ::spbla::cuda_check((x), #x, __FILE__, __LINE__)
#define SPBLA_THROW(st, msg) throw ::spbla::Error((st), (msg))

// ---- context: stream, stream-ordered pool allocator, counters -----------
struct Context {
    int device = -1;
    cudaStream_t stream = 0;
    cudaMemPool_t pool = nullptr;      // temporaries (device default pool)
    cudaMemPool_t mat_pool = nullptr;  // matrix storage (rowptr / colidx of results)
    uint64_t cur_bytes = 0, peak_bytes = 0;
    uint64_t launches = 0;
    int num_sms = kNumSMs;
    size_t smem_optin = 227 * 1024;
    // pinned host scratch for size read-backs
    uint64_t* host_words = nullptr;
};
Context& ctx();
void require_init();

// Two stream-ordered pools: matrix storage (`mat`) and temporaries.  Keeping
// the long-lived result arrays apart from the scratch of an operation lets a
// repeated MxM reuse the freed result block exactly instead of fragmenting it
// with temporaries (a pool miss maps fresh memory: ~60 ms per GB on B200).
void* dev_alloc(size_t bytes, bool mat = false);
void dev_free(void* p, size_t bytes);
// true if dev_alloc(bytes, mat) can be served without evicting the cache: a
// cached block of its size class, or free device (+ pool) memory with a
// margin of max(2 GB, 1/16 of the device)
bool dev_can_alloc(size_t bytes, bool mat);
// give the size-class cache's blocks back to the pools (Finalize, OOM retry)
void release_cached_blocks();
// read `n` uint64 words from device memory (synchronises the stream)
void trace_mark(const char* what);
void read_words(const uint64_t* dev, uint64_t* host, int n);
// wait for the library stream by polling (no thread sleep; see context.cu)
void stream_sync_spin();
// read_words plus up to 128 more bytes from dev2 into host2, one synchronisation
void read_words2(const uint64_t* dev, uint64_t* host, int n, const void* dev2, void* host2, size_t bytes2);
void memset_async(void* p, int v, size_t bytes);
void copy_async(void* dst, const void* src, size_t bytes, cudaMemcpyKind kind);
inline void count_launch(int n = 1) { ctx().launches += n; }
// Optional per-kernel CUDA-event timing on the launching stream (bench.py's
// roofline evidence): ktime_begin returns -1 when timing is off.
int ktime_begin(const char* name, cudaStream_t s);
void ktime_end(int slot);
void check_launch(const char* name);

// RAII device buffer in the pool.
template <typename T>
struct DevBuf {
    T* p = nullptr;
    size_t n = 0;
    DevBuf() {}
    explicit DevBuf(size_t count, bool mat = false) { alloc(count, mat); }
    void alloc(size_t count, bool mat = false) {
        release();
        n = count;
        if (count) p = (T*)dev_alloc(count * sizeof(T), mat);
    }
    void release() {
        if (p) dev_free(p, n * sizeof(T));
        p = nullptr;
        n = 0;
    }
    T* detach() { T* q = p; p = nullptr; n = 0; return q; }
    ~DevBuf() { release(); }
    DevBuf(const DevBuf&) = delete;
    DevBuf& operator=(const DevBuf&) = delete;
};

constexpr bool kMat = true;  // DevBuf(count, kMat): storage that becomes a matrix's

// ---- matrix --------------------------------------------------------------
}  // namespace spbla

struct spbla_Matrix_t {
    spbla::idx_t nrows = 0, ncols = 0;
    uint64_t nnz = 0;
    spbla::off_t64* rowptr = nullptr;  // nrows+1 (always allocated for owned)
    spbla::idx_t* colidx = nullptr;    // nnz
    size_t rowptr_cap = 0, colidx_cap = 0;  // allocated element counts
    bool owned = true;
};

namespace spbla {

typedef spbla_Matrix_t Matrix;

// Install new storage into m (frees the old one).  rowptr must hold nrows+1.
void matrix_replace(Matrix* m, off_t64* rowptr, size_t rowptr_cap, idx_t* colidx,
                    size_t colidx_cap, uint64_t nnz);
void matrix_set_empty(Matrix* m);
void matrix_release(Matrix* m);

// Lightweight by-value view passed to kernels.
struct CsrView {
    idx_t nrows, ncols;
    const off_t64* __restrict__ rowptr;
    const idx_t* __restrict__ colidx;
};
inline CsrView view(const Matrix* m) { return CsrView{m->nrows, m->ncols, m->rowptr, m->colidx}; }

// ---- in-house primitives (scan.cu) ----------------------------------------
// Exclusive prefix sum out[i] = sum_{j<i} in[i]; out has n+1 entries, out[n]
// = total.  Single-pass decoupled look-back; returns nothing (total stays on
// the device at out[n]).
void exclusive_scan_u32(const uint32_t* in, uint64_t* out, size_t n);
void exclusive_scan_u64(const uint64_t* in, uint64_t* out, size_t n);

// ---- row engine (rowsort.cu) --------------------------------------------
// Produce, for every output row r in [0, nrows), the sorted duplicate-free
// union of a per-row list of column "segments" (MxM: B rows; Build /
// Transpose: one bucket), then compact into CSR.  See DESIGN.md §4.2.
struct SegSource {
    // Descriptor mode (kind = 0, MxM): row r's NON-EMPTY segments are
    // desc[dbase[r] + r + j], j < nseg[r], each {ptr lo, ptr hi, len, end}
    // with end = inclusive prefix of the row's segment lengths (written by
    // the upper-bound pass: C[r] first when accumulating, then B[k] for k in
    // A[r]).  Staging a row is then a plain copy.  List mode (kind = 1,
    // Build / Transpose): one segment lst[lrp[r] .. lrp[r+1]).
    int kind;
    const off_t64* __restrict__ dbase;
    const uint32_t* __restrict__ nseg;
    const uint4* __restrict__ desc;
    const off_t64* __restrict__ lrp;
    const idx_t* __restrict__ lst;
};
// ub: per-row upper bound of entries (device, nrows).  Installs the result
// in `out` (nrows x ncols).  dedup=false promises rows are duplicate-free.
// range (nullable): per-row [min col, max col] of the row's segments, needed
// (and computed by MxM) for rows with ub > kRangeMinUb; null means [0, ncols).
#ifndef SPBLA_WARP_MAX
#define SPBLA_WARP_MAX 128  // (rows of 129-256 products: the 32-thread hash bin H0; duplicate-heavy ones: W8)
#endif
constexpr uint64_t kRangeMinUb = SPBLA_WARP_MAX;
// Bit 63 of a row's ub: the producer expects the row to be duplicate-heavy
// (closure steps: products >> the row's current length); the engine masks it.
constexpr uint64_t kUbDupFlag = uint64_t(1) << 63;
// Bit 62: the row's only segment is already a sorted duplicate-free row (the
// accumulate input C[r] of a row with no B products): the engine copies it.
constexpr uint64_t kUbCopyFlag = uint64_t(1) << 62;
constexpr uint64_t kUbValue = kUbCopyFlag - 1;  // the count without the flags
void row_engine(const SegSource& src, idx_t nrows, idx_t ncols, const uint64_t* ub, const uint2* range,
                Matrix* out);

// ---- device helpers ------------------------------------------------------
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }

template <typename T>
__device__ __forceinline__ T warp_inclusive_scan(T v) {
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        T t = __shfl_up_sync(0xffffffffu, v, d);
        if ((int)lane_id() >= d) v += t;
    }
    return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(0xffffffffu, v, d);
    return v;
}

// Block-wide exclusive scan of one value per thread (blockDim multiple of 32,
// <= 1024).  `sh` needs 33 words of T.  Returns exclusive prefix; *total set.
template <typename T>
__device__ __forceinline__ T block_exclusive_scan(T v, T* sh, T* total) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int nw = blockDim.x >> 5;
    T inc = warp_inclusive_scan(v);
    if (lane == 31) sh[warp] = inc;
    __syncthreads();
    if (warp == 0) {
        T w = lane < nw ? sh[lane] : T(0);
        T wi = warp_inclusive_scan(w);
        if (lane < nw) sh[lane] = wi - w;
        if (lane == nw - 1) sh[32] = wi;
    }
    __syncthreads();
    T r = inc - v + sh[warp];
    *total = sh[32];
    __syncthreads();
    return r;
}

__host__ __device__ inline uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

}  // namespace spbla
