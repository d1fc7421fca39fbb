// Library context: device binding, stream, stream-ordered memory pool with
// byte accounting (peak device memory is part of the BASELINE metric), and
// matrix storage helpers.
#include "common.cuh"

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>
#include <chrono>
#include <cstdlib>
#include <unordered_map>

namespace spbla {

static Context g_ctx;
Context& ctx() { return g_ctx; }

void require_init() {
    if (g_ctx.device < 0) SPBLA_THROW(SPBLA_STATUS_INVALID_STATE, "spbla_Initialize was not called");
}

void cuda_check(cudaError_t e, const char* what, const char* file, int line) {
    if (e == cudaSuccess) return;
    char buf[512];
    std::snprintf(buf, sizeof(buf), "%s failed: %s (%s:%d)", what, cudaGetErrorString(e), file, line);
    if (e == cudaErrorMemoryAllocation) {
        (void)cudaGetLastError();
        throw Error(SPBLA_STATUS_OUT_OF_MEMORY, buf);
    }
    throw Error(SPBLA_STATUS_DEVICE_ERROR, buf);
}

void check_launch(const char* name) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
        char buf[256];
        std::snprintf(buf, sizeof(buf), "kernel %s launch failed: %s", name, cudaGetErrorString(e));
        throw Error(SPBLA_STATUS_DEVICE_ERROR, buf);
    }
}

// Size-class cache on top of the stream-ordered pools.  cudaMallocFromPoolAsync
// is cheap when a freed block of the right size is at hand, but with varying
// sizes it assembles large requests by remapping the pool's physical pages
// into fresh address ranges -- measured on the configs[3] closure loop: 25-130
// ms for a 44-516 MB request with the pool's reservation unchanged.  Freed
// blocks therefore go to per-class free lists (8 classes per power of two,
// <= 12.5% rounding) and are handed out again in stream order: all library
// work runs on one stream (SetStream orders a new stream after the old one),
// so a block freed by earlier work is safe for any later work.  Cached blocks
// go back to the pool on an allocation failure and at Finalize.
namespace {
// one cache for both pools: with exact size classes a block serves any
// later request of its class, matrix storage or scratch
std::unordered_map<size_t, std::vector<void*>> g_free;

size_t size_class(size_t b) {
    if (b <= 4096) return 4096;
    int e = 63 - __builtin_clzll(b);  // 2^e <= b < 2^(e+1)
    const size_t step = size_t(1) << (e - 3);
    return (b + step - 1) / step * step;
}
}  // namespace

void release_cached_blocks() {
    for (auto& kv : g_free)
        for (void* p : kv.second) cudaFreeAsync(p, g_ctx.stream);
    g_free.clear();
}

void* dev_alloc(size_t bytes, bool mat) {
    require_init();
    void* p = nullptr;
    if (bytes == 0) return nullptr;
    const size_t cb = size_class(bytes);
    auto& fl = g_free[cb];
    if (!fl.empty()) {
        p = fl.back();
        fl.pop_back();
    } else {
        cudaMemPool_t pool = mat ? g_ctx.mat_pool : g_ctx.pool;
        static int trace = -1;
        if (trace < 0) trace = std::getenv("SPBLA_TRACE") != nullptr;
        const auto t0 = std::chrono::steady_clock::now();
        cudaError_t e = cudaMallocFromPoolAsync(&p, cb, pool, g_ctx.stream);
        if (e != cudaSuccess) {
            (void)cudaGetLastError();
            // give the cached blocks and the pools' free memory back and retry once
            release_cached_blocks();
            cudaStreamSynchronize(g_ctx.stream);
            cudaMemPoolTrimTo(g_ctx.pool, 0);
            cudaMemPoolTrimTo(g_ctx.mat_pool, 0);
            e = cudaMallocFromPoolAsync(&p, cb, pool, g_ctx.stream);
            if (e != cudaSuccess) {
                (void)cudaGetLastError();
                char buf[128];
                std::snprintf(buf, sizeof(buf), "device allocation of %zu bytes failed", bytes);
                throw Error(SPBLA_STATUS_OUT_OF_MEMORY, buf);
            }
        }
        if (trace) {
            const double ms = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
            if (ms > 1.0) {
                uint64_t r = 0, u = 0;
                cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &r);
                cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &u);
                std::fprintf(stderr, "[trace] slow alloc %.3f ms: %zu bytes (%s pool: reserved %.3f GB, used %.3f GB)\n",
                             ms, cb, mat ? "matrix" : "scratch", r / 1e9, u / 1e9);
            }
        }
    }
    g_ctx.cur_bytes += bytes;
    if (g_ctx.cur_bytes > g_ctx.peak_bytes) g_ctx.peak_bytes = g_ctx.cur_bytes;
    return p;
}

bool dev_can_alloc(size_t bytes, bool mat) {
    require_init();
    const size_t cb = size_class(bytes);
    auto it = g_free.find(cb);
    if (it != g_free.end() && !it->second.empty()) return true;  // a cached block of the class
    size_t fr = 0, tot = 0;
    if (cudaMemGetInfo(&fr, &tot) != cudaSuccess) {
        (void)cudaGetLastError();
        return false;
    }
    cudaMemPool_t pool = mat ? g_ctx.mat_pool : g_ctx.pool;
    uint64_t r = 0, u = 0;
    cudaMemPoolGetAttribute(pool, cudaMemPoolAttrReservedMemCurrent, &r);
    cudaMemPoolGetAttribute(pool, cudaMemPoolAttrUsedMemCurrent, &u);
    const size_t margin = std::max<size_t>(size_t(2) << 30, tot / 16);  // headroom for the rest of the operation
    return fr + (r > u ? r - u : 0) >= cb + margin;
}

void dev_free(void* p, size_t bytes) {
    if (!p) return;
    // (the caller passes the size it allocated; matrices record it as their capacity)
    g_free[size_class(bytes)].push_back(p);
    g_ctx.cur_bytes -= bytes;
}

// SPBLA_TRACE=1: synchronise and print wall-clock per phase plus pool
// reservation (diagnostics only; off by default).
void trace_mark(const char* what) {
    static int on = -1;
    if (on < 0) on = std::getenv("SPBLA_TRACE") != nullptr;
    if (!on) return;
    static auto last = std::chrono::steady_clock::now();
    cudaStreamSynchronize(g_ctx.stream);
    auto now = std::chrono::steady_clock::now();
    uint64_t r = 0, u = 0, r2 = 0, u2 = 0;
    cudaMemPoolGetAttribute(g_ctx.pool, cudaMemPoolAttrReservedMemCurrent, &r);
    cudaMemPoolGetAttribute(g_ctx.pool, cudaMemPoolAttrUsedMemCurrent, &u);
    cudaMemPoolGetAttribute(g_ctx.mat_pool, cudaMemPoolAttrReservedMemCurrent, &r2);
    cudaMemPoolGetAttribute(g_ctx.mat_pool, cudaMemPoolAttrUsedMemCurrent, &u2);
    r += r2;
    u += u2;
    std::fprintf(stderr, "[trace] %-14s %9.3f ms  pool reserved %.2f GB used %.2f GB\n", what,
                 std::chrono::duration<double, std::milli>(now - last).count(), r / 1e9, u / 1e9);
    last = now;
}

// Wait for the library stream by polling an event instead of
// cudaStreamSynchronize: the runtime's default (blocking/yield) wait puts the
// host thread to sleep at every size read-back, and on the GPU boxes the
// wake-up costs 0.1-1 ms and occasionally tens of ms (measured on the configs[3]
// closure, 12 read-backs per step: 16 voluntary context switches per step,
// 8-15 ms medians with 40-230 ms outliers; tools/stall_probe.py).  The read-backs
// are short waits on a GPU that is about to finish, so spinning is the cheap
// choice.
void stream_sync_spin() {
    static cudaEvent_t ev = nullptr;
    static int dev = -1;
    if (dev != g_ctx.device) {
        if (ev) cudaEventDestroy(ev);
        CUDA_CHECK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
        dev = g_ctx.device;
    }
    CUDA_CHECK(cudaEventRecord(ev, g_ctx.stream));
    for (;;) {
        const cudaError_t e = cudaEventQuery(ev);
        if (e == cudaSuccess) return;
        if (e != cudaErrorNotReady) CUDA_CHECK(e);
    }
}

void read_words(const uint64_t* dev, uint64_t* host, int n) {
    CUDA_CHECK(cudaMemcpyAsync(g_ctx.host_words, dev, n * sizeof(uint64_t), cudaMemcpyDeviceToHost,
                               g_ctx.stream));
    stream_sync_spin();
    std::memcpy(host, g_ctx.host_words, n * sizeof(uint64_t));
}

void read_words2(const uint64_t* dev, uint64_t* host, int n, const void* dev2, void* host2, size_t bytes2) {
    if (n > 8 || bytes2 > 128) throw Error(SPBLA_STATUS_INVALID_ARGUMENT, "read_words2: too many bytes");
    unsigned char* hw = reinterpret_cast<unsigned char*>(g_ctx.host_words);
    CUDA_CHECK(cudaMemcpyAsync(hw, dev, n * sizeof(uint64_t), cudaMemcpyDeviceToHost, g_ctx.stream));
    CUDA_CHECK(cudaMemcpyAsync(hw + 128, dev2, bytes2, cudaMemcpyDeviceToHost, g_ctx.stream));
    stream_sync_spin();
    std::memcpy(host, hw, n * sizeof(uint64_t));
    std::memcpy(host2, hw + 128, bytes2);
}

void memset_async(void* p, int v, size_t bytes) {
    if (bytes) CUDA_CHECK(cudaMemsetAsync(p, v, bytes, g_ctx.stream));
}

void copy_async(void* dst, const void* src, size_t bytes, cudaMemcpyKind kind) {
    if (bytes) CUDA_CHECK(cudaMemcpyAsync(dst, src, bytes, kind, g_ctx.stream));
}

void matrix_release(Matrix* m) {
    if (m->owned) {
        dev_free(m->rowptr, m->rowptr_cap * sizeof(off_t64));
        dev_free(m->colidx, m->colidx_cap * sizeof(idx_t));
    }
    m->rowptr = nullptr;
    m->colidx = nullptr;
    m->rowptr_cap = m->colidx_cap = 0;
    m->nnz = 0;
    m->owned = true;
}

void matrix_replace(Matrix* m, off_t64* rowptr, size_t rowptr_cap, idx_t* colidx,
                    size_t colidx_cap, uint64_t nnz) {
    matrix_release(m);
    m->rowptr = rowptr;
    m->rowptr_cap = rowptr_cap;
    m->colidx = colidx;
    m->colidx_cap = colidx_cap;
    m->nnz = nnz;
    m->owned = true;
}

void matrix_set_empty(Matrix* m) {
    DevBuf<off_t64> rp(size_t(m->nrows) + 1, kMat);
    memset_async(rp.p, 0, rp.n * sizeof(off_t64));
    size_t cap = rp.n;
    matrix_replace(m, rp.detach(), cap, nullptr, 0, 0);
}

struct KRec {
    std::string name;
    cudaStream_t stream;
    cudaEvent_t a, b;
};
static bool g_ktime_on = false;
static std::vector<KRec> g_krec;
static std::vector<cudaEvent_t> g_kevpool;
static size_t g_kev_used = 0;

static cudaEvent_t kev() {
    if (g_kev_used == g_kevpool.size()) {
        cudaEvent_t e;
        CUDA_CHECK(cudaEventCreate(&e));
        g_kevpool.push_back(e);
    }
    return g_kevpool[g_kev_used++];
}

int ktime_begin(const char* name, cudaStream_t s) {
    if (!g_ktime_on) return -1;
    KRec r{name, s, kev(), kev()};
    CUDA_CHECK(cudaEventRecord(r.a, s));
    g_krec.push_back(r);
    return int(g_krec.size()) - 1;
}

void ktime_end(int slot) {
    if (slot < 0) return;
    CUDA_CHECK(cudaEventRecord(g_krec[slot].b, g_krec[slot].stream));
}

void ktime_enable(bool on) {
    // events are created up front: a cudaEventCreate inside a timed step
    // showed up as a slow first timed step
    while (on && g_kevpool.size() < 8192) {
        cudaEvent_t e;
        CUDA_CHECK(cudaEventCreate(&e));
        g_kevpool.push_back(e);
    }
    g_ktime_on = on;
    g_krec.clear();
    g_kev_used = 0;
}

void ktime_query(const char* name, double* total_ms, uint64_t* launches) {
    double t = 0;
    uint64_t n = 0;
    for (auto& r : g_krec) {
        if (r.name != name) continue;
        CUDA_CHECK(cudaEventSynchronize(r.b));
        float ms = 0;
        CUDA_CHECK(cudaEventElapsedTime(&ms, r.a, r.b));
        t += ms;
        ++n;
    }
    *total_ms = t;
    *launches = n;
}

}  // namespace spbla
