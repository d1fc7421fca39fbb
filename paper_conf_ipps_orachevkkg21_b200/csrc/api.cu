// The C ABI (include/spbla_b200.h): argument checks and exception ->
// status translation around the device implementations.
#include "common.cuh"

#include <cstring>

#include <cstdio>
#include <new>
#include <string>

namespace spbla {
void mxm(Matrix* C, const Matrix* A, const Matrix* B, bool accumulate, uint32_t dup_ratio = 0);
int transitive_closure(Matrix* C);
int transitive_closure_incremental(Matrix* C, const Matrix* D);
void ewise_add(Matrix* C, const Matrix* A, const Matrix* B);
void kronecker(Matrix* K, const Matrix* A, const Matrix* B);
void transpose(Matrix* T, const Matrix* M);
void reduce_to_column(Matrix* V, const Matrix* M);
void submatrix(Matrix* R, const Matrix* M, idx_t i0, idx_t j0, idx_t nr, idx_t nc);
void matrix_build(Matrix* m, const idx_t* rows, const idx_t* cols, uint64_t n, uint32_t hints);
void matrix_extract_pairs(const Matrix* m, idx_t* rows, idx_t* cols, uint32_t hints);
void matrix_export(const Matrix* m, off_t64* rowptr, idx_t* colidx, uint32_t hints);
void matrix_export_block(const Matrix* m, off_t64* rowptr_out, idx_t* colidx_out, off_t64 offset);
void matrix_export_block_multi(const Matrix* m, off_t64* const* rowptr_out, idx_t* const* colidx_out, uint32_t ndst,
                               off_t64 offset);
void matrix_import(Matrix* m, const off_t64* rowptr, const idx_t* colidx, uint64_t nnz, uint32_t hints);
void matrix_duplicate(const Matrix* m, Matrix* d);
void matrix_assemble(Matrix* m, uint32_t nblocks, const idx_t* nrows, const off_t64* const* rowptr,
                     const idx_t* const* colidx, const uint64_t* nnz);
void validate_csr(const off_t64* rowptr, const idx_t* colidx, idx_t nrows, idx_t ncols, uint64_t nnz);
void ktime_enable(bool on);
void ktime_query(const char* name, double* total_ms, uint64_t* launches);
void engine_thresholds(uint64_t* out, uint32_t* n);
void set_out_of_place_compaction(bool on);
}  // namespace spbla

using namespace spbla;

static thread_local std::string g_last_error;

template <typename F>
static spbla_Status guarded(F&& f) {
    try {
        f();
        g_last_error.clear();
        return SPBLA_STATUS_SUCCESS;
    } catch (const Error& e) {
        g_last_error = e.what();
        return e.status;
    } catch (const std::bad_alloc&) {
        g_last_error = "host allocation failed";
        return SPBLA_STATUS_ERROR;
    } catch (const std::exception& e) {
        g_last_error = e.what();
        return SPBLA_STATUS_ERROR;
    }
}

#define NEED(cond, msg) \
    do { if (!(cond)) SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, msg); } while (0)

extern "C" {

spbla_Status spbla_Initialize(int device) {
    return guarded([&] {
        Context& c = ctx();
        if (c.device == device) return;
        NEED(c.device < 0, "already initialised on another device");
        int n = 0;
        CUDA_CHECK(cudaGetDeviceCount(&n));
        NEED(device >= 0 && device < n, "no such CUDA device");
        CUDA_CHECK(cudaSetDevice(device));
        cudaDeviceProp prop;
        CUDA_CHECK(cudaGetDeviceProperties(&prop, device));
        if (prop.major != 10)
            SPBLA_THROW(SPBLA_STATUS_DEVICE_ERROR, "this build targets sm_100a (B200); device is not compute 10.x");
        c.num_sms = prop.multiProcessorCount;
        c.smem_optin = prop.sharedMemPerBlockOptin;
        CUDA_CHECK(cudaDeviceGetDefaultMemPool(&c.pool, device));
        uint64_t thr = UINT64_MAX;  // keep freed blocks cached in the pool
        CUDA_CHECK(cudaMemPoolSetAttribute(c.pool, cudaMemPoolAttrReleaseThreshold, &thr));
        if (!c.mat_pool) {
            cudaMemPoolProps props = {};
            props.allocType = cudaMemAllocationTypePinned;
            props.handleTypes = cudaMemHandleTypeNone;
            props.location.type = cudaMemLocationTypeDevice;
            props.location.id = device;
            CUDA_CHECK(cudaMemPoolCreate(&c.mat_pool, &props));
            CUDA_CHECK(cudaMemPoolSetAttribute(c.mat_pool, cudaMemPoolAttrReleaseThreshold, &thr));
        }
        CUDA_CHECK(cudaMallocHost(&c.host_words, 256));
        c.stream = 0;
        c.device = device;
    });
}

spbla_Status spbla_Finalize(void) {
    return guarded([&] {
        Context& c = ctx();
        if (c.device < 0) return;
        release_cached_blocks();
        CUDA_CHECK(cudaStreamSynchronize(c.stream));
        cudaMemPoolTrimTo(c.pool, 0);
        if (c.mat_pool) cudaMemPoolDestroy(c.mat_pool);
        c.mat_pool = nullptr;
        if (c.host_words) cudaFreeHost(c.host_words);
        c.host_words = nullptr;
        c.device = -1;
        c.stream = 0;
    });
}

spbla_Status spbla_SetStream(void* stream) {
    return guarded([&] {
        require_init();
        Context& c = ctx();
        cudaStream_t ns = (cudaStream_t)stream;
        if (ns != c.stream) {
            // work already queued on the old stream (and the stream-ordered
            // frees of storage it uses) must precede everything issued on the
            // new one: the new stream waits for the old stream's tail
            cudaEvent_t ev;
            CUDA_CHECK(cudaEventCreateWithFlags(&ev, cudaEventDisableTiming));
            CUDA_CHECK(cudaEventRecord(ev, c.stream));
            CUDA_CHECK(cudaStreamWaitEvent(ns, ev, 0));
            CUDA_CHECK(cudaEventDestroy(ev));
        }
        c.stream = ns;
    });
}

spbla_Status spbla_GetStream(void** stream) {
    return guarded([&] {
        NEED(stream, "null argument");
        *stream = (void*)ctx().stream;
    });
}

spbla_Status spbla_Synchronize(void) {
    return guarded([&] {
        require_init();
        CUDA_CHECK(cudaStreamSynchronize(ctx().stream));
    });
}

spbla_Status spbla_GetMemoryStats(uint64_t* cur, uint64_t* peak) {
    return guarded([&] {
        if (cur) *cur = ctx().cur_bytes;
        if (peak) *peak = ctx().peak_bytes;
    });
}

spbla_Status spbla_GetPoolStats(uint64_t* reserved, uint64_t* used) {
    return guarded([&] {
        require_init();
        uint64_t r = 0, u = 0;
        for (cudaMemPool_t pl : {ctx().pool, ctx().mat_pool}) {
            uint64_t a = 0, b = 0;
            CUDA_CHECK(cudaMemPoolGetAttribute(pl, cudaMemPoolAttrReservedMemCurrent, &a));
            CUDA_CHECK(cudaMemPoolGetAttribute(pl, cudaMemPoolAttrUsedMemCurrent, &b));
            r += a;
            u += b;
        }
        if (reserved) *reserved = r;
        if (used) *used = u;
    });
}

spbla_Status spbla_ResetPeakMemory(void) {
    return guarded([&] { ctx().peak_bytes = ctx().cur_bytes; });
}

const char* spbla_GetLastErrorMessage(void) { return g_last_error.c_str(); }
const char* spbla_GetVersion(void) { return "spbla_b200 0.1 (sm_100a)"; }
uint64_t spbla_GetLaunchCount(void) { return ctx().launches; }

spbla_Status spbla_SetKernelTiming(int enable) {
    return guarded([&] {
        require_init();
        ktime_enable(enable != 0);
    });
}

spbla_Status spbla_GetKernelTiming(const char* name, double* total_ms, uint64_t* launches) {
    return guarded([&] {
        NEED(name && total_ms && launches, "null argument");
        ktime_query(name, total_ms, launches);
    });
}

spbla_Status spbla_GetEngineThresholds(uint64_t* thresholds, uint32_t* n) {
    return guarded([&] {
        NEED(thresholds && n, "null argument");
        engine_thresholds(thresholds, n);
    });
}

spbla_Status spbla_SetOutOfPlaceCompaction(int enable) {
    return guarded([&] { set_out_of_place_compaction(enable != 0); });
}
void spbla_ResetLaunchCount(void) { ctx().launches = 0; }

spbla_Status spbla_Matrix_New(spbla_Matrix* matrix, spbla_Index nrows, spbla_Index ncols) {
    return guarded([&] {
        require_init();
        NEED(matrix, "null matrix out-pointer");
        NEED(nrows < 0xFFFFFFFFu && ncols < 0xFFFFFFFFu, "dimension must be < 2^32-1");
        Matrix* m = new Matrix;
        m->nrows = nrows;
        m->ncols = ncols;
        try {
            matrix_set_empty(m);
        } catch (...) {
            delete m;
            throw;
        }
        *matrix = m;
    });
}

spbla_Status spbla_Matrix_Free(spbla_Matrix matrix) {
    return guarded([&] {
        NEED(matrix, "null matrix");
        if (ctx().device >= 0) matrix_release(matrix);
        delete matrix;
    });
}

spbla_Status spbla_Matrix_Duplicate(spbla_Matrix matrix, spbla_Matrix* duplicate) {
    return guarded([&] {
        require_init();
        NEED(matrix && duplicate, "null argument");
        Matrix* d = new Matrix;
        try {
            matrix_duplicate(matrix, d);
        } catch (...) {
            delete d;
            throw;
        }
        *duplicate = d;
    });
}

spbla_Status spbla_Matrix_Nrows(spbla_Matrix m, spbla_Index* v) {
    return guarded([&] { NEED(m && v, "null argument"); *v = m->nrows; });
}
spbla_Status spbla_Matrix_Ncols(spbla_Matrix m, spbla_Index* v) {
    return guarded([&] { NEED(m && v, "null argument"); *v = m->ncols; });
}
spbla_Status spbla_Matrix_Nvals(spbla_Matrix m, uint64_t* v) {
    return guarded([&] { NEED(m && v, "null argument"); *v = m->nnz; });
}

spbla_Status spbla_Matrix_Build(spbla_Matrix m, const spbla_Index* rows, const spbla_Index* cols,
                                uint64_t nvals, uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(m, "null matrix");
        matrix_build(m, rows, cols, nvals, hints);
    });
}

spbla_Status spbla_Matrix_ExtractPairs(spbla_Matrix m, spbla_Index* rows, spbla_Index* cols, uint64_t* nvals,
                                       uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(m && nvals, "null argument");
        if (*nvals < m->nnz) {
            *nvals = m->nnz;
            SPBLA_THROW(SPBLA_STATUS_INVALID_ARGUMENT, "ExtractPairs: buffers too small");
        }
        NEED(m->nnz == 0 || (rows && cols), "null pair buffers");
        matrix_extract_pairs(m, rows, cols, hints);
        *nvals = m->nnz;
    });
}

spbla_Status spbla_Matrix_ExportCSR(spbla_Matrix m, spbla_Offset* rowptr, spbla_Index* colidx, uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(m, "null matrix");
        NEED(m->nnz == 0 || colidx || !rowptr, "null colidx buffer");
        matrix_export(m, rowptr, colidx, hints);
    });
}

spbla_Status spbla_Matrix_ExportRowBlock(spbla_Matrix m, spbla_Offset* rowptr, spbla_Index* colidx,
                                        spbla_Offset offset) {
    return guarded([&] {
        require_init();
        NEED(m && rowptr, "null argument");
        NEED(m->nnz == 0 || colidx, "null colidx buffer");
        matrix_export_block(m, rowptr, colidx, offset);
    });
}

spbla_Status spbla_Matrix_ExportRowBlockMulti(spbla_Matrix m, spbla_Offset* const* rowptrs, spbla_Index* const* colidxs,
                                             uint32_t ndst, spbla_Offset offset) {
    return guarded([&] {
        require_init();
        NEED(m && (ndst == 0 || (rowptrs && colidxs)), "null argument");
        for (uint32_t k = 0; k < ndst; ++k) NEED(rowptrs[k] && (m->nnz == 0 || colidxs[k]), "null destination");
        if (ndst) matrix_export_block_multi(m, rowptrs, colidxs, ndst, offset);
    });
}

spbla_Status spbla_PeerBufferCreate(uint64_t bytes, void** ptr, void* handle) {
    return guarded([&] {
        require_init();
        NEED(ptr && handle && bytes, "null argument or zero size");
        void* p = nullptr;
        CUDA_CHECK(cudaMalloc(&p, bytes));
        cudaIpcMemHandle_t h;
        const cudaError_t e = cudaIpcGetMemHandle(&h, p);
        if (e != cudaSuccess) {
            (void)cudaGetLastError();
            cudaFree(p);
            SPBLA_THROW(SPBLA_STATUS_DEVICE_ERROR, "cudaIpcGetMemHandle failed");
        }
        static_assert(sizeof(h) == SPBLA_PEER_HANDLE_BYTES, "IPC handle size");
        std::memcpy(handle, &h, sizeof(h));
        *ptr = p;
    });
}

spbla_Status spbla_PeerBufferOpen(const void* handle, void** ptr) {
    return guarded([&] {
        require_init();
        NEED(ptr && handle, "null argument");
        cudaIpcMemHandle_t h;
        std::memcpy(&h, handle, sizeof(h));
        void* p = nullptr;
        // mapped for the library's device; peer access to the owner's GPU is
        // enabled as needed (fails cleanly when the GPUs cannot reach each other)
        const cudaError_t e = cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess);
        if (e != cudaSuccess) {
            (void)cudaGetLastError();
            SPBLA_THROW(SPBLA_STATUS_DEVICE_ERROR, std::string("cudaIpcOpenMemHandle: ") + cudaGetErrorString(e));
        }
        *ptr = p;
    });
}

spbla_Status spbla_PeerBufferClose(void* ptr) {
    return guarded([&] {
        if (ptr) CUDA_CHECK(cudaIpcCloseMemHandle(ptr));
    });
}

spbla_Status spbla_PeerBufferFree(void* ptr) {
    return guarded([&] {
        if (ptr) {
            CUDA_CHECK(cudaDeviceSynchronize());  // (peers may be mid-write only outside the protocol)
            CUDA_CHECK(cudaFree(ptr));
        }
    });
}

spbla_Status spbla_Matrix_ImportCSR(spbla_Matrix m, const spbla_Offset* rowptr, const spbla_Index* colidx,
                                    uint64_t nvals, uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(m && rowptr, "null argument");
        NEED(nvals == 0 || colidx, "null colidx");
        matrix_import(m, rowptr, colidx, nvals, hints);
    });
}

spbla_Status spbla_Matrix_Wrap(spbla_Matrix* matrix, spbla_Index nrows, spbla_Index ncols,
                               const spbla_Offset* rowptr, const spbla_Index* colidx, uint64_t nvals,
                               uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(matrix && rowptr, "null argument");
        NEED(nvals == 0 || colidx, "null colidx");
        NEED(!(hints & SPBLA_HINT_HOST_MEMORY), "Wrap takes device arrays only");
        if (hints & SPBLA_HINT_VALIDATE) validate_csr(rowptr, colidx, nrows, ncols, nvals);
        Matrix* m = new Matrix;
        m->nrows = nrows;
        m->ncols = ncols;
        m->nnz = nvals;
        m->rowptr = const_cast<off_t64*>(rowptr);
        m->colidx = const_cast<idx_t*>(colidx);
        m->owned = false;
        *matrix = m;
    });
}

spbla_Status spbla_Matrix_DevicePointers(spbla_Matrix m, const spbla_Offset** rowptr, const spbla_Index** colidx) {
    return guarded([&] {
        NEED(m, "null matrix");
        if (rowptr) *rowptr = m->rowptr;
        if (colidx) *colidx = m->colidx;
    });
}

spbla_Status spbla_Matrix_AssembleRowBlocks(spbla_Matrix m, uint32_t nblocks, const spbla_Index* nrows,
                                            const spbla_Offset* const* rowptr, const spbla_Index* const* colidx,
                                            const uint64_t* nnz) {
    return guarded([&] {
        require_init();
        NEED(m && (nblocks == 0 || (nrows && rowptr && colidx && nnz)), "null argument");
        matrix_assemble(m, nblocks, nrows, rowptr, colidx, nnz);
    });
}

spbla_Status spbla_MxM(spbla_Matrix C, spbla_Matrix A, spbla_Matrix B, uint32_t hints) {
    return guarded([&] {
        require_init();
        NEED(C && A && B, "null matrix");
        mxm(C, A, B, (hints & SPBLA_HINT_ACCUMULATE) != 0, (hints & SPBLA_HINT_CLOSURE_STEP) ? 4u : 0u);
    });
}

spbla_Status spbla_Matrix_EWiseAdd(spbla_Matrix C, spbla_Matrix A, spbla_Matrix B, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(C && A && B, "null matrix");
        ewise_add(C, A, B);
    });
}

spbla_Status spbla_Kronecker(spbla_Matrix K, spbla_Matrix A, spbla_Matrix B, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(K && A && B, "null matrix");
        NEED(K != A && K != B, "Kronecker output must not alias an input");
        kronecker(K, A, B);
    });
}

spbla_Status spbla_Matrix_Transpose(spbla_Matrix T, spbla_Matrix M, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(T && M, "null matrix");
        NEED(T != M, "Transpose output must not alias the input");
        transpose(T, M);
    });
}

spbla_Status spbla_Matrix_ExtractSubMatrix(spbla_Matrix R, spbla_Matrix M, spbla_Index i, spbla_Index j,
                                           spbla_Index nrows, spbla_Index ncols, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(R && M, "null matrix");
        NEED(R != M, "ExtractSubMatrix output must not alias the input");
        submatrix(R, M, i, j, nrows, ncols);
    });
}

spbla_Status spbla_Matrix_Reduce(spbla_Matrix V, spbla_Matrix M, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(V && M, "null matrix");
        NEED(V != M, "Reduce output must not alias the input");
        reduce_to_column(V, M);
    });
}

spbla_Status spbla_TransitiveClosure(spbla_Matrix C, int* iterations, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(C, "null matrix");
        NEED(C->owned, "closure: matrix is a non-owning view");
        int it = transitive_closure(C);
        if (iterations) *iterations = it;
    });
}

spbla_Status spbla_TransitiveClosureIncremental(spbla_Matrix C, spbla_Matrix D, int* iterations, uint32_t hints) {
    (void)hints;
    return guarded([&] {
        require_init();
        NEED(C && D, "null matrix");
        NEED(C->owned, "closure: matrix is a non-owning view");
        int it = transitive_closure_incremental(C, D);
        if (iterations) *iterations = it;
    });
}

}  // extern "C"
