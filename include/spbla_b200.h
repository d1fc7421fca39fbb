/*
 * spbla_b200.h — C ABI of the B200-native sparse Boolean linear algebra hot
 * path (SPbLA, Orachev et al., IPPS'21 workshop paper; PAPER.md).
 *
 * Semiring (§II l.210-211): values {1, 0}; '+' is logical OR, 'x' is
 * logical AND, 0 (false) is the identity of '+'.
 *
 * Storage (§III-A "cuBool" l.253-257): value-free CSR.  A matrix
 * M of size m x n is a row-offset array `rowptr` (m+1 entries) and a
 * column-index array `colidx` (nnz(M) entries); a stored pair (i, j) means
 * M[i][j] = 1.  Column indices are spbla_Index (uint32_t) as in the paper;
 * row offsets are spbla_Offset (uint64_t) — a deliberate departure from the
 * paper's 32-bit offsets so one B200 (180 GB HBM3e) can hold results with
 * more than 2^32 stored values.  Within every row the column
 * indices are strictly increasing (sorted, duplicate-free); every operation
 * below produces that form and may assume it of its inputs.
 *
 * Operation list: PAPER.md §II l.228-239.
 *
 * Conventions for every entry point:
 *  - Returns SPBLA_STATUS_SUCCESS (0) or an error code; on error no output
 *    matrix is modified (exception: a failed non-accumulating MxM leaves C
 *    empty, its old content having been released to lower the memory peak),
 *    and spbla_GetLastErrorMessage() describes the error.
 *  - All device work is enqueued on the library stream (spbla_SetStream; the
 *    legacy default stream until set).  Entry points that must learn a result
 *    size on the host (Build, MxM, EWiseAdd, Transpose, ExtractSubMatrix,
 *    Reduce, TransitiveClosure) synchronise that stream once or twice; the
 *    peer-buffer calls (PeerBufferCreate/Open/Close/Free: cudaMalloc, CUDA
 *    IPC) are synchronous; all others (AssembleRowBlocks included) are
 *    asynchronous.
 *  - Pointer arguments flagged with SPBLA_HINT_HOST_MEMORY are host memory;
 *    otherwise they are device memory of the current device.  Caller-owned
 *    buffers stay caller-owned; matrices own their storage unless created by
 *    spbla_Matrix_Wrap.
 *  - Output matrices must be distinct from input matrices except where noted
 *    (MxM with ACCUMULATE reads C before replacing it; A, B may alias each
 *    other and C).
 *  - Not thread-safe: one host thread per library instance (one process per
 *    GPU, as in the multi-GPU design).
 */
#ifndef SPBLA_B200_H
#define SPBLA_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef uint32_t spbla_Index;   /* row / column index (PAPER.md l.256-257 IndexType) */
typedef uint64_t spbla_Offset;  /* row offset into colidx */

typedef struct spbla_Matrix_t* spbla_Matrix;

typedef enum {
    SPBLA_STATUS_SUCCESS = 0,
    SPBLA_STATUS_ERROR = 1,
    SPBLA_STATUS_DEVICE_ERROR = 2,        /* CUDA runtime/kernel failure */
    SPBLA_STATUS_INVALID_ARGUMENT = 3,    /* null pointer, bad flag, non-owned write */
    SPBLA_STATUS_INVALID_STATE = 4,       /* library not initialised */
    SPBLA_STATUS_DIM_MISMATCH = 5,        /* operand shapes incompatible */
    SPBLA_STATUS_INDEX_OUT_OF_BOUNDS = 6, /* a pair / range outside the matrix */
    SPBLA_STATUS_OUT_OF_MEMORY = 7,       /* device allocation failed */
    SPBLA_STATUS_NOT_IMPLEMENTED = 8
} spbla_Status;

typedef enum {
    SPBLA_HINT_NO = 0,
    SPBLA_HINT_HOST_MEMORY = 1u << 0,   /* pointer arguments are host memory */
    SPBLA_HINT_ACCUMULATE = 1u << 1,    /* MxM: C += A x B instead of C = A x B */
    SPBLA_HINT_SORTED = 1u << 2,        /* Build: pairs sorted by (row, col) ... */
    SPBLA_HINT_NO_DUPLICATES = 1u << 3, /* ... and duplicate-free: skip the sort */
    SPBLA_HINT_VALIDATE = 1u << 4,      /* Import/Wrap: check the CSR invariants */
    SPBLA_HINT_CLOSURE_STEP = 1u << 5   /* MxM with ACCUMULATE: a closure step C += C x C (or a
                                           row shard of one); rows whose products exceed 4x
                                           their current length skip the hash bins (mostly
                                           repeated columns) -- a scheduling hint, the result
                                           is the same */
} spbla_Hint;

/* ---- library state --------------------------------------------------- */

/* Bind the library to CUDA device `device` (cudaSetDevice) and create the
 * stream-ordered memory pool.  Idempotent for the same device. */
spbla_Status spbla_Initialize(int device);
/* Free pooled memory; matrices must have been freed. */
spbla_Status spbla_Finalize(void);
/* Enqueue all further work on `stream` (a cudaStream_t, may be 0).  When
 * the stream changes, the new stream first waits (an event) for all work
 * already queued on the old one, so matrices and pooled scratch still in use
 * there are never reused early. */
spbla_Status spbla_SetStream(void* stream);
spbla_Status spbla_GetStream(void** stream);
/* Synchronise the library stream. */
spbla_Status spbla_Synchronize(void);
/* Bytes currently held by matrices and scratch, and the high-water mark
 * since the last spbla_ResetPeakMemory. */
spbla_Status spbla_GetMemoryStats(uint64_t* current_bytes, uint64_t* peak_bytes);
spbla_Status spbla_ResetPeakMemory(void);
/* Bytes the stream-ordered pool has reserved from the device / hands out. */
spbla_Status spbla_GetPoolStats(uint64_t* reserved_bytes, uint64_t* used_bytes);
const char* spbla_GetLastErrorMessage(void);
const char* spbla_GetVersion(void);
/* Number of kernels the library has launched since the last reset (the
 * bench's "gpu_launches" evidence). */
uint64_t spbla_GetLaunchCount(void);
void spbla_ResetLaunchCount(void);
/* Per-kernel CUDA-event timing on each kernel's launching stream (bench.py's
 * roofline evidence).  enable != 0 clears previous records and starts
 * recording; spbla_GetKernelTiming sums the recorded launches of the named
 * kernel group and synchronises on their end events.  Groups: "mxm_ub"
 * (B-row records + upper-bound pass), "warp_bins" (W1..W8), "H0".."H6"
 * (block hash bins), "dense" (bitmap bin of the heaviest rows), "dense_ovf"
 * (small bitmap kernel: duplicate-heavy and fallen-back rows), "compact",
 * "ewise_split", "ewise_merge", "kron". */
spbla_Status spbla_SetKernelTiming(int enable);
spbla_Status spbla_GetKernelTiming(const char* name, double* total_ms, uint64_t* launches);
/* Upper-bound ("ub") limits of the row engine's bins, ascending (11 values):
 * warp bins W1, W2, W4, W8 (32 E products), hash bins H0..H6; rows above the
 * last go to the bitmap ("dense") bin.  *n: capacity in, count out. */
spbla_Status spbla_GetEngineThresholds(uint64_t* thresholds, uint32_t* n);
/* Final step of the row engine (MxM, Build, Transpose, closure steps): the
 * rows are produced at capacity offsets and then moved to their CSR offsets.
 * enable != 0 (the default; environment SPBLA_INPLACE_COMPACT=1 starts with
 * 0): when the device has room for it (free memory >= the result plus
 * max(2 GB, 1/16 of the device)), the move goes into a new exact-size buffer
 * -- a plain streaming copy, but the result and the scratch coexist for the
 * copy; otherwise, and with enable == 0, the move is in place (no second
 * buffer; tiles ordered by their overlaps, DESIGN.md §4.2 step 5).  Results
 * are identical either way.  Process-wide; never fails. */
spbla_Status spbla_SetOutOfPlaceCompaction(int enable);

/* ---- matrix life cycle --------------------------- */

/* Create an empty (all-zero) nrows x ncols matrix (l.229). */
spbla_Status spbla_Matrix_New(spbla_Matrix* matrix, spbla_Index nrows, spbla_Index ncols);
/* Delete a matrix and free its storage (l.230). */
spbla_Status spbla_Matrix_Free(spbla_Matrix matrix);
/* Deep copy into a new matrix. */
spbla_Status spbla_Matrix_Duplicate(spbla_Matrix matrix, spbla_Matrix* duplicate);
spbla_Status spbla_Matrix_Nrows(spbla_Matrix matrix, spbla_Index* nrows);
spbla_Status spbla_Matrix_Ncols(spbla_Matrix matrix, spbla_Index* ncols);
spbla_Status spbla_Matrix_Nvals(spbla_Matrix matrix, uint64_t* nvals);

/* Fill matrix with values {(i,j)_k}_k (l.231): replaces the content with
 * M[i][j] = 1 for each of the `nvals` pairs (rows[k], cols[k]); duplicate
 * pairs collapse.  Pairs need no order (hints SORTED|NO_DUPLICATES skip the
 * sort).  Host or device arrays (SPBLA_HINT_HOST_MEMORY).  Errors:
 * INDEX_OUT_OF_BOUNDS if any pair lies outside the matrix. */
spbla_Status spbla_Matrix_Build(spbla_Matrix matrix, const spbla_Index* rows,
                                const spbla_Index* cols, uint64_t nvals, uint32_t hints);

/* Read matrix values {(i,j) | M[i][j] = 1} (l.232) in row-major order into
 * caller buffers of capacity *nvals; on return *nvals = nnz(M).  Errors:
 * INVALID_ARGUMENT if the capacity is too small (then *nvals = nnz(M)). */
spbla_Status spbla_Matrix_ExtractPairs(spbla_Matrix matrix, spbla_Index* rows,
                                       spbla_Index* cols, uint64_t* nvals, uint32_t hints);

/* Copy the CSR arrays out: rowptr (nrows+1 offsets) and colidx (nnz). */
spbla_Status spbla_Matrix_ExportCSR(spbla_Matrix matrix, spbla_Offset* rowptr,
                                    spbla_Index* colidx, uint32_t hints);
/* Replace the content by a copy of CSR arrays (must satisfy the invariants;
 * SPBLA_HINT_VALIDATE checks them on the device). */
spbla_Status spbla_Matrix_ImportCSR(spbla_Matrix matrix, const spbla_Offset* rowptr,
                                    const spbla_Index* colidx, uint64_t nvals, uint32_t hints);
/* Create a NON-OWNING matrix over caller device arrays (zero copy).  The
 * caller keeps them alive and unmodified until spbla_Matrix_Free; the view
 * may be used only as an operation input. */
spbla_Status spbla_Matrix_Wrap(spbla_Matrix* matrix, spbla_Index nrows, spbla_Index ncols,
                               const spbla_Offset* rowptr, const spbla_Index* colidx,
                               uint64_t nvals, uint32_t hints);
/* Borrow the device pointers of a matrix (valid until it is modified/freed). */
spbla_Status spbla_Matrix_DevicePointers(spbla_Matrix matrix, const spbla_Offset** rowptr,
                                         const spbla_Index** colidx);
/* Write `matrix` as one row block of a larger CSR matrix (PAPER.md l.253-257
 * storage; DESIGN.md §7 row partitioning): rowptr[i] = matrix.rowptr[i] +
 * offset for i in [0, nrows] (nrows + 1 entries) and colidx[0, nvals) =
 * matrix.colidx -- device arrays owned by the caller (typically the shard's
 * slice of an all-gather buffer), asynchronous on the library stream.
 * Errors: null matrix / rowptr, null colidx for a non-empty matrix. */
spbla_Status spbla_Matrix_ExportRowBlock(spbla_Matrix matrix, spbla_Offset* rowptr, spbla_Index* colidx,
                                        spbla_Offset offset);
/* spbla_Matrix_ExportRowBlock into ndst destination pairs (rowptrs[k],
 * colidxs[k]) with one kernel that loads the block once and stores it ndst
 * times -- the push all-gather over peer memory: the
 * destinations are every rank's slice of its gathered buffers, mapped into
 * this process by CUDA IPC, so on an NVSwitch box the stores go over NVLink.
 * Asynchronous on the library stream; the caller synchronises before the
 * destination owners read.  Errors: null matrix, null arrays or entries. */
spbla_Status spbla_Matrix_ExportRowBlockMulti(spbla_Matrix matrix, spbla_Offset* const* rowptrs,
                                             spbla_Index* const* colidxs, uint32_t ndst, spbla_Offset offset);
/* Peer buffers for the push all-gather: device memory of the
 * library's GPU that other processes map through CUDA IPC.
 * PeerBufferCreate: cudaMalloc of `bytes` (not the pools: IPC needs a whole
 * allocation), *ptr its device address, `handle` receives the
 * SPBLA_PEER_HANDLE_BYTES-byte IPC handle (plain bytes, for any transport).
 * PeerBufferOpen: maps another process's buffer from its handle for the
 * library's device (peer access enabled as needed); DEVICE_ERROR when the
 * GPUs cannot reach each other -- the caller falls back to broadcasts.
 * PeerBufferClose unmaps (PeerBufferOpen's pointer), PeerBufferFree frees
 * (PeerBufferCreate's pointer, after a device synchronisation); the owner
 * frees only after every peer has closed its mapping. */
#define SPBLA_PEER_HANDLE_BYTES 64
spbla_Status spbla_PeerBufferCreate(uint64_t bytes, void** ptr, void* handle);
spbla_Status spbla_PeerBufferOpen(const void* handle, void** ptr);
spbla_Status spbla_PeerBufferClose(void* ptr);
spbla_Status spbla_PeerBufferFree(void* ptr);
/* Concatenate row blocks (block b: nrows[b] rows, device arrays rowptr[b]
 * starting at 0 and colidx[b] with nnz[b] values) into `matrix` (replaced;
 * its ncols is kept; sum nrows[b] must equal its nrows).  Used to assemble a
 * row-partitioned matrix from all-gathered shards. */
spbla_Status spbla_Matrix_AssembleRowBlocks(spbla_Matrix matrix, uint32_t nblocks,
                                            const spbla_Index* nrows,
                                            const spbla_Offset* const* rowptr,
                                            const spbla_Index* const* colidx,
                                            const uint64_t* nnz);

/* ---- operations ---------------------------------- */

/* Matrix-matrix multiplication (l.236): C = A x B, or C += A x B with
 * SPBLA_HINT_ACCUMULATE.  A: m x k, B: k x n, C: m x n.  C may alias A
 * and/or B (closure step C += C x C).  Row-wise Gustavson with per-row
 * binning. */
spbla_Status spbla_MxM(spbla_Matrix C, spbla_Matrix A, spbla_Matrix B, uint32_t hints);

/* Element-wise addition (l.237): C = A + B (C may alias A or B, which
 * gives M += N).  Global merge path. */
spbla_Status spbla_Matrix_EWiseAdd(spbla_Matrix C, spbla_Matrix A, spbla_Matrix B,
                                   uint32_t hints);

/* Kronecker product (l.238): K = A (x) B, K is (mA*mB) x (nA*nB), with
 * K[ia*mB+ib][ja*nB+jb] = A[ia][ja] AND B[ib][jb].  Errors: DIM_MISMATCH
 * if the product shape overflows spbla_Index. */
spbla_Status spbla_Kronecker(spbla_Matrix K, spbla_Matrix A, spbla_Matrix B, uint32_t hints);

/* Transpose (l.233): T = M^T, T is n x m. */
spbla_Status spbla_Matrix_Transpose(spbla_Matrix T, spbla_Matrix M, uint32_t hints);

/* Sub-matrix extraction (l.234): R = M[i..i+nrows, j..j+ncols]; R must be
 * nrows x ncols.  Errors: INDEX_OUT_OF_BOUNDS if the window leaves M. */
spbla_Status spbla_Matrix_ExtractSubMatrix(spbla_Matrix R, spbla_Matrix M, spbla_Index i,
                                           spbla_Index j, spbla_Index nrows,
                                           spbla_Index ncols, uint32_t hints);

/* Matrix to vector reduce (l.235): V = reduceToColumn(M), V[i] = OR_j M[i][j];
 * V must be m x 1. */
spbla_Status spbla_Matrix_Reduce(spbla_Matrix V, spbla_Matrix M, uint32_t hints);

/* Transitive closure by the loop C += C x C until nnz(C) is unchanged
 * (§I l.117/126: RPQ/CFPQ index creation reduces to transitive
 * closure).  C must be square; replaced in place.  *iterations (nullable)
 * receives the number of C += C x C evaluations, the last one included. */
spbla_Status spbla_TransitiveClosure(spbla_Matrix C, int* iterations, uint32_t hints);

/* Incremental transitive closure (§I l.117, l.126: an RPQ/CFPQ index
 * is updated by adding edges to an already closed relation): C must be
 * square and transitively closed (not checked), D the new edges (same
 * shape, may alias nothing but may overlap C); C is replaced by the closure
 * of C + D, computed semi-naively from the new entries (R11).
 * *iterations (nullable) receives the number of closure steps evaluated,
 * the confirming one included (0 when D adds no entry).  Errors: DIM_MISMATCH
 * on shapes, INVALID_ARGUMENT on a non-owning C. */
spbla_Status spbla_TransitiveClosureIncremental(spbla_Matrix C, spbla_Matrix D, int* iterations, uint32_t hints);

#ifdef __cplusplus
}
#endif
#endif /* SPBLA_B200_H */
