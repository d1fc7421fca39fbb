"""B200-native sparse Boolean linear algebra (SPbLA hot path, PAPER.md).

Thin Python binding over the C ABI of ``include/spbla_b200.h`` (the
``libspbla_b200.so`` built from ``csrc/`` for sm_100a).  Functions keep the
C names (``Matrix_New``, ``Matrix_Build``, ``Matrix_ExtractPairs``, ``MxM``,
``Matrix_EWiseAdd``, ``Kronecker``, ``Matrix_Transpose``,
``Matrix_ExtractSubMatrix``, ``Matrix_Reduce``, ``TransitiveClosure``) and
only marshal arguments; every step runs in the CUDA library.  PyTorch
provides device memory, the stream and ``torch.distributed`` (see
``dist.py``).
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _capi
from ._capi import (HINT_ACCUMULATE, HINT_CLOSURE_STEP, HINT_HOST_MEMORY, HINT_NO,  # noqa: F401
                    HINT_NO_DUPLICATES, HINT_SORTED, HINT_VALIDATE)

__all__ = [
    "SpblaError", "Initialize", "Finalize", "SetStream", "Synchronize", "memory_stats",
    "reset_peak_memory", "launch_count", "reset_launch_count", "Matrix", "Matrix_New",
    "Matrix_Build", "Matrix_ExtractPairs", "MxM", "Matrix_EWiseAdd", "Kronecker",
    "Matrix_Transpose", "Matrix_ExtractSubMatrix", "Matrix_Reduce", "TransitiveClosure", "TransitiveClosureIncremental",
]


class SpblaError(RuntimeError):
    def __init__(self, status: int, where: str, msg: str):
        self.status = status
        super().__init__(f"{where}: {_capi.STATUS_NAMES.get(status, status)}: {msg}")


def _lib():
    return _capi.load()


def _check(status: int, where: str):
    if status != 0:
        msg = _lib().spbla_GetLastErrorMessage()
        raise SpblaError(status, where, msg.decode() if msg else "")


_device = None


def Initialize(device: int = 0, stream=None):
    """Bind the library to ``cuda:device`` and to ``stream`` (a
    torch.cuda.Stream or raw cudaStream_t; default: torch's current stream)."""
    global _device
    import torch
    _check(_lib().spbla_Initialize(int(device)), "spbla_Initialize")
    _device = int(device)
    if stream is None:
        with torch.cuda.device(device):
            stream = torch.cuda.current_stream()
    SetStream(stream)


def _ensure():
    if _device is None:
        import torch
        Initialize(torch.cuda.current_device())


def Finalize():
    global _device
    _check(_lib().spbla_Finalize(), "spbla_Finalize")
    _device = None


def SetStream(stream):
    raw = getattr(stream, "cuda_stream", stream)
    _check(_lib().spbla_SetStream(ctypes.c_void_p(int(raw or 0))), "spbla_SetStream")


def Synchronize():
    _check(_lib().spbla_Synchronize(), "spbla_Synchronize")


def memory_stats():
    cur, peak = ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib().spbla_GetMemoryStats(ctypes.byref(cur), ctypes.byref(peak)), "spbla_GetMemoryStats")
    return int(cur.value), int(peak.value)


def pool_stats():
    """(reserved, used) bytes of the library's stream-ordered pool."""
    r, u = ctypes.c_uint64(), ctypes.c_uint64()
    _check(_lib().spbla_GetPoolStats(ctypes.byref(r), ctypes.byref(u)), "spbla_GetPoolStats")
    return int(r.value), int(u.value)


def reset_peak_memory():
    _check(_lib().spbla_ResetPeakMemory(), "spbla_ResetPeakMemory")


def launch_count() -> int:
    return int(_lib().spbla_GetLaunchCount())


def reset_launch_count():
    _lib().spbla_ResetLaunchCount()


def set_kernel_timing(enable: bool):
    _check(_lib().spbla_SetKernelTiming(1 if enable else 0), "spbla_SetKernelTiming")


def kernel_timing(name: str):
    """(total ms, launches) of a kernel group recorded since set_kernel_timing(True)."""
    ms, n = ctypes.c_double(), ctypes.c_uint64()
    _check(_lib().spbla_GetKernelTiming(name.encode(), ctypes.byref(ms), ctypes.byref(n)),
           "spbla_GetKernelTiming")
    return float(ms.value), int(n.value)


def engine_thresholds():
    buf = (ctypes.c_uint64 * 16)()
    n = ctypes.c_uint32(16)
    _check(_lib().spbla_GetEngineThresholds(buf, ctypes.byref(n)), "spbla_GetEngineThresholds")
    return [int(buf[i]) for i in range(n.value)]


def set_out_of_place_compaction(enable: bool = True):
    """spbla_SetOutOfPlaceCompaction: engine compaction into a new buffer when
    memory allows (results never change)."""
    _check(_lib().spbla_SetOutOfPlaceCompaction(int(bool(enable))), "spbla_SetOutOfPlaceCompaction")


PEER_HANDLE_BYTES = 64


class PeerBuffer:
    """Device memory that other processes map through CUDA IPC
    (spbla_PeerBufferCreate / Open / Close / Free): the gathered buffers of
    the push all-gather (dist.PeerGather)."""

    def __init__(self, nbytes: int = 0, handle: bytes = None):
        self.ptr, self.owner = 0, handle is None
        p = ctypes.c_void_p()
        if handle is None:
            h = ctypes.create_string_buffer(PEER_HANDLE_BYTES)
            _check(_lib().spbla_PeerBufferCreate(int(nbytes), ctypes.byref(p), h), "spbla_PeerBufferCreate")
            self.handle = h.raw
        else:
            h = ctypes.create_string_buffer(bytes(handle), PEER_HANDLE_BYTES)
            _check(_lib().spbla_PeerBufferOpen(h, ctypes.byref(p)), "spbla_PeerBufferOpen")
            self.handle = bytes(handle)
        self.ptr = int(p.value or 0)

    def tensor(self, dtype, n: int):
        """torch view of the first n elements (owner's buffer, this device)."""
        import torch
        ts = {torch.int64: "<i8", torch.int32: "<i4"}[dtype]

        class _Cai:
            def __init__(self, ptr, n, typestr):
                self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False),
                                                 "version": 3, "strides": None}
        return torch.as_tensor(_Cai(self.ptr, n, ts), device=f"cuda:{_device}")

    def close(self):
        if self.ptr:
            fn = _lib().spbla_PeerBufferFree if self.owner else _lib().spbla_PeerBufferClose
            _check(fn(ctypes.c_void_p(self.ptr)), "spbla_PeerBufferFree/Close")
        self.ptr = 0


def _ptr(a):
    """Raw address of a torch tensor / numpy array, and whether it is host memory."""
    if a is None:
        return None, False
    if isinstance(a, np.ndarray):
        return a.ctypes.data, True
    return a.data_ptr(), (not a.is_cuda)


def _as_u32(a):
    import torch
    if isinstance(a, np.ndarray):
        return np.ascontiguousarray(a, dtype=np.uint32)
    if isinstance(a, torch.Tensor):
        if a.dtype not in (torch.int32,):
            a = a.to(torch.int32)
        return a.contiguous()
    return np.ascontiguousarray(np.asarray(a), dtype=np.uint32)


class Matrix:
    """Owning handle of a device CSR Boolean matrix (spbla_Matrix)."""

    __slots__ = ("_h", "_keep", "__weakref__")

    def __init__(self, handle, keep=None):
        self._h = handle
        self._keep = keep  # tensors a wrapped (non-owning) view depends on

    # -- life cycle ------------------------------------------------------
    @classmethod
    def new(cls, nrows: int, ncols: int) -> "Matrix":
        _ensure()
        h = ctypes.c_void_p()
        _check(_lib().spbla_Matrix_New(ctypes.byref(h), nrows, ncols), "spbla_Matrix_New")
        return cls(h)

    @classmethod
    def from_pairs(cls, nrows, ncols, rows, cols, hints: int = 0) -> "Matrix":
        m = cls.new(nrows, ncols)
        m.build(rows, cols, hints)
        return m

    @classmethod
    def from_csr(cls, nrows, ncols, rowptr, colidx, hints: int = 0) -> "Matrix":
        m = cls.new(nrows, ncols)
        m.import_csr(rowptr, colidx, hints)
        return m

    @classmethod
    def wrap(cls, nrows, ncols, rowptr, colidx, nvals=None, hints: int = 0) -> "Matrix":
        """Zero-copy view over torch device tensors (rowptr int64, colidx int32)."""
        _ensure()
        h = ctypes.c_void_p()
        n = int(colidx.numel()) if nvals is None else int(nvals)
        _check(_lib().spbla_Matrix_Wrap(ctypes.byref(h), nrows, ncols, rowptr.data_ptr(),
                                        colidx.data_ptr() if n else None, n, hints),
               "spbla_Matrix_Wrap")
        return cls(h, keep=(rowptr, colidx))

    def free(self):
        if self._h is not None and self._h.value:
            _check(_lib().spbla_Matrix_Free(self._h), "spbla_Matrix_Free")
        self._h = None
        self._keep = None

    def __del__(self):
        try:
            if self._h is not None and self._h.value and _capi._lib is not None:
                _capi._lib.spbla_Matrix_Free(self._h)
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.free()

    @property
    def handle(self):
        return self._h

    def duplicate(self) -> "Matrix":
        h = ctypes.c_void_p()
        _check(_lib().spbla_Matrix_Duplicate(self._h, ctypes.byref(h)), "spbla_Matrix_Duplicate")
        return Matrix(h)

    # -- shape -------------------------------------------------------------
    @property
    def nrows(self) -> int:
        v = ctypes.c_uint32()
        _check(_lib().spbla_Matrix_Nrows(self._h, ctypes.byref(v)), "spbla_Matrix_Nrows")
        return int(v.value)

    @property
    def ncols(self) -> int:
        v = ctypes.c_uint32()
        _check(_lib().spbla_Matrix_Ncols(self._h, ctypes.byref(v)), "spbla_Matrix_Ncols")
        return int(v.value)

    @property
    def nvals(self) -> int:
        v = ctypes.c_uint64()
        _check(_lib().spbla_Matrix_Nvals(self._h, ctypes.byref(v)), "spbla_Matrix_Nvals")
        return int(v.value)

    @property
    def shape(self):
        return (self.nrows, self.ncols)

    # -- data in / out -------------------------------------------------------
    def build(self, rows, cols, hints: int = 0):
        r, c = _as_u32(rows), _as_u32(cols)
        pr, host_r = _ptr(r)
        pc, host_c = _ptr(c)
        if host_r != host_c:
            raise ValueError("rows and cols must both be host or both be device arrays")
        n = int(r.shape[0])
        if host_r:
            hints |= HINT_HOST_MEMORY
        _check(_lib().spbla_Matrix_Build(self._h, pr if n else None, pc if n else None, n, hints),
               "spbla_Matrix_Build")

    def extract_pairs(self, device: bool = False):
        """(rows, cols) in row-major order: uint32 numpy arrays, or int32
        device tensors with ``device=True``."""
        n = self.nvals
        nv = ctypes.c_uint64(n)
        if device:
            import torch
            r = torch.empty(max(n, 1), dtype=torch.int32, device=f"cuda:{_device}")
            c = torch.empty(max(n, 1), dtype=torch.int32, device=f"cuda:{_device}")
            _check(_lib().spbla_Matrix_ExtractPairs(self._h, r.data_ptr(), c.data_ptr(), ctypes.byref(nv), 0),
                   "spbla_Matrix_ExtractPairs")
            return r[:n], c[:n]
        r = np.empty(max(n, 1), dtype=np.uint32)
        c = np.empty(max(n, 1), dtype=np.uint32)
        _check(_lib().spbla_Matrix_ExtractPairs(self._h, r.ctypes.data, c.ctypes.data, ctypes.byref(nv),
                                                HINT_HOST_MEMORY), "spbla_Matrix_ExtractPairs")
        return r[:n], c[:n]

    def to_csr(self):
        """(rowptr uint64, colidx uint32) numpy arrays (device -> host copy)."""
        rp = np.empty(self.nrows + 1, dtype=np.uint64)
        n = self.nvals
        ci = np.empty(max(n, 1), dtype=np.uint32)
        _check(_lib().spbla_Matrix_ExportCSR(self._h, rp.ctypes.data, ci.ctypes.data, HINT_HOST_MEMORY),
               "spbla_Matrix_ExportCSR")
        return rp, ci[:n]

    def export_csr(self, rowptr, colidx, hints: int = 0):
        """Copy into caller buffers (torch device tensors or numpy arrays)."""
        prp, host = _ptr(rowptr)
        pci, _ = _ptr(colidx)
        if host:
            hints |= HINT_HOST_MEMORY
        _check(_lib().spbla_Matrix_ExportCSR(self._h, prp, pci, hints), "spbla_Matrix_ExportCSR")

    def import_csr(self, rowptr, colidx, hints: int = 0):
        prp, host = _ptr(rowptr)
        pci, _ = _ptr(colidx)
        n = int(colidx.shape[0])
        if host:
            hints |= HINT_HOST_MEMORY
        _check(_lib().spbla_Matrix_ImportCSR(self._h, prp, pci if n else None, n, hints),
               "spbla_Matrix_ImportCSR")

    def device_pointers(self):
        rp, ci = ctypes.c_void_p(), ctypes.c_void_p()
        _check(_lib().spbla_Matrix_DevicePointers(self._h, ctypes.byref(rp), ctypes.byref(ci)),
               "spbla_Matrix_DevicePointers")
        return int(rp.value or 0), int(ci.value or 0)

    def device_tensors(self):
        """Borrowed torch views (rowptr int64 [nrows+1], colidx int32 [nvals])
        of the matrix storage; valid until the matrix is modified or freed."""
        import torch
        rp, ci = self.device_pointers()
        n, m = self.nvals, self.nrows
        dev = f"cuda:{_device}"

        class _Cai:
            def __init__(self, ptr, n, typestr):
                self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False),
                                                 "version": 3, "strides": None}
        trp = torch.as_tensor(_Cai(rp, m + 1, "<i8"), device=dev)
        tci = (torch.as_tensor(_Cai(ci, n, "<i4"), device=dev) if n
               else torch.empty(0, dtype=torch.int32, device=dev))
        return trp, tci

    def export_row_block(self, rowptr, colidx, offset: int):
        """Write this matrix as one row block of a larger CSR matrix into the
        device tensors rowptr (int64, nrows+1: entries + offset) and colidx
        (int32, nvals)."""
        n = self.nvals
        _check(_lib().spbla_Matrix_ExportRowBlock(self._h, rowptr.data_ptr(), colidx.data_ptr() if n else None,
                                                  int(offset)), "spbla_Matrix_ExportRowBlock")

    def export_row_block_multi(self, dsts, offset: int):
        """export_row_block into several destinations with one kernel
        (spbla_Matrix_ExportRowBlockMulti): dsts = [(rowptr_ptr, colidx_ptr)]
        raw device addresses -- peer-mapped buffers of other ranks included."""
        nd = len(dsts)
        rps = (ctypes.c_void_p * max(nd, 1))(*[int(a) for a, _ in dsts])
        cis = (ctypes.c_void_p * max(nd, 1))(*[int(b) for _, b in dsts])
        _check(_lib().spbla_Matrix_ExportRowBlockMulti(self._h, rps, cis, nd, int(offset)),
               "spbla_Matrix_ExportRowBlockMulti")

    def assemble_row_blocks(self, blocks):
        """Replace content by the concatenation of row blocks
        [(nrows_b, rowptr_b tensor, colidx_b tensor, nnz_b), ...] (device)."""
        nb = len(blocks)
        nr = (ctypes.c_uint32 * nb)(*[int(b[0]) for b in blocks])
        rps = (ctypes.c_void_p * nb)(*[b[1].data_ptr() for b in blocks])
        cis = (ctypes.c_void_p * nb)(*[b[2].data_ptr() for b in blocks])
        nz = (ctypes.c_uint64 * nb)(*[int(b[3]) for b in blocks])
        _check(_lib().spbla_Matrix_AssembleRowBlocks(self._h, nb, nr, rps, cis, nz),
               "spbla_Matrix_AssembleRowBlocks")

    def __repr__(self):
        if self._h is None:
            return "Matrix(<freed>)"
        return f"Matrix({self.nrows}x{self.ncols}, nvals={self.nvals})"


# ---- C-named functions ---------------------------------

def Matrix_New(nrows: int, ncols: int) -> Matrix:
    return Matrix.new(nrows, ncols)


def Matrix_Build(m: Matrix, rows, cols, hints: int = 0):
    m.build(rows, cols, hints)


def Matrix_ExtractPairs(m: Matrix, device: bool = False):
    return m.extract_pairs(device)


def MxM(C: Matrix, A: Matrix, B: Matrix, accumulate: bool = False, closure_step: bool = False):
    """C = A x B, or C += A x B; closure_step (with
    accumulate): scheduling hint for a closure step C += C x C."""
    hints = (HINT_ACCUMULATE if accumulate else 0) | (HINT_CLOSURE_STEP if closure_step else 0)
    _check(_lib().spbla_MxM(C.handle, A.handle, B.handle, hints), "spbla_MxM")


def Matrix_EWiseAdd(C: Matrix, A: Matrix, B: Matrix):
    """C = A + B."""
    _check(_lib().spbla_Matrix_EWiseAdd(C.handle, A.handle, B.handle, 0), "spbla_Matrix_EWiseAdd")


def Kronecker(K: Matrix, A: Matrix, B: Matrix):
    """K = A (x) B."""
    _check(_lib().spbla_Kronecker(K.handle, A.handle, B.handle, 0), "spbla_Kronecker")


def Matrix_Transpose(T: Matrix, M: Matrix):
    _check(_lib().spbla_Matrix_Transpose(T.handle, M.handle, 0), "spbla_Matrix_Transpose")


def Matrix_ExtractSubMatrix(R: Matrix, M: Matrix, i: int, j: int, nrows: int, ncols: int):
    _check(_lib().spbla_Matrix_ExtractSubMatrix(R.handle, M.handle, i, j, nrows, ncols, 0),
           "spbla_Matrix_ExtractSubMatrix")


def Matrix_Reduce(V: Matrix, M: Matrix):
    _check(_lib().spbla_Matrix_Reduce(V.handle, M.handle, 0), "spbla_Matrix_Reduce")


def TransitiveClosure(C: Matrix) -> int:
    it = ctypes.c_int(0)
    _check(_lib().spbla_TransitiveClosure(C.handle, ctypes.byref(it), 0), "spbla_TransitiveClosure")
    return int(it.value)


def TransitiveClosureIncremental(C: Matrix, D: Matrix) -> int:
    """C (transitively closed) <- closure(C + D); returns the closure steps."""
    it = ctypes.c_int(0)
    _check(_lib().spbla_TransitiveClosureIncremental(C.handle, D.handle, ctypes.byref(it), 0),
           "spbla_TransitiveClosureIncremental")
    return int(it.value)


# convenience constructors ---------------------------------------------------

def mxm(A: Matrix, B: Matrix) -> Matrix:
    C = Matrix.new(A.nrows, B.ncols)
    MxM(C, A, B)
    return C


def ewise_add(A: Matrix, B: Matrix) -> Matrix:
    C = Matrix.new(A.nrows, A.ncols)
    Matrix_EWiseAdd(C, A, B)
    return C


def kronecker(A: Matrix, B: Matrix) -> Matrix:
    K = Matrix.new(A.nrows * B.nrows, A.ncols * B.ncols)
    Kronecker(K, A, B)
    return K


def transpose(M: Matrix) -> Matrix:
    T = Matrix.new(M.ncols, M.nrows)
    Matrix_Transpose(T, M)
    return T


def reduce_to_column(M: Matrix) -> Matrix:
    V = Matrix.new(M.nrows, 1)
    Matrix_Reduce(V, M)
    return V


def submatrix(M: Matrix, i: int, j: int, nrows: int, ncols: int) -> Matrix:
    R = Matrix.new(nrows, ncols)
    Matrix_ExtractSubMatrix(R, M, i, j, nrows, ncols)
    return R


def closure(M: Matrix):
    C = M.duplicate()
    it = TransitiveClosure(C)
    return C, it
