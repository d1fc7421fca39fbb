"""CPU oracle for the SPbLA Boolean hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_ipps_orachevkkg21_b200``) never imports it and
shares no code with it.

The arithmetic lives in ``spbla_oracle.cpp`` (plain C++, ``std::set`` per
output row; every function cites the PAPER.md passage it follows).  This
module only compiles it with g++ and marshals numpy arrays through ctypes.

CSR convention on this side: ``rowptr`` uint64 [nrows+1], ``colidx`` uint32
[nnz], rows sorted and duplicate-free.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "spbla_oracle.cpp")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

_u64p = ctypes.POINTER(ctypes.c_uint64)
_u32p = ctypes.POINTER(ctypes.c_uint32)


def build_lib(force: bool = False) -> str:
    """Compile the oracle shared library (g++ -O2)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = ctypes.CDLL(build_lib())
        vp = ctypes.c_void_p
        u32, u64 = ctypes.c_uint32, ctypes.c_uint64
        lib.ocsr_free.argtypes = [vp]
        lib.ocsr_nvals.argtypes = [vp]
        lib.ocsr_nvals.restype = u64
        lib.ocsr_nrows.argtypes = [vp]
        lib.ocsr_nrows.restype = u32
        lib.ocsr_ncols.argtypes = [vp]
        lib.ocsr_ncols.restype = u32
        lib.ocsr_copy.argtypes = [vp, _u64p, _u32p]
        lib.oracle_build.argtypes = [u32, u32, _u32p, _u32p, u64, ctypes.POINTER(ctypes.c_int)]
        lib.oracle_build.restype = vp
        lib.oracle_mxm.argtypes = [u32, u32, u32, _u64p, _u32p, _u64p, _u32p, _u64p, _u32p]
        lib.oracle_mxm.restype = vp
        lib.oracle_mxm_rows.argtypes = [u32, _u64p, _u32p, _u64p, _u32p, _u64p, _u32p, _u32p, u32]
        lib.oracle_mxm_rows.restype = vp
        lib.oracle_ewise_add.argtypes = [u32, u32, _u64p, _u32p, _u64p, _u32p]
        lib.oracle_ewise_add.restype = vp
        lib.oracle_kronecker.argtypes = [u32, u32, _u64p, _u32p, u32, u32, _u64p, _u32p]
        lib.oracle_kronecker.restype = vp
        lib.oracle_transpose.argtypes = [u32, u32, _u64p, _u32p]
        lib.oracle_transpose.restype = vp
        lib.oracle_reduce.argtypes = [u32, u32, _u64p, _u32p]
        lib.oracle_reduce.restype = vp
        lib.oracle_submatrix.argtypes = [u32, u32, _u64p, _u32p, u32, u32, u32, u32]
        lib.oracle_submatrix.restype = vp
        lib.oracle_closure.argtypes = [u32, _u64p, _u32p, ctypes.POINTER(ctypes.c_int)]
        lib.oracle_closure.restype = vp
        _lib = lib
        return lib


class Csr:
    """A Boolean CSR matrix held in numpy arrays (oracle side)."""

    __slots__ = ("nrows", "ncols", "rowptr", "colidx")

    def __init__(self, nrows, ncols, rowptr, colidx):
        self.nrows = int(nrows)
        self.ncols = int(ncols)
        self.rowptr = np.ascontiguousarray(rowptr, dtype=np.uint64)
        self.colidx = np.ascontiguousarray(colidx, dtype=np.uint32)

    @property
    def nvals(self) -> int:
        return int(self.colidx.shape[0])

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.nrows, self.ncols), dtype=bool)
        rows = np.repeat(np.arange(self.nrows), np.diff(self.rowptr.astype(np.int64)))
        d[rows, self.colidx.astype(np.int64)] = True
        return d

    def pairs(self):
        rows = np.repeat(np.arange(self.nrows, dtype=np.uint32),
                         np.diff(self.rowptr.astype(np.int64)))
        return rows, self.colidx.copy()

    def __eq__(self, other):
        return (self.nrows == other.nrows and self.ncols == other.ncols
                and np.array_equal(self.rowptr, other.rowptr)
                and np.array_equal(self.colidx, other.colidx))


def _p64(a):
    return a.ctypes.data_as(_u64p)


def _p32(a):
    return a.ctypes.data_as(_u32p)


def _take(ptr) -> Csr:
    lib = _load()
    nr, nc, nv = lib.ocsr_nrows(ptr), lib.ocsr_ncols(ptr), lib.ocsr_nvals(ptr)
    rp = np.empty(nr + 1, dtype=np.uint64)
    ci = np.empty(max(nv, 1), dtype=np.uint32)
    lib.ocsr_copy(ptr, _p64(rp), _p32(ci))
    lib.ocsr_free(ptr)
    return Csr(nr, nc, rp, ci[:nv])


def build(nrows: int, ncols: int, rows, cols) -> Csr:
    lib = _load()
    r = np.ascontiguousarray(rows, dtype=np.uint32)
    c = np.ascontiguousarray(cols, dtype=np.uint32)
    st = ctypes.c_int(0)
    p = lib.oracle_build(nrows, ncols, _p32(r), _p32(c), r.shape[0], ctypes.byref(st))
    if st.value != 0:
        raise IndexError("oracle_build: index out of range")
    return _take(p)


def from_dense(d) -> Csr:
    d = np.asarray(d, dtype=bool)
    r, c = np.nonzero(d)
    return build(d.shape[0], d.shape[1], r, c)


def mxm(a: Csr, b: Csr, c: Csr | None = None) -> Csr:
    """C = A x B, or C + A x B when ``c`` is given (accumulate)."""
    assert a.ncols == b.nrows
    if c is not None:
        assert c.nrows == a.nrows and c.ncols == b.ncols
    lib = _load()
    p = lib.oracle_mxm(a.nrows, a.ncols, b.ncols, _p64(a.rowptr), _p32(a.colidx),
                       _p64(b.rowptr), _p32(b.colidx),
                       _p64(c.rowptr) if c is not None else None,
                       _p32(c.colidx) if c is not None else None)
    return _take(p)


def mxm_rows(a: Csr, b: Csr, rows, c: Csr | None = None) -> Csr:
    """Rows ``rows`` of (C +) A x B, as a len(rows) x ncols matrix."""
    lib = _load()
    s = np.ascontiguousarray(rows, dtype=np.uint32)
    p = lib.oracle_mxm_rows(b.ncols, _p64(a.rowptr), _p32(a.colidx),
                            _p64(b.rowptr), _p32(b.colidx),
                            _p64(c.rowptr) if c is not None else None,
                            _p32(c.colidx) if c is not None else None,
                            _p32(s), s.shape[0])
    return _take(p)


def ewise_add(a: Csr, b: Csr) -> Csr:
    assert a.nrows == b.nrows and a.ncols == b.ncols
    lib = _load()
    return _take(lib.oracle_ewise_add(a.nrows, a.ncols, _p64(a.rowptr), _p32(a.colidx),
                                      _p64(b.rowptr), _p32(b.colidx)))


def kronecker(a: Csr, b: Csr) -> Csr:
    lib = _load()
    return _take(lib.oracle_kronecker(a.nrows, a.ncols, _p64(a.rowptr), _p32(a.colidx),
                                      b.nrows, b.ncols, _p64(b.rowptr), _p32(b.colidx)))


def transpose(a: Csr) -> Csr:
    lib = _load()
    return _take(lib.oracle_transpose(a.nrows, a.ncols, _p64(a.rowptr), _p32(a.colidx)))


def reduce_to_column(a: Csr) -> Csr:
    lib = _load()
    return _take(lib.oracle_reduce(a.nrows, a.ncols, _p64(a.rowptr), _p32(a.colidx)))


def submatrix(a: Csr, i0: int, j0: int, nr: int, nc: int) -> Csr:
    assert i0 + nr <= a.nrows and j0 + nc <= a.ncols
    lib = _load()
    return _take(lib.oracle_submatrix(a.nrows, a.ncols, _p64(a.rowptr), _p32(a.colidx),
                                      i0, j0, nr, nc))


def closure(a: Csr):
    """(C, iterations): C += C x C from C = A until nnz(C) is unchanged."""
    assert a.nrows == a.ncols
    lib = _load()
    it = ctypes.c_int(0)
    p = lib.oracle_closure(a.nrows, _p64(a.rowptr), _p32(a.colidx), ctypes.byref(it))
    return _take(p), it.value
