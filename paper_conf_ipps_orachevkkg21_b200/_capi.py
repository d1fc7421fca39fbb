"""ctypes declarations of the C ABI in ``include/spbla_b200.h``.

Argument marshalling only: every operation runs in ``libspbla_b200.so``.
Importing this module fails loudly if the library has not been built —
there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import os

from ._build import LIB

_u32, _u64, _int, _vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p
_pu32 = ctypes.POINTER(ctypes.c_uint32)
_pu64 = ctypes.POINTER(ctypes.c_uint64)

# name -> (restype, argtypes); order follows include/spbla_b200.h
SIGNATURES = {
    "spbla_Initialize": (_int, [_int]),
    "spbla_Finalize": (_int, []),
    "spbla_SetStream": (_int, [_vp]),
    "spbla_GetStream": (_int, [ctypes.POINTER(_vp)]),
    "spbla_Synchronize": (_int, []),
    "spbla_GetMemoryStats": (_int, [_pu64, _pu64]),
    "spbla_ResetPeakMemory": (_int, []),
    "spbla_GetPoolStats": (_int, [_pu64, _pu64]),
    "spbla_GetLastErrorMessage": (ctypes.c_char_p, []),
    "spbla_GetVersion": (ctypes.c_char_p, []),
    "spbla_GetLaunchCount": (_u64, []),
    "spbla_ResetLaunchCount": (None, []),
    "spbla_SetKernelTiming": (_int, [_int]),
    "spbla_GetKernelTiming": (_int, [ctypes.c_char_p, ctypes.POINTER(ctypes.c_double), _pu64]),
    "spbla_GetEngineThresholds": (_int, [_pu64, _pu32]),
    "spbla_SetOutOfPlaceCompaction": (_int, [_int]),
    "spbla_Matrix_New": (_int, [ctypes.POINTER(_vp), _u32, _u32]),
    "spbla_Matrix_Free": (_int, [_vp]),
    "spbla_Matrix_Duplicate": (_int, [_vp, ctypes.POINTER(_vp)]),
    "spbla_Matrix_Nrows": (_int, [_vp, _pu32]),
    "spbla_Matrix_Ncols": (_int, [_vp, _pu32]),
    "spbla_Matrix_Nvals": (_int, [_vp, _pu64]),
    "spbla_Matrix_Build": (_int, [_vp, _vp, _vp, _u64, _u32]),
    "spbla_Matrix_ExtractPairs": (_int, [_vp, _vp, _vp, _pu64, _u32]),
    "spbla_Matrix_ExportCSR": (_int, [_vp, _vp, _vp, _u32]),
    "spbla_Matrix_ImportCSR": (_int, [_vp, _vp, _vp, _u64, _u32]),
    "spbla_Matrix_Wrap": (_int, [ctypes.POINTER(_vp), _u32, _u32, _vp, _vp, _u64, _u32]),
    "spbla_Matrix_DevicePointers": (_int, [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp)]),
    "spbla_Matrix_ExportRowBlock": (_int, [_vp, _vp, _vp, _u64]),
    "spbla_Matrix_ExportRowBlockMulti": (_int, [_vp, ctypes.POINTER(_vp), ctypes.POINTER(_vp), _u32, _u64]),
    "spbla_PeerBufferCreate": (_int, [_u64, ctypes.POINTER(_vp), _vp]),
    "spbla_PeerBufferOpen": (_int, [_vp, ctypes.POINTER(_vp)]),
    "spbla_PeerBufferClose": (_int, [_vp]),
    "spbla_PeerBufferFree": (_int, [_vp]),
    "spbla_Matrix_AssembleRowBlocks": (_int, [_vp, _u32, _pu32, ctypes.POINTER(_vp), ctypes.POINTER(_vp), _pu64]),
    "spbla_MxM": (_int, [_vp, _vp, _vp, _u32]),
    "spbla_Matrix_EWiseAdd": (_int, [_vp, _vp, _vp, _u32]),
    "spbla_Kronecker": (_int, [_vp, _vp, _vp, _u32]),
    "spbla_Matrix_Transpose": (_int, [_vp, _vp, _u32]),
    "spbla_Matrix_ExtractSubMatrix": (_int, [_vp, _vp, _u32, _u32, _u32, _u32, _u32]),
    "spbla_Matrix_Reduce": (_int, [_vp, _vp, _u32]),
    "spbla_TransitiveClosure": (_int, [_vp, ctypes.POINTER(_int), _u32]),
    "spbla_TransitiveClosureIncremental": (_int, [_vp, _vp, ctypes.POINTER(_int), _u32]),
}

HINT_NO = 0
HINT_HOST_MEMORY = 1 << 0
HINT_ACCUMULATE = 1 << 1
HINT_SORTED = 1 << 2
HINT_NO_DUPLICATES = 1 << 3
HINT_VALIDATE = 1 << 4
HINT_CLOSURE_STEP = 1 << 5

STATUS_NAMES = {
    0: "SUCCESS", 1: "ERROR", 2: "DEVICE_ERROR", 3: "INVALID_ARGUMENT", 4: "INVALID_STATE",
    5: "DIM_MISMATCH", 6: "INDEX_OUT_OF_BOUNDS", 7: "OUT_OF_MEMORY", 8: "NOT_IMPLEMENTED",
}

_lib = None


def load():
    """Load libspbla_b200.so (raises if it was not built)."""
    global _lib
    if _lib is not None:
        return _lib
    lib_path = os.environ.get("SPBLA_LIB_PATH", LIB)  # debug builds (tools/probe.sh) only
    if not os.path.exists(lib_path):
        raise ImportError(
            f"{LIB} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
            "(the CUDA library is the only implementation; there is no fallback)")
    lib = ctypes.CDLL(lib_path)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    _lib = lib
    return lib
