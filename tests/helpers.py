"""Shared helpers for the GPU parity tests (CUDA path vs oracle)."""
import numpy as np

import oracle


def gpu_lib():
    import torch
    import paper_conf_ipps_orachevkkg21_b200 as sp
    sp.Initialize(0)
    torch.cuda.set_device(0)
    return sp


def both_from_pairs(sp, nrows, ncols, r, c):
    """Same seeded pairs -> (device Matrix built by Matrix_Build, oracle Csr)."""
    import torch
    rn = r.numpy() if hasattr(r, "numpy") else np.asarray(r)
    cn = c.numpy() if hasattr(c, "numpy") else np.asarray(c)
    rt = torch.as_tensor(rn.astype(np.int32)).cuda()
    ct = torch.as_tensor(cn.astype(np.int32)).cuda()
    M = sp.Matrix.from_pairs(nrows, ncols, rt, ct)
    O = oracle.build(nrows, ncols, rn.astype(np.uint32), cn.astype(np.uint32))
    return M, O


def assert_same(M, O, what=""):
    """Bit-exact CSR equality: identical rowptr and colidx."""
    assert M.nrows == O.nrows and M.ncols == O.ncols, f"{what}: shape {M.shape} vs {(O.nrows, O.ncols)}"
    rp, ci = M.to_csr()
    assert rp.shape == O.rowptr.shape, f"{what}: rowptr length"
    if not np.array_equal(rp, O.rowptr):
        bad = np.nonzero(rp != O.rowptr)[0][:5]
        raise AssertionError(f"{what}: rowptr differs at {bad}: {rp[bad]} vs {O.rowptr[bad]}")
    if not np.array_equal(ci, O.colidx):
        bad = np.nonzero(ci != O.colidx)[0][:5]
        raise AssertionError(f"{what}: colidx differs at {bad} (nnz {len(ci)} vs {len(O.colidx)})")


def csr_is_valid(rp, ci, ncols):
    """Properties that hold at any size: offsets start at 0, non-decreasing,
    end at nnz; columns in range, strictly increasing inside every row."""
    rp = rp.astype(np.int64)
    if rp[0] != 0 or rp[-1] != len(ci) or np.any(np.diff(rp) < 0):
        return False
    if len(ci) == 0:
        return True
    if int(ci.max()) >= ncols:
        return False
    d = np.diff(ci.astype(np.int64))
    row_start = np.zeros(len(ci), dtype=bool)
    starts = rp[:-1][np.diff(rp) > 0]
    row_start[starts] = True
    return bool(np.all((d > 0) | row_start[1:]))
