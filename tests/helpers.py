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


def dag_reach_and_depth(n, src, dst):
    """Reachability (paths of length >= 1) and the longest shortest-path
    length D of a DAG whose edges v -> u all have u < v: processing v in
    increasing order, reach(v) = U_{u in out(v)} ({u} U reach(u)) with
    dist_v(w) = 1 + min over those u (0 for w = u itself).  Independent of the
    oracle and of the CUDA path (a different algorithm than C += C.C)."""
    src = np.asarray(src, np.int64)
    dst = np.asarray(dst, np.int64)
    assert np.all(dst < src), "labeled_dag edges point to smaller ids"
    o = np.argsort(src, kind="stable")
    d = dst[o]
    st = np.searchsorted(src[o], np.arange(n + 1))
    reach, dist = [None] * n, [None] * n
    empty_t, empty_d = np.zeros(0, np.int64), np.zeros(0, np.int32)
    D = 0
    for v in range(n):
        kids = d[st[v]:st[v + 1]]
        if len(kids) == 0:
            reach[v], dist[v] = empty_t, empty_d
            continue
        pt, pd = [kids], [np.ones(len(kids), np.int32)]
        for u in kids.tolist():
            pt.append(reach[u])
            pd.append(dist[u] + 1)
        t = np.concatenate(pt)
        dd = np.concatenate(pd)
        oo = np.lexsort((dd, t))
        t, dd = t[oo], dd[oo]
        first = np.empty(len(t), bool)
        first[0] = True
        first[1:] = t[1:] != t[:-1]
        reach[v], dist[v] = t[first], dd[first]
        D = max(D, int(dist[v].max()))
    lens = np.array([len(x) for x in reach], np.int64)
    rp = np.zeros(n + 1, np.uint64)
    rp[1:] = np.cumsum(lens)
    return oracle.Csr(n, n, rp, np.concatenate(reach).astype(np.uint32)), D
