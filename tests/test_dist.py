"""Row-partitioned multi-GPU protocol (dist.py) on CPU: world_size 2, gloo,
the oracle as the local multiply.  Checks that partitioning + the exact-size
all-gather of CSR row blocks (each rank writes its block into its slice, one
broadcast per rank) reproduce the single-process results of MxM and of the
closure loop (rows, nnz and iteration count)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import spgen
from paper_conf_ipps_orachevkkg21_b200 import dist as spdist


class OracleOps:
    """The dist.py ops on CPU tensors with the oracle as the local multiply."""

    def shape_nnz(self, M):
        return M.nrows, M.nvals

    def device(self, M):
        return torch.device("cpu")

    def nvals(self, M):
        return M.nvals

    def export_block(self, M, rowptr, colidx, offset):
        rowptr.copy_(torch.as_tensor(M.rowptr.astype(np.int64) + offset))
        if M.nvals:
            colidx.copy_(torch.as_tensor(M.colidx.astype(np.int64)).to(torch.int32))

    def wrap(self, nrows, ncols, rowptr, colidx, nnz):
        return oracle.Csr(nrows, ncols, rowptr.numpy().astype(np.uint64),
                          colidx[:nnz].numpy().astype(np.uint32))

    def mxm(self, C, A, B, accumulate, closure_step=False):
        return oracle.mxm(A, B, C if accumulate else None)


def rows_of(M, r0, r1):
    rp = M.rowptr[r0:r1 + 1] - M.rowptr[r0]
    ci = M.colidx[int(M.rowptr[r0]):int(M.rowptr[r1])]
    return oracle.Csr(r1 - r0, M.ncols, rp, ci)


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        ops = OracleOps()
        # MxM on an R-MAT, product-balanced rows
        n = 1 << 10
        r, c = spgen.rmat_pairs(10, 8, 0.45, 0.22, 0.22, seed=3)
        A = oracle.build(n, n, r.numpy(), c.numpy())
        lens = np.diff(A.rowptr.astype(np.int64))
        ub = np.add.reduceat(lens[A.colidx.astype(np.int64)], A.rowptr[:-1].astype(np.int64)) if A.nvals else lens
        ub[lens == 0] = 0
        bounds = spdist.product_balanced_bounds(torch.as_tensor(ub), world)
        r0, r1 = bounds[rank], bounds[rank + 1]
        Al = rows_of(A, r0, r1)
        Cl = spdist.distributed_mxm(ops, Al, Al, n, n)
        full = oracle.mxm(A, A)
        ok_mxm = Cl == rows_of(full, r0, r1)
        # closure of an edge-labelled DAG
        m = 700
        (a0, b0), (a1, b1) = spgen.labeled_dag(m, 0.25, seed=5)
        G = oracle.build(m, m, np.concatenate([a0.numpy(), a1.numpy()]), np.concatenate([b0.numpy(), b1.numpy()]))
        gb = spdist.product_balanced_bounds(torch.as_tensor(np.diff(G.rowptr.astype(np.int64))), world)
        s0, s1 = gb[rank], gb[rank + 1]
        Cl2, it = spdist.distributed_closure(ops, rows_of(G, s0, s1), m)
        ref, ref_it = oracle.closure(G)
        ok_clo = (Cl2 == rows_of(ref, s0, s1)) and it == ref_it
        # degenerate split: rank 1 owns no rows (empty CSR block in the
        # padded all-gather, 0-row local multiply)
        eb = [0, n, n]
        Ae = rows_of(A, eb[rank], eb[rank + 1])
        Ce = spdist.distributed_mxm(ops, Ae, Ae, n, n)
        ok_mxm = ok_mxm and Ce == rows_of(full, eb[rank], eb[rank + 1])
        q.put((rank, bool(ok_mxm), bool(ok_clo), bounds, it, ref_it))
    finally:
        dist.destroy_process_group()


def test_row_partitioned_protocol_gloo_ws2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, ok_mxm, ok_clo, bounds, it, ref_it in res:
        assert ok_mxm, f"rank {rank}: distributed MxM rows differ"
        assert ok_clo, f"rank {rank}: distributed closure differs ({it} vs {ref_it} iterations)"
        assert bounds[0] == 0 and bounds[-1] == 1024 and bounds[1] > 0


def test_product_balanced_bounds():
    w = torch.tensor([100, 0, 0, 1, 1, 1, 100, 5, 5, 5], dtype=torch.int64)
    b = spdist.product_balanced_bounds(w, 3)
    assert b[0] == 0 and b[-1] == 10 and all(x <= y for x, y in zip(b, b[1:]))
    assert spdist.product_balanced_bounds(torch.zeros(0, dtype=torch.int64), 2) == [0, 0, 0]
    # each block's weight is within one max-row of the ideal share
    cw = np.cumsum(w.numpy() + 1)
    for i in range(1, 3):
        assert abs(cw[b[i] - 1] - cw[-1] * i / 3) <= 101
