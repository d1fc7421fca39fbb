"""Row-partitioned multi-GPU driver: one process per GPU,
``torch.distributed`` over NCCL for the plumbing.

A and C are row-partitioned; B is assembled on every rank from the row
shards each rank owns (an all-gather of CSR blocks over NVLink — the "B
broadcast" of the north star), then every rank multiplies its own rows.  The
transitive closure all-gathers the new C shards every iteration and tests the
fixed point with an all-reduce of nnz.

The local operations go through an ``ops`` object so the host-side protocol
(partitioning, padded all-gather of variable-size CSR blocks, fixed-point
loop) is exercised by world_size-2 gloo tests on CPU with the oracle as the
local multiply; production uses :class:`CudaOps` (the CUDA library).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def product_balanced_bounds(row_weight: torch.Tensor, world: int):
    """Row boundaries [b0=0, b1, ..., bN=nrows] splitting rows into ``world``
    contiguous blocks of near-equal total weight (weight = products + 1 per
    row, so empty rows still spread)."""
    n = int(row_weight.numel())
    w = row_weight.to(torch.float64).cpu() + 1.0
    cum = torch.cumsum(w, 0)
    total = float(cum[-1]) if n else 0.0
    bounds = [0]
    for r in range(1, world):
        target = total * r / world
        b = int(torch.searchsorted(cum, torch.tensor([target], dtype=torch.float64))[0]) + 1 if n else 0
        bounds.append(min(max(b, bounds[-1]), n))
    bounds.append(n)
    return bounds


def allgather_csr(rowptr: torch.Tensor, colidx: torch.Tensor, group=None):
    """All-gather variable-size CSR row blocks.  ``rowptr`` (int64, starts at
    0, nrows+1) and ``colidx`` (int32) of this rank's block; returns
    [(nrows_b, rowptr_b, colidx_b, nnz_b)] for every rank in rank order.
    Blocks are padded to the largest one for the collective."""
    world = dist.get_world_size(group)
    dev = rowptr.device
    if dev.type == "cuda" and dist.get_backend(group) == "gloo":
        # gloo path (CPU tests / single-GPU multi-rank runs): collective on host copies
        blocks = allgather_csr(rowptr.cpu(), colidx.cpu(), group)
        return [(nr, rp.to(dev), ci.to(dev), nz) for nr, rp, ci, nz in blocks]
    nrows = rowptr.numel() - 1
    nnz = colidx.numel()
    sizes = torch.tensor([nrows, nnz], dtype=torch.int64, device=dev)
    all_sizes = torch.empty(world * 2, dtype=torch.int64, device=dev)
    dist.all_gather_into_tensor(all_sizes, sizes, group=group)
    all_sizes = all_sizes.view(world, 2).cpu().tolist()
    max_rows = max(s[0] for s in all_sizes)
    max_nnz = max(max(s[1] for s in all_sizes), 1)
    rp = torch.zeros(max_rows + 1, dtype=torch.int64, device=dev)
    rp[:nrows + 1] = rowptr
    ci = torch.zeros(max_nnz, dtype=torch.int32, device=dev)
    ci[:nnz] = colidx
    rp_all = torch.empty(world * (max_rows + 1), dtype=torch.int64, device=dev)
    ci_all = torch.empty(world * max_nnz, dtype=torch.int32, device=dev)
    dist.all_gather_into_tensor(rp_all, rp, group=group)
    dist.all_gather_into_tensor(ci_all, ci, group=group)
    out = []
    for b, (nr, nz) in enumerate(all_sizes):
        rpb = rp_all[b * (max_rows + 1): b * (max_rows + 1) + nr + 1]
        cib = ci_all[b * max_nnz: b * max_nnz + nz]
        out.append((nr, rpb, cib, nz))
    return out


class CudaOps:
    """Local operations on the CUDA library (production path)."""

    def __init__(self, sp):
        self.sp = sp

    def csr(self, M):
        return M.device_tensors()

    def nvals(self, M):
        return M.nvals

    def assemble(self, blocks, nrows, ncols):
        B = self.sp.Matrix.new(nrows, ncols)
        B.assemble_row_blocks(blocks)
        return B

    def mxm(self, C, A, B, accumulate, closure_step=False):
        if C is None:
            C = self.sp.Matrix.new(A.nrows, B.ncols)
        self.sp.MxM(C, A, B, accumulate=accumulate, closure_step=closure_step)
        return C


def allreduce_int(x: int, group=None, op=dist.ReduceOp.SUM, device=None) -> int:
    """All-reduce of one integer (host tensor for gloo, device tensor for NCCL)."""
    dev = "cpu" if dist.get_backend(group) == "gloo" else (device or "cuda")
    t = torch.tensor([x], dtype=torch.int64, device=dev)
    dist.all_reduce(t, op=op, group=group)
    return int(t)


def gather_rows(ops, M_local, nrows_total, ncols, group=None):
    rp, ci = ops.csr(M_local)
    blocks = allgather_csr(rp, ci, group)
    return ops.assemble(blocks, nrows_total, ncols)


def distributed_mxm(ops, A_local, B_local, nrows_B, ncols_B, group=None, C_local=None, accumulate=False):
    """C_local (+)= A_local x B with B the row-concatenation of every rank's
    B_local (assembled by an all-gather)."""
    B = gather_rows(ops, B_local, nrows_B, ncols_B, group)
    return ops.mxm(C_local, A_local, B, accumulate)


def distributed_closure(ops, C_local, n, group=None, max_iters=10_000):
    """C += C x C to the fixed point with C row-partitioned: every iteration
    all-gathers the C shards (B = C), updates the local rows, and all-reduces
    nnz to detect the fixed point.  Returns (C_local, iterations)."""
    dev = ops.csr(C_local)[0].device
    prev = allreduce_int(ops.nvals(C_local), group, device=dev)
    it = 0
    while it < max_iters:
        B = gather_rows(ops, C_local, n, n, group)
        C_local = ops.mxm(C_local, C_local, B, True, closure_step=True)
        it += 1
        cur = allreduce_int(ops.nvals(C_local), group, device=dev)
        if cur == prev:
            break
        prev = cur
    return C_local, it
