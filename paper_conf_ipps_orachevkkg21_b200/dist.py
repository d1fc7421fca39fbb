"""Row-partitioned multi-GPU driver: one process per GPU,
``torch.distributed`` over NCCL for the plumbing.

A and C are row-partitioned; B is assembled on every rank from the row
shards each rank owns (an all-gather of CSR blocks over NVLink — the "B
broadcast" of the north star), then every rank multiplies its own rows.  The
transitive closure all-gathers the new C shards every iteration and tests the
fixed point with an all-reduce of nnz.

The local operations go through an ``ops`` object so the host-side protocol
(partitioning, exact-size all-gather of CSR row blocks, fixed-point loop) is exercised by world_size-2 gloo tests on CPU with the oracle as the
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


def allgather_rows(ops, M_local, nrows_total, ncols, group=None):
    """All-gather a row-partitioned matrix (every rank's block of rows, in
    rank order) into ONE CSR: the block sizes are exchanged first, every rank
    writes its own block straight into its slice of the gathered rowptr /
    colidx buffers (offsets shifted on the device by ``ops.export_block``),
    and one broadcast per rank fills the other slices -- exact sizes, no
    padding and no second copy.  Returns the gathered matrix (``ops.wrap``)."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    nrows, nnz = ops.shape_nnz(M_local)
    dev = ops.device(M_local)
    gloo = dist.get_backend(group) == "gloo"
    sdev = "cpu" if gloo else dev
    sizes = torch.tensor([nrows, nnz], dtype=torch.int64, device=sdev)
    all_sizes = [torch.empty_like(sizes) for _ in range(world)]
    dist.all_gather(all_sizes, sizes, group=group)
    all_sizes = [tuple(int(v) for v in t.cpu()) for t in all_sizes]
    assert sum(s[0] for s in all_sizes) == nrows_total, "row blocks do not cover the matrix"
    total = sum(s[1] for s in all_sizes)
    rbase = [0] * world
    nbase = [0] * world
    for b in range(1, world):
        rbase[b] = rbase[b - 1] + all_sizes[b - 1][0]
        nbase[b] = nbase[b - 1] + all_sizes[b - 1][1]
    rp_all = torch.empty(nrows_total + 1, dtype=torch.int64, device=dev)
    ci_all = torch.empty(max(total, 1), dtype=torch.int32, device=dev)
    ops.export_block(M_local, rp_all[rbase[rank]:rbase[rank] + nrows + 1], ci_all[nbase[rank]:nbase[rank] + nnz],
                     nbase[rank])
    for b, (nr, nz) in enumerate(all_sizes):
        # (block b's first offset equals block b-1's last: overlapping
        # slices receive identical values)
        for t in (rp_all[rbase[b]:rbase[b] + nr + 1], ci_all[nbase[b]:nbase[b] + nz]):
            if t.numel() == 0:
                continue
            if gloo and t.device.type != "cpu":  # gloo (CPU tests, one-GPU multi-rank runs): via host
                h = t.cpu()
                dist.broadcast(h, src=b, group=group)
                if b != rank:
                    t.copy_(h)
            else:
                dist.broadcast(t, src=b, group=group)
    return ops.wrap(nrows_total, ncols, rp_all, ci_all, total)


class PeerGather:
    """All-gather of CSR row blocks by pushing over peer memory:
    every rank holds two pairs of gathered buffers (rowptr, colidx; double
    buffered so a push never lands in a buffer a peer may still be reading)
    allocated by the library as IPC-shareable device memory, maps every other
    rank's buffers into its address space once (CUDA IPC, opened for its own
    GPU with peer access enabled as needed), and each step writes its own block
    into its slice of EVERY rank's current buffer with one kernel
    (``spbla_Matrix_ExportRowBlockMulti``: the block is loaded once and stored
    world times -- on an NVSwitch box the peer stores go over NVLink), then
    synchronises the device and meets the other ranks at a barrier.  No
    collective library moves the data; NCCL/gloo only carry the block sizes,
    the one-off 64-byte IPC handles and the barrier.

    ``ok`` becomes False (on every rank: an all-reduced flag) when any rank
    cannot map another's buffers; the caller then uses the broadcast
    all-gather."""

    def __init__(self, sp, group=None):
        self.sp = sp
        self.group = group
        self.cap = (0, 0)
        self.own = None    # [parity] -> (PeerBuffer rowptr, PeerBuffer colidx)
        self.peers = None  # [rank][parity] -> (rowptr address, colidx address)
        self.mapped = []
        self.parity = 0
        self.ok = True

    def _release(self):
        for m in self.mapped:  # unmap the peers' buffers, then (after every
            m.close()          # rank has) free our own
        self.mapped = []
        if self.own is not None:
            dist.barrier(group=self.group)
            for pair in self.own:
                for buf in pair:
                    buf.close()
        self.own = self.peers = None

    def _alloc(self, rows_cap, nnz_cap):
        world = dist.get_world_size(self.group)
        rank = dist.get_rank(self.group)
        self._release()
        own = [(self.sp.PeerBuffer(rows_cap * 8), self.sp.PeerBuffer(nnz_cap * 4)) for _ in range(2)]
        objs = [None] * world
        dist.all_gather_object(objs, [[b.handle for b in pair] for pair in own], group=self.group)
        peers, ok = [], True
        for b in range(world):
            if b == rank:
                peers.append([(rp.ptr, ci.ptr) for rp, ci in own])
                continue
            try:
                pair_ptrs = []
                for hrp, hci in objs[b]:
                    mrp, mci = self.sp.PeerBuffer(handle=hrp), self.sp.PeerBuffer(handle=hci)
                    self.mapped += [mrp, mci]
                    pair_ptrs.append((mrp.ptr, mci.ptr))
                peers.append(pair_ptrs)
            except Exception:  # (the GPUs cannot reach each other)
                ok = False
                break
        dev_flag = "cpu" if dist.get_backend(self.group) == "gloo" else "cuda"
        flag = torch.tensor([0 if ok else 1], dtype=torch.int64, device=dev_flag)
        dist.all_reduce(flag, group=self.group)
        self.own, self.peers, self.cap = own, peers, (rows_cap, nnz_cap)
        self.ok = int(flag) == 0
        if not self.ok:
            self._release()

    def gather(self, ops, M_local, nrows_total, ncols):
        world = dist.get_world_size(self.group)
        rank = dist.get_rank(self.group)
        nrows, nnz = ops.shape_nnz(M_local)
        dev = ops.device(M_local)
        sdev = "cpu" if dist.get_backend(self.group) == "gloo" else dev
        sizes = torch.tensor([nrows, nnz], dtype=torch.int64, device=sdev)
        all_sizes = [torch.empty_like(sizes) for _ in range(world)]
        dist.all_gather(all_sizes, sizes, group=self.group)
        all_sizes = [tuple(int(v) for v in t.cpu()) for t in all_sizes]
        assert sum(s[0] for s in all_sizes) == nrows_total, "row blocks do not cover the matrix"
        total = sum(s[1] for s in all_sizes)
        rbase = [0] * world
        nbase = [0] * world
        for b in range(1, world):
            rbase[b] = rbase[b - 1] + all_sizes[b - 1][0]
            nbase[b] = nbase[b - 1] + all_sizes[b - 1][1]
        if nrows_total + 1 > self.cap[0] or max(total, 1) > self.cap[1]:
            # (every rank sees the same sizes: a collective decision; the
            # closure's growing C gets 1.5x headroom)
            self._alloc(nrows_total + 1, max(int(total * 1.5), total, 1))
            if not self.ok:
                return None
        p = self.parity
        self.parity ^= 1
        dsts = [(self.peers[b][p][0] + 8 * rbase[rank], self.peers[b][p][1] + 4 * nbase[rank])
                for b in range(world)]
        ops.export_block_multi(M_local, dsts, nbase[rank])
        torch.cuda.synchronize(dev)
        dist.barrier(group=self.group)
        rp, ci = self.own[p]
        return ops.wrap(nrows_total, ncols, rp.tensor(torch.int64, nrows_total + 1),
                        ci.tensor(torch.int32, max(total, 1)), total)


class CudaOps:
    """Local operations on the CUDA library (production path).  peer=True:
    B is all-gathered by pushing over peer memory (:class:`PeerGather`),
    falling back to the broadcast all-gather when the ranks cannot map each
    other's memory."""

    def __init__(self, sp, peer=True):
        self.sp = sp
        self.peer = PeerGather(sp) if peer else None

    def export_block_multi(self, M, dsts, offset):
        M.export_row_block_multi(dsts, offset)

    def shape_nnz(self, M):
        return M.nrows, M.nvals

    def device(self, M):
        return M.device_tensors()[0].device

    def nvals(self, M):
        return M.nvals

    def export_block(self, M, rowptr, colidx, offset):
        M.export_row_block(rowptr, colidx, offset)

    def wrap(self, nrows, ncols, rowptr, colidx, nnz):
        return self.sp.Matrix.wrap(nrows, ncols, rowptr, colidx, nvals=nnz)

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
    peer = getattr(ops, "peer", None)
    if peer is not None and peer.ok and group is None:
        B = peer.gather(ops, M_local, nrows_total, ncols)
        if B is not None:
            return B
    return allgather_rows(ops, M_local, nrows_total, ncols, group)


def distributed_mxm(ops, A_local, B_local, nrows_B, ncols_B, group=None, C_local=None, accumulate=False):
    """C_local (+)= A_local x B with B the row-concatenation of every rank's
    B_local (assembled by an all-gather)."""
    B = gather_rows(ops, B_local, nrows_B, ncols_B, group)
    return ops.mxm(C_local, A_local, B, accumulate)


def distributed_closure(ops, C_local, n, group=None, max_iters=10_000):
    """C += C x C to the fixed point with C row-partitioned: every iteration
    all-gathers the C shards (B = C), updates the local rows, and all-reduces
    nnz to detect the fixed point.  Returns (C_local, iterations)."""
    dev = ops.device(C_local)
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
