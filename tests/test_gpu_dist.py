"""The production multi-GPU path on the CUDA library (one GPU here):
``spbla_Matrix_AssembleRowBlocks`` bit-exact round trip, and the
row-partitioned ``distributed_mxm`` / ``distributed_closure`` of dist.py with
:class:`CudaOps` at world_size 2 (two processes sharing cuda:0, gloo for the
collectives), with B all-gathered either by the peer-memory push kernel or by
broadcasts, every rank's rows compared with the oracle."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import spgen
from helpers import assert_same, gpu_lib

pytestmark = pytest.mark.gpu


def rows_of(M, r0, r1):
    rp = M.rowptr[r0:r1 + 1] - M.rowptr[r0]
    ci = M.colidx[int(M.rowptr[r0]):int(M.rowptr[r1])]
    return oracle.Csr(r1 - r0, M.ncols, rp, ci)


def device_block(sp, M, r0, r1):
    rp, ci = M.device_tensors()
    b, e = int(rp[r0]), int(rp[r1])
    return (r1 - r0, (rp[r0:r1 + 1] - b).contiguous(), ci[b:e].contiguous(), e - b)


def test_assemble_row_blocks_roundtrip():
    sp = gpu_lib()
    n = 1 << 14
    r, c = spgen.rmat_pairs(14, 8, 0.45, 0.22, 0.22, seed=11)
    A = sp.Matrix.from_pairs(n, n, r.cuda(), c.cuda())
    O = oracle.build(n, n, r.numpy(), c.numpy())
    cuts = [0, 5000, 5000, 12000, n]  # includes an empty block
    blocks = [device_block(sp, A, a, b) for a, b in zip(cuts[:-1], cuts[1:])]
    B = sp.Matrix.new(n, n)
    B.assemble_row_blocks(blocks)
    assert_same(B, O, "assembled row blocks")
    assert_same(sp.mxm(B, B), oracle.mxm(O, O), "A.A on the assembled matrix")


def test_export_row_block_multi_and_peer_buffers():
    """spbla_Matrix_ExportRowBlockMulti writes one row block (offsets shifted)
    into many destinations at once -- 11 here, so the kernel's 8-destination
    batches split -- including same-process IPC buffers; a garbage IPC handle
    is a clean DEVICE_ERROR."""
    sp = gpu_lib()
    n = 1 << 12
    r, c = spgen.rmat_pairs(12, 8, 0.45, 0.22, 0.22, seed=9)
    A = sp.Matrix.from_pairs(n, n, r.cuda(), c.cuda())
    rp, ci = A.device_tensors()
    off = 12345
    dsts = [(torch.zeros(n + 1, dtype=torch.int64, device="cuda"), torch.zeros(A.nvals, dtype=torch.int32, device="cuda"))
            for _ in range(10)]
    pb_rp, pb_ci = sp.PeerBuffer((n + 1) * 8), sp.PeerBuffer(A.nvals * 4)
    ptrs = [(a.data_ptr(), b.data_ptr()) for a, b in dsts] + [(pb_rp.ptr, pb_ci.ptr)]
    A.export_row_block_multi(ptrs, off)
    torch.cuda.synchronize()
    for a, b in dsts + [(pb_rp.tensor(torch.int64, n + 1), pb_ci.tensor(torch.int32, A.nvals))]:
        assert torch.equal(a, rp + off) and torch.equal(b, ci)
    pb_rp.close()
    pb_ci.close()
    with pytest.raises(sp.SpblaError):
        sp.PeerBuffer(handle=bytes(64))


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def worker(rank, world, port, q, peer):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_orachevkkg21_b200 as sp
        from paper_conf_ipps_orachevkkg21_b200 import dist as spdist
        sp.Initialize(0)
        torch.cuda.set_device(0)
        ops = spdist.CudaOps(sp, peer=peer)
        n = 1 << 13
        r, c = spgen.rmat_pairs(13, 12, 0.45, 0.22, 0.22, seed=3)
        O = oracle.build(n, n, r.numpy(), c.numpy())
        lens = np.diff(O.rowptr.astype(np.int64))
        ub = np.zeros(n, np.int64)
        nzr = lens > 0
        ub[nzr] = np.add.reduceat(lens[O.colidx.astype(np.int64)], O.rowptr[:-1].astype(np.int64)[nzr])
        bounds = spdist.product_balanced_bounds(torch.as_tensor(ub), world)
        r0, r1 = bounds[rank], bounds[rank + 1]
        sel = (r.numpy() >= r0) & (r.numpy() < r1)
        Al = sp.Matrix.from_pairs(r1 - r0, n, torch.as_tensor(r.numpy()[sel] - r0).cuda(),
                                  torch.as_tensor(c.numpy()[sel]).cuda())
        Cl = spdist.distributed_mxm(ops, Al, Al, n, n)
        rp, ci = Cl.to_csr()
        want = rows_of(oracle.mxm(O, O), r0, r1)
        ok_mxm = np.array_equal(rp, want.rowptr) and np.array_equal(ci, want.colidx)
        # closure of an edge-labelled DAG, row-partitioned
        m = 3000
        (a0, b0), (a1, b1) = spgen.labeled_dag(m, 0.25, seed=5)
        src = np.concatenate([a0.numpy(), a1.numpy()])
        dst = np.concatenate([b0.numpy(), b1.numpy()])
        G = oracle.build(m, m, src, dst)
        gb = spdist.product_balanced_bounds(torch.as_tensor(np.diff(G.rowptr.astype(np.int64))), world)
        s0, s1 = gb[rank], gb[rank + 1]
        sel = (src >= s0) & (src < s1)
        Gl = sp.Matrix.from_pairs(s1 - s0, m, torch.as_tensor(src[sel] - s0).cuda(), torch.as_tensor(dst[sel]).cuda())
        Cl2, it = spdist.distributed_closure(ops, Gl, m)
        ref, ref_it = oracle.closure(G)
        rp2, ci2 = Cl2.to_csr()
        want2 = rows_of(ref, s0, s1)
        ok_clo = np.array_equal(rp2, want2.rowptr) and np.array_equal(ci2, want2.colidx) and it == ref_it
        used_peer = ops.peer is not None and ops.peer.ok and ops.peer.own is not None
        if ops.peer is not None:
            ops.peer._release()
        q.put((rank, bool(ok_mxm), bool(ok_clo), it, ref_it, None, used_peer))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, False, False, 0, 0, repr(e), False))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("peer", [True, False], ids=["peer_push", "broadcast"])
def test_distributed_cuda_ws2(peer):
    """peer_push: B all-gathered by the push kernel over peer memory (CUDA IPC
    between the two processes; on one GPU the mapping is same-device);
    broadcast: one NCCL/gloo broadcast per rank."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    procs = [ctx.Process(target=worker, args=(r, 2, port, q, peer)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    for rank, ok_mxm, ok_clo, it, ref_it, err, used_peer in res:
        assert err is None, f"rank {rank}: {err}"
        assert used_peer == peer, f"rank {rank}: peer push used = {used_peer}"
        assert ok_mxm, f"rank {rank}: distributed MxM rows differ"
        assert ok_clo, f"rank {rank}: distributed closure differs ({it} vs {ref_it} iterations)"
