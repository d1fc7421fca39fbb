"""Host-parallel driver of the UNCHANGED oracle — TEST INFRASTRUCTURE ONLY.

Row-wise Gustavson rows are independent (§II l.236: row i of
C = A x B is the OR of the rows B_k, k in A_i), so the oracle's own
``mxm_rows`` (``spbla_oracle.cpp``, one ``std::set`` per row) can be
evaluated over contiguous row chunks on every host core.  No arithmetic
lives here: chunking, threads and a comparison callback only.  ctypes
releases the GIL around the foreign call, so a thread pool runs the chunks
truly in parallel.

Used by the full-size parity tests (tests/test_gpu_fullsize.py) and by
bench.py's ``cpu_baseline`` / ``--impl reference`` leg.
"""
from __future__ import annotations

import os
from concurrent.futures import ThreadPoolExecutor

import numpy as np

from . import Csr, mxm_rows


def host_cores() -> int:
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def row_products(a: Csr, b: Csr) -> np.ndarray:
    """Products per row of A x B (sum of |B_k| over k in A_i), int64.  Only a
    size count for chunking — not part of the multiply."""
    blen = np.diff(b.rowptr.astype(np.int64))
    per = blen[a.colidx.astype(np.int64)] if a.nvals else np.zeros(0, np.int64)
    cs = np.concatenate([[0], np.cumsum(per)])
    rp = a.rowptr.astype(np.int64)
    return cs[rp[1:]] - cs[rp[:-1]]


def chunk_bounds(weight: np.ndarray, target: float) -> list[tuple[int, int]]:
    """Contiguous row ranges of about ``target`` total weight (+1 per row)."""
    n = len(weight)
    if n == 0:
        return []
    cum = np.cumsum(weight.astype(np.float64) + 1.0)
    nch = max(1, int(np.ceil(cum[-1] / max(target, 1.0))))
    cuts = np.searchsorted(cum, cum[-1] * np.arange(1, nch) / nch, side="right")
    edges = np.unique(np.concatenate([[0], cuts, [n]]))
    return [(int(s), int(e)) for s, e in zip(edges[:-1], edges[1:]) if e > s]


def mxm_rows_chunked(a: Csr, b: Csr, chunks, consume, c: Csr | None = None, threads: int | None = None):
    """For every (r0, r1) in ``chunks``: R = oracle.mxm_rows(a, b, [r0, r1),
    c), then ``consume(r0, r1, R)`` (called from the worker thread; must be
    thread-safe).  At most 2*threads chunks are in flight."""
    threads = threads or host_cores()

    def work(ch):
        r0, r1 = ch
        R = mxm_rows(a, b, np.arange(r0, r1, dtype=np.uint32), c)
        return consume(r0, r1, R)

    out = []
    with ThreadPoolExecutor(max_workers=threads) as ex:
        futs = []
        for ch in chunks:
            futs.append(ex.submit(work, ch))
            if len(futs) >= 2 * threads:
                out.append(futs.pop(0).result())
        out.extend(f.result() for f in futs)
    return out


def build_chunked(nrows: int, ncols: int, rows, cols, block_rows: int = 1 << 16,
                  threads: int | None = None) -> Csr:
    """``oracle.build`` over row blocks of the pair list (PAPER.md l.231,
    duplicates collapse): the pairs are only partitioned by row block here;
    each block is built by the unchanged oracle and the blocks' CSR arrays
    are concatenated with their row offsets shifted."""
    from . import build
    r = np.ascontiguousarray(rows, dtype=np.int64)
    c = np.ascontiguousarray(cols, dtype=np.uint32)
    if r.size and (r.min() < 0 or r.max() >= nrows):
        raise IndexError("build_chunked: row index out of range")
    blk = r // block_rows
    order = np.argsort(blk, kind="stable")
    nblk = (nrows + block_rows - 1) // block_rows
    starts = np.searchsorted(blk[order], np.arange(nblk + 1))
    threads = threads or host_cores()

    def one(b):
        sel = order[starts[b]:starts[b + 1]]
        r0 = b * block_rows
        nr = min(block_rows, nrows - r0)
        return build(nr, ncols, (r[sel] - r0).astype(np.uint32), c[sel])

    with ThreadPoolExecutor(max_workers=threads) as ex:
        parts = list(ex.map(one, range(nblk)))
    rps, base = [np.zeros(1, np.uint64)], np.uint64(0)
    for p in parts:
        rps.append(p.rowptr[1:] + base)
        base += np.uint64(p.nvals)
    ci = np.concatenate([p.colidx for p in parts]) if parts else np.zeros(0, np.uint32)
    return Csr(nrows, ncols, np.concatenate(rps), ci)
