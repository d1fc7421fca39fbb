"""Seeded synthetic input generators shared by the oracle tests, the CUDA parity
tests and ``bench.py``.

This module holds NO arithmetic of the method (no multiply, merge, Kronecker
or closure): it only draws index pairs.  Every draw is a counter-based hash
(SplitMix64 finaliser over ``(seed, stream, counter)``) evaluated with plain
int64 torch ops, so the same call returns bit-identical pairs on the CPU and
on a CUDA device (integer ops only; no device RNG state).  The recipes and the
parameters chosen for each BASELINE.json config are stated in DESIGN.md §3.

Workload shapes follow the paper's evaluation (§Evaluation, Tables
I and III: RDF / graph-database graphs with 10^5..10^7 vertices and 2..10
edges per vertex; power-law degree structure) and BASELINE.json ``configs``.
"""
from __future__ import annotations

import torch

_M64 = (1 << 64) - 1


def _s64(x: int) -> int:
    """Reinterpret an unsigned 64-bit constant as a signed int64 literal."""
    x &= _M64
    return x - (1 << 64) if x >= (1 << 63) else x


_GOLDEN = _s64(0x9E3779B97F4A7C15)
_MIX1 = _s64(0xBF58476D1CE4E5B9)
_MIX2 = _s64(0x94D049BB133111EB)


def _lsr(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 tensor (torch's >> is arithmetic)."""
    return (x >> s) & ((1 << (64 - s)) - 1)


def _mix(z: torch.Tensor) -> torch.Tensor:
    z = (z ^ _lsr(z, 30)) * _MIX1
    z = (z ^ _lsr(z, 27)) * _MIX2
    return z ^ _lsr(z, 31)


def _mix_int(z: int) -> int:
    """Pure-Python reference of ``_mix`` (used by the generator self-test)."""
    z &= _M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & _M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & _M64
    return z ^ (z >> 31)


def hash64(seed: int, stream: int, counter: torch.Tensor) -> torch.Tensor:
    """64 random bits per element of ``counter`` (int64), as int64."""
    key = _mix_int((seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03 + 1) & _M64)
    return _mix(counter * _GOLDEN + _s64(key))


def hash64_int(seed: int, stream: int, counter: int) -> int:
    key = _mix_int((seed * 0x9E3779B97F4A7C15 + stream * 0xD1B54A32D192ED03 + 1) & _M64)
    return _mix_int((counter * 0x9E3779B97F4A7C15 + key) & _M64)


def uniform_below(seed: int, stream: int, counter: torch.Tensor, bound) -> torch.Tensor:
    """Integers in [0, bound) from the top 31 bits of the hash (bound < 2^31
    or an int64 tensor of per-element bounds < 2^31)."""
    h31 = _lsr(hash64(seed, stream, counter), 33)
    return (h31 * bound) >> 31


def _arange(n: int, device) -> torch.Tensor:
    return torch.arange(n, dtype=torch.int64, device=device)


def scramble(v: torch.Tensor, bits: int, seed: int) -> torch.Tensor:
    """Seeded bijection on [0, 2^bits): odd-multiplier affine maps and
    xor-shifts, each invertible mod 2^bits (Graph500-style relabelling that
    removes R-MAT's artificial locality)."""
    if bits == 0:
        return v
    mask = (1 << bits) - 1
    k1 = (hash64_int(seed, 101, 0) >> 33) | 1
    k2 = (hash64_int(seed, 102, 0) >> 33) | 1
    c1 = hash64_int(seed, 103, 0) & mask
    c2 = hash64_int(seed, 104, 0) & mask
    s = max(1, bits // 2)
    v = (v * k1 + c1) & mask
    v = v ^ (v >> s)
    v = (v * k2 + c2) & mask
    v = v ^ (v >> max(1, s - 1))
    return (v * k1 + c2) & mask


def uniform_pairs(nrows: int, ncols: int, per_row: int, seed: int, device="cpu"):
    """Erdős–Rényi-style CSR input: every row draws ``per_row`` columns
    uniformly (duplicates possible; ``Matrix_Build`` merges them)."""
    e = _arange(nrows * per_row, device)
    rows = e // per_row
    cols = uniform_below(seed, 1, e, ncols)
    return rows.to(torch.int32), cols.to(torch.int32)


def random_pairs(nrows: int, ncols: int, nvals: int, seed: int, device="cpu"):
    """``nvals`` pairs uniform over the whole nrows x ncols grid."""
    e = _arange(nvals, device)
    rows = uniform_below(seed, 2, e, nrows)
    cols = uniform_below(seed, 3, e, ncols)
    return rows.to(torch.int32), cols.to(torch.int32)


def rmat_pairs(scale: int, edge_factor: int, a: float, b: float, c: float,
               seed: int, device="cpu", scramble_ids: bool = True):
    """R-MAT (Chakrabarti et al.) edge list on 2^scale vertices with
    ``edge_factor * 2^scale`` draws.  Each level picks a quadrant with
    probabilities (a, b, c, 1-a-b-c) by comparing 53 hash bits against
    integer thresholds (exact, identical on every device)."""
    n = 1 << scale
    m = n * edge_factor
    e = _arange(m, device)
    ta = int(a * (1 << 53))
    tab = int((a + b) * (1 << 53))
    tabc = int((a + b + c) * (1 << 53))
    r = torch.zeros(m, dtype=torch.int64, device=device)
    cc = torch.zeros(m, dtype=torch.int64, device=device)
    for lvl in range(scale):
        u = _lsr(hash64(seed, 1000 + lvl, e), 11)
        rbit = (u >= tab).to(torch.int64)
        cbit = (((u >= ta) & (u < tab)) | (u >= tabc)).to(torch.int64)
        r |= rbit << lvl
        cc |= cbit << lvl
        del u, rbit, cbit
    if scramble_ids:
        r = scramble(r, scale, seed)
        cc = scramble(cc, scale, seed)
    return r.to(torch.int32), cc.to(torch.int32)


def labeled_dag(n: int, extra_prob: float, seed: int, device="cpu"):
    """Edge-labelled taxonomy-shaped graph (the paper's CFPQ/RPQ RDF graphs:
    subClassOf / type hierarchies, Table III).  Label 0: every vertex
    v>0 has one edge v -> parent, parent uniform in [0, v) (random recursive
    tree).  Label 1: with probability ``extra_prob`` a second edge v -> u,
    u uniform in [0, v).  Returns [(rows, cols) for label 0, for label 1]."""
    v = torch.arange(1, n, dtype=torch.int64, device=device)
    p0 = uniform_below(seed, 11, v, v)
    keep = _lsr(hash64(seed, 12, v), 11) < int(extra_prob * (1 << 53))
    v1 = v[keep]
    p1 = uniform_below(seed, 13, v1, v1)
    return [(v.to(torch.int32), p0.to(torch.int32)),
            (v1.to(torch.int32), p1.to(torch.int32))]


def rsm_pairs(states: int, nlabels: int, per_state: int, seed: int, device="cpu"):
    """Recursive-state-machine (query automaton) adjacency, §I
    (tensor-product RPQ/CFPQ): ``states`` x ``states`` Boolean matrix with
    ``per_state`` transitions out of every state, drawn uniformly."""
    e = _arange(states * per_state, device)
    rows = e // per_state
    cols = uniform_below(seed, 21 + nlabels, e, states)
    return rows.to(torch.int32), cols.to(torch.int32)
