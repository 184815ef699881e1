"""Seeded, counter-based synthetic inputs shared by the oracle side and the CUDA side.

This module holds NONE of the method's arithmetic (no sums, no distances, no gradients): it only maps
(seed, global element index) -> a value.  Every value is produced with integer ops plus at most one
exactly-rounded float conversion, so torch-CPU, torch-CUDA and NumPy (via ``.numpy()``) see identical
bits, and a row shard ``[r0, r1)`` of a matrix regenerates exactly the rows of the full matrix
(DESIGN.md §4).  Hash: Wellons' ``lowbias32`` applied to (seed, hi32(i), lo32(i)).
"""
from __future__ import annotations

import torch

_M32 = 0xFFFFFFFF
_CHUNK = 1 << 24  # elements per generation slice (bounds int64 temporaries to ~128 MiB)


def _lowbias32(x: torch.Tensor) -> torch.Tensor:
    # int64 tensors holding values in [0, 2^32); products wrap in two's complement and are masked.
    x = x & _M32
    x = x ^ (x >> 16)
    x = (x * 0x7FEB352D) & _M32
    x = x ^ (x >> 15)
    x = (x * 0x846CA68B) & _M32
    x = x ^ (x >> 16)
    return x


def _lowbias32_int(x: int) -> int:
    x &= _M32
    x ^= x >> 16
    x = (x * 0x7FEB352D) & _M32
    x ^= x >> 15
    x = (x * 0x846CA68B) & _M32
    x ^= x >> 16
    return x


def hash32(seed: int, idx: torch.Tensor) -> torch.Tensor:
    """32-bit hash of (seed, idx) for an int64 index tensor; result int64 in [0, 2^32)."""
    s = _lowbias32_int(seed)
    hi = idx >> 32
    lo = idx & _M32
    return _lowbias32(lo ^ _lowbias32(hi ^ s))


def _indices(offset: int, n: int, device) -> torch.Tensor:
    return torch.arange(offset, offset + n, dtype=torch.int64, device=device)


def _fill(out: torch.Tensor, offset: int, fn) -> torch.Tensor:
    flat = out.view(-1)
    n = flat.numel()
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        flat[s:e] = fn(_indices(offset + s, e - s, out.device)).to(out.dtype)
    return out


def _empty(shape, dtype, device):
    return torch.empty(tuple(shape), dtype=dtype, device=device)


# ---------------------------------------------------------------- element kinds

def uniform_f32(seed, shape, offset=0, device="cpu", lo=0.0, scale=1.0):
    """fp32 values lo + scale * (h >> 8) * 2^-24 (exact when scale is a power of two)."""
    def fn(i):
        u = (hash32(seed, i) >> 8).to(torch.float64) * (2.0 ** -24)
        return u * scale + lo
    return _fill(_empty(shape, torch.float32, device), offset, fn)


def uniform_f64(seed, shape, offset=0, device="cpu", lo=0.0, scale=1.0):
    """fp64 values lo + scale * u, u = (h1 >> 11 : h2) * 2^-53 from two hashes (53 random bits, exact)."""
    def fn(i):
        h1 = hash32(seed, i) >> 11                       # 21 bits
        h2 = hash32(seed ^ 0x5bd1e995, i)                 # 32 bits
        u = ((h1 << 32) | h2).to(torch.float64) * (2.0 ** -53)
        return u * scale + lo
    return _fill(_empty(shape, torch.float64, device), offset, fn)


def exact_f32(seed, shape, offset=0, device="cpu"):
    """fp32 values k * 2^-8, k in [0, 256): sums of <= 65,536 of them are exact in fp32."""
    def fn(i):
        return (hash32(seed, i) >> 24).to(torch.float64) * (2.0 ** -8)
    return _fill(_empty(shape, torch.float32, device), offset, fn)


def small_int_f32(seed, shape, lo=0, hi=15, offset=0, device="cpu"):
    """fp32 holding integers in [lo, hi]."""
    span = hi - lo + 1

    def fn(i):
        return (hash32(seed, i) % span + lo).to(torch.float64)
    return _fill(_empty(shape, torch.float32, device), offset, fn)


def int_uniform(seed, shape, lo, hi, dtype=torch.int32, offset=0, device="cpu"):
    """Integers in [lo, hi] (hi - lo < 2^32)."""
    span = hi - lo + 1
    assert 0 < span <= (1 << 32)

    def fn(i):
        return hash32(seed, i) % span + lo
    return _fill(_empty(shape, dtype, device), offset, fn)


def int64_wide(seed, shape, offset=0, device="cpu"):
    """Full-range int64 values (two 32-bit hashes); sums of these wrap mod 2^64."""
    def fn(i):
        a = hash32(seed, i)
        b = hash32(seed ^ 0x5BD1E995, i)
        return (a << 32) | b  # wraps into the signed range
    return _fill(_empty(shape, torch.int64, device), offset, fn)


def arange_matrix(shape, dtype=torch.int64, offset=0, device="cpu"):
    """m[r, c] = offset + r * C + c, cast (wrapping) to dtype."""
    def fn(i):
        if dtype == torch.int32:
            return ((i & _M32) ^ 0x80000000) - 0x80000000  # two's-complement wrap to int32
        return i
    return _fill(_empty(shape, dtype, device), offset, fn)


def ones(shape, dtype, device="cpu"):
    return torch.ones(tuple(shape), dtype=dtype, device=device)


# ---------------------------------------------------------------- workload recipes

def kmeans_inputs(N, D, K, seed=5, row_offset=0, device="cpu", integer=False):
    """Centroids U[-8,8)^D and points = centroid[z_i] + noise.

    ``integer=True`` draws integer coordinates in [-8, 8] so every fp32 squared distance is exact.
    ``row_offset`` lets a shard regenerate points [row_offset, row_offset + N) of the full set.
    """
    if integer:
        ctr = int_uniform(seed, (K, D), -8, 8, dtype=torch.int64, device=device).to(torch.float32)
        z = int_uniform(seed + 1, (N,), 0, K - 1, dtype=torch.int64, offset=row_offset, device=device)
        noise = int_uniform(seed + 2, (N, D), -2, 2, dtype=torch.int64, offset=row_offset * D,
                            device=device).to(torch.float32)
        x = ctr.index_select(0, z) + noise
        x.clamp_(-8, 8)
        return x.contiguous(), ctr
    ctr = uniform_f32(seed, (K, D), device=device, lo=-8.0, scale=16.0)
    z = int_uniform(seed + 1, (N,), 0, K - 1, dtype=torch.int64, offset=row_offset, device=device)
    x = _empty((N, D), torch.float32, device)
    flat = x.view(-1)
    n = N * D
    base = row_offset * D
    for s in range(0, n, _CHUNK):
        e = min(n, s + _CHUNK)
        i = _indices(base + s, e - s, device)
        acc = torch.zeros(e - s, dtype=torch.float64, device=device)
        for j in range(4):  # Irwin-Hall(4) - 2: mean 0, var 1/3; exact in fp64, one rounding to fp32
            acc += (hash32(seed + 10 + j, i) >> 8).to(torch.float64) * (2.0 ** -24)
        rows = (torch.arange(s, e, device=device) // D)
        cols = (torch.arange(s, e, device=device) % D)
        c = ctr.to(torch.float64)[z[rows], cols]
        flat[s:e] = (c + acc - 2.0).to(torch.float32)
    return x, ctr


def logreg_inputs(B, Rb, C, seed=6, batch_offset=0, device="cpu", y_zero=False):
    """x U[0,1)^(B*Rb x C), y in {0,1}^(B*Rb), w U[-1/16,1/16)^C."""
    n_rows = B * Rb
    r0 = batch_offset * Rb
    x = uniform_f32(seed, (n_rows, C), offset=r0 * C, device=device)
    if y_zero:
        y = torch.zeros(n_rows, dtype=torch.float32, device=device)
    else:
        y = int_uniform(seed + 1, (n_rows,), 0, 1, dtype=torch.int64, offset=r0,
                        device=device).to(torch.float32)
    w = uniform_f32(seed + 2, (C,), device=device, lo=-1.0 / 16, scale=1.0 / 8)
    return x, y, w


def _pair_clz(h: torch.Tensor) -> torch.Tensor:
    """Number of leading all-zero bit PAIRS of a 32-bit value (0..16), integer ops only."""
    k = torch.zeros_like(h)
    for j in range(1, 17):
        k += (h < (1 << (32 - 2 * j))).to(h.dtype)
    return k


def pagerank_inputs(N, avg_deg=16, seed=7, max_deg=1024, device="cpu"):
    """A directed multigraph of N nodes as the CSR of IN-neighbours: row n lists every w with an edge
    w -> n (Fig 5: `n.nbrs`), plus each node's out-degree and a previous PageRank vector.

    In-degrees follow a doubling-class power law (integer ops only): with k = leading zero bit pairs of
    a hash (P(k >= j) = 4^-j) and base = dmin * 2^k, d_n = min(max_deg, base + hash' mod base), mean
    about 2.25 * dmin, dmin = max(1, round(avg_deg / 2.25)). Neighbours are uniform over [0, N).
    Returns (rowptr int64 [N+1], colidx int32 [E], pr float32 [N], outdeg int32 [N])."""
    dmin = max(1, int(round(avg_deg / 2.25)))
    i = _indices(0, N, device)
    k = torch.clamp(_pair_clz(hash32(seed, i)), max=20)
    base = dmin * (torch.ones_like(k) << k)
    deg = torch.clamp(base + hash32(seed + 1, i) % base, max=max_deg)
    rowptr = torch.zeros(N + 1, dtype=torch.int64, device=device)
    rowptr[1:] = torch.cumsum(deg, 0)
    E = int(rowptr[-1])
    colidx = _empty((E,), torch.int32, device)
    _fill(colidx, 0, lambda j: hash32(seed + 2, j) % N)
    outdeg = torch.bincount(colidx.long(), minlength=N).to(torch.int32)
    pr = uniform_f32(seed + 3, (N,), device=device, lo=0.5, scale=1.0) * (1.0 / N)
    return rowptr, colidx, pr.contiguous(), outdeg
