"""Oracle: sumRows / sumCols and their Split(k) partials — TEST INFRASTRUCTURE ONLY (see oracle/__init__).

Definitions (plain, no blocking or reordering beyond the definition):
  sumRows  out[r] = Σ_{c<C} m[r,c]           PAPER.md Fig 1 L68-70 ("m mapRows { r => r reduce + }"), L93-97
  sumCols  out[c] = Σ_{r<R} m[r,c]           PAPER.md Fig 1 L68-70 ("m mapCols { c => c reduce + }")
  Split(k) partial[s][o] = Σ over the s-th contiguous chunk of ⌈N/k⌉ inner indices
                                              PAPER.md §IV-A, Fig 6c; G12
  sumWeightedRows/Cols: the inner pattern is zipWith(v)(*) then reduce(+)
                                              PAPER.md Fig 15; G9
  sumRowsCols: both counts of the Naive Bayes classifier ("the number of words per document and the
  number of documents for each ... word") over one matrix, out = [sumRows | sumCols]
                                              PAPER.md §VI-E; S8 RC
Floating point: fp64 (``math.fsum`` = the correctly rounded exact sum in the literal evaluator).
Integers: exact Python / unsigned NumPy arithmetic, wrapped to the element width (G19).
"""
from __future__ import annotations

import math

import numpy as np

_CHUNK_ELEMS = 1 << 22


def wrap(value: int, bits: int) -> int:
    """Two's-complement wrap of an exact integer to ``bits`` bits (G19)."""
    mask = (1 << bits) - 1
    v = value & mask
    return v - (1 << bits) if v >> (bits - 1) else v


def _is_int(a: np.ndarray) -> bool:
    return np.issubdtype(a.dtype, np.integer)


def _bits(a: np.ndarray) -> int:
    return a.dtype.itemsize * 8


# ------------------------------------------------------------------ literal evaluator (small shapes)

def sum_rows_literal(m: np.ndarray) -> list:
    """Pure-Python nested loops: Map over rows, Reduce over the row (Fig 1 L70)."""
    R, C = m.shape
    rows = m.tolist()
    if _is_int(m):
        return [wrap(sum(int(v) for v in rows[r]), _bits(m)) for r in range(R)]
    return [math.fsum(float(v) for v in rows[r]) for r in range(R)]


def sum_cols_literal(m: np.ndarray) -> list:
    """Pure-Python nested loops: Map over columns, Reduce down the column (Fig 1 L69)."""
    R, C = m.shape
    rows = m.tolist()
    if _is_int(m):
        return [wrap(sum(int(rows[r][c]) for r in range(R)), _bits(m)) for c in range(C)]
    return [math.fsum(float(rows[r][c]) for r in range(R)) for c in range(C)]


def sum_weighted_rows_literal(m: np.ndarray, v: np.ndarray) -> list:
    """out[r] = Σ_c m[r,c]·v[c]  (Fig 15 with rows; zipWith(*) then reduce(+))."""
    R, C = m.shape
    rows, vv = m.tolist(), v.tolist()
    if _is_int(m):
        return [wrap(sum(int(rows[r][c]) * int(vv[c]) for c in range(C)), _bits(m)) for r in range(R)]
    return [math.fsum(float(rows[r][c]) * float(vv[c]) for c in range(C)) for r in range(R)]


def sum_weighted_cols_literal(m: np.ndarray, v: np.ndarray) -> list:
    """out[c] = Σ_r m[r,c]·v[r]  (Fig 15: column c zipWith v, then reduce)."""
    R, C = m.shape
    rows, vv = m.tolist(), v.tolist()
    if _is_int(m):
        return [wrap(sum(int(rows[r][c]) * int(vv[r]) for r in range(R)), _bits(m)) for c in range(C)]
    return [math.fsum(float(rows[r][c]) * float(vv[r]) for r in range(R)) for c in range(C)]


# ------------------------------------------------------------------ vectorised evaluator (large shapes)

def _acc_reduce(block: np.ndarray, axis: int) -> np.ndarray:
    """One NumPy reduction in the exact/fp64 accumulator domain (library primitive)."""
    if _is_int(block):
        # unsigned arithmetic wraps mod 2^64, which is exact for the mod-2^bits result we need
        return np.add.reduce(block.astype(np.int64).view(np.uint64), axis=axis, dtype=np.uint64)
    return np.add.reduce(block.astype(np.float64), axis=axis, dtype=np.float64)


def _finish(acc: np.ndarray, like: np.ndarray) -> np.ndarray:
    if _is_int(like):
        bits = _bits(like)
        if bits == 64:
            return acc.view(np.int64).copy()
        return (acc & np.uint64((1 << bits) - 1)).astype(np.int64).astype(np.uint32).view(np.int32)
    return acc


def sum_rows(m: np.ndarray) -> np.ndarray:
    """out[r] = Σ_c m[r,c]; fp64 (float input) or wrapped integers. Row chunks bound memory."""
    R, C = m.shape
    step = max(1, _CHUNK_ELEMS // max(C, 1))
    parts = [_acc_reduce(m[r:r + step], axis=1) for r in range(0, R, step)]
    acc = np.concatenate(parts) if parts else _acc_reduce(m, axis=1)
    return _finish(acc, m)


def sum_cols(m: np.ndarray) -> np.ndarray:
    """out[c] = Σ_r m[r,c]; partial column sums over row chunks are added in row order."""
    R, C = m.shape
    step = max(1, _CHUNK_ELEMS // max(C, 1))
    acc = None
    for r in range(0, R, step):
        part = _acc_reduce(m[r:r + step], axis=0)
        acc = part if acc is None else acc + part
    if acc is None:
        acc = _acc_reduce(m, axis=0)
    return _finish(acc, m)


def sum_rows_cols(m: np.ndarray) -> np.ndarray:
    """[sumRows(m) | sumCols(m)] — the two Naive Bayes counts (§VI-E), concatenated."""
    return np.concatenate([sum_rows(m), sum_cols(m)])


def sum_rows_cols_literal(m: np.ndarray) -> list:
    return sum_rows_literal(m) + sum_cols_literal(m)


def sum_weighted_rows(m: np.ndarray, v: np.ndarray) -> np.ndarray:
    """out[r] = Σ_c m[r,c]·v[c] (fp32·fp32 products are exact in fp64)."""
    if _is_int(m):
        prod = (m.astype(np.int64).view(np.uint64) * v.astype(np.int64).view(np.uint64)[None, :])
        return _finish(np.add.reduce(prod, axis=1, dtype=np.uint64), m)
    return np.add.reduce(m.astype(np.float64) * v.astype(np.float64)[None, :], axis=1)


def sum_weighted_cols(m: np.ndarray, v: np.ndarray) -> np.ndarray:
    """out[c] = Σ_r m[r,c]·v[r]."""
    if _is_int(m):
        prod = (m.astype(np.int64).view(np.uint64) * v.astype(np.int64).view(np.uint64)[:, None])
        return _finish(np.add.reduce(prod, axis=0, dtype=np.uint64), m)
    return np.add.reduce(m.astype(np.float64) * v.astype(np.float64)[:, None], axis=0)


def sum_abs_rows(m: np.ndarray) -> np.ndarray:
    """Σ_c |m[r,c]| in fp64 — the scale of the fp32 tolerance bound for signed data."""
    return np.add.reduce(np.abs(m.astype(np.float64)), axis=1)


def sum_abs_cols(m: np.ndarray) -> np.ndarray:
    return np.add.reduce(np.abs(m.astype(np.float64)), axis=0)


# ------------------------------------------------------------------ Split(k) white box

def split_chunks(n: int, k: int) -> list:
    """Contiguous chunks of ⌈n/k⌉ indices (L543-544, G12): [(start, end), ...]."""
    chunk = -(-n // k)
    return [(s, min(n, s + chunk)) for s in range(0, n, chunk)]


def split_partials(m: np.ndarray, pattern: str, k: int) -> np.ndarray:
    """partial[s][o] for Split(k) of the inner (Reduce) level (Fig 6c).

    pattern 'rows': inner = columns; 'cols': inner = rows.  Result [G, outer] in fp64 / uint64.
    """
    R, C = m.shape
    if pattern == "rows":
        return np.stack([_acc_reduce(m[:, s:e], axis=1) for s, e in split_chunks(C, k)])
    return np.stack([_acc_reduce(m[s:e, :], axis=0) for s, e in split_chunks(R, k)])
