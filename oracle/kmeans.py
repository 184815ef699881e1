"""Oracle: k-means assignment step — TEST INFRASTRUCTURE ONLY (see oracle/__init__).

The nest (BASELINE.json config 4; the triply nested form of PAPER.md L606-610, related to the
MSMBuilder clustering case study L1256-1271):
    points mapRows { x_i => (0 until K) argmin { k => (x_i zipWith c_k)((a,b) => (a-b)^2) reduce + } }
i.e.  a[i] = min{ k : Σ_d (x[i,d] − c[k,d])² is minimal }   — ties go to the lowest k (G20).
The paper has no k-means and fixes no precision, so the decision is taken in fp64 as written (DESIGN.md
reading G25): d(i,k) = Σ_{d=0}^{D-1} (x_id − c_kd)² evaluated left to right in IEEE fp64 — each
difference, square and add rounded to nearest, no fused multiply-add — and a[i] is the lowest k whose
d(i,k) is minimal. (This equals the exact-real argmin except when two exact distances lie within the
fp64 rounding error of each other, ~D·2^-53 relative; tests pin that against exact rationals.)

The centroid update that follows an assignment is Table I's groupBy (L292) followed
by a Reduce per group:
    points groupBy { i => a_i }  map { g => ((g map x) reduce +, g.size) }
i.e. for k in [0, K):  U[k, d] = Σ_{i : a_i = k} x[i, d]  (d < D),  U[k, D] = |{i : a_i = k}|.
Points whose a_i lies outside [0, K) belong to no group (reading G23). fp64 sums, exact counts.
"""
from __future__ import annotations

import math

import numpy as np


def distance_literal(xi, ck) -> float:
    """d = Σ_d (x_d − c_d)² left to right in fp64 (Python floats are IEEE doubles; every op rounds)."""
    d = 0.0
    for a, b in zip(xi, ck):
        t = float(a) - float(b)
        d = d + t * t
    return d


def assign_literal(x: np.ndarray, c: np.ndarray) -> list:
    """Pure-Python triple loop, outer Map over points, argmin over centroids, Reduce over dims."""
    xs, cs = x.tolist(), c.tolist()
    out = []
    for xi in xs:
        best_k, best_d = -1, None
        for k, ck in enumerate(cs):
            d = distance_literal(xi, ck)
            if best_d is None or d < best_d:       # strict: the first (lowest) k wins ties
                best_k, best_d = k, d
        out.append(best_k)
    return out


def distances(x: np.ndarray, c: np.ndarray, chunk: int = 4096) -> np.ndarray:
    """d[i,k] = Σ_d (x[i,d] − c[k,d])², the same fp64 operations in the same order as
    distance_literal (one elementwise subtract, square and add per d, over all (i, k) at once)."""
    x64, c64 = x.astype(np.float64), c.astype(np.float64)
    out = np.empty((x.shape[0], c.shape[0]), dtype=np.float64)
    for s in range(0, x.shape[0], chunk):
        xs = x64[s:s + chunk]
        acc = np.zeros((xs.shape[0], c.shape[0]), dtype=np.float64)
        for d in range(x.shape[1]):
            t = xs[:, None, d] - c64[None, :, d]
            acc += t * t
        out[s:s + chunk] = acc
    return out


def assign(x: np.ndarray, c: np.ndarray, chunk: int = 4096) -> np.ndarray:
    """Vectorised a[i]: ``np.argmin`` returns the first minimum, i.e. the lowest k on ties."""
    out = np.empty(x.shape[0], dtype=np.int32)
    for s in range(0, x.shape[0], chunk):
        out[s:s + chunk] = np.argmin(distances(x[s:s + chunk], c), axis=1)
    return out


def update_literal(x: np.ndarray, a: np.ndarray, K: int) -> list:
    """Pure-Python groupBy then Reduce: rows [Σ_{a_i = k} x_i (math.fsum per dim) ..., count_k]."""
    xs, aa = x.tolist(), [int(v) for v in a.tolist()]
    D = x.shape[1]
    groups = {k: [] for k in range(K)}
    for xi, k in zip(xs, aa):
        if 0 <= k < K:
            groups[k].append(xi)
    return [[math.fsum(float(p[d]) for p in groups[k]) for d in range(D)] + [float(len(groups[k]))]
            for k in range(K)]


def update(x: np.ndarray, a: np.ndarray, K: int) -> np.ndarray:
    """Vectorised: U[k] = (np.add.reduce over the rows with a_i = k in fp64, count) -> [K, D+1] fp64."""
    N, D = x.shape
    out = np.zeros((K, D + 1), dtype=np.float64)
    x64 = x.astype(np.float64)
    a = np.asarray(a).astype(np.int64)
    for k in range(K):
        mask = a == k
        out[k, :D] = np.add.reduce(x64[mask], axis=0) if mask.any() else 0.0
        out[k, D] = float(mask.sum())
    return out


def update_scale(x: np.ndarray, a: np.ndarray, K: int) -> np.ndarray:
    """Σ_{a_i = k} |x[i, d]| — the scale of the fp32 tolerance bound for signed data."""
    return update(np.abs(x.astype(np.float64)), a, K)[:, :-1]
