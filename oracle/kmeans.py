"""Oracle: k-means assignment step — TEST INFRASTRUCTURE ONLY (see oracle/__init__).

The nest (BASELINE.json config 4; the triply nested form of PAPER.md L606-610, related to the
MSMBuilder clustering case study L1256-1271):
    points mapRows { x_i => (0 until K) argmin { k => (x_i zipWith c_k)((a,b) => (a-b)^2) reduce + } }
i.e.  a[i] = min{ k : Σ_d (x[i,d] − c[k,d])² is minimal }   — ties go to the lowest k (G20).
fp64: the difference of two fp32 values and its square are exact in fp64, so the literal evaluator's
``math.fsum`` distance is the correctly rounded exact distance.
"""
from __future__ import annotations

import math

import numpy as np


def assign_literal(x: np.ndarray, c: np.ndarray) -> list:
    """Pure-Python triple loop, outer Map over points, argmin over centroids, Reduce over dims."""
    xs, cs = x.tolist(), c.tolist()
    out = []
    for xi in xs:
        best_k, best_d = -1, None
        for k, ck in enumerate(cs):
            d = math.fsum((float(a) - float(b)) ** 2 for a, b in zip(xi, ck))
            if best_d is None or d < best_d:       # strict: the first (lowest) k wins ties
                best_k, best_d = k, d
        out.append(best_k)
    return out


def distances(x: np.ndarray, c: np.ndarray, chunk: int = 4096) -> np.ndarray:
    """d[i,k] = Σ_d (x[i,d] − c[k,d])² in fp64 (NumPy reduction as the library primitive)."""
    x64, c64 = x.astype(np.float64), c.astype(np.float64)
    out = np.empty((x.shape[0], c.shape[0]), dtype=np.float64)
    for s in range(0, x.shape[0], chunk):
        diff = x64[s:s + chunk, None, :] - c64[None, :, :]
        out[s:s + chunk] = np.add.reduce(diff * diff, axis=2)
    return out


def assign(x: np.ndarray, c: np.ndarray, chunk: int = 4096) -> np.ndarray:
    """Vectorised a[i]: ``np.argmin`` returns the first minimum, i.e. the lowest k on ties."""
    out = np.empty(x.shape[0], dtype=np.int32)
    for s in range(0, x.shape[0], chunk):
        out[s:s + chunk] = np.argmin(distances(x[s:s + chunk], c), axis=1)
    return out
