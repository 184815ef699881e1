"""Oracle: batched logistic-regression gradient — TEST INFRASTRUCTURE ONLY (see oracle/__init__).

The three-level nest (BASELINE.json config 5; G22):
    batches map { b => rows(b) reduce { i =>
        e_i = σ((x_i zipWith w)(*) reduce +) − y_i          // L2 Reduce (dot)
        x_i map { x_ij => x_ij * e_i } } }                    // L2 Map; L1 Reduce adds the vectors
i.e.  g[b,j] = Σ_{i=b·Rb}^{(b+1)·Rb−1} x[i,j] · (σ(Σ_k x[i,k] w[k]) − y[i]),  σ(z) = 1/(1+e^{−z}),
the gradient of Σ_i [softplus(z_i) − y_i z_i] with respect to w over each mini-batch. B = 1 is the
full-batch gradient.  fp64 throughout (``math.exp`` / ``np.exp``).
"""
from __future__ import annotations

import math

import numpy as np


def sigmoid(z: float) -> float:
    return 1.0 / (1.0 + math.exp(-z)) if z >= 0 else math.exp(z) / (1.0 + math.exp(z))


def grad_literal(x: np.ndarray, y: np.ndarray, w: np.ndarray, B: int) -> list:
    """Pure-Python loops in the nest's order: Map over batches, Reduce over rows, Map/Reduce over cols."""
    n, C = x.shape
    Rb = n // B
    xs, ys, ws = x.tolist(), y.tolist(), w.tolist()
    g = []
    for b in range(B):
        terms = [[] for _ in range(C)]
        for i in range(b * Rb, (b + 1) * Rb):
            z = math.fsum(float(xs[i][k]) * float(ws[k]) for k in range(C))
            e = sigmoid(z) - float(ys[i])
            for j in range(C):
                terms[j].append(float(xs[i][j]) * e)
        g.append([math.fsum(t) for t in terms])
    return g


def residuals(x: np.ndarray, y: np.ndarray, w: np.ndarray) -> np.ndarray:
    """e_i = σ(x_i·w) − y_i in fp64 (matrix-vector product as the library primitive)."""
    z = x.astype(np.float64) @ w.astype(np.float64)
    return 1.0 / (1.0 + np.exp(-z)) - y.astype(np.float64)


def grad(x: np.ndarray, y: np.ndarray, w: np.ndarray, B: int, chunk_batches: int = 64) -> np.ndarray:
    """Vectorised g[B, C] in fp64."""
    n, C = x.shape
    Rb = n // B
    out = np.empty((B, C), dtype=np.float64)
    for b0 in range(0, B, chunk_batches):
        b1 = min(B, b0 + chunk_batches)
        xs = x[b0 * Rb:b1 * Rb].astype(np.float64)
        e = residuals(x[b0 * Rb:b1 * Rb], y[b0 * Rb:b1 * Rb], w)
        out[b0:b1] = np.add.reduce((xs * e[:, None]).reshape(b1 - b0, Rb, C), axis=1)
    return out


def grad_scales(x: np.ndarray, y: np.ndarray, w: np.ndarray, B: int):
    """(Σ_i |x_ij e_i|, Σ_i |x_ij|) per (b, j): the two scales of the fp32 tolerance of DESIGN.md §5
    (relative error of the accumulated terms, and the absolute error of each fp32 residual e_i)."""
    n, C = x.shape
    Rb = n // B
    x64 = np.abs(x.astype(np.float64))
    e = np.abs(residuals(x, y, w))
    return (np.add.reduce((x64 * e[:, None]).reshape(B, Rb, C), axis=1),
            np.add.reduce(x64.reshape(B, Rb, C), axis=1))
