"""Pins for oracle/kmeans.py and oracle/logreg.py (closed forms, special cases, library routines)."""
import math

import numpy as np
import pytest
import torch

from oracle import kmeans, logreg
from synth import gen


# ------------------------------------------------------------------ k-means assignment

def test_points_equal_to_centroids():
    _, c = gen.kmeans_inputs(4, 16, 8)
    c = c.numpy()
    perm = np.array([3, 1, 7, 0, 0, 5, 2, 6, 4])
    x = c[perm]
    assert kmeans.assign(x, c).tolist() == perm.tolist()
    assert kmeans.assign_literal(x, c) == perm.tolist()


def test_single_centroid():
    x, c = gen.kmeans_inputs(50, 5, 1)
    assert kmeans.assign(x.numpy(), c.numpy()).tolist() == [0] * 50


def test_one_dimension_nearest():
    c = np.array([[-3.0], [0.5], [2.0], [7.0]], dtype=np.float32)
    x = np.array([[-10.0], [-1.25], [-1.0], [1.0], [1.25], [1.5], [4.5], [4.75], [100.0]], dtype=np.float32)
    # midpoints -1.25, 1.25, 4.5 are ties -> lowest index
    assert kmeans.assign(x, c).tolist() == [0, 0, 1, 1, 1, 2, 2, 3, 3]
    assert kmeans.assign_literal(x, c) == [0, 0, 1, 1, 1, 2, 2, 3, 3]


def test_tie_goes_to_lowest_index():
    c = np.array([[1, 0], [0, 1], [-1, 0], [0, -1]], dtype=np.float32)
    x = np.zeros((1, 2), dtype=np.float32)
    assert kmeans.assign(x, c).tolist() == [0]
    x2 = np.array([[0.0, -1.0]], dtype=np.float32)
    c2 = np.array([[5, 5], [0, -1], [0, -1]], dtype=np.float32)
    assert kmeans.assign_literal(x2, c2) == [1]


def test_integer_data_exact_and_library():
    x, c = gen.kmeans_inputs(300, 12, 7, integer=True)
    x, c = x.numpy(), c.numpy()
    a = kmeans.assign(x, c)
    assert a.tolist() == kmeans.assign_literal(x, c)
    d = torch.cdist(torch.from_numpy(x).double(), torch.from_numpy(c).double()) ** 2
    # squared integer distances are exact: recompute with exact ints and compare argmin with ties
    xi, ci = x.astype(np.int64), c.astype(np.int64)
    exact = ((xi[:, None, :] - ci[None, :, :]) ** 2).sum(-1)
    assert a.tolist() == np.argmin(exact, axis=1).tolist()
    assert np.allclose(d.numpy(), exact, rtol=1e-12)


def test_random_data_vs_cdist():
    x, c = gen.kmeans_inputs(2000, 64, 32)
    x, c = x.numpy(), c.numpy()
    a = kmeans.assign(x, c)
    d = torch.cdist(torch.from_numpy(x).double(), torch.from_numpy(c).double())
    assert a.tolist() == torch.argmin(d, dim=1).tolist()
    assert kmeans.assign_literal(x[:40], c) == a[:40].tolist()


def test_vectorised_distances_bitwise_literal():
    # the vectorised oracle performs the literal's fp64 operations in the literal's order (G25)
    rng = np.random.default_rng(5)
    for D, K in [(64, 32), (7, 5), (128, 3)]:
        x = (rng.standard_normal((40, D)) * rng.choice([1e-3, 1.0, 1e3], size=(40, D))).astype(np.float32)
        c = (rng.standard_normal((K, D)) * 4).astype(np.float32)
        d = kmeans.distances(x, c)
        for i in range(0, 40, 7):
            for k in range(K):
                assert d[i, k] == kmeans.distance_literal(x[i].tolist(), c[k].tolist())


def test_fp64_decision_is_the_exact_argmin_away_from_ties():
    # pin of reading G25 against exact rational arithmetic: |d64 - d| <= D * 2^-52 * d (each of the D
    # squares and adds rounds once, differences of fp32 values are exact in fp64 at these magnitudes),
    # and the fp64 argmin is the exact argmin whenever the exact margin exceeds twice that bound
    from fractions import Fraction
    rng = np.random.default_rng(6)
    D, K = 16, 6
    x = rng.uniform(-8, 8, (60, D)).astype(np.float32)
    c = rng.uniform(-8, 8, (K, D)).astype(np.float32)
    d64 = kmeans.distances(x, c)
    a = kmeans.assign(x, c)
    for i in range(60):
        exact = [sum((Fraction(float(p)) - Fraction(float(q))) ** 2 for p, q in zip(x[i], c[k])) for k in range(K)]
        for k in range(K):
            assert abs(Fraction(d64[i, k]) - exact[k]) <= Fraction(D, 2 ** 52) * exact[k]
        order = sorted(range(K), key=lambda k: (exact[k], k))
        margin = exact[order[1]] - exact[order[0]]
        if margin > Fraction(2 * D, 2 ** 52) * exact[order[1]]:
            assert a[i] == order[0]


def test_exact_midpoint_ties_go_to_lowest_index():
    # dyadic coordinates: x = (c_a + c_b)/2 is exactly equidistant from c_a and c_b, and every fp64
    # operation on these values is exact, so the tie is real and the lower index wins (G20)
    rng = np.random.default_rng(7)
    D, K = 64, 32
    c = (rng.integers(-64, 64, (K, D)) / 4.0).astype(np.float32)
    pairs = [(3, 17), (20, 5), (0, 31), (9, 8)]
    x = np.stack([(c[p] + c[q]) / 2 for p, q in pairs]).astype(np.float32)
    d = kmeans.distances(x, c)
    for row, (p, q) in enumerate(pairs):
        assert d[row, p] == d[row, q]
    a = kmeans.assign(x, c)
    for row, (p, q) in enumerate(pairs):
        if d[row].min() == d[row, p]:
            assert a[row] == min(p, q)
    assert kmeans.assign_literal(x, c) == a.tolist()


# ------------------------------------------------------------------ logistic-regression gradient

def test_w_zero_closed_form():
    B, Rb, C = 3, 20, 9
    x, y, _ = gen.logreg_inputs(B, Rb, C)
    x, y = x.numpy(), y.numpy()
    w = np.zeros(C, dtype=np.float32)
    g = logreg.grad(x, y, w, B)
    ref = (x.astype(np.float64) * (0.5 - y.astype(np.float64))[:, None]).reshape(B, Rb, C).sum(1)
    assert np.allclose(g, ref, rtol=1e-14, atol=0)


def test_all_ones_symmetry():
    B, Rb, C = 2, 10, 7
    x = np.ones((B * Rb, C), dtype=np.float32)
    _, y, w = gen.logreg_inputs(B, Rb, C)
    g = logreg.grad(x, y.numpy(), w.numpy(), B)
    for b in range(B):
        assert np.allclose(g[b], g[b][0], rtol=1e-15)
    # sigma(sum w) - y summed over rows
    s = 1.0 / (1.0 + math.exp(-float(w.double().sum())))
    assert math.isclose(g[0][0], sum(s - float(v) for v in y[:Rb]), rel_tol=1e-12)


@pytest.mark.parametrize("B", [1, 3])
def test_autograd_and_literal(B):
    Rb, C = 8, 11
    x, y, w = gen.logreg_inputs(B, Rb, C, seed=12)
    g = logreg.grad(x.numpy(), y.numpy(), w.numpy(), B)
    assert np.allclose(g, np.array(logreg.grad_literal(x.numpy(), y.numpy(), w.numpy(), B)), rtol=1e-13)
    for b in range(B):
        wt = w.double().clone().requires_grad_(True)
        xb, yb = x[b * Rb:(b + 1) * Rb].double(), y[b * Rb:(b + 1) * Rb].double()
        z = xb @ wt
        loss = (torch.nn.functional.softplus(z) - yb * z).sum()
        loss.backward()
        assert np.allclose(g[b], wt.grad.numpy(), rtol=1e-12, atol=1e-14)


def test_finite_differences():
    Rb, C = 6, 5
    x, y, w = gen.logreg_inputs(1, Rb, C, seed=13)
    x64, y64, w64 = x.double().numpy(), y.double().numpy(), w.double().numpy()

    def loss(wv):
        z = x64 @ wv
        return float(np.sum(np.logaddexp(0.0, z) - y64 * z))
    g = logreg.grad(x.numpy(), y.numpy(), w.numpy(), 1)[0]
    h = 1e-6
    for j in range(C):
        e = np.zeros(C)
        e[j] = h
        fd = (loss(w64 + e) - loss(w64 - e)) / (2 * h)
        assert math.isclose(fd, g[j], rel_tol=1e-6, abs_tol=1e-9)


# ---------------------------------------------------------------- k-means update (groupBy + Reduce)

def test_update_closed_forms():
    from oracle import sums
    rng = np.random.default_rng(7)
    x = rng.integers(-50, 50, size=(300, 12)).astype(np.float32)
    # one group holding every point: the sums are sumCols (independently pinned), the count is N
    u = kmeans.update(x, np.zeros(300, dtype=np.int32), 1)
    assert np.array_equal(u[0, :12], sums.sum_cols(x)) and u[0, 12] == 300
    # a_i = i mod K on arange data: closed form Σ_{i ≡ k} (i*D + d)
    N, D, K = 100, 3, 7
    xa = np.arange(N * D, dtype=np.float32).reshape(N, D)
    ua = kmeans.update(xa, np.arange(N) % K, K)
    for k in range(K):
        ids = list(range(k, N, K))
        assert ua[k, D] == len(ids)
        for d in range(D):
            assert ua[k, d] == sum(i * D + d for i in ids)
    # invalid keys belong to no group; counts of valid keys sum to their number; groups partition
    a = rng.integers(-2, 9, size=300)
    u = kmeans.update(x, a, 7)
    valid = (a >= 0) & (a < 7)
    assert u[:, 12].sum() == valid.sum()
    assert np.array_equal(u[:, :12].sum(axis=0), sums.sum_cols(x[valid]))


def test_update_literal_matches_vectorised():
    rng = np.random.default_rng(3)
    x = rng.standard_normal((57, 5)).astype(np.float32)
    a = rng.integers(-1, 4, size=57)
    lit = np.array(kmeans.update_literal(x, a, 4))
    vec = kmeans.update(x, a, 4)
    assert np.allclose(lit, vec, rtol=1e-14, atol=1e-12)
    assert np.array_equal(lit[:, -1], vec[:, -1])


def test_update_after_assign_is_a_lloyd_step():
    # Lloyd: the new centroids U[:, :D] / U[:, D] never increase the assignment's total squared distance
    x, c = gen.kmeans_inputs(2000, 8, 5, seed=21)
    x, c = x.numpy(), c.numpy()
    a = kmeans.assign(x, c)
    u = kmeans.update(x, a, 5)
    newc = np.where(u[:, -1:] > 0, u[:, :-1] / np.maximum(u[:, -1:], 1), c.astype(np.float64))
    before = ((x.astype(np.float64) - c.astype(np.float64)[a]) ** 2).sum()
    after = ((x.astype(np.float64) - newc[a]) ** 2).sum()
    assert after <= before + 1e-9
