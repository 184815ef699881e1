"""Pins of the PageRank-step oracle (Fig 5) against closed forms, an invariant and a library."""
import numpy as np
import pytest
import torch

from oracle import pagerank as opr
from synth import gen


def test_ring_closed_form():
    # each node's only in-neighbour is its predecessor (out-degree 1): out[n] = (1-d)/N + d*pr[n-1]
    N = 7
    rowptr = np.arange(N + 1)
    colidx = (np.arange(N) - 1) % N
    pr = np.arange(1, N + 1, dtype=np.float64) / 28.0
    out = opr.step(rowptr, colidx, pr, np.ones(N, dtype=np.int32))
    assert np.allclose(out, (1 - opr.DAMP) / N + opr.DAMP * pr[(np.arange(N) - 1) % N], rtol=1e-15)


def test_complete_graph_uniform_is_fixed_point():
    # K_m with self loops: every node has all m nodes as in-neighbours, out-degree m; pr = 1/m is stationary
    m = 9
    rowptr = np.arange(0, m * m + 1, m)
    colidx = np.tile(np.arange(m), m)
    out = opr.step(rowptr, colidx, np.full(m, 1.0 / m), np.full(m, m))
    assert np.allclose(out, 1.0 / m, rtol=1e-15)
    assert opr.step_literal(rowptr, colidx, np.full(m, 1.0 / m), np.full(m, m)) == pytest.approx([1.0 / m] * m, rel=1e-15)


def test_mass_conservation_and_library():
    # with out-degree = occurrences in colidx, Σ_n out[n] = (1-d) + d * Σ_{w: deg(w) > 0} pr[w]
    rowptr, colidx, pr, outdeg = (t.numpy() for t in gen.pagerank_inputs(3000, avg_deg=12, seed=3, max_deg=200))
    out = opr.step(rowptr, colidx, pr, outdeg)
    has_out = outdeg > 0
    assert abs(out.sum() - ((1 - opr.DAMP) + opr.DAMP * pr.astype(np.float64)[has_out].sum())) < 1e-12
    # the same step as a sparse matrix-vector product (scipy as the library primitive)
    sp = pytest.importorskip("scipy.sparse")
    A = sp.csr_matrix((np.ones(len(colidx)), colidx, rowptr), shape=(3000, 3000))
    x = np.where(has_out, pr.astype(np.float64) / np.maximum(outdeg, 1), 0.0)
    assert np.allclose(out, (1 - opr.DAMP) / 3000 + opr.DAMP * (A @ x), rtol=1e-13)


def test_literal_matches_vectorised_with_empty_rows():
    rowptr = np.array([0, 0, 3, 3, 5, 5])
    colidx = np.array([1, 3, 1, 0, 1])
    outdeg = np.bincount(colidx, minlength=5)
    outdeg[outdeg == 0] = 1
    pr = np.array([0.1, 0.2, 0.3, 0.25, 0.15])
    lit = np.array(opr.step_literal(rowptr, colidx, pr, outdeg))
    assert np.allclose(lit, opr.step(rowptr, colidx, pr, outdeg), rtol=1e-15)
    assert lit[0] == lit[2] == lit[4] == (1 - opr.DAMP) / 5   # nodes without in-neighbours


def test_generator_shape():
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(5000, avg_deg=16, seed=7, max_deg=1024)
    deg = torch.diff(rowptr)
    assert int(deg.min()) >= 1 and int(deg.max()) <= 1024
    assert 12 <= float(deg.float().mean()) <= 20               # ~avg_deg
    assert int(outdeg.sum()) == len(colidx) and int(colidx.min()) >= 0 and int(colidx.max()) < 5000
    assert torch.equal(gen.pagerank_inputs(5000, seed=7)[1], colidx)  # deterministic


def test_shard_rows_match_full_step():
    # rows [lo, hi) of the step from the shard's CSR alone (numNodes stays the graph's N)
    rowptr, colidx, pr, outdeg = (t.numpy() for t in gen.pagerank_inputs(800, avg_deg=5, seed=4, max_deg=50))
    full = opr.step(rowptr, colidx, pr, outdeg)
    lo, hi = 300, 555
    part = opr.step(rowptr[lo:hi + 1] - rowptr[lo], colidx[rowptr[lo]:rowptr[hi]], pr, outdeg)
    assert np.array_equal(part, full[lo:hi])
