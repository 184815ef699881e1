"""GPU parity for the three-level nests (k-means assignment, batched logistic-regression gradient)
through the C-ABI against the fp64 oracle.

Tolerances:
  logreg  |g - g64| <= 1e-5 * Σ_i|x_ij e_i|   (z and e_i in fp64, fp32 products and 4-term sums)
  kmeans  index-exact on every input: the decision is the fp64 distance as written (G25);
          the kernel's fp32 screen settles only points whose margin beats its rigorous error bound
          and recomputes the rest in fp64 with the oracle's operations
"""
import numpy as np
import pytest
import torch

from oracle import kmeans as okm
from oracle import logreg as olr
from oracle import select as osel
from synth import gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def npp(cuda_device):
    from paper_conf_micro_leebsro14_b200 import npp as _npp
    return _npp


def _check_logreg(g, x, y, w, B):
    xn, yn, wn = x.cpu().numpy(), y.cpu().numpy(), w.cpu().numpy()
    want = olr.grad(xn, yn, wn, B)
    s_rel, _ = olr.grad_scales(xn, yn, wn, B)
    err = np.abs(g.cpu().numpy().astype(np.float64) - want)
    tol = 1e-5 * s_rel
    bad = np.argwhere(err > tol)
    assert bad.size == 0, (bad[:4], err[tuple(bad[0])], tol[tuple(bad[0])])


@pytest.mark.parametrize("B,Rb,C", [(1, 1000, 256), (3, 70, 12), (16, 4096, 256), (2, 31, 256),
                                    (7, 33, 100), (300, 64, 256), (1, 1 << 18, 256), (64, 32, 4)])
def test_logreg_parity(npp, cuda_device, B, Rb, C):
    x, y, w = gen.logreg_inputs(B, Rb, C, seed=6, device=cuda_device)
    p = npp.Plan("LOGREG_GRAD", (B, Rb, C), "f32", "AUTO")
    assert p.mapping == osel.select("LOGREG_GRAD", (B, Rb, C), "f32", npp.limits_query(0), "AUTO")
    for _ in range(2):  # the second run checks that the workspace came back zeroed
        g = p.execute([x, y, w], p.new_out())
        torch.cuda.synchronize()
        _check_logreg(g, x, y, w, B)


def test_logreg_y_zero_and_w_zero(npp, cuda_device):
    B, Rb, C = 8, 512, 256
    x, y, w = gen.logreg_inputs(B, Rb, C, seed=7, device=cuda_device, y_zero=True)
    p = npp.Plan("LOGREG_GRAD", (B, Rb, C), "f32", "AUTO")
    g = p.execute([x, y, w], p.new_out())
    torch.cuda.synchronize()
    _check_logreg(g, x, y, w, B)
    w0 = torch.zeros_like(w)
    g0 = p.execute([x, y, w0], p.new_out())
    torch.cuda.synchronize()
    want = (x.double() * 0.5).view(B, Rb, C).sum(1)  # closed form: e = 1/2 - 0
    assert torch.allclose(g0.double(), want, rtol=1e-6, atol=0)


def test_logreg_full_size(npp, cuda_device):
    # BASELINE.json config 5: [16M, 256] fp32 (16 GiB), B = 4096 batches of 4096 rows; every batch's
    # gradient is compared with the oracle (64 batches at a time)
    B, Rb, C = 4096, 4096, 256
    free, _ = torch.cuda.mem_get_info()
    if free < 24 * (1 << 30):
        pytest.skip("needs 24 GiB free")
    x, y, w = gen.logreg_inputs(B, Rb, C, seed=6, device=cuda_device)
    p = npp.Plan("LOGREG_GRAD", (B, Rb, C), "f32", "AUTO")
    g = p.execute([x, y, w], p.new_out())
    torch.cuda.synchronize()
    nb = 64
    for b0 in range(0, B, nb):
        rows = slice(b0 * Rb, (b0 + nb) * Rb)
        _check_logreg(g[b0:b0 + nb], x[rows], y[rows], w, nb)
    del x


@pytest.mark.parametrize("N,D,K", [(10000, 64, 32), (1000, 12, 5), (4099, 128, 96), (127, 4, 1),
                                   (20000, 64, 256), (129, 32, 33), (5000, 128, 128), (3000, 8, 256)])
def test_kmeans_integer_data_exact(npp, cuda_device, N, D, K):
    x, c = gen.kmeans_inputs(N, D, K, integer=True, device=cuda_device)
    p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "AUTO")
    assert p.mapping == osel.select("KMEANS_ASSIGN", (N, D, K), "f32", npp.limits_query(0), "AUTO")
    a = p.execute([x, c], p.new_out())
    torch.cuda.synchronize()
    assert a.cpu().numpy().tolist() == okm.assign(x.cpu().numpy(), c.cpu().numpy()).tolist()


@pytest.mark.parametrize("N,D,K", [(50000, 64, 32), (3000, 16, 7), (20000, 128, 128), (7777, 4, 3), (9000, 96, 32),
                                   (4097, 72, 20), (6000, 100, 64)])
def test_kmeans_random_data_exact(npp, cuda_device, N, D, K):
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device)
    p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "AUTO")
    a = p.execute([x, c], p.new_out())
    torch.cuda.synchronize()
    assert np.array_equal(a.cpu().numpy(), okm.assign(x.cpu().numpy(), c.cpu().numpy()))


def test_kmeans_unclustered_data_exact(npp, cuda_device):
    # points uniform in the centroids' box (no cluster structure): many small margins, so the fp64
    # recheck of near ties runs often
    N, D, K = 60000, 64, 32
    _, c = gen.kmeans_inputs(16, D, K, device=cuda_device)
    x = gen.uniform_f32(31, (N, D), lo=-8.0, scale=16.0, device=cuda_device)
    a = npp.kmeans_assign(x, c)
    torch.cuda.synchronize()
    assert np.array_equal(a.cpu().numpy(), okm.assign(x.cpu().numpy(), c.cpu().numpy()))


def test_kmeans_exact_and_near_ties(npp, cuda_device):
    # dyadic midpoints of centroid pairs are exactly equidistant (the lower index wins), and points
    # nudged by one ulp towards either side of a midpoint are decided by the fp64 distances
    N, D, K = 4096, 64, 32
    g = torch.Generator().manual_seed(9)
    c = (torch.randint(-64, 64, (K, D), generator=g).float() / 4.0)
    pa = torch.randint(0, K, (N,), generator=g)
    pb = (pa + torch.randint(1, K, (N,), generator=g)) % K
    x = (c[pa] + c[pb]) / 2
    nudge = torch.randint(0, 3, (N, 1), generator=g).float() - 1.0  # one ulp towards c_b, none, towards c_a
    direction = torch.sign(c[pb] - c[pa]) * nudge
    inf = torch.full_like(x, float("inf"))
    x = torch.nextafter(x, torch.where(direction > 0, inf, torch.where(direction < 0, -inf, x)))
    x, c = x.contiguous().to(cuda_device), c.contiguous().to(cuda_device)
    a = npp.kmeans_assign(x, c)
    torch.cuda.synchronize()
    want = okm.assign(x.cpu().numpy(), c.cpu().numpy())
    assert np.array_equal(a.cpu().numpy(), want)
    # the exact ties really occur and go to the lower index
    ties = (nudge.squeeze(1) == 0).numpy()
    d = okm.distances(x.cpu().numpy(), c.cpu().numpy())
    exact_tie = ties & (d[np.arange(N), pa.numpy()] == d.min(1))
    assert exact_tie.sum() > 100
    assert np.all(want[exact_tie] == np.minimum(pa.numpy(), pb.numpy())[exact_tie])


def test_kmeans_full_size_exact(npp, cuda_device):
    # BASELINE.json config 4: 4M points x 64 dims x 32 centroids, every assignment checked
    N, D, K = 1 << 22, 64, 32
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device)
    p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "AUTO")
    a = p.execute([x, c], p.new_out())
    torch.cuda.synchronize()
    a = a.cpu().numpy()
    cn = c.cpu().numpy()
    step = 1 << 19
    for s0 in range(0, N, step):
        want = okm.assign(x[s0:s0 + step].cpu().numpy(), cn)
        assert np.array_equal(a[s0:s0 + step], want), s0


def test_kmeans_two_streams_distinct_centroids(npp, cuda_device):
    """The centroids live in one constant bank per device: interleaved executes of two plans on two
    streams, with different centroids and no host sync in between, must each see their own."""
    N = 1 << 16
    xa, ca = gen.kmeans_inputs(N, 64, 32, seed=21, integer=True, device=cuda_device)
    xb, cb = gen.kmeans_inputs(N, 32, 7, seed=22, integer=True, device=cuda_device)
    pa = npp.Plan("KMEANS_ASSIGN", (N, 64, 32), "f32", "AUTO")
    pb = npp.Plan("KMEANS_ASSIGN", (N, 32, 7), "f32", "AUTO")
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()
    outs = []
    for _ in range(8):
        oa, ob = pa.new_out(), pb.new_out()
        with torch.cuda.stream(sa):
            pa.execute([xa, ca], oa, stream=sa)
        with torch.cuda.stream(sb):
            pb.execute([xb, cb], ob, stream=sb)
        outs.append((oa, ob))
    torch.cuda.synchronize()
    wa = okm.assign(xa.cpu().numpy(), ca.cpu().numpy()).tolist()
    wb = okm.assign(xb.cpu().numpy(), cb.cpu().numpy()).tolist()
    for oa, ob in outs:
        assert oa.cpu().numpy().tolist() == wa
        assert ob.cpu().numpy().tolist() == wb


def test_kmeans_points_on_centroids(npp, cuda_device):
    _, c = gen.kmeans_inputs(4, 64, 32, device=cuda_device)
    perm = torch.randint(0, 32, (5000,), generator=torch.Generator().manual_seed(1)).to(cuda_device)
    x = c.index_select(0, perm).contiguous()
    p = npp.Plan("KMEANS_ASSIGN", (5000, 64, 32), "f32", "AUTO")
    a = p.execute([x, c], p.new_out())
    torch.cuda.synchronize()
    assert torch.equal(a.long(), perm)


def test_unsupported_shapes(npp, cuda_device):
    with pytest.raises(npp.NppError) as e:
        npp.Plan("LOGREG_GRAD", (4, 64, 512), "f32", "AUTO")
    assert e.value.status == npp.ERR_UNSUPPORTED
    with pytest.raises(npp.NppError) as e:
        npp.Plan("KMEANS_ASSIGN", (100, 6, 3), "f32", "AUTO")
    assert e.value.status == npp.ERR_UNSUPPORTED
    # the direct 3-level family executes mappings without Split; a Split on a reduce level is unsupported
    lit = npp.Plan("KMEANS_ASSIGN", (100, 64, 3), "f32", "LITERAL").mapping
    split = dict(lit, levels=[lit["levels"][0], lit["levels"][1], dict(lit["levels"][2], span=npp.SPLIT_K, factor=2)])
    with pytest.raises(npp.NppError) as e:
        npp.Plan("KMEANS_ASSIGN", (100, 64, 3), "f32", mapping=split)
    assert e.value.status == npp.ERR_UNSUPPORTED
    with pytest.raises(npp.NppError) as e:
        npp.Plan("LOGREG_GRAD", (4, 64, 256), "f32", "LITERAL")
    assert e.value.status == npp.ERR_UNSUPPORTED


# ---------------------------------------------------------------- k-means centroid update (class KU)

def _check_update(u, x, a, K):
    """Sums within 1e-5 * Σ|x| of the fp64 oracle per element (signed data); counts exact."""
    xn, an = x.cpu().numpy(), a.cpu().numpy()
    want = okm.update(xn, an, K)
    scale = okm.update_scale(xn, an, K)
    got = u.cpu().numpy().astype(np.float64)
    assert np.array_equal(got[:, -1], want[:, -1]), "counts"
    err = np.abs(got[:, :-1] - want[:, :-1])
    bad = np.argwhere(err > 1e-5 * scale + 1e-30)
    assert bad.size == 0, (bad[:4], got[tuple(bad[0])], want[tuple(bad[0])])


@pytest.mark.parametrize("N,D,K", [(1, 4, 1), (127, 8, 3), (129, 64, 32), (3000, 64, 32), (10007, 60, 34),
                                   (5000, 4, 256), (70000, 16, 128), (200000, 64, 32), (33, 32, 64),
                                   (100003, 32, 64), (65536, 64, 7), (300, 32, 9)])
def test_kmeans_update_parity(npp, cuda_device, N, D, K):
    # random keys in [-1, K] (the out-of-range ones belong to no group), ragged last tile, every
    # warp-row / flush boundary; back-to-back executes (plain and PDL-overlapped) leave the workspace zero
    x, _ = gen.kmeans_inputs(N, D, max(K, 1), seed=40 + K, device=cuda_device)
    a = gen.int_uniform(41, (N,), -1, K, device=cuda_device)
    p = npp.Plan("KMEANS_UPDATE", (N, D, K))
    assert p.mapping == osel.select("KMEANS_UPDATE", (N, D, K), "f32", npp.limits_query(0), "AUTO")
    assert p.mapping["kernel_class"] == npp.CLASS_KMUPDATE
    outs = [p.execute([x, a], p.new_out()), p.execute([x, a], p.new_out(), overlap=True)]
    torch.cuda.synchronize()
    for u in outs:
        _check_update(u, x, a, K)
    assert int(p.workspace.count_nonzero()) == 0


@pytest.mark.parametrize("D,K", [(64, 32), (32, 64), (16, 128)])
def test_kmeans_update_skewed_keys(npp, cuda_device, D, K):
    # degenerate clusterings: every point in one group, then two groups of 1:1000 size (the key-owner
    # path puts a whole tile on one warp)
    N = 70001
    x, _ = gen.kmeans_inputs(N, D, K, seed=42, device=cuda_device)
    for a in (torch.full((N,), K - 1, dtype=torch.int32, device=cuda_device),
              torch.where(gen.int_uniform(43, (N,), 0, 999, device=cuda_device) == 0, 3, K - 2).to(torch.int32)):
        _check_update(npp.kmeans_update(x, a, K), x, a, K)


def test_kmeans_update_integer_exact(npp, cuda_device):
    # integer coordinates: every partial sum is an exact fp32 integer (|U| < 2^24), so bit-exact
    # (keys: the oracle's own assignment of the points — no oracle input comes from the CUDA path)
    N, D, K = 50000, 64, 32
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device, integer=True)
    xn = x.cpu().numpy()
    an = okm.assign(xn, c.cpu().numpy())
    u = npp.kmeans_update(x, torch.from_numpy(an).to(cuda_device), K)
    torch.cuda.synchronize()
    assert np.array_equal(u.cpu().numpy().astype(np.float64), okm.update(xn, an, K))


def test_lloyd_step_full_size(npp, cuda_device):
    # one Lloyd iteration on the BASELINE.json k-means configuration (4M x 64 x 32): assignment, then
    # the update, both on the GPU, checked by invariants that hold for any assignment. Parity at this
    # size uses the generator's own cluster labels z as keys (a synthetic input, not a CUDA result):
    # the first 1M points through a second plan against the oracle
    N, D, K = 1 << 22, 64, 32
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device)
    a = npp.kmeans_assign(x, c)
    u = npp.kmeans_update(x, a, K)
    n1 = 1 << 20
    z = gen.int_uniform(5 + 1, (n1,), 0, K - 1, dtype=torch.int32, device=cuda_device)  # kmeans_inputs' labels
    u1 = npp.Plan("KMEANS_UPDATE", (n1, D, K)).execute([x[:n1], z], torch.empty(K, D + 1, device=cuda_device))
    torch.cuda.synchronize()
    _check_update(u1, x[:n1], z, K)
    un = u.cpu().numpy().astype(np.float64)
    assert un[:, -1].sum() == N                                           # every point in one group
    colsum = x.double().sum(0).cpu().numpy()                              # Σ_k U[k] = Σ_i x_i
    assert np.all(np.abs(un[:, :-1].sum(0) - colsum) <= 1e-5 * x.double().abs().sum(0).cpu().numpy())
    counts = torch.bincount(a.long(), minlength=K).cpu().numpy()
    assert np.array_equal(un[:, -1], counts)


def test_kmeans_update_plan_rules(npp, cuda_device):
    for strategy in ("LITERAL", "1D", "TB_T", "WARP"):
        with pytest.raises(npp.NppError) as e:
            npp.Plan("KMEANS_UPDATE", (100, 64, 32), "f32", strategy)
        assert e.value.status == npp.ERR_UNSUPPORTED
    for shape in [(100, 66, 4), (100, 128, 4), (100, 64, 33), (100, 8, 257)]:
        with pytest.raises(npp.NppError) as e:
            npp.Plan("KMEANS_UPDATE", shape)
        assert e.value.status == npp.ERR_UNSUPPORTED
    p = npp.Plan("KMEANS_UPDATE", (0, 8, 3))   # no points: every group empty
    u = p.execute([torch.empty(0, 8, device=cuda_device), torch.empty(0, dtype=torch.int32, device=cuda_device)],
                  torch.full((3, 9), 5.0, device=cuda_device))
    torch.cuda.synchronize()
    assert float(u.abs().sum()) == 0.0


# ---------------------------------------------------------------- PageRank step (class PR, Fig 5)

def _check_pr(out, rowptr, colidx, pr, outdeg):
    from oracle import pagerank as opr
    want = opr.step(rowptr.cpu().numpy(), colidx.cpu().numpy(), pr.cpu().numpy(), outdeg.cpu().numpy())
    got = out.cpu().numpy().astype(np.float64)
    err = np.abs(got - want)
    bad = np.nonzero(err > 1e-5 * want)[0]   # every term is positive: relative 1e-5
    assert bad.size == 0, (bad[:5], got[bad[:5]], want[bad[:5]])


@pytest.mark.parametrize("N,avg,maxd", [(1, 3, 8), (7, 1, 4), (1000, 2, 64), (5000, 16, 1024), (20000, 5, 300),
                                        (100000, 40, 1024), (3000, 16, 4096)])
def test_pagerank_parity(npp, cuda_device, N, avg, maxd):
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(N, avg_deg=avg, seed=N % 97, max_deg=maxd, device=cuda_device)
    E = colidx.numel()
    p = npp.Plan("PAGERANK", (N, E))
    assert p.mapping == osel.select("PAGERANK", (N, E), "f32", npp.limits_query(0), "AUTO")
    assert p.mapping["kernel_class"] == npp.CLASS_PAGERANK
    outs = [p.execute([rowptr, colidx, pr, outdeg], p.new_out()),
            p.execute([rowptr, colidx, pr, outdeg], p.new_out(), overlap=True)]
    torch.cuda.synchronize()
    for o in outs:
        _check_pr(o, rowptr, colidx, pr, outdeg)
    assert int(p.workspace[:256].count_nonzero()) == 0   # the claim counter re-armed itself


def test_pagerank_edge_cases(npp, cuda_device):
    from oracle import pagerank as opr
    # no edges: every node gets (1 - d) / N; rows of very different lengths in one chunk
    N = 1000
    rowptr = torch.zeros(N + 1, dtype=torch.int64, device=cuda_device)
    out = npp.pagerank_step(rowptr, torch.empty(0, dtype=torch.int32, device=cuda_device),
                            torch.full((N,), 1.0 / N, device=cuda_device), torch.ones(N, dtype=torch.int32, device=cuda_device))
    torch.cuda.synchronize()
    assert torch.allclose(out.double().cpu(), torch.full((N,), (1 - opr.DAMP) / N, dtype=torch.float64), rtol=1e-6)
    # complete graph with uniform PageRank is a fixed point (oracle pin, now on the GPU)
    m = 300
    rowptr = torch.arange(0, m * m + 1, m, dtype=torch.int64, device=cuda_device)
    colidx = torch.arange(m, dtype=torch.int32, device=cuda_device).repeat(m)
    out = npp.pagerank_step(rowptr, colidx, torch.full((m,), 1.0 / m, device=cuda_device),
                            torch.full((m,), m, dtype=torch.int32, device=cuda_device))
    torch.cuda.synchronize()
    assert torch.allclose(out.cpu(), torch.full((m,), 1.0 / m), rtol=1e-5)
    for strategy in ("LITERAL", "1D"):
        with pytest.raises(npp.NppError) as e:
            npp.Plan("PAGERANK", (100, 1000), "f32", strategy)
        assert e.value.status == npp.ERR_UNSUPPORTED


def test_pagerank_segmented_row_structure(npp, cuda_device):
    # the segmented mapping (mean in-degree >= 8, S8 PR): empty rows between non-empty ones,
    # rows ending exactly on a 32-edge batch boundary, rows longer than a claim's 8 batches, a claim whose
    # rows are all empty, and a row count that is not a multiple of 31
    degs = ([0, 0, 37, 1, 0, 64, 5, 0, 32, 31, 33, 1000, 0] * 40 + [0] * 31 + [2000, 1, 0, 95] * 3)[:611]
    N = len(degs)
    rowptr = torch.tensor([0] + list(np.cumsum(degs)), dtype=torch.int64, device=cuda_device)
    E = int(rowptr[-1])
    colidx = gen.int_uniform(11, (E,), 0, N - 1, device=cuda_device)
    pr = gen.uniform_f32(12, (N,), device=cuda_device, lo=0.5)
    outdeg = torch.bincount(colidx.long(), minlength=N).clamp(min=1).to(torch.int32)
    p = npp.Plan("PAGERANK", (N, E))
    assert p.mapping["levels"][1]["span"] == osel.SPLIT and p.mapping["claim_tiles"] == 31
    out = p.execute([rowptr, colidx, pr, outdeg], p.new_out())
    torch.cuda.synchronize()
    _check_pr(out, rowptr, colidx, pr, outdeg)
    assert int(p.workspace[:256].count_nonzero()) == 0
    # mean in-degree < 8: the row-group mapping
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(5000, avg_deg=3, seed=3, max_deg=64, device=cuda_device)
    p = npp.Plan("PAGERANK", (5000, colidx.numel()))
    assert p.mapping["levels"][1]["span"] == osel.ALL


def test_pagerank_full_size(npp, cuda_device):
    # the bench workload: 4M nodes, power-law in-degrees (mean ~16, cap 1024), ~63M edges
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(1 << 22, avg_deg=16, seed=7, max_deg=1024, device=cuda_device)
    out = npp.pagerank_step(rowptr, colidx, pr, outdeg)
    torch.cuda.synchronize()
    _check_pr(out, rowptr, colidx, pr, outdeg)


def test_pagerank_shard_rows(npp, cuda_device):
    # the multi-GPU form: rows [lo, hi) from the shard's CSR against the whole pr / outdeg ({rows, E, N})
    rowptr, colidx, pr, outdeg = gen.pagerank_inputs(50000, avg_deg=12, seed=5, max_deg=2000, device=cuda_device)
    lo, hi = 12345, 40000
    lrp = (rowptr[lo:hi + 1] - rowptr[lo]).contiguous()
    lci = colidx[int(rowptr[lo]):int(rowptr[hi])].contiguous()
    out = npp.pagerank_shard(lrp, lci, pr, outdeg, lo, hi)
    torch.cuda.synchronize()
    _check_pr(out, lrp, lci, pr, outdeg)


@pytest.mark.parametrize("N,D,K", [(5000, 64, 32), (3000, 100, 33), (777, 8, 5), (1 << 18, 64, 32)])
def test_kmeans_literal_mapping_exact(npp, cuda_device, N, D, K):
    # strategy LITERAL: Algorithm 1 + ControlDOP exactly (e.g. L0 = (y, 1, Span(n)), L1 = (z, 16, all),
    # L2 = (x, 64, all)), executed by the direct 3-level family; index-exact like AUTO
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device)
    p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", "LITERAL")
    assert p.mapping == osel.select("KMEANS_ASSIGN", (N, D, K), "f32", npp.limits_query(0), "LITERAL")
    assert p.mapping["staged"] == 0 and p.launches == 1
    a = p.execute([x, c], p.new_out())
    torch.cuda.synchronize()
    assert np.array_equal(a.cpu().numpy(), okm.assign(x.cpu().numpy(), c.cpu().numpy()))


@pytest.mark.parametrize("N,D,K", [(300, 8, 5), (4096, 32, 16)])
def test_kmeans_every_enumerated_mapping(npp, cuda_device, N, D, K):
    # the Fig 17 space of the three-level nest: every hard-feasible Algorithm 1 candidate without Split
    # executes through npp_plan_with_mapping and returns the oracle's assignment; Split candidates are
    # rejected as unsupported
    x, c = gen.kmeans_inputs(N, D, K, device=cuda_device)
    x[:16] = (c[torch.arange(16, device=cuda_device) % K] + c[(torch.arange(16, device=cuda_device) + 1) % K]) / 2
    want = okm.assign(x.cpu().numpy(), c.cpu().numpy())
    recs = npp.enumerate_mappings("KMEANS_ASSIGN", (N, D, K), "f32", npp.limits_query(0))
    ran = 0
    for rec in recs:
        if any(l["span"] == npp.SPLIT_K for l in rec["levels"]):
            with pytest.raises(npp.NppError) as e:
                npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", mapping=rec)
            assert e.value.status == npp.ERR_UNSUPPORTED
            continue
        p = npp.Plan("KMEANS_ASSIGN", (N, D, K), "f32", mapping=rec)
        a = p.execute([x, c], p.new_out())
        torch.cuda.synchronize()
        assert np.array_equal(a.cpu().numpy(), want), rec["levels"]
        ran += 1
    assert ran > 100
