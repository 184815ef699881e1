"""The input generator: deterministic, shard-invariant, in range."""
import torch

from synth import gen


def test_shard_invariance():
    full = gen.uniform_f32(3, (64, 40))
    a = gen.uniform_f32(3, (20, 40), offset=0)
    b = gen.uniform_f32(3, (44, 40), offset=20 * 40)
    assert torch.equal(full, torch.cat([a, b]))


def test_ranges_and_exactness():
    u = gen.uniform_f32(1, (1000,))
    assert float(u.min()) >= 0.0 and float(u.max()) < 1.0
    assert torch.equal(u.double() * 2 ** 24, (u.double() * 2 ** 24).round())
    e = gen.exact_f32(1, (1000,))
    assert torch.equal(e.double() * 256, (e.double() * 256).round()) and float(e.max()) < 1.0
    i = gen.int_uniform(2, (1000,), -1000, 1000)
    assert int(i.min()) >= -1000 and int(i.max()) <= 1000 and i.dtype == torch.int32


def test_arange_and_hash_determinism():
    a = gen.arange_matrix((3, 4), torch.int64)
    assert a.flatten().tolist() == list(range(12))
    h1 = gen.hash32(5, torch.arange(10))
    h2 = gen.hash32(5, torch.arange(10))
    assert torch.equal(h1, h2) and int(h1.max()) < 2 ** 32 and len(set(h1.tolist())) == 10


def test_kmeans_logreg_recipes():
    x, c = gen.kmeans_inputs(100, 8, 4)
    assert x.shape == (100, 8) and c.shape == (4, 8)
    xs, cs = gen.kmeans_inputs(50, 8, 4, row_offset=50)
    assert torch.equal(xs, x[50:]) and torch.equal(cs, c)
    xi, ci = gen.kmeans_inputs(64, 8, 4, integer=True)
    assert torch.equal(xi, xi.round()) and float(xi.abs().max()) <= 8
    X, y, w = gen.logreg_inputs(4, 8, 16)
    assert X.shape == (32, 16) and set(y.tolist()) <= {0.0, 1.0} and float(w.abs().max()) <= 1 / 16


def test_uniform_f64_is_53_bit_and_counter_based():
    # 53 random bits in [0, 1), identical for any offset split (shards regenerate the same values)
    full = gen.uniform_f64(5, (4, 1000))
    part = gen.uniform_f64(5, (2, 1000), offset=2000)
    assert torch.equal(full[2:], part)
    assert float(full.min()) >= 0.0 and float(full.max()) < 1.0
    frac = (full * 2.0 ** 53)
    assert torch.equal(frac, torch.floor(frac))
    assert (frac % 2 == 1).any()  # the low bit is used
