"""Test helper: the tile schedule a mapping record prescribes (S8/S9), derived from the
record's fields alone — grid G, claim_tiles U, static_tiles Ts, per-level chunks and grids — the way
the kernels read them. Used by the CPU property tests of the R2 rule (tests/test_r2_properties.py) and
by the GPU white-box trace tests (tests/test_gpu_trace.py). No method arithmetic lives here.
"""
from __future__ import annotations

X = 0
ESZ = {"f32": 4, "i32": 4, "i64": 8, "f64": 8}


def cdiv(a, b):
    return -(-a // b)


def staged_geometry(pattern, shape, dtype, rec):
    """(To, Ti, BR, W, align) of a staged sum record. align: the whole-outer-tile rules (RX one-row tiles,
    MX-narrow strips), whose static split is aligned to whole outer tiles."""
    esz = ESZ[dtype]
    To, Ti = rec["levels"][0]["grid"], rec["levels"][1]["grid"]
    rows = pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    if rows:
        BR = rec["levels"][0]["chunk"]
        W = rec["levels"][1]["chunk"] if Ti > 1 else shape[1]
        # a one-row tile of a whole row has W = C; round W up to the tile width the kernel uses
        if Ti == 1:
            W = {1: 32768, 8: 4096, 32: 1024}[BR] // esz
        align = BR == 1
    else:
        W = rec["levels"][0]["chunk"]
        BR = rec["levels"][1]["chunk"] if Ti > 1 else {256 // esz: 128, 1024 // esz: 32}[W]
        align = W == 256 // esz
    return To, Ti, BR, W, align


def static_ranges(G, Ts, Ti, align):
    """Block b's static range [s0, s1) of tiles (kernel formula of kern_sum_tma.cu)."""
    out = []
    for b in range(G):
        if align:
            s0, s1 = (b * (Ts // Ti) // G) * Ti, ((b + 1) * (Ts // Ti) // G) * Ti
        else:
            s0, s1 = b * Ts // G, (b + 1) * Ts // G
        out.append((s0, s1))
    return out


def pool_units(T, Ts, U, Ti, G):
    """The claim-pool ranges of [Ts, T) in claim order (S8): units of U tiles, the last
    F = min(G, T - Ts) tiles one at a time when U < Ti."""
    F = min(G, T - Ts) if U < Ti else 0
    big = [(c, min(T - F, c + U)) for c in range(Ts, T - F, U)]
    return big + [(t, t + 1) for t in range(T - F, T)]


def contiguous_ranges(T, P, G):
    """Block b of the contiguous-range families (LR, KM, KU): tiles [b*P, min(T, (b+1)*P))."""
    return [(b * P, min(T, (b + 1) * P)) for b in range(G)]


def rc_regions(rec):
    """SUM_ROWS_COLS: (gr, gc, nreg, G, block ranges over regions [b*nreg/G, (b+1)*nreg/G))."""
    gr, gc = rec["levels"][0]["grid"], rec["levels"][1]["grid"]
    nreg, G = gr * gc, rec["grid"]
    return gr, gc, nreg, G, [(b * nreg // G, (b + 1) * nreg // G) for b in range(G)]
