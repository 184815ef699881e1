"""Oracle: brute-force mapping selector — TEST INFRASTRUCTURE ONLY (see oracle/__init__).

Follows PAPER.md §IV step by step, with the readings of DESIGN.md §2/§3 where the paper is silent:
  nest descriptor (levels, sync, accesses)   §IV intro L396-403, L454-455; Fig 8 L683-692   (S1)
  candidate space Dim × Size × Span          Alg 1 L748-753, L772-777                        (S2)
  hard constraints (HL, HG, HW limits)       Table II; L642-662                      (S3)
  soft constraints and derived weights       Table II; L664-716                               (S4)
  best = max score, then DOP, then …         L734-741, Alg 1 L790-792                         (S5)
  ControlDOP                                 Alg 1; L798-809                         (S6)
  forced 1D / thread-block-thread / warp     L99-115; Fig 7; L1052-1055    (S7)
  runtime parameter step (AUTO)              L810-817                                         (S8)
Written as plain nested loops over the whole candidate space (no pruning, no memoisation).

W_C/W_B and the tie-break key are readings pinned by invariance, R2 by schedule properties.
"""
from __future__ import annotations

import itertools

# logical dims (S2): x varies fastest
X, Y, Z = 0, 1, 2
# span codes (S9 / record)
ONE, ALL, SPAN_N, SPLIT = 0, 1, 2, 3
# kernel classes (S9)
RX, MX, KM, LR, EMPTY, RC, KU, PR = 0, 1, 2, 3, 4, 5, 6, 7

SIZE_SET = [1 << i for i in range(11)]          # {1,2,4,...,1024}  Alg 1
W_C, W_B = 8, 1                                  # DESIGN.md G3
MIN_BLOCK_SIZE = 64                              # Table II SG, L563; G5
UNKNOWN_SIZE = 1000                              # L699-700; G17
T_BLOCK, U_MIN = 256, 8                          # DESIGN.md S8
MAX_GRID = (1 << 31) - 1                         # DESIGN.md S3 H6

PATTERNS = ("SUM_ROWS", "SUM_COLS", "KMEANS_ASSIGN", "LOGREG_GRAD",
            "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS", "SUM_ROWS_COLS", "KMEANS_UPDATE", "PAGERANK")
DTYPE_SIZE = {"f32": 4, "i32": 4, "i64": 8, "f64": 8}

B200 = dict(sm_count=148, max_threads_per_sm=2048, max_threads_per_block=1024,
            max_block_dim=(1024, 1024, 64), warp_size=32, max_blocks_per_sm=32,
            regs_per_sm=65536, regs_per_block=65536, regs_per_thread=32,
            smem_per_block=232448)
# Tesla K20c: 13 SMs x 2048 threads
K20C = dict(sm_count=13, max_threads_per_sm=2048, max_threads_per_block=1024,
            max_block_dim=(1024, 1024, 64), warp_size=32, max_blocks_per_sm=16,
            regs_per_sm=65536, regs_per_block=65536, regs_per_thread=32,
            smem_per_block=49152)


class NoFeasibleMapping(Exception):
    pass


class Unsupported(Exception):
    pass


def cdiv(a: int, b: int) -> int:
    return -(-a // b)


def pow2ceil(v: int) -> int:
    p = 1
    while p < v:
        p *= 2
    return p


def prod(xs) -> int:
    r = 1
    for v in xs:
        r *= v
    return r


# ------------------------------------------------------------------ S1 nest descriptor

def build_nest(pattern: str, shape) -> dict:
    """Levels (N, sync) outermost first and accesses (contig level, exec-count mask)."""
    if pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS"):
        R, C = shape
        levels = [(R, False), (C, True)]            # Map rows / Reduce row (Fig 1 L70)
        acc = [(0, (0,)), (1, (0, 1))]              # out[r], m[r,c]
        if pattern == "SUM_WEIGHTED_ROWS":
            acc.append((1, (0, 1)))                 # v[c]
    elif pattern in ("SUM_COLS", "SUM_WEIGHTED_COLS"):
        R, C = shape
        levels = [(C, False), (R, True)]            # Map cols / Reduce column (Fig 1 L69)
        acc = [(0, (0,)), (0, (0, 1))]              # out[c], m[r,c] (stride-1 index is c = L0)
        if pattern == "SUM_WEIGHTED_COLS":
            acc.append((1, (0, 1)))                 # v[r]
    elif pattern == "SUM_ROWS_COLS":                 # Naive Bayes counts, §VI-E
        R, C = shape
        levels = [(R, True), (C, True)]             # rows Reduce (column sums), cols Reduce (row sums)
        acc = [(0, (0,)), (1, (1,)), (1, (0, 1))]   # out_rows[r], out_cols[c], m[r,c]
    elif pattern == "KMEANS_UPDATE":                 # groupBy (Table I) + Reduce per group
        N, D, K = shape
        if K < 1:
            raise ValueError("KMEANS_UPDATE needs K >= 1")
        levels = [(N, True), (D, False)]            # points: Reduce into K groups; dims: Map
        acc = [(1, (0, 1)), (0, (0,)), (1, (1,))]   # x[i,d], a[i], U[k,d]
        return {"pattern": pattern, "levels": levels, "accesses": acc, "K": K}
    elif pattern == "PAGERANK":                      # Fig 5 L348-361 over the CSR of in-neighbours
        N, E = shape[0], shape[1]                   # {N, E} or {rows, E, N}: L0 = the rows computed
        if E < 0:
            raise ValueError("PAGERANK needs E >= 0")
        inner = max(1, cdiv(E, N)) if N > 0 else 1  # the average in-degree stands for the inner size
        levels = [(N, False), (inner, True)]         # nodes: Map; neighbours: Map + Reduce
        acc = [(0, (0,)), (0, (0,)), (1, (0, 1)), (-1, (0, 1)), (-1, (0, 1))]  # rowptr, out, colidx, 2 gathers
        return {"pattern": pattern, "levels": levels, "accesses": acc, "E": E,
                "nodes": shape[2] if len(shape) == 3 else N}
    elif pattern == "KMEANS_ASSIGN":
        N, D, K = shape
        levels = [(N, False), (K, True), (D, True)]
        acc = [(0, (0,)), (2, (0, 1, 2)), (2, (0, 1, 2))]   # a[i], x[i,d], c[k,d]
    elif pattern == "LOGREG_GRAD":
        B, Rb, C = shape
        levels = [(B, False), (Rb, True), (C, True)]       # L2 holds Map_j and Reduce_k (HG)
        acc = [(1, (0, 1)), (2, (0, 1, 2)), (2, (0, 1, 2)), (2, (0, 1, 2)), (2, (0, 2))]
    else:
        raise ValueError(pattern)
    return {"pattern": pattern, "levels": levels, "accesses": acc}


def _eff(n: int) -> int:
    return UNKNOWN_SIZE if n < 0 else n


# ------------------------------------------------------------------ S6 DOP (G7)

def level_dop(n: int, b: int, span: int, factor: int) -> int:
    n = _eff(n)
    if span == ONE:
        return n
    if span == ALL:
        return min(b, n)
    if span == SPAN_N:
        return cdiv(n, factor)
    return factor * min(b, cdiv(n, factor))          # SPLIT


def mapping_dop(nest, blocks, spans, factors) -> int:
    return prod(level_dop(nest["levels"][l][0], blocks[l], spans[l], factors[l])
                for l in range(len(blocks)))


def level_blocks(n: int, b: int, span: int, factor: int, vec: int = 1) -> int:
    """Blocks along a level (Fig 6 caption L450-452): ONE ⌈N/b⌉, Span(n) ⌈N/(b·n)⌉, ALL 1, Split ⌈N/⌈N/k⌉⌉."""
    return cdiv(_eff(n), level_chunk(n, b, span, factor, vec))


def level_chunk(n: int, b: int, span: int, factor: int, vec: int = 1) -> int:
    n = _eff(n)
    if span == ONE:
        return b * vec
    if span == SPAN_N:
        return b * vec * factor
    if span == ALL:
        return max(n, 1)
    return cdiv(n, factor)


# ------------------------------------------------------------------ S3 hard constraints

def acc_bytes(pattern: str, dtype: str) -> int:
    if pattern in ("KMEANS_ASSIGN", "LOGREG_GRAD", "KMEANS_UPDATE", "PAGERANK"):
        return 8
    return 4 if dtype == "i32" else 8


def staging_bytes(nest) -> int:
    if nest["pattern"] == "KMEANS_ASSIGN":
        (N, _), (K, _), (D, _) = nest["levels"]
        return 4 * _eff(K) * _eff(D) + 4 * _eff(K)
    return 0


def smem_model(nest, dtype, blocks) -> int:
    par_reduce = any(sync and b > 1 for (n, sync), b in zip(nest["levels"], blocks))
    return (prod(blocks) * acc_bytes(nest["pattern"], dtype) if par_reduce else 0) + staging_bytes(nest)


def hard_ok(nest, dtype, lim, dims, blocks, spans) -> bool:
    for (n, sync), s in zip(nest["levels"], spans):
        if sync and s != ALL:                               # H1: HL (Table II), HG (L651-656)
            return False
    tb = prod(blocks)
    if tb > lim["max_threads_per_block"]:                    # H2 (L661-662)
        return False
    for d, b in zip(dims, blocks):
        if b > lim["max_block_dim"][d]:                     # H3 (L661-662)
            return False
    if tb * lim["regs_per_thread"] > lim["regs_per_block"]:  # H4 (north_star: registers)
        return False
    if smem_model(nest, dtype, blocks) > lim["smem_per_block"]:  # H5 (north_star: shared memory)
        return False
    grid = prod(level_blocks(n, b, s, 1) for (n, _), b, s in zip(nest["levels"], blocks, spans))
    if grid > MAX_GRID:                                      # H6
        return False
    return True


# ------------------------------------------------------------------ S4 soft constraints

def score(nest, lim, dims, blocks) -> int:
    total = 0
    for contig, mask in nest["accesses"]:
        if contig < 0:
            continue
        weight = W_C * prod(_eff(nest["levels"][l][0]) for l in mask)
        # SL: sequential accesses -> Dim(x) and block size multiple of WARP_SIZE (Table II)
        if dims[contig] == X and blocks[contig] % lim["warp_size"] == 0:
            total += weight
    # SG: threads in block >= MIN_BLOCK_SIZE (Table II), weighted by the whole nest's execution count
    if prod(blocks) >= MIN_BLOCK_SIZE:
        total += W_B * prod(_eff(n) for n, _ in nest["levels"])
    return total


# ------------------------------------------------------------------ S2 + S5 search (Algorithm 1)

def search(nest, dtype, lim, restrict_1d=False):
    """Brute force over CandSet (Alg 1) with the S5 key; returns (dims, blocks, spans, score)."""
    L = len(nest["levels"])
    best = None
    best_key = None
    for dims in itertools.permutations(range(L)):             # lexicographic
        for blocks in itertools.product(SIZE_SET, repeat=L):
            if restrict_1d and any(b != 1 for b in blocks[1:]):
                continue
            for spans in itertools.product((ONE, ALL), repeat=L):
                if restrict_1d and any(s != ALL for s in spans[1:]):
                    continue
                if not hard_ok(nest, dtype, lim, dims, blocks, spans):
                    continue
                sc = score(nest, lim, dims, blocks)
                dop = mapping_dop(nest, blocks, spans, [1] * L)
                key = (sc, dop, -prod(blocks))
                if best_key is None or key > best_key:           # strict: first (lex-smallest) wins ties
                    best_key, best = key, (tuple(dims), tuple(blocks), tuple(spans), sc)
    if best is None:
        raise NoFeasibleMapping(nest["pattern"])
    return best


# ------------------------------------------------------------------ S6 ControlDOP

def control_dop(nest, lim, blocks, spans):
    L = len(blocks)
    spans = list(spans)
    factors = [1] * L
    min_dop = lim["sm_count"] * lim["max_threads_per_sm"]      # L799-801
    max_dop = 100 * min_dop                                    # L801-803
    dop = mapping_dop(nest, blocks, spans, factors)
    if dop < min_dop:                                          # Alg 1
        best_l, best_nb = -1, 1
        for l in range(L):
            n, sync = nest["levels"][l]
            nb = cdiv(_eff(n), blocks[l])
            if sync and spans[l] == ALL and nb >= 2 and nb > best_nb:
                best_l, best_nb = l, nb
        if best_l >= 0:
            k = min(cdiv(min_dop, dop), best_nb)
            if k >= 2:
                spans[best_l], factors[best_l] = SPLIT, k
    elif dop > max_dop:                                        # Alg 1
        for l in range(L):
            if spans[l] == ONE:
                n = min(cdiv(dop, max_dop), cdiv(_eff(nest["levels"][l][0]), blocks[l]))
                if n >= 2:
                    spans[l], factors[l] = SPAN_N, n
                break
    return spans, factors


def min_max_dop(lim):
    m = lim["sm_count"] * lim["max_threads_per_sm"]
    return m, 100 * m


# ------------------------------------------------------------------ S7 forced strategies

def forced(nest, dtype, lim, strategy):
    if len(nest["levels"]) != 2:
        raise Unsupported(strategy)
    if strategy == "1D":
        dims, blocks, spans, _ = search(nest, dtype, lim, restrict_1d=True)
    elif strategy == "TB_T":                                   # Fig 7a
        dims, blocks, spans = (Y, X), (1, min(1024, pow2ceil(_eff(nest["levels"][1][0])))), (ONE, ALL)
    elif strategy == "WARP":                                   # Fig 7b, fn 4 L621-622
        dims, blocks, spans = (Y, X), (16, 32), (ONE, ALL)
    else:
        raise ValueError(strategy)
    if not hard_ok(nest, dtype, lim, dims, blocks, spans):
        raise NoFeasibleMapping(strategy)
    return dims, blocks, spans


# ------------------------------------------------------------------ S8 runtime step (R2)

def slots(lim, threads_per_block: int) -> int:
    per_sm = min(lim["max_blocks_per_sm"], lim["max_threads_per_sm"] // threads_per_block,
                 lim["regs_per_sm"] // (threads_per_block * lim["regs_per_thread"]))
    return lim["sm_count"] * max(1, per_sm)


STAGE_ROWS = 32                                   # DESIGN.md S8 (staged): BR


def staged_eligible(nest, dtype, dims) -> bool:
    """DESIGN.md S8: (weighted) sums whose row pitch is a multiple of 16 B and whose stride-1 level of m
    is on x."""
    pattern = nest["pattern"]
    if pattern not in ("SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"):
        return False
    rows = pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    C = nest["levels"][1][0] if rows else nest["levels"][0][0]
    contig_level = 1 if rows else 0
    return C % (16 // DTYPE_SIZE[dtype]) == 0 and dims[contig_level] == X


def staged_tiles(nest, dtype):
    """DESIGN.md S8 staged: tile = BR rows x W columns (32 KB) of 1 KB chunks (BC elements each).
    Narrow tiles: 32 rows x 1 KB. Wide tiles (SUM_ROWS, row pitch a multiple of 4 KB): 8 rows x 4 KB. Outer tiles:
    BR-row bands (SUM_ROWS) or W-column strips (SUM_COLS). Returns (BR, BC, W, To, Ti)."""
    esz = DTYPE_SIZE[dtype]
    BC = 1024 // esz
    O, I = nest["levels"][0][0], nest["levels"][1][0]
    rows = nest["pattern"] in ("SUM_ROWS", "SUM_WEIGHTED_ROWS")
    C = I if rows else O
    wide = rows and (C * esz) % 4096 == 0
    BR, W = (8, 4 * BC) if wide else (STAGE_ROWS, BC)
    if nest["pattern"] == "SUM_ROWS" and (C * esz) % 32768 == 0 and 65536 <= C * esz <= 32768 * WHOLE_UNIT_MAX:
        BR, W = 1, 32 * BC          # RX one-row tiles: whole-row static split, no row is ever cut
    if nest["pattern"] == "SUM_COLS" and C * esz >= 65536 and cdiv(I, 128) <= WHOLE_UNIT_MAX:
        BR, W = 128, 256 // esz     # MX-narrow strips: whole-strip static split, no strip is ever cut
    if rows:
        return BR, BC, W, cdiv(O, BR), cdiv(I, W)
    return BR, BC, W, cdiv(O, W), cdiv(I, BR)


POOL_DIV = 8                                      # DESIGN.md S8 balance rule
POOL_UNIT = 4
POOL_UNIT_SHORT = 8                               # outer tiles of 9..512 tiles
POOL_UNIT_SHORT_TI_MAX = 512
WHOLE_UNIT_MAX = 8


def balance(To, Ti, lim):
    """DESIGN.md S8 balance rule over T = To*Ti tiles: G = min(SMs, T) persistent blocks; pool claim
    unit U = Ti if Ti <= 8, else 8 if Ti <= 512, else 4; Ts = U*floor((T - floor(T/8))/U) tiles split statically (block b
    streams [b*Ts/G, (b+1)*Ts/G)); the units of [Ts, T) are claimed in order by whichever block is
    free. Returns (G, U, Ts)."""
    T = To * Ti
    G = min(lim["sm_count"], T)
    U = Ti if Ti <= WHOLE_UNIT_MAX else (POOL_UNIT_SHORT if Ti <= POOL_UNIT_SHORT_TI_MAX else POOL_UNIT)
    return G, U, U * ((T - T // POOL_DIV) // U)


def pool_claims(T, Ts, U, Ti, G):
    """DESIGN.md S8 claim order of the pool [Ts, T): units of U tiles, except that when U < Ti the last
    F = min(G, T - Ts) tiles are claimed one at a time. Returns the list of claimed [start, end) ranges
    in claim order."""
    F = min(G, T - Ts) if U < Ti else 0
    out = []
    for c in range(Ts, T - F, U):
        out.append((c, min(T - F, c + U)))
    for j in range(F):
        out.append((T - F + j, T - F + j + 1))
    return out


def r2_staged(nest, dtype, lim):
    """DESIGN.md S8, staged family: persistent blocks (one per SM) stream BR x W tiles in outer-major
    order (static range + pool, balance()); the inner level is Split(Ti)."""
    esz = DTYPE_SIZE[dtype]
    BR, BC, W, To, Ti = staged_tiles(nest, dtype)
    wide = W > BC
    I = nest["levels"][1][0]
    G, CL, _ = balance(To, Ti, lim)
    if nest["pattern"] in ("SUM_ROWS", "SUM_WEIGHTED_ROWS"):  # 8 warps; narrow: 4 rows/warp, wide: 1
        blocks = (8, 32)
        spans = (ONE if wide else SPAN_N, ALL if Ti == 1 else SPLIT)
        factors = (1 if wide else 4, Ti)
        chunks = (BR, W if Ti > 1 else I)
        vec = 16 // esz
    else:                                 # one thread per column of a tile (W columns, 256/W row groups)
        blocks = (W, 256 // W)
        spans = (ONE, ALL if Ti == 1 else SPLIT)
        factors = (1, Ti)
        chunks = (W, BR if Ti > 1 else I)
        vec = 1
    return blocks, spans, factors, vec, chunks, G, CL


def r2_staged_static(nest, dtype, lim) -> int:
    """Ts of the balance rule for a staged sum: the tiles split statically (the rest is the pool)."""
    _, _, _, To, Ti = staged_tiles(nest, dtype)
    return balance(To, Ti, lim)[2]


RC_COL_TILES_MAX = 32                             # DESIGN.md S8 RC: column tiles of one region


def rc_tiling(R, C, dtype, lim):
    """DESIGN.md S8 RC region rule. The ceil(R/32) x ceil(C/BC) tile grid is cut into regions of cr row
    bands x cc column tiles (cc <= 32). Written as the plain double loop over gc and gr:
    for gc in [ceil(Tc/32), max(that, min(Tc, S))], gr in [1, min(Tr, S // gc')], with cc = ceil(Tc/gc),
    gc' = ceil(Tc/cc), cr = ceil(Tr/gr), gr' = ceil(Tr/cr), nreg = gr'*gc', G = min(S, nreg):
    minimise (ceil(nreg/G)*cr*cc, nreg, gc'), the first minimum winning.
    Returns dict(BC, Tr, Tc, cr, cc, gr, gc, nreg, G)."""
    S = lim["sm_count"]
    BC = 1024 // DTYPE_SIZE[dtype]
    Tr, Tc = cdiv(R, STAGE_ROWS), cdiv(C, BC)
    gc_lo = cdiv(Tc, RC_COL_TILES_MAX)
    best, best_key = None, None
    for gc in range(gc_lo, max(gc_lo, min(Tc, S)) + 1):
        cc = cdiv(Tc, gc)
        gce = cdiv(Tc, cc)
        for gr in range(1, min(Tr, max(1, S // gce)) + 1):
            cr = cdiv(Tr, gr)
            gre = cdiv(Tr, cr)
            nreg = gre * gce
            G = min(S, nreg)
            key = (cdiv(nreg, G) * cr * cc, nreg, gce)
            if best_key is None or key < best_key:
                best_key = key
                best = dict(BC=BC, Tr=Tr, Tc=Tc, cr=cr, cc=cc, gr=gre, gc=gce, nreg=nreg, G=G)
    return best


def r2_rowscols(nest, dtype, lim):
    """DESIGN.md S8 RC: columns on x, one thread per column of a 1 KB tile (256/BC row halves), the
    regions of rc_tiling as Split levels. Returns (dims, blocks, spans, factors, vec, chunks, staged, G,
    claim)."""
    (R, _), (C, _) = nest["levels"]
    t = rc_tiling(R, C, dtype, lim)
    dims = (Y, X)
    blocks = (256 // t["BC"], t["BC"])
    spans = (SPLIT if t["gr"] > 1 else ALL, SPLIT if t["gc"] > 1 else ALL)
    factors = (t["gr"], t["gc"])
    chunks = (STAGE_ROWS * t["cr"] if t["gr"] > 1 else R, t["BC"] * t["cc"] if t["gc"] > 1 else C)
    staged = 1 if C % (16 // DTYPE_SIZE[dtype]) == 0 else 0
    return dims, blocks, spans, factors, 1, chunks, staged, t["G"], t["cr"] * t["cc"]


def r2_pagerank(nest, lim):
    """DESIGN.md S8 PR: mean in-degree m = ceil(E/N). m >= 8 (segmented): warps claim chunks of 31 rows, the
    chunk's edges split over 32 lanes (Split), min(8*SMs, chunks) blocks. m < 8 (row groups): V = min(32,
    pow2 >= ceil(m/4)) lanes per row on x, 256/V row groups on y, warp claims of 4*32/V rows, min(4*SMs,
    chunks) blocks. Returns (dims, blocks, spans, factors, vec, chunks, G, chunk)."""
    (N, _), (inner, _) = nest["levels"]
    if inner >= 8:                                 # segmented: 8 warps x 32 lanes, 31 rows per claim
        chunk = 31
        G = min(8 * lim["sm_count"], cdiv(N, chunk))
        return (Y, X), (8, 32), (SPAN_N, SPLIT), (chunk, 32), 1, (chunk, inner), G, chunk
    V = min(32, pow2ceil(cdiv(inner, 4)))          # four edges per lane for a row of average length
    RPB = 256 // V
    chunk = 4 * (32 // V)                          # a warp's claim: 4 rows per group
    G = min(4 * lim["sm_count"], cdiv(N, chunk))
    return (Y, X), (RPB, V), (SPAN_N, ALL), (4, 1), 1, (chunk, inner), G, chunk


def r2_kmupdate(nest, lim):
    """DESIGN.md S8 KU: 96-point tiles, contiguous ranges of P tiles, 12 warps x 32 lanes (2 dims per lane).
    Returns (dims, blocks, spans, factors, vec, chunks, G, P)."""
    (N, _), (D, _) = nest["levels"]
    K = nest["K"]
    if D % 4 != 0 or D < 4 or D > 64 or K < 1 or K > 256 or K * D > 2048:
        raise Unsupported("KMEANS_UPDATE AUTO needs D % 4 == 0, 4 <= D <= 64, 1 <= K <= 256, K*D <= 2048")
    T = cdiv(N, KU_TILE)
    P = cdiv(T, min(lim["sm_count"], T))
    G = cdiv(T, P)
    spans = (SPLIT if G > 1 else ALL, ALL)
    chunks = (KU_TILE * P if G > 1 else N, D)
    return (Y, X), (12, 32), spans, (G, 1), 2, chunks, G, P


KU_TILE = 96                                      # DESIGN.md S8 KU: points per tile (8 per consumer warp)


def r2_logreg(nest, lim, dims):
    """DESIGN.md S8, LOGREG_GRAD staged: 32-row tiles of one batch, contiguous tile ranges."""
    (B, _), (Rb, _), (C, _) = nest["levels"]
    if dims[2] != X or C % 4 != 0 or C > 256:
        raise Unsupported("LOGREG_GRAD AUTO needs C % 4 == 0, C <= 256 and L2 on x")
    Ti = cdiv(Rb, 32)
    tiles = B * Ti
    P = cdiv(tiles, min(lim["sm_count"], tiles))
    G = cdiv(tiles, P)
    blocks = (1, 8, 32)
    spans = (ONE, ALL if Ti == 1 else SPLIT, ALL)
    factors = (1, Ti, 1)
    chunks = (1, 32 if Ti > 1 else Rb, C)
    return blocks, spans, factors, 4, chunks, G, P


KM_REGS = 80                                      # DESIGN.md S8 KM: the kernels' register cap


def km_sets(K: int, lim) -> int:
    """DESIGN.md S8 KM: warp sets (256 threads each) taking tiles round robin — 3 when the centroids are
    one 32-chunk (K <= 32) and a 768-thread block of KM_REGS registers fits, else 2."""
    fits3 = lim["max_threads_per_block"] >= 768 and 768 * KM_REGS <= lim["regs_per_block"]
    return 3 if cdiv(K, 32) == 1 and fits3 else 2


def km_smem_bytes(K: int, D: int, S: int) -> int:
    """DESIGN.md S8 KM shared memory: 1 KB alignment pad + 256 B barriers + ||c||² [32⌈K/32⌉] fp32 +
    exchange words [S sets x (2 if S == 2 else 1) areas][4 groups][TP] x 8 B + a 3-deep ring of 64 KB."""
    TP = 256 if D <= 64 else 128
    return 1024 + 256 + 4 * 32 * cdiv(K, 32) + S * (2 if S == 2 else 1) * 4 * TP * 8 + 3 * 65536


def r2_kmeans(nest, lim):
    """DESIGN.md S8, KMEANS_ASSIGN staged: TP-point tiles, TP/64 points per thread, 4 centroid groups,
    km_sets(K) warp sets taking tiles round robin."""
    (N, _), (K, _), (D, _) = nest["levels"]
    if D % 4 != 0 or D < 4 or D > 128 or K > 256 or 32 * cdiv(K, 32) * D > 16384:
        raise Unsupported("KMEANS_ASSIGN AUTO needs D % 4 == 0, 4 <= D <= 128, K <= 256, Kpad*D <= 16384")
    TP = 256 if D <= 64 else 128                 # points per tile: 4 (or 2) per thread
    T = cdiv(N, TP)
    P = cdiv(T, min(lim["sm_count"], T))
    G = cdiv(T, P)
    S = km_sets(K, lim)
    if (256 * S > lim["max_threads_per_block"] or 256 * S * KM_REGS > lim["regs_per_block"]
            or km_smem_bytes(K, D, S) > lim["smem_per_block"]):
        raise Unsupported("KMEANS_ASSIGN AUTO needs a 512-thread block of 80 registers and its shared memory")
    blocks = (64 * S, 4, 1)                      # S sets of 64 x 4 threads take tiles round robin
    spans = (SPAN_N, ALL, ALL)
    factors = (TP // 64, 1, 1)
    chunks = (S * TP, K, D)
    return blocks, spans, factors, 4, chunks, G, P


def r2_sums(nest, dtype, lim, dims):
    """DESIGN.md S8 (unstaged) for the 2-level sums: returns (blocks, spans, factors, vec, chunks)."""
    pattern = nest["pattern"]
    O, I = nest["levels"][0][0], nest["levels"][1][0]
    C = I if pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS") else O
    contig_level = 1 if pattern in ("SUM_ROWS", "SUM_WEIGHTED_ROWS") else 0
    x_level = 0 if dims[0] == X else 1
    v0 = 16 // DTYPE_SIZE[dtype]
    vec = v0 if (x_level == contig_level and C % v0 == 0) else 1
    S = slots(lim, T_BLOCK)
    if x_level == 1:                                           # class RX
        bx = min(32, pow2ceil(cdiv(I, vec)))
        by = T_BLOCK // bx
        g = cdiv(O, by)
        if g >= S:
            k, n = 1, cdiv(g, S)
        else:
            n = 1
            k = max(1, min(S // g, cdiv(I, bx * vec * U_MIN)))
        chunk_i = vec * cdiv(cdiv(I, k), vec)
        k = cdiv(I, chunk_i)
        blocks = (by, bx)
        spans = (ONE if n == 1 else SPAN_N, ALL if k == 1 else SPLIT)
        factors = (n, k)
        chunks = (by * n, chunk_i if k > 1 else I)
    else:                                                      # class MX
        bx = min(32, pow2ceil(cdiv(O, vec)))
        by = T_BLOCK // bx
        g = cdiv(O, bx * vec)
        if g >= S:
            k, n = 1, cdiv(g, S)
        else:
            n = 1
            k = max(1, min(S // g, cdiv(I, by * U_MIN)))
        chunk_i = cdiv(I, k)
        k = cdiv(I, chunk_i)
        blocks = (bx, by)
        spans = (ONE if n == 1 else SPAN_N, ALL if k == 1 else SPLIT)
        factors = (n, k)
        chunks = (bx * vec * n, chunk_i if k > 1 else I)
    return blocks, spans, factors, vec, chunks


# ------------------------------------------------------------------ S9 record

def kernel_class(pattern, dims):
    if pattern == "KMEANS_ASSIGN":
        return KM
    if pattern == "LOGREG_GRAD":
        return LR
    if pattern == "SUM_ROWS_COLS":
        return RC
    if pattern == "KMEANS_UPDATE":
        return KU
    if pattern == "PAGERANK":
        return PR
    return RX if dims[1] == X else MX


TEMP_NONE, TEMP_MALLOC, TEMP_PREALLOC = 0, 1, 2     # DESIGN.md S10


def temp_layout(nest, dims):
    """DESIGN.md S10 (§V-A, Fig 11): a weighted sum's inner zipWith result goes to one
    preallocated [outer x inner] buffer laid out for the mapping: outer level on x -> offset m, stride
    M (Fig 11b); otherwise offset m*N, stride 1 (Fig 11a). Returns (temp, (outer stride, inner stride))."""
    if nest["pattern"] not in ("SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"):
        return TEMP_NONE, (0, 0)
    M, N = _eff(nest["levels"][0][0]), _eff(nest["levels"][1][0])
    return TEMP_PREALLOC, ((1, M) if dims[0] == X else (N, 1))


def make_record(nest, dtype, lim, dims, blocks, spans, factors, vec, score_, chunks=None, staged=0,
                persistent_grid=None, claim_tiles=0, temp=(TEMP_NONE, (0, 0)), static_tiles=0):
    L = len(blocks)
    levels = []
    for l in range(L):
        n = nest["levels"][l][0]
        v = vec if dims[l] == X else 1
        ch = chunks[l] if chunks is not None else level_chunk(n, blocks[l], spans[l], factors[l], v)
        levels.append(dict(dim=dims[l], block=blocks[l], span=spans[l],
                           factor=(factors[l] if spans[l] in (SPAN_N, SPLIT) else 1),
                           chunk=ch, grid=cdiv(_eff(n), ch)))
    grid = prod(lv["grid"] for lv in levels) if persistent_grid is None else persistent_grid
    block3 = [1, 1, 1]
    for l in range(L):
        block3[dims[l]] = blocks[l]
    rec = dict(nlevels=L, kernel_class=kernel_class(nest["pattern"], dims), vec=vec, staged=staged,
               levels=levels, score=score_, dop=mapping_dop(nest, blocks, spans, factors),
               threads=grid * prod(blocks), grid=grid, block=block3,
               smem_bytes=smem_model(nest, dtype, blocks), workspace_bytes=0, claim_tiles=claim_tiles,
               temp=temp[0], temp_stride=[temp[1][0], temp[1][1]], static_tiles=static_tiles)
    if nest["pattern"] == "LOGREG_GRAD" and staged:  # tickets [B] + fp64 accumulators [B x C]
        B, C = _eff(nest["levels"][0][0]), _eff(nest["levels"][2][0])
        rec["workspace_bytes"] = 256 * cdiv(4 * B, 256) + 256 * cdiv(8 * B * C, 256)
    if nest["pattern"] in ("SUM_ROWS", "SUM_COLS", "SUM_WEIGHTED_ROWS", "SUM_WEIGHTED_COLS"):
        if staged:  # pool counters (256 B) + tickets [To] + accumulators [O] (S8 staged)
            O = _eff(nest["levels"][0][0])
            To = staged_tiles(nest, dtype)[3]   # tickets [To] u32, then accumulators [O]
            rec["workspace_bytes"] = (256 + 256 * cdiv(4 * To, 256)
                                      + 256 * cdiv(O * acc_bytes(nest["pattern"], dtype), 256))
        elif levels[1]["grid"] >= 2:
            O = _eff(nest["levels"][0][0])
            part = levels[1]["grid"] * O * acc_bytes(nest["pattern"], dtype)
            tick = levels[0]["grid"] * 4
            rec["workspace_bytes"] = 256 * cdiv(part, 256) + 256 * cdiv(tick, 256)
    if nest["pattern"] == "PAGERANK" and persistent_grid is not None:  # claim counter + contrib [N] f32
        rec["workspace_bytes"] = 256 + 256 * cdiv(4 * nest["nodes"], 256)
    if nest["pattern"] == "KMEANS_UPDATE" and staged:  # ticket (256 B) + fp64 accumulators [K x (D+1)]
        rec["workspace_bytes"] = 256 + 256 * cdiv(8 * nest["K"] * (_eff(nest["levels"][1][0]) + 1), 256)
    if nest["pattern"] == "SUM_ROWS_COLS" and persistent_grid is not None:
        # S9 RC: tickets [gr] + tickets [gc] (u32), accumulators [R] + [C] of the accumulator type
        R, C = nest["levels"][0][0], nest["levels"][1][0]
        t = rc_tiling(R, C, dtype, lim)
        ab = acc_bytes(nest["pattern"], dtype)
        rec["workspace_bytes"] = (256 * cdiv(4 * t["gr"], 256) + 256 * cdiv(4 * t["gc"], 256)
                                  + 256 * cdiv(R * ab, 256) + 256 * cdiv(C * ab, 256))
    if temp[0] == TEMP_PREALLOC:   # S10: the [outer x inner] buffer after partials and tickets
        M, N = _eff(nest["levels"][0][0]), _eff(nest["levels"][1][0])
        rec["workspace_bytes"] += 256 * cdiv(M * N * DTYPE_SIZE[dtype], 256)
    elif temp[0] == TEMP_MALLOC:   # S10: an error flag
        rec["workspace_bytes"] += 256
    return rec


# ------------------------------------------------------------------ entry point

def enumerate_mappings(pattern: str, shape, dtype: str, lim: dict) -> list:
    """DESIGN.md S2/S3/S6/S9: every hard-feasible candidate of Algorithm 1's CandSet (L772-777), in
    enumeration order, each with ControlDOP applied and recorded as LITERAL records it (its S4 score)."""
    nest = build_nest(pattern, shape)
    L = len(nest["levels"])
    out = []
    for dims in itertools.permutations(range(L)):
        for blocks in itertools.product(SIZE_SET, repeat=L):
            for spans in itertools.product((ONE, ALL), repeat=L):
                if not hard_ok(nest, dtype, lim, dims, blocks, spans):
                    continue
                sc = score(nest, lim, dims, blocks)
                sp, factors = control_dop(nest, lim, blocks, spans)
                out.append(make_record(nest, dtype, lim, dims, blocks, sp, factors, 1, sc,
                                       temp=temp_layout(nest, dims)))
    return out


def select(pattern: str, shape, dtype: str, lim: dict, strategy: str = "AUTO") -> dict:
    """The mapping record for (pattern, shape, dtype, limits, strategy) per DESIGN.md §3."""
    nest = build_nest(pattern, shape)
    L = len(nest["levels"])
    if any(n == 0 or n < -1 for n, _ in nest["levels"]):
        raise ValueError("sizes must be >= 1 (or -1 = unknown)")
    unknown = any(n < 0 for n, _ in nest["levels"])
    if strategy in ("1D", "TB_T", "WARP"):
        dims, blocks, spans = forced(nest, dtype, lim, strategy)
        return make_record(nest, dtype, lim, dims, blocks, spans, [1] * L, 1,
                           score(nest, lim, dims, blocks), temp=temp_layout(nest, dims))
    dims, blocks, spans, sc = search(nest, dtype, lim)
    spans, factors = control_dop(nest, lim, blocks, spans)
    if strategy == "LITERAL":
        return make_record(nest, dtype, lim, dims, blocks, spans, factors, 1, sc, temp=temp_layout(nest, dims))
    if strategy != "AUTO":
        raise ValueError(strategy)
    if unknown:
        raise Unsupported("AUTO needs known sizes")
    if pattern == "LOGREG_GRAD":
        b3, s3, f3, vec, chunks, G, P = r2_logreg(nest, lim, dims)
        return make_record(nest, dtype, lim, dims, b3, s3, f3, vec, sc, chunks, staged=1,
                           persistent_grid=G, claim_tiles=P)
    if pattern == "KMEANS_ASSIGN":
        b3, s3, f3, vec, chunks, G, P = r2_kmeans(nest, lim)
        return make_record(nest, dtype, lim, dims, b3, s3, f3, vec, sc, chunks, staged=1,
                           persistent_grid=G, claim_tiles=P)
    if pattern == "PAGERANK":
        d2, b2, s2, f2, vec, chunks, G, CH = r2_pagerank(nest, lim)
        return make_record(nest, dtype, lim, d2, b2, s2, f2, vec, sc, chunks, staged=0,
                           persistent_grid=G, claim_tiles=CH)
    if pattern == "KMEANS_UPDATE":
        d2, b2, s2, f2, vec, chunks, G, P = r2_kmupdate(nest, lim)
        return make_record(nest, dtype, lim, d2, b2, s2, f2, vec, sc, chunks, staged=1,
                           persistent_grid=G, claim_tiles=P)
    if pattern == "SUM_ROWS_COLS":
        d2, b2, s2, f2, vec, chunks, staged, G, CL = r2_rowscols(nest, dtype, lim)
        return make_record(nest, dtype, lim, d2, b2, s2, f2, vec, sc, chunks, staged=staged,
                           persistent_grid=G, claim_tiles=CL)
    if staged_eligible(nest, dtype, dims):
        b2, s2, f2, vec, chunks, G, CL = r2_staged(nest, dtype, lim)
        return make_record(nest, dtype, lim, dims, b2, s2, f2, vec, sc, chunks, staged=1,
                           persistent_grid=G, claim_tiles=CL, static_tiles=r2_staged_static(nest, dtype, lim))
    b2, s2, f2, vec, chunks = r2_sums(nest, dtype, lim, dims)
    return make_record(nest, dtype, lim, dims, b2, s2, f2, vec, sc, chunks)
