// select.cpp — the mapping analysis of PAPER.md §IV as deterministic integer logic (CUDA-free).
//
//   S1 nest descriptor            §IV intro P:L396-403, L454-455; Fig 8
//   S2 candidate space            Algorithm 1
//   S3 hard constraints           Table II P:L559-565 (HL, HG); P:L658-662 (GPU limits)
//   S4 soft constraints, weights  Table II (SL, SG)
//   S5 selection key              P:L734-741; Alg 1 P:L790-792 (ties made deterministic, G2)
//   S6 ControlDOP                 Alg 1
//   S7 forced prior-work mappings P:L99-115; Fig 7
//   S8 runtime step R2            P:L810-817 ("block sizes and span/split factors can be
//                                 dynamically changed without recompiling the code")
//   S9 mapping record             grid/chunk/workspace for the kernel families (§IV-E)
// Every rule is spelled out in DESIGN.md §3; oracle/select.py implements the same document
// independently and tests/test_select_parity.py compares the two records field by field.
#include "select.hpp"

#include <algorithm>
#include <climits>
#include <cstdlib>
#include <cstdio>

namespace npp {

namespace {

constexpr int kSizeSetLen = 11;          // {1,2,...,1024}  Alg 1
constexpr int64_t kWC = 8;               // coalescing intrinsic weight (G3)
constexpr int64_t kWB = 1;               // min-block-size intrinsic weight (G3)
constexpr int kMinBlockSize = 64;        // Table II SG (G5)
constexpr int64_t kUnknownSize = 1000;   // P:L699-700 (G17)
constexpr int kTBlock = 256;             // R2 threads per block (S8)
constexpr int64_t kUMin = 8;             // R2 minimum loads per lane per chunk (S8)
constexpr int64_t kMaxGrid = (int64_t(1) << 31) - 1;  // H6

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline int64_t eff(int64_t n) { return n < 0 ? kUnknownSize : n; }
inline int64_t pow2ceil(int64_t v) {
  int64_t p = 1;
  while (p < v) p <<= 1;
  return p;
}

int64_t prod_blocks(const Nest& n, const Choice& c) {
  int64_t p = 1;
  for (int l = 0; l < n.L; ++l) p *= c.blocks[l];
  return p;
}

// G7: DOP contributed by one level
int64_t level_dop(int64_t N, int b, int span, int64_t factor) {
  N = eff(N);
  switch (span) {
    case NPP_SPAN_ONE: return N;
    case NPP_SPAN_ALL: return b < N ? b : N;
    case NPP_SPAN_N: return cdiv(N, factor);
    default: {  // Split(k)
      int64_t per = cdiv(N, factor);
      return factor * (b < per ? b : per);
    }
  }
}

int64_t mapping_dop(const Nest& n, const Choice& c) {
  int64_t d = 1;
  for (int l = 0; l < n.L; ++l) d *= level_dop(n.N[l], c.blocks[l], c.spans[l], c.factors[l]);
  return d;
}

// S9: indices of level l one thread block covers
int64_t level_chunk(int64_t N, int b, int span, int64_t factor, int vec) {
  N = eff(N);
  switch (span) {
    case NPP_SPAN_ONE: return int64_t(b) * vec;
    case NPP_SPAN_N: return int64_t(b) * vec * factor;
    case NPP_SPAN_ALL: return N > 0 ? N : 1;
    default: {  // Split(k): contiguous chunks of ceil(N/k) (G12), rounded up to the vector width
      int64_t ch = cdiv(N, factor);
      return cdiv(ch, vec) * vec;
    }
  }
}

int acc_bytes(int pattern, int dtype) {
  if (pattern == NPP_KMEANS_ASSIGN || pattern == NPP_LOGREG_GRAD || pattern == NPP_KMEANS_UPDATE ||
      pattern == NPP_PAGERANK)
    return 8;
  return dtype == NPP_I32 ? 4 : 8;
}

int64_t staging_bytes(const Nest& n) {
  if (n.pattern == NPP_KMEANS_ASSIGN) return 4 * eff(n.N[1]) * eff(n.N[2]) + 4 * eff(n.N[1]);
  return 0;
}

int64_t smem_model(const Nest& n, int dtype, const Choice& c) {
  bool par_reduce = false;
  for (int l = 0; l < n.L; ++l) par_reduce |= (n.sync[l] && c.blocks[l] > 1);
  return (par_reduce ? prod_blocks(n, c) * acc_bytes(n.pattern, dtype) : 0) + staging_bytes(n);
}

bool key_greater(int64_t s1, int64_t d1, int64_t p1, int64_t s2, int64_t d2, int64_t p2) {
  if (s1 != s2) return s1 > s2;
  if (d1 != d2) return d1 > d2;
  return p1 < p2;  // smaller Π b wins
}

// Alg 1 SEARCH with the S5 key. restrict_1d: b_l = 1 and Span(all) for l >= 1 (S7 1D).
// S2: every candidate of Algorithm 1's CandSet (L772-777) in enumeration order — dims permutations
// lexicographic, then block sizes (level 0 most significant), then spans (ONE < ALL) — that passes the
// hard constraints (S3). `visit(c)` sees each one.
template <typename Visit>
void for_each_candidate(const Nest& n, int dtype, const npp_limits& lim, bool restrict_1d, Visit visit) {
  static const int perms2[2][2] = {{0, 1}, {1, 0}};
  static const int perms3[6][3] = {{0, 1, 2}, {0, 2, 1}, {1, 0, 2}, {1, 2, 0}, {2, 0, 1}, {2, 1, 0}};
  const int nperm = n.L == 1 ? 1 : (n.L == 2 ? 2 : 6);
  int total_sizes = 1, total_spans = 1;
  for (int l = 0; l < n.L; ++l) {
    total_sizes *= kSizeSetLen;
    total_spans *= 2;
  }
  for (int p = 0; p < nperm; ++p) {
    Choice c;
    for (int l = 0; l < n.L; ++l) c.dims[l] = n.L == 1 ? 0 : (n.L == 2 ? perms2[p][l] : perms3[p][l]);
    for (int si = 0; si < total_sizes; ++si) {  // lexicographic, level 0 most significant
      int rem = si;
      for (int l = n.L - 1; l >= 0; --l) {
        c.blocks[l] = 1 << (rem % kSizeSetLen);
        rem /= kSizeSetLen;
      }
      if (restrict_1d) {
        bool ok = true;
        for (int l = 1; l < n.L; ++l) ok &= c.blocks[l] == 1;
        if (!ok) continue;
      }
      for (int sp = 0; sp < total_spans; ++sp) {  // ONE(0) < ALL(1), level 0 most significant
        for (int l = 0; l < n.L; ++l) c.spans[l] = (sp >> (n.L - 1 - l)) & 1 ? NPP_SPAN_ALL : NPP_SPAN_ONE;
        if (restrict_1d) {
          bool ok = true;
          for (int l = 1; l < n.L; ++l) ok &= c.spans[l] == NPP_SPAN_ALL;
          if (!ok) continue;
        }
        for (int l = 0; l < n.L; ++l) c.factors[l] = 1;
        if (!hard_ok(n, dtype, lim, c)) continue;
        visit(c);
      }
    }
  }
}

bool search(const Nest& n, int dtype, const npp_limits& lim, bool restrict_1d, Choice* best,
            int64_t* best_score) {
  int64_t bs = 0, bd = 0, bp = 0;
  bool found = false;
  for_each_candidate(n, dtype, lim, restrict_1d, [&](const Choice& c) {
    const int64_t s = score(n, lim, c);
    const int64_t d = mapping_dop(n, c);
    const int64_t pb = prod_blocks(n, c);
    if (!found || key_greater(s, d, pb, bs, bd, bp)) {  // strict: first (lex-smallest) wins ties
      found = true;
      bs = s;
      bd = d;
      bp = pb;
      *best = c;
    }
  });
  *best_score = bs;
  return found;
}

// S6 ControlDOP
void control_dop(const Nest& n, const npp_limits& lim, Choice* c) {
  const int64_t min_dop = int64_t(lim.sm_count) * lim.max_threads_per_sm;
  const int64_t max_dop = 100 * min_dop;
  for (int l = 0; l < n.L; ++l) c->factors[l] = 1;
  const int64_t dop = mapping_dop(n, *c);
  if (dop < min_dop) {  // Span(all) -> Split(k)
    int best_l = -1;
    int64_t best_nb = 1;
    for (int l = 0; l < n.L; ++l) {
      const int64_t nb = cdiv(eff(n.N[l]), c->blocks[l]);
      if (n.sync[l] && c->spans[l] == NPP_SPAN_ALL && nb >= 2 && nb > best_nb) {
        best_l = l;
        best_nb = nb;
      }
    }
    if (best_l >= 0) {
      int64_t k = cdiv(min_dop, dop);
      if (k > best_nb) k = best_nb;
      if (k >= 2) {
        c->spans[best_l] = NPP_SPLIT_K;
        c->factors[best_l] = k;
      }
    }
  } else if (dop > max_dop) {  // Span(1) -> Span(n)
    for (int l = 0; l < n.L; ++l) {
      if (c->spans[l] != NPP_SPAN_ONE) continue;
      int64_t nn = cdiv(dop, max_dop);
      const int64_t cap = cdiv(eff(n.N[l]), c->blocks[l]);
      if (nn > cap) nn = cap;
      if (nn >= 2) {
        c->spans[l] = NPP_SPAN_N;
        c->factors[l] = nn;
      }
      break;
    }
  }
}

int64_t slots(const npp_limits& lim, int threads_per_block) {
  int64_t per_sm = lim.max_blocks_per_sm;
  const int64_t by_threads = lim.max_threads_per_sm / threads_per_block;
  const int64_t by_regs = lim.regs_per_sm / (int64_t(threads_per_block) * lim.regs_per_thread);
  if (by_threads < per_sm) per_sm = by_threads;
  if (by_regs < per_sm) per_sm = by_regs;
  if (per_sm < 1) per_sm = 1;
  return int64_t(lim.sm_count) * per_sm;
}

// S8 staged family: plain sums, 16-B row pitch, stride-1 level of m on x.
bool staged_eligible(const Nest& n, int dtype, const Choice& c) {
  if (!is_sum_pattern(n.pattern)) return false;
  const int contig_level = is_rows_pattern(n.pattern) ? 1 : 0;
  return n.cols % (16 / dtype_size(dtype)) == 0 && c.dims[contig_level] == NPP_DIM_X;
}

// S8 staged family: persistent blocks (one per SM) stream BR x W tiles in outer-major order
// (static range + pool); the inner level is Split(Ti).
void r2_staged(const Nest& n, int dtype, const npp_limits& lim, Choice* c) {
  const bool rows = is_rows_pattern(n.pattern);
  const int64_t R = rows ? n.N[0] : n.N[1];
  const StagedTiling t = staged_tiling(n.pattern, R, n.cols, dtype);
  const StagedBalance bal = staged_balance(t.To, t.Ti, lim.sm_count);
  c->claim_tiles = bal.U;
  c->static_tiles = bal.Ts;
  c->persistent_grid = bal.G;
  c->staged = 1;
  if (rows) {  // 8 warps; narrow: 4 rows per warp, wide: 1 row per warp
    c->blocks[0] = 8;
    c->blocks[1] = 32;
    c->spans[0] = t.wide ? NPP_SPAN_ONE : NPP_SPAN_N;
    c->factors[0] = t.wide ? 1 : 4;
    c->chunks[0] = t.BR;
    c->chunks[1] = t.Ti > 1 ? t.W : n.N[1];
    c->vec = 16 / dtype_size(dtype);
  } else {  // one thread per column of each 1 KB chunk (W / BC chunks per tile row)
    c->blocks[0] = int(t.wide ? t.W : t.BC);
    c->blocks[1] = int(256 / c->blocks[0]);
    c->spans[0] = NPP_SPAN_ONE;
    c->factors[0] = 1;
    c->chunks[0] = t.W;
    c->chunks[1] = t.Ti > 1 ? t.BR : n.N[1];
    c->vec = 1;
  }
  c->spans[1] = t.Ti == 1 ? NPP_SPAN_ALL : NPP_SPLIT_K;
  c->factors[1] = t.Ti;
}

// S8 LOGREG_GRAD staged: 32-row tiles of one batch, contiguous tile ranges (class LR).
bool r2_logreg(const Nest& n, const npp_limits& lim, Choice* c) {
  const int64_t B = n.N[0], Rb = n.N[1], C = n.N[2];
  if (c->dims[2] != NPP_DIM_X || C % 4 != 0 || C > 256) return false;
  const int64_t Ti = cdiv(Rb, 32), tiles = B * Ti;
  const int64_t per_block = cdiv(tiles, std::min<int64_t>(lim.sm_count, tiles));
  c->claim_tiles = per_block;
  c->persistent_grid = cdiv(tiles, per_block);
  c->staged = 1;
  c->vec = 4;
  c->blocks[0] = 1, c->blocks[1] = 8, c->blocks[2] = 32;
  c->spans[0] = NPP_SPAN_ONE, c->factors[0] = 1, c->chunks[0] = 1;
  c->spans[1] = Ti == 1 ? NPP_SPAN_ALL : NPP_SPLIT_K, c->factors[1] = Ti, c->chunks[1] = Ti > 1 ? 32 : Rb;
  c->spans[2] = NPP_SPAN_ALL, c->factors[2] = 1, c->chunks[2] = C;
  return true;
}

// S8 KMEANS_ASSIGN staged: TP-point tiles, TP/64 points per thread, 4 centroid groups, 2 warp sets (class KM).
bool r2_kmeans(const Nest& n, const npp_limits& lim, Choice* c) {
  const int64_t N = n.N[0], K = n.N[1], D = n.N[2];
  if (D % 4 != 0 || D < 4 || D > 128 || K > 256 || 32 * cdiv(K, 32) * D > 16384) return false;
  const int64_t TP = D <= 64 ? 256 : 128;  // points per tile: 4 (or 2) per thread
  const int64_t T = cdiv(N, TP);
  const int64_t per_block = cdiv(T, std::min<int64_t>(lim.sm_count, T));
  c->claim_tiles = per_block;
  c->persistent_grid = cdiv(T, per_block);
  c->staged = 1;
  c->vec = 4;
  // S sets of 64 x 4 threads take tiles round robin: 3 when the centroids are one 32-chunk and a
  // 768-thread block of kKmRegs registers fits, else 2; a block covers S tiles at once
  constexpr int64_t kKmRegs = 80;
  const bool fits3 = lim.max_threads_per_block >= 768 && 768 * kKmRegs <= lim.regs_per_block;
  const int64_t S = cdiv(K, 32) == 1 && fits3 ? 3 : 2;
  const int64_t km_smem = 1024 + 256 + 4 * 32 * cdiv(K, 32) + S * (S == 2 ? 2 : 1) * 4 * TP * 8 + 3 * 65536;
  if (256 * S > lim.max_threads_per_block || 256 * S * kKmRegs > lim.regs_per_block || km_smem > lim.smem_per_block)
    return false;
  c->blocks[0] = int(64 * S), c->blocks[1] = 4, c->blocks[2] = 1;
  c->spans[0] = NPP_SPAN_N, c->factors[0] = TP / 64, c->chunks[0] = S * TP;
  c->spans[1] = NPP_SPAN_ALL, c->factors[1] = 1, c->chunks[1] = K;
  c->spans[2] = NPP_SPAN_ALL, c->factors[2] = 1, c->chunks[2] = D;
  return true;
}

// S8 (unstaged) for the 2-level sums: keep LITERAL's dims, re-choose blocks / vec / factors / chunks.
void r2_sums(const Nest& n, int dtype, const npp_limits& lim, Choice* c) {
  const bool rows = n.pattern == NPP_SUM_ROWS || n.pattern == NPP_SUM_WEIGHTED_ROWS;
  const int64_t O = n.N[0], I = n.N[1], C = n.cols;
  const int contig_level = rows ? 1 : 0;
  const int x_level = c->dims[0] == NPP_DIM_X ? 0 : 1;
  const int v0 = 16 / dtype_size(dtype);
  const int vec = (x_level == contig_level && C % v0 == 0) ? v0 : 1;
  const int64_t S = slots(lim, kTBlock);
  int64_t k, nn;
  c->vec = vec;
  if (x_level == 1) {  // class RX: inner Reduce on x
    const int64_t bx = std::min<int64_t>(32, pow2ceil(cdiv(I, vec)));
    const int64_t by = kTBlock / bx;
    const int64_t g = cdiv(O, by);
    if (g >= S) {
      k = 1;
      nn = cdiv(g, S);
    } else {
      nn = 1;
      k = std::min<int64_t>(S / g, cdiv(I, bx * vec * kUMin));
      if (k < 1) k = 1;
    }
    const int64_t chunk_i = vec * cdiv(cdiv(I, k), vec);
    k = cdiv(I, chunk_i);
    c->blocks[0] = int(by);
    c->blocks[1] = int(bx);
    c->chunks[0] = by * nn;
    c->chunks[1] = k > 1 ? chunk_i : I;
  } else {  // class MX: outer Map on x, inner Reduce on y
    const int64_t bx = std::min<int64_t>(32, pow2ceil(cdiv(O, vec)));
    const int64_t by = kTBlock / bx;
    const int64_t g = cdiv(O, bx * vec);
    if (g >= S) {
      k = 1;
      nn = cdiv(g, S);
    } else {
      nn = 1;
      k = std::min<int64_t>(S / g, cdiv(I, by * kUMin));
      if (k < 1) k = 1;
    }
    const int64_t chunk_i = cdiv(I, k);
    k = cdiv(I, chunk_i);
    c->blocks[0] = int(bx);
    c->blocks[1] = int(by);
    c->chunks[0] = bx * vec * nn;
    c->chunks[1] = k > 1 ? chunk_i : I;
  }
  c->spans[0] = nn == 1 ? NPP_SPAN_ONE : NPP_SPAN_N;
  c->factors[0] = nn;
  c->spans[1] = k == 1 ? NPP_SPAN_ALL : NPP_SPLIT_K;
  c->factors[1] = k;
}

// S8 RC: both outputs from one pass; columns on x (the stride-1 level of m and of the column output),
// one thread per column of a 1 KB tile (two row halves for 8-byte types), regions from rc_tiling.
void r2_rowscols(const Nest& n, int dtype, const npp_limits& lim, Choice* c) {
  const int64_t R = n.N[0], C = n.N[1];
  const RcTiling t = rc_tiling(R, C, dtype, lim.sm_count);
  c->dims[0] = NPP_DIM_Y, c->dims[1] = NPP_DIM_X;
  c->blocks[0] = int(256 / t.BC), c->blocks[1] = int(t.BC);
  c->spans[0] = t.gr > 1 ? NPP_SPLIT_K : NPP_SPAN_ALL, c->factors[0] = t.gr;
  c->chunks[0] = t.gr > 1 ? kStageRows * t.cr : R;
  c->spans[1] = t.gc > 1 ? NPP_SPLIT_K : NPP_SPAN_ALL, c->factors[1] = t.gc;
  c->chunks[1] = t.gc > 1 ? t.BC * t.cc : C;
  c->vec = 1;
  c->staged = C % (16 / dtype_size(dtype)) == 0 ? 1 : 0;  // TMA needs a 16-B row pitch
  c->persistent_grid = t.G;
  c->claim_tiles = t.cr * t.cc;
}

// S8 KMEANS_UPDATE (class KU): 96-point tiles, contiguous ranges of P tiles, 12 warps one point at a
// time with 2 dims per lane on x.
constexpr int64_t kKuTile = 96;  // S8 KU: points per tile (8 per consumer warp, 12 warps)
bool r2_kmupdate(const Nest& n, const npp_limits& lim, Choice* c) {
  const int64_t N = n.N[0], D = n.N[1], K = n.K;
  if (D % 4 != 0 || D < 4 || D > 64 || K < 1 || K > 256 || K * D > 2048) return false;
  const int64_t T = cdiv(N, kKuTile);
  const int64_t P = cdiv(T, std::min<int64_t>(lim.sm_count, T));
  c->dims[0] = NPP_DIM_Y, c->dims[1] = NPP_DIM_X;
  c->blocks[0] = 12, c->blocks[1] = 32;
  c->persistent_grid = cdiv(T, P);
  c->claim_tiles = P;
  c->spans[0] = c->persistent_grid > 1 ? NPP_SPLIT_K : NPP_SPAN_ALL, c->factors[0] = c->persistent_grid;
  c->chunks[0] = c->persistent_grid > 1 ? kKuTile * P : N;
  c->spans[1] = NPP_SPAN_ALL, c->factors[1] = 1, c->chunks[1] = D;
  c->vec = 2;
  c->staged = 1;
  return true;
}

// S8 PAGERANK (class PR): V = min(32, pow2 >= ceil(ceil(E/N)/2)) lanes per row on x, 256/V row groups on y,
// rows claimed by warps in chunks of 4*32/V; min(4*SMs, chunks) blocks.
void r2_pagerank(const Nest& n, const npp_limits& lim, Choice* c) {
  const int64_t N = n.N[0], inner = n.N[1];  // inner = mean in-degree ceil(E/N)
  c->dims[0] = NPP_DIM_Y, c->dims[1] = NPP_DIM_X;
  c->vec = 1;
  c->staged = 0;
  if (inner >= 8) {  // segmented: warps claim 31 rows, the chunk's edges split over 32 lanes
    const int64_t chunk = 31;
    c->blocks[0] = 8, c->blocks[1] = 32;
    c->spans[0] = NPP_SPAN_N, c->factors[0] = chunk, c->chunks[0] = chunk;
    c->spans[1] = NPP_SPLIT_K, c->factors[1] = 32, c->chunks[1] = inner;
    c->persistent_grid = std::min<int64_t>(8 * int64_t(lim.sm_count), cdiv(N, chunk));  // 8 x 256 threads per SM
    c->claim_tiles = chunk;
    return;
  }
  const int64_t V = std::min<int64_t>(32, pow2ceil(cdiv(inner, 4)));  // four edges per lane on average
  const int64_t RPB = 256 / V, chunk = 4 * (32 / V);  // a warp's claim: 4 rows per group
  const int64_t units = cdiv(N, chunk);
  c->blocks[0] = int(RPB), c->blocks[1] = int(V);
  c->spans[0] = NPP_SPAN_N, c->factors[0] = 4, c->chunks[0] = chunk;
  c->spans[1] = NPP_SPAN_ALL, c->factors[1] = 1, c->chunks[1] = inner;
  c->persistent_grid = std::min<int64_t>(4 * int64_t(lim.sm_count), units);  // 4 x 256 threads per SM
  c->claim_tiles = chunk;
}

int kernel_class_of(const Nest& n, const Choice& c) {
  if (n.pattern == NPP_KMEANS_ASSIGN) return NPP_CLASS_KMEANS;
  if (n.pattern == NPP_LOGREG_GRAD) return NPP_CLASS_LOGREG;
  if (n.pattern == NPP_SUM_ROWS_COLS) return NPP_CLASS_RC;
  if (n.pattern == NPP_KMEANS_UPDATE) return NPP_CLASS_KMUPDATE;
  if (n.pattern == NPP_PAGERANK) return NPP_CLASS_PAGERANK;
  return c.dims[1] == NPP_DIM_X ? NPP_CLASS_RX : NPP_CLASS_MX;
}

}  // namespace

thread_local std::string g_error;

void set_error(const std::string& msg) { g_error = msg; }

// S8 balance rule (S8): G = min(SMs, T) persistent blocks over T tiles in order. The pool
// unit is U = Ti when an outer tile has at most kWholeUnitMax tiles (a claim then covers whole outer
// tiles), else kPoolUnitShort for outer tiles of at most kPoolUnitShortTiMax tiles (fewer contributors
// per cut outer tile: sumCols [8K,8K] 43.3 -> 42.6 us, profiles/r01/unit/sweep.log) and kPoolUnit
// beyond (sumCols [64K,1K] is 0.35 us slower with 8). Ts = U * floor((T - floor(T / kPoolDiv)) / U) tiles are split statically:
// block b streams [b*Ts/G, (b+1)*Ts/G); the units of [Ts, T) are claimed in order from a counter by
// whichever block is free, which absorbs the per-SM bandwidth differences of a static split.
// (NPP_POOL_DIV / NPP_POOL_UNIT override the constants for measurements; tests never set them.)
StagedBalance staged_balance(int64_t To, int64_t Ti, int sm_count) {
  static const int64_t div = [] {
    const char* e = getenv("NPP_POOL_DIV");
    return e ? std::max<int64_t>(1, atoll(e)) : kPoolDiv;
  }();
  static const int64_t unit = [] {
    const char* e = getenv("NPP_POOL_UNIT");
    return e ? std::max<int64_t>(1, atoll(e)) : int64_t(0);
  }();
  StagedBalance b;
  const int64_t T = To * Ti;
  b.G = std::min<int64_t>(sm_count, T);
  b.U = Ti <= kWholeUnitMax ? Ti : (unit ? unit : (Ti <= kPoolUnitShortTiMax ? kPoolUnitShort : kPoolUnit));
  b.Ts = b.U * ((T - T / div) / b.U);
  return b;
}

StagedTiling staged_tiling(int pattern, int64_t R, int64_t C, int dtype) {
  StagedTiling t;
  const int64_t esz = dtype_size(dtype);
  t.BC = 1024 / esz;
  t.wide = is_rows_pattern(pattern) && (C * esz) % 4096 == 0;  // MX measured faster with 1 KB strips
  t.BR = t.wide ? 8 : kStageRows;
  t.W = t.wide ? 4 * t.BC : t.BC;
  if (pattern == NPP_SUM_ROWS && (C * esz) % 32768 == 0 && C * esz >= 65536 && C * esz <= 32768 * kWholeUnitMax) {
    // RX one-row tiles (S8): 1 row x 32 KB, a row is 2-8 tiles, the pool unit is a whole row and the
    // static split is aligned to whole rows: no row is ever cut (no combine)
    t.wide = true;
    t.r1 = true;
    t.BR = 1;
    t.W = 32 * t.BC;
  }
  if (pattern == NPP_SUM_COLS && C * esz >= 65536 && cdiv(R, kStageRowsNarrowMx) <= kWholeUnitMax) {
    // MX-narrow strips (S8): 128 rows x 256 B tiles, so an outer strip is <= 8 tiles, the pool unit is a
    // whole strip and the static split is aligned to whole strips: no strip is ever cut (no combine)
    t.wide = true;
    t.BR = kStageRowsNarrowMx;
    t.W = 256 / esz;
  }
  if (is_rows_pattern(pattern)) {
    t.To = cdiv(R, t.BR);
    t.Ti = cdiv(C, t.W);
  } else {
    t.To = cdiv(C, t.W);
    t.Ti = cdiv(R, t.BR);
  }
  return t;
}

// S8 RC region rule: over gc in [ceil(Tc/32), max(that, min(Tc, S))] and gr in [1, min(Tr, S/gc')]
// (gc', gr' the region counts after rounding the region sizes cc = ceil(Tc/gc), cr = ceil(Tr/gr)),
// minimise (ceil(nreg/G) * cr * cc = tiles of the busiest block, nreg, gc'); first minimum wins.
RcTiling rc_tiling(int64_t R, int64_t C, int dtype, int sm_count) {
  RcTiling best{};
  const int64_t S = sm_count;
  best.BC = 1024 / dtype_size(dtype);
  best.Tr = cdiv(R, kStageRows);
  best.Tc = cdiv(C, best.BC);
  const int64_t gc_lo = cdiv(best.Tc, kRcColTilesMax);
  const int64_t gc_hi = std::max(gc_lo, std::min(best.Tc, S));
  int64_t kc = -1, kn = 0, kg = 0;
  for (int64_t gc = gc_lo; gc <= gc_hi; ++gc) {
    const int64_t cc = cdiv(best.Tc, gc), gce = cdiv(best.Tc, cc);
    const int64_t gr_hi = std::min(best.Tr, std::max<int64_t>(1, S / gce));
    for (int64_t gr = 1; gr <= gr_hi; ++gr) {
      const int64_t cr = cdiv(best.Tr, gr), gre = cdiv(best.Tr, cr);
      const int64_t nreg = gre * gce, G = std::min(S, nreg);
      const int64_t cost = cdiv(nreg, G) * cr * cc;
      if (kc < 0 || cost < kc || (cost == kc && (nreg < kn || (nreg == kn && gce < kg)))) {
        kc = cost, kn = nreg, kg = gce;
        best.cr = cr, best.cc = cc, best.gr = gre, best.gc = gce, best.nreg = nreg, best.G = G;
      }
    }
  }
  return best;
}

int dtype_size(int dtype) { return (dtype == NPP_I64 || dtype == NPP_F64) ? 8 : 4; }

bool is_rows_pattern(int p) { return p == NPP_SUM_ROWS || p == NPP_SUM_WEIGHTED_ROWS; }

bool is_sum_pattern(int p) {
  return p == NPP_SUM_ROWS || p == NPP_SUM_COLS || p == NPP_SUM_WEIGHTED_ROWS ||
         p == NPP_SUM_WEIGHTED_COLS;
}

int build_nest(int pattern, const int64_t* shape, int ndim, Nest* out) {
  if (!shape) {
    set_error("shape is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  Nest n;
  n.pattern = pattern;
  auto need = [&](int d) {
    if (ndim != d) {
      char buf[96];
      std::snprintf(buf, sizeof buf, "pattern %d expects %d sizes, got %d", pattern, d, ndim);
      set_error(buf);
      return false;
    }
    return true;
  };
  switch (pattern) {
    case NPP_SUM_ROWS:
    case NPP_SUM_WEIGHTED_ROWS:
      if (!need(2)) return NPP_ERR_INVALID_ARG;
      n.L = 2;
      n.N[0] = shape[0], n.sync[0] = false;  // Map rows
      n.N[1] = shape[1], n.sync[1] = true;   // Reduce along the row (Fig 1)
      n.acc[n.nacc++] = {0, 0x1u};           // out[r]
      n.acc[n.nacc++] = {1, 0x3u};           // m[r,c]
      if (pattern == NPP_SUM_WEIGHTED_ROWS) n.acc[n.nacc++] = {1, 0x3u};  // v[c]
      n.cols = shape[1];
      break;
    case NPP_SUM_COLS:
    case NPP_SUM_WEIGHTED_COLS:
      if (!need(2)) return NPP_ERR_INVALID_ARG;
      n.L = 2;
      n.N[0] = shape[1], n.sync[0] = false;  // Map columns
      n.N[1] = shape[0], n.sync[1] = true;   // Reduce down the column (Fig 1)
      n.acc[n.nacc++] = {0, 0x1u};           // out[c]
      n.acc[n.nacc++] = {0, 0x3u};           // m[r,c]: stride-1 index is c, i.e. level 0
      if (pattern == NPP_SUM_WEIGHTED_COLS) n.acc[n.nacc++] = {1, 0x3u};  // v[r]
      n.cols = shape[1];
      break;
    case NPP_SUM_ROWS_COLS:  // both levels Reduce: rows for the column sums, columns for the row sums
      if (!need(2)) return NPP_ERR_INVALID_ARG;
      n.L = 2;
      n.N[0] = shape[0], n.sync[0] = true;
      n.N[1] = shape[1], n.sync[1] = true;
      n.acc[n.nacc++] = {0, 0x1u};  // out_rows[r]
      n.acc[n.nacc++] = {1, 0x2u};  // out_cols[c]
      n.acc[n.nacc++] = {1, 0x3u};  // m[r,c]
      n.cols = shape[1];
      break;
    case NPP_KMEANS_UPDATE:  // shape {N, D, K}: groupBy over points (a Reduce into K groups), Map over dims
      if (!need(3)) return NPP_ERR_INVALID_ARG;
      n.L = 2;
      n.N[0] = shape[0], n.sync[0] = true;
      n.N[1] = shape[1], n.sync[1] = false;
      n.K = shape[2];
      if (n.K < 1) {
        set_error("KMEANS_UPDATE needs K >= 1");
        return NPP_ERR_INVALID_ARG;
      }
      n.acc[n.nacc++] = {1, 0x3u};  // x[i,d]
      n.acc[n.nacc++] = {0, 0x1u};  // a[i]
      n.acc[n.nacc++] = {1, 0x2u};  // U[k,d]
      n.cols = shape[1];
      break;
    case NPP_PAGERANK:  // shape {N, E} or {rows, E, N}: Map over nodes, Map+Reduce over in-neighbours (Fig 5)
      if (ndim != 2 && ndim != 3) {
        set_error("PAGERANK expects {N, E} or {rows, E, N}");
        return NPP_ERR_INVALID_ARG;
      }
      if (shape[1] < 0 || (ndim == 3 && shape[2] < shape[0])) {
        set_error("PAGERANK needs E >= 0 and rows <= N");
        return NPP_ERR_INVALID_ARG;
      }
      n.L = 2;
      n.N[0] = shape[0], n.sync[0] = false;
      n.E = shape[1];
      n.N[1] = shape[0] > 0 ? std::max<int64_t>(1, cdiv(shape[1], shape[0])) : 1, n.sync[1] = true;
      n.acc[n.nacc++] = {0, 0x1u};   // rowptr[n]
      n.acc[n.nacc++] = {0, 0x1u};   // out[n]
      n.acc[n.nacc++] = {1, 0x3u};   // colidx[j]
      n.acc[n.nacc++] = {-1, 0x3u};  // prevPR(w): a gather
      n.acc[n.nacc++] = {-1, 0x3u};  // w.degree: a gather
      n.cols = ndim == 3 ? shape[2] : shape[0];  // graph nodes (the contrib[] length)
      break;
    case NPP_KMEANS_ASSIGN:  // shape {N, D, K}; levels N / K / D
      if (!need(3)) return NPP_ERR_INVALID_ARG;
      n.L = 3;
      n.N[0] = shape[0], n.sync[0] = false;
      n.N[1] = shape[2], n.sync[1] = true;
      n.N[2] = shape[1], n.sync[2] = true;
      n.acc[n.nacc++] = {0, 0x1u};  // a[i]
      n.acc[n.nacc++] = {2, 0x7u};  // x[i,d]
      n.acc[n.nacc++] = {2, 0x7u};  // c[k,d]
      n.cols = shape[1];
      break;
    case NPP_LOGREG_GRAD:  // shape {B, Rb, C}
      if (!need(3)) return NPP_ERR_INVALID_ARG;
      n.L = 3;
      n.N[0] = shape[0], n.sync[0] = false;
      n.N[1] = shape[1], n.sync[1] = true;
      n.N[2] = shape[2], n.sync[2] = true;  // Map_j + Reduce_k at one level -> Span(all) (HG)
      n.acc[n.nacc++] = {1, 0x3u};  // y[i]
      n.acc[n.nacc++] = {2, 0x7u};  // x[i,k] (dot)
      n.acc[n.nacc++] = {2, 0x7u};  // w[k]
      n.acc[n.nacc++] = {2, 0x7u};  // x[i,j] (update)
      n.acc[n.nacc++] = {2, 0x5u};  // g[b,j]
      n.cols = shape[2];
      break;
    default:
      set_error("unknown pattern");
      return NPP_ERR_INVALID_ARG;
  }
  long double total = 1;
  for (int l = 0; l < n.L; ++l) {
    if (n.N[l] == 0 || n.N[l] < -1 || n.N[l] > (int64_t(1) << 40)) {
      set_error("level sizes must be in [1, 2^40] or -1 (unknown)");
      return NPP_ERR_INVALID_ARG;
    }
    total *= (long double)eff(n.N[l]);
  }
  if (total > (long double)(int64_t(1) << 50)) {
    set_error("nest too large (product of sizes > 2^50)");
    return NPP_ERR_INVALID_ARG;
  }
  *out = n;
  return NPP_OK;
}

int check_limits(const npp_limits* lim) {
  if (!lim) {
    set_error("limits is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  if (lim->sm_count < 1 || lim->max_threads_per_sm < 1 || lim->warp_size < 1 ||
      lim->max_blocks_per_sm < 1 || lim->regs_per_sm < 1 || lim->regs_per_thread < 1) {
    set_error("limits: sm_count, max_threads_per_sm, warp_size, max_blocks_per_sm, regs_per_sm and "
              "regs_per_thread must be >= 1");
    return NPP_ERR_INVALID_ARG;
  }
  return NPP_OK;
}

bool hard_ok(const Nest& n, int dtype, const npp_limits& lim, const Choice& c) {
  for (int l = 0; l < n.L; ++l) {  // H1: Reduce -> Span(all) (HL); one span per level (HG)
    const bool all_like = c.spans[l] == NPP_SPAN_ALL || c.spans[l] == NPP_SPLIT_K;
    if (n.sync[l] && !all_like) return false;
  }
  const int64_t tb = prod_blocks(n, c);
  if (tb > lim.max_threads_per_block) return false;                       // H2
  for (int l = 0; l < n.L; ++l) {
    if (c.dims[l] < 0 || c.dims[l] > 2) return false;
    if (c.blocks[l] < 1 || c.blocks[l] > lim.max_block_dim[c.dims[l]]) return false;  // H3
  }
  if (tb * lim.regs_per_thread > lim.regs_per_block) return false;        // H4
  if (smem_model(n, dtype, c) > lim.smem_per_block) return false;         // H5
  int64_t grid = 1;                                                       // H6
  for (int l = 0; l < n.L; ++l) {
    const int span = c.spans[l] == NPP_SPLIT_K ? NPP_SPAN_ALL
                                               : (c.spans[l] == NPP_SPAN_N ? NPP_SPAN_ONE : c.spans[l]);
    grid *= cdiv(eff(n.N[l]), level_chunk(n.N[l], c.blocks[l], span, 1, 1));
    if (grid > kMaxGrid) return false;
  }
  return true;
}

int64_t score(const Nest& n, const npp_limits& lim, const Choice& c) {
  int64_t total = 0;
  for (int a = 0; a < n.nacc; ++a) {
    const Access& ac = n.acc[a];
    if (ac.contig < 0) continue;
    int64_t w = kWC;
    for (int l = 0; l < n.L; ++l)
      if (ac.mask & (1u << l)) w *= eff(n.N[l]);
    // SL: sequential accesses -> Dim(x) and block size a multiple of WARP_SIZE
    if (c.dims[ac.contig] == NPP_DIM_X && c.blocks[ac.contig] % lim.warp_size == 0) total += w;
  }
  if (prod_blocks(n, c) >= kMinBlockSize) {  // SG: threads per block >= MIN_BLOCK_SIZE
    int64_t w = kWB;
    for (int l = 0; l < n.L; ++l) w *= eff(n.N[l]);
    total += w;
  }
  return total;
}

int record_from_choice(const Nest& n, int dtype, const npp_limits& lim, Choice c, int64_t score_value,
                       npp_mapping* out) {
  npp_mapping m{};
  m.nlevels = n.L;
  m.kernel_class = kernel_class_of(n, c);
  m.vec = c.vec;
  int64_t grid = 1, tb = 1;
  for (int l = 0; l < n.L; ++l) {
    npp_level& lv = m.level[l];
    const int v = c.dims[l] == NPP_DIM_X ? c.vec : 1;
    lv.dim = c.dims[l];
    lv.block = c.blocks[l];
    lv.span = c.spans[l];
    lv.factor = (c.spans[l] == NPP_SPAN_N || c.spans[l] == NPP_SPLIT_K) ? c.factors[l] : 1;
    lv.chunk = c.chunks[l] > 0 ? c.chunks[l] : level_chunk(n.N[l], c.blocks[l], c.spans[l], lv.factor, v);
    lv.grid = cdiv(eff(n.N[l]), lv.chunk);
    grid *= lv.grid;
    tb *= c.blocks[l];
  }
  m.score = score_value;
  m.dop = mapping_dop(n, c);
  if (c.persistent_grid > 0) grid = c.persistent_grid;  // staged: persistent blocks, dynamic tiles
  m.grid = grid;
  m.threads = grid * tb;
  m.block[0] = m.block[1] = m.block[2] = 1;
  for (int l = 0; l < n.L; ++l) m.block[c.dims[l]] = c.blocks[l];
  m.smem_bytes = int32_t(smem_model(n, dtype, c));
  m.workspace_bytes = 0;
  m.staged = c.staged;
  m.claim_tiles = c.claim_tiles;
  m.static_tiles = c.static_tiles;
  m.temp = c.temp;
  m.temp_stride[0] = c.temp_stride[0];
  m.temp_stride[1] = c.temp_stride[1];
  if (n.pattern == NPP_LOGREG_GRAD && c.staged) {  // tickets [B] + fp64 accumulators [B x C]
    m.workspace_bytes = 256 * cdiv(4 * eff(n.N[0]), 256) + 256 * cdiv(8 * eff(n.N[0]) * eff(n.N[2]), 256);
  } else if (n.pattern == NPP_PAGERANK && c.persistent_grid > 0) {
    m.workspace_bytes = 256 + 256 * cdiv(4 * n.cols, 256);  // S9 PR: claim counter + contrib [nodes] f32
  } else if (n.pattern == NPP_KMEANS_UPDATE && c.staged) {
    // S9 KU: ticket (256 B) + fp64 accumulators [K x (D+1)]
    m.workspace_bytes = 256 + 256 * cdiv(8 * n.K * (eff(n.N[1]) + 1), 256);
  } else if (n.pattern == NPP_SUM_ROWS_COLS && c.persistent_grid > 0) {
    // S9 RC: tickets [gr] + tickets [gc] (u32) + accumulators [R] + [C] of the accumulator type
    const RcTiling t = rc_tiling(n.N[0], n.N[1], dtype, lim.sm_count);
    const int64_t ab = acc_bytes(n.pattern, dtype);
    m.workspace_bytes = 256 * cdiv(4 * t.gr, 256) + 256 * cdiv(4 * t.gc, 256) + 256 * cdiv(n.N[0] * ab, 256) +
                        256 * cdiv(n.N[1] * ab, 256);
  } else if (is_sum_pattern(n.pattern) && c.staged) {
    // pool counters (256 B) + tickets [To] + accumulators [O] of the accumulator type
    const StagedTiling t = staged_tiling(n.pattern, is_rows_pattern(n.pattern) ? n.N[0] : n.N[1], n.cols, dtype);
    m.workspace_bytes =
        256 + 256 * cdiv(4 * t.To, 256) + 256 * cdiv(eff(n.N[0]) * acc_bytes(n.pattern, dtype), 256);
  } else if (is_sum_pattern(n.pattern) && m.level[1].grid >= 2) {
    const int64_t part = m.level[1].grid * eff(n.N[0]) * acc_bytes(n.pattern, dtype);
    const int64_t tick = m.level[0].grid * 4;
    m.workspace_bytes = 256 * cdiv(part, 256) + 256 * cdiv(tick, 256);
  }
  if (c.temp == NPP_TEMP_PREALLOC)  // S10: the [outer x inner] buffer after partials and tickets
    m.workspace_bytes += 256 * cdiv(eff(n.N[0]) * eff(n.N[1]) * dtype_size(dtype), 256);
  else if (c.temp == NPP_TEMP_MALLOC)  // S10: one error flag (a device malloc that returned NULL)
    m.workspace_bytes += 256;
  *out = m;
  return NPP_OK;
}

void temp_layout(const Nest& n, Choice* c) {
  if (n.pattern != NPP_SUM_WEIGHTED_ROWS && n.pattern != NPP_SUM_WEIGHTED_COLS) return;
  c->temp = NPP_TEMP_PREALLOC;
  if (c->dims[0] == NPP_DIM_X) {  // Fig 11b
    c->temp_stride[0] = 1;
    c->temp_stride[1] = eff(n.N[0]);
  } else {  // Fig 11a
    c->temp_stride[0] = eff(n.N[1]);
    c->temp_stride[1] = 1;
  }
}

int select_mapping(const Nest& n, int dtype, const npp_limits& lim, int strategy, npp_mapping* out) {
  bool unknown = false;
  for (int l = 0; l < n.L; ++l) unknown |= n.N[l] < 0;
  Choice c;
  int64_t sc = 0;
  if (strategy == NPP_MAP_1D || strategy == NPP_MAP_TB_THREAD || strategy == NPP_MAP_WARP) {
    if (n.L != 2) {
      set_error("forced prior-work mappings (Fig 7) are defined for 2-level nests only");
      return NPP_ERR_UNSUPPORTED;
    }
    if (strategy == NPP_MAP_1D) {  // only the outermost level is parallel
      if (!search(n, dtype, lim, true, &c, &sc)) {
        set_error("no feasible 1D mapping");
        return NPP_ERR_NO_FEASIBLE_MAPPING;
      }
    } else if (strategy == NPP_MAP_TB_THREAD) {  // Fig 7a
      c.dims[0] = NPP_DIM_Y, c.blocks[0] = 1, c.spans[0] = NPP_SPAN_ONE;
      c.dims[1] = NPP_DIM_X, c.spans[1] = NPP_SPAN_ALL;
      c.blocks[1] = int(std::min<int64_t>(1024, pow2ceil(eff(n.N[1]))));
    } else {  // Fig 7b, footnote 4 P:L621-622
      c.dims[0] = NPP_DIM_Y, c.blocks[0] = 16, c.spans[0] = NPP_SPAN_ONE;
      c.dims[1] = NPP_DIM_X, c.blocks[1] = 32, c.spans[1] = NPP_SPAN_ALL;
    }
    if (!hard_ok(n, dtype, lim, c)) {
      set_error("forced mapping violates a hard constraint on this device");
      return NPP_ERR_NO_FEASIBLE_MAPPING;
    }
    temp_layout(n, &c);  // the paper's generated code preallocates with the mapping's layout (S10)
    return record_from_choice(n, dtype, lim, c, score(n, lim, c), out);
  }
  if (strategy != NPP_MAP_AUTO && strategy != NPP_MAP_LITERAL) {
    set_error("unknown strategy");
    return NPP_ERR_INVALID_ARG;
  }
  if (!search(n, dtype, lim, false, &c, &sc)) {
    set_error("no candidate mapping satisfies the hard constraints (Algorithm 1 CandSet is empty)");
    return NPP_ERR_NO_FEASIBLE_MAPPING;
  }
  control_dop(n, lim, &c);
  if (strategy == NPP_MAP_LITERAL) {
    temp_layout(n, &c);
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (unknown) {
    set_error("strategy AUTO needs known sizes (use LITERAL for -1 sizes)");
    return NPP_ERR_UNSUPPORTED;
  }
  if (n.pattern == NPP_LOGREG_GRAD) {
    if (!r2_logreg(n, lim, &c)) {
      set_error("LOGREG_GRAD AUTO needs C % 4 == 0, C <= 256 and the column level on x");
      return NPP_ERR_UNSUPPORTED;
    }
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (n.pattern == NPP_KMEANS_ASSIGN) {
    if (!r2_kmeans(n, lim, &c)) {
      set_error("KMEANS_ASSIGN AUTO needs D % 4 == 0, 4 <= D <= 128, K <= 256, 32*ceil(K/32)*D <= 16384 and a "
                "device that holds its 512-thread (80-register) block and shared memory");
      return NPP_ERR_UNSUPPORTED;
    }
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (n.pattern == NPP_SUM_ROWS_COLS) {
    r2_rowscols(n, dtype, lim, &c);
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (n.pattern == NPP_PAGERANK) {
    r2_pagerank(n, lim, &c);
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (n.pattern == NPP_KMEANS_UPDATE) {
    if (!r2_kmupdate(n, lim, &c)) {
      set_error("KMEANS_UPDATE AUTO needs D % 4 == 0, 4 <= D <= 64, 1 <= K <= 256 and K*D <= 2048");
      return NPP_ERR_UNSUPPORTED;
    }
    return record_from_choice(n, dtype, lim, c, sc, out);
  }
  if (staged_eligible(n, dtype, c))
    r2_staged(n, dtype, lim, &c);
  else
    r2_sums(n, dtype, lim, &c);
  return record_from_choice(n, dtype, lim, c, sc, out);
}

}  // namespace npp

extern "C" int npp_select(int pattern, const int64_t* shape, int ndim, int dtype, const npp_limits* limits,
                          int strategy, npp_mapping* out) {
  using namespace npp;
  if (!out) {
    set_error("out is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  if (dtype < NPP_F32 || dtype > NPP_F64) {
    set_error("unknown dtype");
    return NPP_ERR_INVALID_ARG;
  }
  int st = check_limits(limits);
  if (st) return st;
  Nest n;
  st = build_nest(pattern, shape, ndim, &n);
  if (st) return st;
  if ((pattern == NPP_KMEANS_ASSIGN || pattern == NPP_LOGREG_GRAD || pattern == NPP_KMEANS_UPDATE ||
       pattern == NPP_PAGERANK) &&
      dtype != NPP_F32) {
    set_error("k-means, logreg and PageRank are defined for f32");
    return NPP_ERR_UNSUPPORTED;
  }
  return select_mapping(n, dtype, *limits, strategy, out);
}

extern "C" int64_t npp_enumerate(int pattern, const int64_t* shape, int ndim, int dtype, const npp_limits* limits,
                                 npp_mapping* out, int64_t cap) {
  using namespace npp;
  if (cap < 0 || (cap > 0 && !out)) {
    set_error("out is NULL or cap < 0");
    return NPP_ERR_INVALID_ARG;
  }
  if (dtype < NPP_F32 || dtype > NPP_F64) {
    set_error("unknown dtype");
    return NPP_ERR_INVALID_ARG;
  }
  int st = check_limits(limits);
  if (st) return st;
  Nest n;
  st = build_nest(pattern, shape, ndim, &n);
  if (st) return st;
  int64_t count = 0;
  for_each_candidate(n, dtype, *limits, false, [&](const Choice& c0) {
    if (count < cap) {
      Choice c = c0;
      const int64_t s = score(n, *limits, c);
      control_dop(n, *limits, &c);
      temp_layout(n, &c);
      record_from_choice(n, dtype, *limits, c, s, out + count);
    }
    ++count;
  });
  return count;
}
