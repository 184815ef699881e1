// kern_kmeans.cu — class KM: the three-level k-means assignment nest (BASELINE.json config 4):
//     points mapRows { x_i => (0 until K) argmin { k => Σ_d (x_id − c_kd)² } }     ties -> lowest k
// L0 = points (Map), L1 = centroids (argmin Reduce), L2 = dims (Reduce). The mapping keeps L2 on x
// for coalescing, which the staged access satisfies (§V-B): TP-point tiles of x arrive
// by TMA with the 128-byte swizzle (conflict-free per-point reads), while the centroids — read by
// every point — sit in the constant bank for the whole launch.
//   Why the constant bank: every thread of a warp reads the same centroid element at the same time,
//   which is exactly what the constant cache serves; ptxas loads it into uniform registers (LDCU)
//   and the packed FMA takes the uniform register as an operand, so the centroid stream never
//   touches the shared-memory pipe. (With centroids in shared memory the LSU wavefronts, not the
//   FMA pipe, set the pace: profiles/r01/SUMMARY.md.) The S8 limit 32·⌈K/32⌉·D ≤ 16384 floats is
//   the 64 KB constant bank.
//   Thread t of centroid group g (warp-uniform, G = 32/CPT groups) owns points lt + (256/G)·i
//   (i < PPT) of a tile and centroids kc + g·CPT + m (m < CPT) of each 32-centroid chunk kc; it
//   ranks them by s_k = ||c_k||² − 2 x·c_k (same argmin as the squared distance), keeping the first
//   minimum in increasing k; with G = 2 the two groups meet in shared memory (lower k on ties).
//   x·c runs on the packed FP32 pipe (FFMA2, fma.rn.f32x2): even and odd dims accumulate in the two
//   halves of a float2.
//   The dims loop's ceiling is the uniform constant path, not the FMA pipe: one LDCU.64 per 4 FFMA2
//   caps it at ~0.65 of the FFMA2 peak (tools/micro_km_inner.cu). The D > 64 kernel therefore takes 1-2
//   of each thread's 4 pairs per chunk from a broadcast shared-memory copy; the D <= 64 kernels (80-register
//   cap) keep all of them in the constant bank, and with three sets (one 32-chunk) the chunk loop is a
//   compile-time single pass, so the argmin state is born after the dims loop.
// The path is FP32-FMA-bound: 2·N·K·D flops against 4·D bytes of x per point.
#include <cstdint>
#include <mutex>
#include <type_traits>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

constexpr int kMaxStages = 3;
constexpr int kBoxCols = 32;  // 128 B of floats: the 128-B swizzle span
// ping-pong: SETS sets of 8 warps take tiles round robin, so one set's per-tile epilogue (argmin, group
// combine, set barrier) overlaps the other sets' FMA streams. Three sets (24 warps, 768 threads at the
// 80-register cap) when the centroids are one 32-chunk, which all sets read at once from the constant
// cache; with more chunks the sets sit in different chunks and three of them overrun the constant
// cache (K = 256: 3x slower), so two. Exchange areas per set: 2 (tile parity, one set barrier per tile)
// with two sets; 1 with three (shared memory), plus a second set barrier before the words are rewritten.
// exchange areas per set: 2 (tile parity) with two sets over several chunks, else 1
__host__ __device__ constexpr int km_par(int sets, bool one) { return sets == 2 && !one ? 2 : 1; }
#ifndef NPP_KM_JUNROLL
#define NPP_KM_JUNROLL 2
#endif
constexpr int kJUnroll = NPP_KM_JUNROLL;          // 4-dim steps per iteration of the dims loop
constexpr int kConsumerWarps = 8;                 // per set
constexpr int kConsumers = kConsumerWarps * 32;   // per set
constexpr int kSmemHeader = 256;
constexpr int kMaxBoxes = 4;  // D <= 128: four 32-float boxes per point row
constexpr int kMaxStageBytes = 64 * 1024;
constexpr int kSmemLimit = 227 * 1024;
constexpr int kConstFloats = 16384;  // DESIGN.md S8: 32·⌈K/32⌉·D ≤ 16384


// centroids as pairs of −2c: km_pairs[(k/2)·D + d] = (−2c[k & ~1][d], −2c[k | 1][d]), padded rows zero
// (the scaling by −2 is exact). One packed FFMA2 advances two centroids' chains with one (broadcast) x
// element; a chain starts at ||c_k||², so each accumulator half ends as the score ||c_k||² − 2 x·c_k.
__constant__ __align__(16) float2 km_pairs[kConstFloats / 2];
__device__ float2 km_pack_buf[kConstFloats / 2];  // staging for the copy into the constant bank

__global__ void npp_kmeans_pack_kernel(const float* __restrict__ c, int K, int Kp, int D) {
  const int n = Kp / 2 * D;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int k2 = i / D, d = i - k2 * D;
    const int k = 2 * k2;
    km_pack_buf[i] = make_float2(k < K ? -2.f * c[k * D + d] : 0.f, k + 1 < K ? -2.f * c[(k + 1) * D + d] : 0.f);
  }
}

__host__ __device__ inline int64_t km_kpad(int64_t K) { return (K + 31) / 32 * 32; }
__host__ __device__ inline int km_boxes(int64_t D) { return int((D + kBoxCols - 1) / kBoxCols); }
// shared-memory pairs: LDSP of each thread's 4 pairs per 32-chunk come from a shared-memory copy
// (csm[chunk][d][group][LS] float2, LS = LDSP rounded up to a power of two), the rest from the constant
// bank, so the two operand paths share the load: in the bare dims loop the LDCU stream alone caps FFMA2
// at ~0.63-0.69 of peak, the LDS broadcast alone at ~0.74, half and half at ~0.82 (profiles/r02/kmeans/
// micro_inner.log). In the full kernels it pays only where registers are left for the extra operands:
// the D > 64 kernel (2 pairs with three sets, 1 with two); the D <= 64 kernels at the 80-register cap
// are fastest with every pair from the constant bank (profiles/r02/kmeans/lds_pairs.log).
__host__ __device__ constexpr int km_ls(int ldsp) { return ldsp == 0 ? 0 : ldsp == 1 ? 1 : ldsp == 2 ? 2 : 4; }
__host__ __device__ inline int64_t km_csm_bytes(int64_t K, int64_t D, int ldsp) {
  return km_kpad(K) * D * km_ls(ldsp);  // (Kp/32) chunks x D x 4 groups x LS pairs x 8 B
}
__host__ __device__ inline int64_t km_rest_bytes(int64_t K, int64_t D, int tp, int sets, bool one, int ldsp) {
  // alignment pad + barriers (full, released) + ||c||² + exchange words [sets x parities][4 groups][tp]
  // + the shared-memory pairs
  const int par = km_par(sets, one);
  return 1024 + kSmemHeader + km_kpad(K) * 4 + int64_t(sets) * par * 4 * tp * 8 + km_csm_bytes(K, D, ldsp);
}
// ring depth: 3 x 64 KB tiles when they fit
__host__ __device__ inline int km_stages(int64_t K, int64_t D, int tp, int sets, bool one, int ldsp) {
  return km_rest_bytes(K, D, tp, sets, one, ldsp) + 3 * int64_t(kMaxStageBytes) <= kSmemLimit ? 3 : 2;
}
inline size_t km_smem_bytes(int64_t K, int64_t D, int tp, int sets, bool one, int ldsp) {
  return size_t(km_rest_bytes(K, D, tp, sets, one, ldsp) +
                int64_t(km_stages(K, D, tp, sets, one, ldsp)) * kMaxStageBytes);
}
// the shared-memory pairs of a launch: the kernel's choice where it leaves the 3-deep ring in place,
// else none (every pair from the constant bank)
inline int km_ldsp(int64_t K, int64_t D, int tp, int sets, bool one) {
  const int want = D <= 64 ? 0 : sets == 3 ? 2 : 1;
  return want > 0 && km_stages(K, D, tp, sets, one, want) == 3 ? want : 0;
}

// x·c with even/odd dims in the two halves of an f32x2 accumulator
__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

}  // namespace

// 12-bit monotone codes of non-negative floats (the top 12 bits below the sign: 8 exponent + 4 mantissa
// bits), rounded up or down, so a bound survives the packing into the exchange word (2^-4 relative)
__device__ __forceinline__ unsigned code_up(float v) { return (__float_as_uint(v) + 0x7ffffu) >> 19; }
__device__ __forceinline__ unsigned code_down(float v) { return (__float_as_uint(v) & 0x7fffffffu) >> 19; }
__device__ __forceinline__ float decode12(unsigned c) { return __uint_as_float(c << 19); }

// PPT points per thread, CPT centroids per thread and 32-chunk; G = 32/CPT warp-uniform centroid
// groups; a tile is TP = PPT·256/G points. DT = D when it is known at compile time (the d loop is then
// unrolled with immediate centroid offsets), 0 for any D.
template <int PPT, int CPT, int DT, int SETS, int LDSP, bool ONE>
__device__ __forceinline__ void kmeans_body(const CUtensorMap* mapp, const KmeansArgs& a) {
  constexpr int kSets = SETS, kPar = km_par(SETS, ONE), kThreads = SETS * 256;  // no producer warp (refill below)
  const CUtensorMap& map = *mapp;
  constexpr int G = 32 / CPT;
  static_assert(G == 4, "the exchange word packs four centroid groups");
  constexpr int LP = kConsumers / G;  // threads (and point lanes) per centroid group
  constexpr int TP = PPT * LP;        // points per tile
  constexpr int MPW = TP / kConsumerWarps;  // points of a tile each warp of the set merges (32 or 16)
  static_assert(MPW <= 32 && TP % kConsumerWarps == 0, "a warp merges at most 32 points of a tile");
  extern __shared__ __align__(1024) unsigned char smem[];
  const int D = DT ? DT : int(a.D), K = int(a.K), Kp = int(km_kpad(a.K));
  const int nb = DT ? (DT + kBoxCols - 1) / kBoxCols : km_boxes(a.D);
  constexpr int LS = km_ls(LDSP);
  const int kStages = km_stages(a.K, D, TP, SETS, ONE, LDSP);  // ring depth (2 or 3)
  constexpr bool kBarrierRelease = DT == 0 || SETS == 2;  // see the box release below
  // the 128-byte swizzle is a function of smem address bits [7:9]: boxes must be 1 KB aligned
  const unsigned pad = (1024u - (tma::smem_u32(smem) & 1023u)) & 1023u;
  unsigned char* ring = smem + pad;
  float* cn = reinterpret_cast<float*>(ring + kStages * kMaxStageBytes);  // [Kp] ||c_k||², +inf padded
  // exchange words per (set, tile parity): each group's (best score, {k, margin code, norm code}) per point
  uint2* xch = reinterpret_cast<uint2*>(cn + Kp);  // [kSets * kPar][G][TP]
  // the ring is tracked per 32-float box of a slot, so a box is refilled as soon as the 8 warps of its set
  // are past it (a 64-dim tile frees its first half mid-tile: more lead for the next loads)
  uint64_t* full = reinterpret_cast<uint64_t*>(xch + kSets * kPar * G * TP);  // [kMaxStages][kMaxBoxes]
  unsigned* released = reinterpret_cast<unsigned*>(full + kMaxStages * kMaxBoxes);  // [kMaxStages][kMaxBoxes]
  // shared-memory pairs [Kp/32][D][4 groups][LS] (16-byte aligned: the header is 256 B)
  float2* csm = reinterpret_cast<float2*>(reinterpret_cast<unsigned char*>(full) + kSmemHeader);

  // warp index broadcast from lane 0: ptxas then knows the split is warp-uniform and may use the
  // uniform datapath (LDCU) for the centroid reads after it
  const int warp = __shfl_sync(0xffffffffu, int(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  const long long bid = blockIdx.x;
  const long long T = (a.N + TP - 1) / TP;
  const long long P = a.per_block;
  const long long r0 = bid * P, r1 = (T < r0 + P) ? T : r0 + P;

#ifndef NPP_KM_EARLY
#define NPP_KM_EARLY 2  // 2: the D = 64 kernels (config 4 341.6 -> 339.7 us; the generic-D kernels lose with it)
#endif
  constexpr bool kEarlyIssue = NPP_KM_EARLY == 1 || (NPP_KM_EARLY == 2 && DT != 0);
  const long long n_tiles = r1 - r0;
  auto issue_box = [&](long long t, int slot, int bx) {  // box bx of tile t of the range into slot t % kStages
    if (a.trace && bx == 0) {  // white-box schedule trace (npp_execute_traced)
      a.trace[r0 + t] = int(bid);
      atomicAdd(a.trace + T + r0 + t, 1);
    }
    NPP_CHECK(t >= 0 && t < n_tiles && r0 + t < T && bx < nb && slot < kStages);
    tma::mbar_expect_tx(full + slot * kMaxBoxes + bx, unsigned(TP * 128));
    tma::load_2d(ring + slot * kMaxStageBytes + bx * (TP * 128), &map, bx * kBoxCols, int((r0 + t) * TP),
                 full + slot * kMaxBoxes + bx);
  };
  if (threadIdx.x == 0) {
    for (int i = 0; i < kMaxStages * kMaxBoxes; ++i) {
      tma::mbar_init(full + i, 1);
      released[i] = 0;
    }
    tma::mbar_fence_init();
    // the ring's first tiles load while the block computes ||c||² and the shared-memory pairs below
    if (kEarlyIssue) {
      tma::prefetch_map(&map);
      for (int t = 0; t < kStages && t < n_tiles; ++t)
        for (int bx = 0; bx < nb; ++bx) issue_box(t, t, bx);
    }
  }
  // ||c_k||² (fp32 FMA chain over d); padded rows get +inf and are never selected
  for (int k = threadIdx.x; k < Kp; k += kThreads) {
    float s = 0.f;
    if (k < K)
      for (int d = 0; d < D; ++d) s = fmaf(__ldg(a.c + k * D + d), __ldg(a.c + k * D + d), s);
    cn[k] = k < K ? s : __int_as_float(0x7f800000);
  }
  if constexpr (LDSP > 0) {  // pair m < LDSP of group g in chunk ch at dim d: pair (16 ch + 4 g + m) at d
    const int n = Kp / 32 * D * 4 * LS;
    for (int i = threadIdx.x; i < n; i += kThreads) {
      const int m = i % LS, gg = (i / LS) % 4, d = (i / (4 * LS)) % D, ch = i / (4 * LS * D);
      // from the launch's staging copy (the constant bank's source), not the bank: per-thread constant
      // reads would leave the uniform datapath
      csm[i] = m < LDSP ? km_pack_buf[(16 * ch + 4 * gg + m) * D + d] : make_float2(0.f, 0.f);
    }
  }
  __syncthreads();
  // near-tie bound (DESIGN.md §5 k-means): every fp32 score s_k = fl(||c_k||² − 2 x·c_k) is within
  // γ_{2D+2} (||x|| + ||c_k||)² of its exact value, and the fp64 distance as written (G25) within
  // (D+3) 2^-53 (||x|| + ||c_k||)² of the exact distance; a point whose fp32 margin exceeds twice the
  // sum is decided by its fp32 winner, every other point is recomputed in fp64. (||x|| + ||c||)² <=
  // 2 (||x||² + max_k ||c_k||²) keeps the test free of square roots.
  float cmax = 0.f;
  for (int k = 0; k < K; ++k) cmax = fmaxf(cmax, cn[k]);
  const float cm_up = __fmul_ru(cmax, 1.0001f);  // cn carries γ_D relative error
  const float g2d = float(2 * D + 2) * 5.9604645e-8f;  // (2D+2) u, u = 2^-24
  const float coef = 4.04f * (g2d / (1.f - g2d) + float(D + 3) * 1.1102230e-16f);

  if (!kEarlyIssue && threadIdx.x == 0) {
    tma::prefetch_map(&map);
    for (int t = 0; t < kStages && t < n_tiles; ++t)
      for (int bx = 0; bx < nb; ++bx) issue_box(t, t, bx);
  }

  // centroid group; redux.sync lands in a uniform register, so ptxas treats g as warp-uniform and
  // keeps the centroid reads on the uniform datapath (LDCU)
  const int set = int(__reduce_min_sync(0xffffffffu, unsigned(warp / kConsumerWarps)));
  const int wis = warp % kConsumerWarps;  // warp in set: merges points MPW·wis .. MPW·wis + MPW − 1
  const int g = int(__reduce_min_sync(0xffffffffu, unsigned(wis / (kConsumerWarps / G))));
  const int lt = threadIdx.x % LP;  // point lane: points lt + LP·i
  // 128-byte swizzle: 16-byte chunk j of tile row p lives at chunk j ^ (p & 7); LP is a multiple
  // of 8, so every point of the thread has the key lt & 7
  const unsigned key4 = unsigned(lt & 7) << 4;
  const int nd4 = D / 4;
  const int q0 = g * nd4 / G, q1 = (g + 1) * nd4 / G;  // the group's quarter of the dims for ||x||²

  // merge of this warp's MPW points of tile t (area ar): the four groups' words give the winner
  // (lowest score, then lowest k), the margin to the runner-up (a lower bound) and ||x||² (an upper
  // bound); proven points are written, the rest recomputed in fp64 exactly as the oracle does
  auto merge_share = [&](long long t, int ar) {
    const uint2* exs = xch + ar * G * TP;
    const bool mine = lane < MPW;
    const int pt = MPW * wis + (mine ? lane : 0);
    uint2 w[G];
#pragma unroll
    for (int h = 0; h < G; ++h) w[h] = exs[h * TP + pt];
    // winner: lowest (score, k) — groups interleave centroids, so k decides ties (no dynamic indexing of
    // w[], which would put it in local memory)
    float sb = __uint_as_float(w[0].x);
    unsigned wy = w[0].y;
#pragma unroll
    for (int h = 1; h < G; ++h) {
      const float sh = __uint_as_float(w[h].x);
      if (sh < sb || (sh == sb && (w[h].y >> 24) < (wy >> 24))) sb = sh, wy = w[h].y;
    }
    // margin to the runner-up: the winner group's own runner-up, and every other group's best
    float margin = decode12((wy >> 12) & 0xfffu);
    float xn = cm_up;
#pragma unroll
    for (int h = 0; h < G; ++h) {
      if (w[h].y != wy || w[h].x != __float_as_uint(sb)) margin = fminf(margin, __fsub_rd(__uint_as_float(w[h].x), sb));
      xn = __fadd_ru(xn, decode12(w[h].y & 0xfffu));
    }
    const long long gi = (r0 + t) * TP + pt;
    const bool proven = margin > __fmul_ru(coef, xn);
    const bool valid = mine && gi < a.N;
#if defined(NPP_KM_NO_RECHECK)  // measurement variant: the fp32 winner for every point
    if (valid) a.assign[gi] = int(wy >> 24);
    return;
#elif defined(NPP_KM_MARK_FLAGS)  // measurement variant: near ties reported as -1 - winner
    if (valid) a.assign[gi] = proven ? int(wy >> 24) : -1 - int(wy >> 24);
    return;
#endif
    if (proven && valid) a.assign[gi] = int(wy >> 24);
    unsigned m = __ballot_sync(0xffffffffu, !proven && valid);
    while (m) {  // near ties: the fp64 distance as written (G25), the warp on one point, lane = centroid
      const int src = __ffs(m) - 1;
      m &= m - 1;
      const long long gs = (r0 + t) * TP + MPW * wis + src;
      const float* xr = a.x + gs * D;
      double best = __longlong_as_double(0x7ff0000000000000ll);
      int bestk = 0x7fffffff;
#pragma unroll 1
      for (int k = lane; k < K; k += 32) {
        const float* ck = a.c + (long long)k * D;
        double dist = 0.0;
#pragma unroll 4
        for (int d = 0; d < D; ++d) {
          const double df = __dsub_rn(double(__ldg(xr + d)), double(__ldg(ck + d)));
          dist = __dadd_rn(dist, __dmul_rn(df, df));
        }
        if (dist < best) best = dist, bestk = k;  // k increases per lane: first minimum
      }
#pragma unroll
      for (int off = 16; off >= 1; off >>= 1) {
        const double ob = __shfl_xor_sync(0xffffffffu, best, off);
        const int ok = __shfl_xor_sync(0xffffffffu, bestk, off);
        if (ob < best || (ob == best && ok < bestk)) best = ob, bestk = ok;
      }
      NPP_CHECK(gs < a.N && bestk < K);
      if (lane == 0) a.assign[gs] = bestk;
    }
  };

  // slot = t % kStages and round = t / kStages advance incrementally (no 64-bit division per tile)
  int slot = set % kStages;
  unsigned round = unsigned(set / kStages);
  for (long long t = set; t < n_tiles; t += kSets) {
    const unsigned char* tile = ring + slot * kMaxStageBytes + lt * 128;
    float bs[PPT], s2[PPT];
    int bk[PPT];
    float2 n2[PPT];  // the group's share of ||x||² (even / odd dims)
#pragma unroll
    for (int i = 0; i < PPT; ++i) n2[i] = make_float2(0.f, 0.f);
    // ONE: the centroids are one 32-chunk (always with three sets, S8 KM): the chunk loop then
    // runs once at compile time, and the argmin state is born after the dims loop (fewer live registers)
    constexpr bool kOneChunk = ONE;
    for (int kc = 0; kc < (kOneChunk ? 32 : Kp); kc += 32) {
      const int k0 = kc + g * CPT;  // the thread's first centroid of the chunk
      const bool last_chunk = kc + 32 >= Kp;
      float2 acc[PPT][CPT / 2];  // .x: centroid k0 + 2p, .y: k0 + 2p + 1; starts at (||c||², ||c'||²)
      float2 nkp[CPT / 2];
#pragma unroll
      for (int p = 0; p < CPT / 2; ++p) nkp[p] = *reinterpret_cast<const float2*>(cn + k0 + 2 * p);
      if constexpr (DT == 0) {
#pragma unroll
        for (int i = 0; i < PPT; ++i)
#pragma unroll
          for (int p = 0; p < CPT / 2; ++p) acc[i][p] = nkp[p];
      }
      const float2* cq = km_pairs + (k0 >> 1) * D;  // pairs of −2c: the chain ends at the score
      const float2* cs = csm + ((kc / 32) * D * 4 + g) * LS;  // + d·4·LS + m: the shared-memory pairs
#pragma unroll 1
      for (int bx = 0; bx < nb; ++bx) {
        uint64_t* fb = full + slot * kMaxBoxes + bx;
        if (kc == 0) tma::mbar_wait_warp(fb, round & 1u);
        const unsigned char* tb = tile + bx * (TP * 128);
        const int jn = DT ? ((DT / 4 - 8 * bx) < 8 ? (DT / 4 - 8 * bx) : 8) : min(8, nd4 - 8 * bx);
        // one 4-dim step of the thread's dot products; the very first starts the chains at ||c||²
        auto step = [&](int j, auto first) {
          const int d4 = 8 * bx + j;
          const unsigned char* xb = tb + ((unsigned(j) << 4) ^ key4);
          float4 xv[PPT];
#pragma unroll
          for (int i = 0; i < PPT; ++i) xv[i] = *reinterpret_cast<const float4*>(xb + LP * 128 * i);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            float2 cvs[CPT / 2];  // warp-uniform: broadcast LDS for p < LDSP, LDCU for the rest
            const float2* cd = cs + (4 * d4 + q) * 4 * LS;
            if constexpr (LS == 1) {
              cvs[0] = cd[0];
            } else if constexpr (LS >= 2) {
#pragma unroll
              for (int m = 0; m < LDSP; m += 2) {
                if (m + 1 < LDSP) {
                  const float4 c4 = *reinterpret_cast<const float4*>(cd + m);
                  cvs[m] = make_float2(c4.x, c4.y), cvs[m + 1] = make_float2(c4.z, c4.w);
                } else {
                  cvs[m] = cd[m];
                }
              }
            }
#pragma unroll
            for (int p = LDSP; p < CPT / 2; ++p) cvs[p] = cq[p * D + 4 * d4 + q];
#pragma unroll
            for (int p = 0; p < CPT / 2; ++p) {
              const float2 cv = cvs[p];
#pragma unroll
              for (int i = 0; i < PPT; ++i) {
                const float xs = q == 0 ? xv[i].x : q == 1 ? xv[i].y : q == 2 ? xv[i].z : xv[i].w;
                if constexpr (decltype(first)::value) {
                  if (q == 0) {
                    acc[i][p] = nkp[p];
                  }
                }
                ffma2(acc[i][p], make_float2(xs, xs), cv);
              }
            }
          }
        };
        int j = 0;
        if constexpr (DT != 0) {  // peeled first step (the generic-D path keeps the copies: its uniform
          if (bx == 0) step(j++, std::true_type{});  // datapath does not survive the peel)
        }
#pragma unroll kJUnroll
        for (; j < jn; ++j) step(j, std::false_type{});
        if (kc == 0) {  // the group's quarter of the dims inside this box: its share of ||x||²
          const int lo = max(q0, 8 * bx), hi = min(q1, 8 * bx + jn);
          for (int d4 = lo; d4 < hi; ++d4) {
#pragma unroll
            for (int i = 0; i < PPT; ++i) {
#ifndef NPP_KM_NO_NORM  // measurement variant: skip the norm share (the bound is then wrong)
              const float4 v = *reinterpret_cast<const float4*>(tb + LP * 128 * i + ((unsigned(d4 - 8 * bx) << 4) ^ key4));
              ffma2(n2[i], make_float2(v.x, v.y), make_float2(v.x, v.y));
              ffma2(n2[i], make_float2(v.z, v.w), make_float2(v.z, v.w));
#endif
            }
          }
        }
        // the set is past this box of the slot: the last warp refills it (tile t + kStages). In the
        // generic-D kernels the last box of a multi-box tile is refilled after the set barrier instead
        // (every warp is past it there), so only the earlier boxes pay the release atomics (D = 96: 373 ->
        // 362 us; in the three-set D = 64 kernel the extra code pushes ptxas off the uniform datapath)
        if (last_chunk && !(kBarrierRelease && nb > 1 && bx == nb - 1)) {
          __syncwarp();
          if (lane == 0) {
            __threadfence_block();
            unsigned* rel = released + slot * kMaxBoxes + bx;
            if (atomicAdd(rel, 1u) == kConsumerWarps - 1) {
              __threadfence_block();
              *rel = 0;
              asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
              if (t + kStages < n_tiles) issue_box(t + kStages, slot, bx);
            }
          }
        }
      }
      if (kc == 0) {
#pragma unroll
        for (int i = 0; i < PPT; ++i) bs[i] = s2[i] = __int_as_float(0x7f800000), bk[i] = 0;
      }
#pragma unroll
      for (int p = 0; p < CPT / 2; ++p) {  // increasing k within the thread: strict < keeps the first
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int k = k0 + 2 * p + h;
#pragma unroll
          for (int i = 0; i < PPT; ++i) {
            const float sc = h ? acc[i][p].y : acc[i][p].x;
            s2[i] = fminf(s2[i], fmaxf(sc, bs[i]));  // the runner-up over every other k
            if (sc < bs[i]) bs[i] = sc, bk[i] = k;
          }
        }
      }
    }
    // the words of tile t into area (set, tile parity); the set's barrier then lets every warp merge
    // its share of the tile (the area is rewritten two tiles later, after the next barrier)
    const int ar = kPar == 2 ? set * 2 + int((t / kSets) & 1) : set;
    if (kPar == 1 && t >= kSets)  // every warp of the set is done merging the previous words of this area
      asm volatile("bar.sync %0, %1;" ::"r"(1 + set), "n"(kConsumers) : "memory");
    uint2* ex = xch + (ar * G + g) * TP;
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      const float margin = __fsub_rd(s2[i], bs[i]);
      ex[lt + LP * i] = make_uint2(__float_as_uint(bs[i]), (unsigned(bk[i]) << 24) | (code_down(margin) << 12) |
                                                               code_up(__fadd_ru(n2[i].x, n2[i].y)));
    }
    asm volatile("bar.sync %0, %1;" ::"r"(1 + set), "n"(kConsumers) : "memory");  // this set only
    if (kBarrierRelease && nb > 1 && wis == kConsumerWarps - 1 && lane == 0 && t + kStages < n_tiles) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // the set's reads of the box, then TMA
      issue_box(t + kStages, slot, nb - 1);
    }
    merge_share(t, ar);
    for (slot += kSets; slot >= kStages; slot -= kStages) ++round;
  }
}

// One wrapper per tile shape, each with its own register cap: the cap is what keeps ptxas on the
// uniform datapath (LDCU) for the centroid operands, and the value that does so differs per shape
// (tests/test_sass.py checks the result).
#ifndef NPP_KM_MAXNREG_D64
#define NPP_KM_MAXNREG_D64 80
#endif
#ifndef NPP_KM_MAXNREG_D128
#define NPP_KM_MAXNREG_D128 48
#endif
#ifndef NPP_KM_MAXNREG_D64X
#define NPP_KM_MAXNREG_D64X 80
#endif
template <int SETS, int LDSP>
__global__ void __maxnreg__(NPP_KM_MAXNREG_D64) npp_kmeans_tma_kernel_d64(const __grid_constant__ CUtensorMap map,
                                                                         KmeansArgs a) {
  kmeans_body<4, 8, 0, SETS, LDSP, SETS == 3>(&map, a);  // D <= 64: 256-point tiles
}
template <int SETS, int LDSP>
__global__ void __maxnreg__(NPP_KM_MAXNREG_D64X) npp_kmeans_tma_kernel_d64_exact(
    const __grid_constant__ CUtensorMap map, KmeansArgs a) {
  kmeans_body<4, 8, 64, SETS, LDSP, SETS == 3>(&map, a);  // D = 64 (BASELINE.json config 4): immediate centroid offsets
}
template <int SETS, int LDSP>
__global__ void __maxnreg__(NPP_KM_MAXNREG_D128) npp_kmeans_tma_kernel_d128(
    const __grid_constant__ CUtensorMap map, KmeansArgs a) {
  kmeans_body<2, 8, 0, SETS, LDSP, SETS == 3>(&map, a);  // 64 < D <= 128: 128-point tiles
}

namespace {

// The constant bank is one per device and module: KMEANS_ASSIGN launches on different streams are
// ordered by an event so one launch's centroids are never overwritten while another still runs.
// (Inside a stream capture the ordering is the graph's: captured KMEANS_ASSIGN work must not run
// concurrently with other KMEANS_ASSIGN work.)
std::mutex g_km_mutex;
cudaEvent_t g_km_done[64] = {};

cudaError_t launch_tp(void (*kern)(const CUtensorMap, KmeansArgs), int threads, const CUtensorMap& map,
                      const KmeansArgs& a, int grid, size_t smem, cudaStream_t st) {
  cudaError_t e = ensure_smem(kern, int(smem));
  if (e != cudaSuccess) return e;
  kern<<<grid, threads, smem, st>>>(map, a);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_kmeans(const KmeansArgs& args, const float* x, int grid, cudaStream_t st) {
  KmeansArgs a = args;
  a.x = x;
  // tile: 256 points when D <= 64 (4 points x 64 lanes), else 128 (2 points x 64 lanes); both
  // with 4 centroid groups of 8 (S8)
  const bool small = a.D <= 64;
  const int tp = small ? 256 : 128;
  const int sets = a.sets;  // the record's warp sets (S8 KM): 3 or 2
  if (sets != 2 && sets != 3) return cudaErrorInvalidValue;
  if (sets == 3 && km_kpad(a.K) != 32) return cudaErrorInvalidValue;  // three sets: one 32-chunk (S8 KM)
  const bool one = sets == 3;  // the kernels' ONE (compile-time single chunk)
  const int ldsp = km_ldsp(a.K, a.D, tp, sets, one);  // shared-memory pairs (D > 64 kernel only)
  const size_t smem = km_smem_bytes(a.K, a.D, tp, sets, one, ldsp);
  if (km_kpad(a.K) * a.D > kConstFloats) return cudaErrorInvalidValue;  // S8 bound (constant bank)
  CUtensorMap map;
  cudaError_t e = tma::encode_2d(&map, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.N, a.D, unsigned(kBoxCols),
                                 unsigned(tp), CU_TENSOR_MAP_SWIZZLE_128B);
  if (e != cudaSuccess) return e;
  int dev = 0;
  if ((e = cudaGetDevice(&dev)) != cudaSuccess) return e;
  if (dev < 0 || dev >= 64) return cudaErrorInvalidDevice;
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if ((e = cudaStreamIsCapturing(st, &cap)) != cudaSuccess) return e;
  std::lock_guard<std::mutex> lock(g_km_mutex);
  if (!g_km_done[dev] && (e = cudaEventCreateWithFlags(&g_km_done[dev], cudaEventDisableTiming)) != cudaSuccess)
    return e;
  if (cap == cudaStreamCaptureStatusNone && (e = cudaStreamWaitEvent(st, g_km_done[dev], 0)) != cudaSuccess)
    return e;
  const int Kp = int(km_kpad(a.K)), D = int(a.D);
  npp_kmeans_pack_kernel<<<8, 256, 0, st>>>(a.c, int(a.K), Kp, D);
  if ((e = cudaGetLastError()) != cudaSuccess) return e;
  void* pack = nullptr;
  if ((e = cudaGetSymbolAddress(&pack, km_pack_buf)) != cudaSuccess) return e;
  e = cudaMemcpyToSymbolAsync(km_pairs, pack, size_t(Kp) * D * 4, 0, cudaMemcpyDeviceToDevice, st);
  if (e != cudaSuccess) return e;
  auto kern = a.D == 64 ? (sets == 3 ? npp_kmeans_tma_kernel_d64_exact<3, 0> : npp_kmeans_tma_kernel_d64_exact<2, 0>)
              : small    ? (sets == 3 ? npp_kmeans_tma_kernel_d64<3, 0> : npp_kmeans_tma_kernel_d64<2, 0>)
              : sets == 3 ? (ldsp ? npp_kmeans_tma_kernel_d128<3, 2> : npp_kmeans_tma_kernel_d128<3, 0>)
                          : (ldsp ? npp_kmeans_tma_kernel_d128<2, 1> : npp_kmeans_tma_kernel_d128<2, 0>);
  e = launch_tp(kern, sets * 256, map, a, grid, smem, st);
  if (e != cudaSuccess) return e;
  if (cap == cudaStreamCaptureStatusNone) e = cudaEventRecord(g_km_done[dev], st);
  return e;
}

}  // namespace npp
