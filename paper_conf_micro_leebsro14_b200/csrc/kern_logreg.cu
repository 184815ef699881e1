// kern_logreg.cu — class LR: the three-level nest of the batched logistic-regression gradient
// (BASELINE.json config 5; G22, S8):
//     batches map { b => rows(b) reduce { i => e_i = σ(x_i·w) − y_i ; x_i map (_ * e_i) } }
//     g[b,j] = Σ_{i in b} x[i,j] · (σ(Σ_k x[i,k] w[k]) − y[i])
// L0 = batches, L1 = rows of a batch (Reduce), L2 = columns (Map_j and the dot Reduce_k at one level,
// Span(all) by the Hard Global constraint). The imperfectly nested access pattern (a dot
// product must finish before the same row is reused) is served by shared-memory staging
// (§V-B): each 32-row tile is loaded once by TMA and read twice from shared memory — for
// the dot and for the update — so HBM sees every byte of x exactly once.
//   warp w owns rows 4w..4w+3 of a tile; lane l owns columns 4l..4l+3 and 128+4l..128+4l+3 with w
//   in registers; the dot finishes with warp shuffles; x·e accumulates per lane in fp32 over the
//   tile and in fp64 across tiles; at a batch boundary the eight warps meet in shared memory.
// Work split as the staged sums: block b streams tiles [bP, bP+P) of the batch-major tile order; a
// batch cut by range boundaries adds its fp64 partial with atomics and the last contributor
// (ticket) converts to fp32.
#include <cstdint>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

constexpr int kStages = 4;
constexpr int kTileRows = 32;
constexpr int kMaxCols = 256;
constexpr int kTileBytes = kTileRows * kMaxCols * 4;
constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kThreads = kConsumers + 32;
constexpr int kSmemHeader = 1024;
constexpr int kRedBytes = kConsumerWarps * kMaxCols * 8;
constexpr int kYBox = kTileRows + 4;  // y box starts 16-B aligned (row0 rounded down to 4): 36 floats
constexpr int kYSlot = 256;           // bytes per ring slot of y (TMA destinations are 128-B aligned)
constexpr int kSmemBytes = kSmemHeader + kStages * kTileBytes + kRedBytes + kStages * kYSlot;

__device__ __forceinline__ float warp_sum_f(float v) {
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
  return v;
}

}  // namespace

__global__ void __launch_bounds__(kThreads, 1) npp_logreg_tma_kernel(const __grid_constant__ CUtensorMap map,
                                                                     const __grid_constant__ CUtensorMap ymap,
                                                                     LogregArgs a) {
  extern __shared__ __align__(1024) unsigned char smem[];
  // y of each staged tile (1-D TMA box of 36 floats from row0 & ~3), one 256-B slot per stage
  unsigned char* y_ring = smem + kSmemHeader + kStages * kTileBytes + kRedBytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kStages;
  long long* slot_tile = reinterpret_cast<long long*>(empty + kStages);  // batch b | kFlush
  int* slot_rows = reinterpret_cast<int*>(slot_tile + kStages);            // rows of the tile in batch b
  int* slot_yoff = slot_rows + kStages;                                     // y offset in its y slot
  unsigned* s_last = reinterpret_cast<unsigned*>(slot_yoff + kStages);
  unsigned char* tiles = smem + kSmemHeader;
  double* red = reinterpret_cast<double*>(smem + kSmemHeader + kStages * kTileBytes);  // [8][C]
  constexpr long long kFlush = 1ll << 62;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x;
  const long long C = a.C, Rb = a.Rb, Ti = a.Ti;
  const long long total = a.B * Ti;
  const long long P = a.per_block;
  const long long r0 = bid * P, r1 = (total < r0 + P) ? total : r0 + P;
  const unsigned tile_bytes = unsigned(kTileRows * C * 4);

  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      tma::mbar_init(full + i, 1);
      tma::mbar_init(empty + i, kConsumerWarps);
    }
    tma::mbar_fence_init();
  }
  __syncthreads();

  if (warp == kConsumerWarps) {
    if (lane == 0) {  // ---------------------------------------------- producer
      tma::prefetch_map(&map);
      long long b = r0 / Ti, j = r0 - (r0 / Ti) * Ti;  // batch and row tile, advanced incrementally
      int slot = 0;
      unsigned ph = 0;
      for (long long cur = r0, t = 0; cur < r1; ++cur, ++t) {
        const bool flush = cur + 1 >= r1 || j + 1 == Ti;
        if (t >= kStages) tma::mbar_wait(empty + slot, ph ^ 1u);
        const long long row0 = b * Rb + j * kTileRows;
        slot_tile[slot] = b | (flush ? kFlush : 0);
        slot_rows[slot] = int((Rb - j * kTileRows) < kTileRows ? (Rb - j * kTileRows) : kTileRows);
        slot_yoff[slot] = int(row0 & 3);
        tma::mbar_expect_tx(full + slot, tile_bytes + kYBox * 4);
        tma::load_2d(tiles + slot * kTileBytes, &map, 0, int(row0), full + slot);
        tma::load_1d(y_ring + slot * kYSlot, &ymap, int(row0 & ~3ll), full + slot);
        if (a.trace) {
          a.trace[cur] = int(bid);
          atomicAdd(a.trace + total + cur, 1);
        }
        if (++j == Ti) j = 0, ++b;
        if (++slot == kStages) slot = 0, ph ^= 1u;
      }
    }
    return;  // the producer warp takes no part in the consumer barriers below
  }

  // ------------------------------------------------------------------ consumers
  const int c0 = lane * 4, c1 = 128 + lane * 4;  // this lane's two column quads
  const int Ci = int(C);
  const bool has0 = c0 < Ci, has1 = c1 < Ci;
  float w0[4] = {0, 0, 0, 0}, w1[4] = {0, 0, 0, 0};
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    if (has0) w0[e] = __ldg(a.w + c0 + e);
    if (has1) w1[e] = __ldg(a.w + c1 + e);
  }
  double acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  const long long n_tiles = r1 - r0;
  int slot = 0;
  unsigned ph = 0;
  for (long long t = 0; t < n_tiles; ++t) {
    // y of the tile's rows: lane l holds y[row0 + l] (masked), broadcast by shuffles below
    tma::mbar_wait(full + slot, ph);
    const long long tag = slot_tile[slot];
    const bool flush = (tag & kFlush) != 0;
    const long long b = tag & ~kFlush;
    const int rows_here = slot_rows[slot];
    const int yoff = slot_yoff[slot];
    const float y_lane = lane < rows_here ? reinterpret_cast<const float*>(y_ring + slot * kYSlot)[yoff + lane] : 0.f;
    const float* tile = reinterpret_cast<const float*>(tiles + slot * kTileBytes);
    // dot products of the warp's 4 rows: per-lane fp32 FMA chains over the lane's 8 columns (error
    // <= γ_8 Σ|x w| of the lane's terms) ...
    float4 x0[4], x1[4];
    float dp[4];
#pragma unroll
    for (int rr = 0; rr < 4; ++rr) {
      const int r = warp * 4 + rr;
      x0[rr] = has0 ? *reinterpret_cast<const float4*>(tile + r * Ci + c0) : make_float4(0, 0, 0, 0);
      x1[rr] = has1 ? *reinterpret_cast<const float4*>(tile + r * Ci + c1) : make_float4(0, 0, 0, 0);
      float d = x0[rr].x * w0[0];
      d = fmaf(x0[rr].y, w0[1], d);
      d = fmaf(x0[rr].z, w0[2], d);
      d = fmaf(x0[rr].w, w0[3], d);
      d = fmaf(x1[rr].x, w1[0], d);
      d = fmaf(x1[rr].y, w1[1], d);
      d = fmaf(x1[rr].z, w1[2], d);
      dp[rr] = fmaf(x1[rr].w, w1[3], d);
    }
    // ... finished in fp64 by a transposing butterfly: 6 shuffles leave lane l with the whole dot of
    // row m(l) = 2*bit4(l) + bit3(l), so each lane evaluates one sigmoid, then 4 shuffles share them.
    const bool h16 = (lane & 16) != 0, h8 = (lane & 8) != 0;
    double a0 = double(h16 ? dp[2] : dp[0]), a1 = double(h16 ? dp[3] : dp[1]);
    a0 += double(__shfl_xor_sync(0xffffffffu, h16 ? dp[0] : dp[2], 16));
    a1 += double(__shfl_xor_sync(0xffffffffu, h16 ? dp[1] : dp[3], 16));
    double zd = h8 ? a1 : a0;
    zd += __shfl_xor_sync(0xffffffffu, h8 ? a0 : a1, 8);
    zd += __shfl_xor_sync(0xffffffffu, zd, 4);
    zd += __shfl_xor_sync(0xffffffffu, zd, 2);
    zd += __shfl_xor_sync(0xffffffffu, zd, 1);
    const int my_row = warp * 4 + (h16 ? 2 : 0) + (h8 ? 1 : 0);
    const float yr = __shfl_sync(0xffffffffu, y_lane, my_row);
    // e = σ(z) − y with a relative error of a few ulps: σ(z) = 1/(1+e^-z) for y = 0 and σ(z) − 1 =
    // −σ(−z) for y = 1 (no cancellation; IEEE expf and division, not the __expf/__fdividef
    // approximations); any other label is evaluated in fp64
    float e_row;
    const float z = float(zd);
    if (yr == 0.f) {
      e_row = 1.f / (1.f + expf(-z));
    } else if (yr == 1.f) {
      e_row = -1.f / (1.f + expf(z));
    } else {
      e_row = float(1.0 / (1.0 + exp(-zd)) - double(yr));
    }
    const float e_mine = my_row < rows_here ? e_row : 0.f;
    float p[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#pragma unroll
    for (int rr = 0; rr < 4; ++rr) {
      const float e = __shfl_sync(0xffffffffu, e_mine, ((rr >> 1) << 4) | ((rr & 1) << 3));
      p[0] = fmaf(x0[rr].x, e, p[0]);
      p[1] = fmaf(x0[rr].y, e, p[1]);
      p[2] = fmaf(x0[rr].z, e, p[2]);
      p[3] = fmaf(x0[rr].w, e, p[3]);
      p[4] = fmaf(x1[rr].x, e, p[4]);
      p[5] = fmaf(x1[rr].y, e, p[5]);
      p[6] = fmaf(x1[rr].z, e, p[6]);
      p[7] = fmaf(x1[rr].w, e, p[7]);
    }
    __syncwarp();
    if (lane == 0) tma::mbar_arrive(empty + slot);
    if (++slot == kStages) slot = 0, ph ^= 1u;
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] += double(p[e]);
    if (!flush) continue;

    // ---- batch b ends in this block's range: combine the 8 warps in fixed order
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      if (has0) red[warp * C + c0 + e] = acc[e];
      if (has1) red[warp * C + c1 + e] = acc[4 + e];
    }
#pragma unroll
    for (int e = 0; e < 8; ++e) acc[e] = 0;
    tma::bar_sync_consumers<kConsumers>();
    const long long f0 = b * Ti, f1 = f0 + Ti;  // tiles of batch b
    const bool owned = f0 >= r0 && f1 <= r1;
    for (int c = threadIdx.x; c < C; c += kConsumers) {
      double s = red[c];
#pragma unroll
      for (int ww = 1; ww < kConsumerWarps; ++ww) s += red[ww * C + c];
      if (owned)
        a.g[b * C + c] = float(s);
      else
        atomicAdd(a.acc + b * C + c, s);
    }
    if (!owned) {
      tma::bar_sync_consumers<kConsumers>();
      if (threadIdx.x == 0) {
        const unsigned contributors = unsigned((f1 - 1) / P - f0 / P + 1);
        const unsigned prev = tma::ticket_add(a.tickets + b, 1u);  // release of the block's adds
        *s_last = (prev + 1 == contributors) ? 1u : 0u;
        if (prev + 1 == contributors) a.tickets[b] = 0u;
      }
      tma::bar_sync_consumers<kConsumers>();
      if (*s_last) {
        __threadfence();
        for (int c = threadIdx.x; c < C; c += kConsumers) {
          unsigned long long* pa = reinterpret_cast<unsigned long long*>(a.acc + b * C + c);
          a.g[b * C + c] = float(__longlong_as_double((long long)atomicExch(pa, 0ull)));
        }
      }
    }
    tma::bar_sync_consumers<kConsumers>();  // `red` is reused by the next flush
  }
}

cudaError_t launch_logreg(const LogregArgs& a, const float* x, int grid, cudaStream_t st) {
  cudaError_t e = ensure_smem(npp_logreg_tma_kernel, kSmemBytes);
  if (e != cudaSuccess) return e;
  CUtensorMap map;
  e = tma::encode_2d(&map, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.B * a.Rb, a.C, unsigned(a.C),
                                 unsigned(kTileRows));
  if (e != cudaSuccess) return e;
  CUtensorMap ymap;
  e = tma::encode_1d(&ymap, a.y, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, a.B * a.Rb, unsigned(kYBox));
  if (e != cudaSuccess) return e;
  npp_logreg_tma_kernel<<<grid, kThreads, kSmemBytes, st>>>(map, ymap, a);
  e = cudaGetLastError();
  if (e != cudaSuccess) std::fprintf(stderr, "npp: logreg launch grid=%d smem=%d: %s\n", grid, kSmemBytes, cudaGetErrorString(e));
  return e;
}

}  // namespace npp
