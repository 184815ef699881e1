// kern_kmupdate.cu — class KU: the k-means centroid update that follows an assignment (SURVEY §8f
// NEXT 4), Table I's groupBy followed by a Reduce per group:
//     points groupBy { i => a_i } map { g => ((g map x) reduce +, g.size) }
//     U[k, d] = Σ_{i: a_i = k} x[i, d],  U[k, D] = |{i : a_i = k}|     (a_i outside [0, K): no group)
// The path is HBM-bound (4·D + 4 bytes per point, D adds): tiles of 96 points (x: 2-D TMA box of
// 96 rows x D floats; a: 1-D box of 96 ints) stream through a 4-deep mbarrier ring, one block per
// SM, contiguous tile ranges (S8 KU). The data-dependent key is why this is not a sum family:
// the reduction target of a point is only known when its a_i arrives.
//   Consumer warp w of 12 adds points w, w+12, ... of each tile (8 per tile): lane l owns dims 2l, 2l+1
//   (float2), so a point is one conflict-free 8-byte read of the tile plus a read-modify-write of the
//   warp's OWN fp32 accumulator row k in shared memory (no atomics: shared-memory float atomics are
//   CAS loops on sm_100a). Points go 4 at a time: with distinct keys their 4 row updates are
//   independent and overlap (the serial load-add-store chain per point was the limit: ncu
//   short-scoreboard stalls, 405 -> 235 µs); counts come from one match.any per tile (the lowest lane
//   of each key group adds its size). The kernel stays bound by those read-modify-write chains, so
//   more warps hide more of them: 12 warps (96 KB of copies, 96-point tiles) 198 µs vs 8 warps with
//   128-point tiles 221 µs (profiles/r02/kmeans_update/). Measured and dropped: 8 points per step with
//   repeated keys merged first (331 µs: the merge tests cost more than the overlap gains), half-warp
//   points with float4 lanes one step (279 µs) or two steps (280 µs) at a time, counts updated by lane
//   0 next to each row update instead of the match.any (306 µs: divergent lane-0 branches). Every
//   128 / 8 = 16 tiles (<= 128 points per warp accumulator, so the fp32 error stays below 127u·Σ|x|)
//   the 12 warp copies are folded into one fp64 block accumulator; at the end each block adds it to the
//   fp64 workspace accumulators with RED atomics and a ticket elects the last block, which converts to
//   f32 and re-zeroes (the Split combine of P:L880-883, fused).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

using namespace tma;

#ifndef NPP_KU_STAGES
#define NPP_KU_STAGES 4
#endif
#ifndef NPP_KU_TP  // DESIGN.md S8 KU: 96-point tiles, 12 consumer warps (8 points each per tile)
#define NPP_KU_TP 96
#endif
#ifndef NPP_KU_WARPS
#define NPP_KU_WARPS 12
#endif
constexpr int kStages = NPP_KU_STAGES;
constexpr int kTP = NPP_KU_TP;            // points per tile
constexpr int kXSlot = kTP * 256;         // kTP * D * 4 <= kTP * 256 B (D <= 64)
constexpr int kASlot = (kTP * 4 + 127) / 128 * 128;  // keys (TMA destinations stay 128-B aligned)
constexpr int kConsumerWarps = NPP_KU_WARPS;
constexpr int kPPW = kTP / kConsumerWarps;  // points of a tile per warp
static_assert(kTP % kConsumerWarps == 0 && kPPW % 4 == 0 && kPPW <= 32, "whole 4-point batches per warp");
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kThreads = kConsumers + 32;  // + producer warp
constexpr int kHeader = 1024;
constexpr int kMaxKD = 2048;               // DESIGN.md S8 KU: K*D <= 2048, K <= 256
constexpr int kMaxK = 256;
#ifndef NPP_KU_FLUSH_TILES  // measurement knob only: the fp32 error bound of DESIGN.md §5 assumes <= 128
#define NPP_KU_FLUSH_TILES (128 / (NPP_KU_TP / NPP_KU_WARPS))  // points per warp copy between flushes
#endif
constexpr int kFlushTiles = NPP_KU_FLUSH_TILES;
constexpr int kSmemBytes = kHeader + kStages * (kXSlot + kASlot) + kConsumerWarps * kMaxKD * 4 +
                           kConsumerWarps * kMaxK * 4 + (kMaxKD + kMaxK) * 8;

__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory"); }

}  // namespace

__global__ void __launch_bounds__(kThreads, 1)
    npp_kmupdate_kernel(const __grid_constant__ CUtensorMap xmap, const __grid_constant__ CUtensorMap amap,
                        const KmUpdateArgs a) {
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kStages;
  volatile int* flag = reinterpret_cast<volatile int*>(empty + kStages);
  unsigned char* xring = smem + kHeader;
  unsigned char* aring = xring + kStages * kXSlot;
  float* accw = reinterpret_cast<float*>(aring + kStages * kASlot);           // [8][K*D]
  unsigned* cntw = reinterpret_cast<unsigned*>(accw + kConsumerWarps * kMaxKD);  // [8][K]
  double* bacc = reinterpret_cast<double*>(cntw + kConsumerWarps * kMaxK);     // [K*(D+1)]
  const int D = int(a.D), K = int(a.K), KD = K * D, KD1 = K * (D + 1);

  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long T = (a.N + kTP - 1) / kTP;
  const long long t0 = blockIdx.x * a.per_block;
  const long long t1 = t0 + a.per_block < T ? t0 + a.per_block : T;

  // the producer lane initialises the ring and issues its first kStages tiles before the block barrier,
  // so they load while the consumers zero their accumulator copies
  const unsigned bytes = unsigned(kTP * D * 4 + kTP * 4);  // x box + key box
  long long early = 0;
  auto issue = [&](long long t) {
    const long long i = t - t0;
    const int slot = int(i % kStages);
    if (i >= kStages) mbar_wait(empty + slot, unsigned((i / kStages) & 1) ^ 1u);
    NPP_CHECK(t >= t0 && t < t1 && t * kTP < a.N);
    mbar_expect_tx(full + slot, bytes);
    load_2d(xring + slot * kXSlot, &xmap, 0, int(t * kTP), full + slot);
    load_1d(aring + slot * kASlot, &amap, int(t * kTP), full + slot);
    if (a.trace) {
      a.trace[t] = int(blockIdx.x);
      atomicAdd(a.trace + T + t, 1);
    }
  };
  if (threadIdx.x == kConsumers) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(full + i, 1);
      mbar_init(empty + i, kConsumerWarps);
    }
    mbar_fence_init();
    prefetch_map(&xmap);
    prefetch_map(&amap);
    if (!a.early_reads) asm volatile("griddepcontrol.wait;" ::: "memory");
    for (; early < kStages && t0 + early < t1; ++early) issue(t0 + early);
  }
  if (threadIdx.x < kConsumers) {
    for (int i = threadIdx.x; i < kConsumerWarps * KD; i += kConsumers) accw[i] = 0.f;
    for (int i = threadIdx.x; i < kConsumerWarps * K; i += kConsumers) cntw[i] = 0u;
    for (int i = threadIdx.x; i < KD1; i += kConsumers) bacc[i] = 0.0;
  }
  __syncthreads();

  if (warp == kConsumerWarps) {
    // ------------------------------------------------------------ producer: one elected lane
    if (lane == 0)
      for (long long t = t0 + early; t < t1; ++t) issue(t);
    return;
  }

  // -------------------------------------------------------------- consumers
  float* myacc = accw + warp * KD;
  unsigned* mycnt = cntw + warp * K;
  const bool dim_lane = 2 * lane < D;
  constexpr int kFR = (kMaxKD + kConsumers - 1) / kConsumers;  // flush elements per thread
  int krow[kFR];  // flush: accumulator row of element tid + kConsumers r (no division per flush)
#pragma unroll
  for (int r = 0; r < kFR; ++r) krow[r] = (int(threadIdx.x) + kConsumers * r) / D;
  auto flush = [&]() {  // fold the 8 warp copies into the fp64 block accumulator, zero the copies
    consumers_sync();
#pragma unroll
    for (int r = 0; r < kFR; ++r) {
      const int i = int(threadIdx.x) + kConsumers * r;
      if (i >= KD) break;
      // the 8 warp copies meet in an fp32 pairwise tree (error <= 3u on top of the copies' <= 127u), then
      // one fp64 add (8 fp64 adds per element measured slower)
      float v[kConsumerWarps];
#pragma unroll
      for (int w = 0; w < kConsumerWarps; ++w) {
        v[w] = accw[w * KD + i];
        accw[w * KD + i] = 0.f;
      }
#pragma unroll
      for (int h = 1; h < kConsumerWarps; h *= 2)  // pairwise tree (any copy count)
#pragma unroll
        for (int w = 0; w + h < kConsumerWarps; w += 2 * h) v[w] += v[w + h];
      bacc[i + krow[r]] += double(v[0]);  // row k of [K x (D+1)]
    }
    for (int k = threadIdx.x; k < K; k += kConsumers) {
      unsigned c = 0;
#pragma unroll
      for (int w = 0; w < kConsumerWarps; ++w) {
        c += cntw[w * K + k];
        cntw[w * K + k] = 0u;
      }
      bacc[k * (D + 1) + D] += double(c);
    }
    consumers_sync();
  };
  int since = 0;
  int slot = 0;
  unsigned phase = 0;
  for (long long t = t0; t < t1; ++t, slot = slot + 1 == kStages ? 0 : slot + 1, phase ^= slot == 0 ? 1u : 0u) {
    mbar_wait(full + slot, phase);
    const float* xt = reinterpret_cast<const float*>(xring + slot * kXSlot);
    const int* at = reinterpret_cast<const int*>(aring + slot * kASlot);
    const int np = t + 1 < t1 || t1 * kTP <= a.N ? kTP : int(a.N - t * kTP);  // valid points (TMA zero-fills)
#ifdef NPP_KU_NO_ACC  // measurement variant (wrong results): the stream without the accumulation
    __syncwarp();
    if (lane == 0) mbar_arrive(empty + slot);
    continue;
#endif
    // the warp's kPPW points of the tile are p = warp + W·j: lane j < kPPW reads key j (-1: no group)
    int kl = -1;
    if (lane < kPPW && warp + kConsumerWarps * lane < np) {
      kl = at[warp + kConsumerWarps * lane];
      if (unsigned(kl) >= unsigned(K)) kl = -1;
    }
    // counts: lanes holding equal keys meet in match.any; the lowest of them adds the group's size
    // (after the sums below, so the match latency overlaps them)
    const unsigned same = __match_any_sync(0xffffffffu, kl);
    // sums: 4 points at a time
#pragma unroll
    for (int j0 = 0; j0 < kPPW; j0 += 4) {
      int k[4];
      float2 xv[4];
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        k[q] = __shfl_sync(0xffffffffu, kl, j0 + q);
        xv[q] = make_float2(0.f, 0.f);
        if (k[q] >= 0 && dim_lane)
          xv[q] = *reinterpret_cast<const float2*>(xt + (warp + kConsumerWarps * (j0 + q)) * D + 2 * lane);
      }
      if (!dim_lane) continue;
#pragma unroll
      for (int q = 0; q < 4; ++q) NPP_CHECK(k[q] < K);
      // a repeated key adds its point into the first point of that key (branch-free selects), so
      // the remaining row updates are distinct and their loads may all issue before the stores;
      // with no branches the compiler interleaves consecutive batches
#pragma unroll
      for (int q = 1; q < 4; ++q) {
        bool done = k[q] < 0;
#pragma unroll
        for (int r = 0; r < q; ++r) {
          const bool hit = !done && k[r] == k[q];
          xv[r].x += hit ? xv[q].x : 0.f;
          xv[r].y += hit ? xv[q].y : 0.f;
          done = done || hit;
        }
        k[q] = (k[q] >= 0 && done) ? -1 : k[q];
      }
      float2 v[4];
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (k[q] >= 0) v[q] = *reinterpret_cast<const float2*>(myacc + k[q] * D + 2 * lane);
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (k[q] >= 0) {
          v[q].x += xv[q].x;
          v[q].y += xv[q].y;
          *reinterpret_cast<float2*>(myacc + k[q] * D + 2 * lane) = v[q];
        }
    }
    if (kl >= 0 && __ffs(same) - 1 == lane) mycnt[kl] += unsigned(__popc(same));
    __syncwarp();
    if (lane == 0) mbar_arrive(empty + slot);
    if (++since == kFlushTiles) {
      flush();
      since = 0;
    }
  }
  if (since) flush();

  // ---- block result -> fp64 workspace accumulators; the last block converts (fused Split combine)
  asm volatile("griddepcontrol.wait;" ::: "memory");  // workspace / out: after the previous grid
  for (int i = threadIdx.x; i < KD1; i += kConsumers) {
    const double v = bacc[i];
    if (v != 0.0) atomicAdd(a.acc + i, v);
  }
  consumers_sync();
  if (threadIdx.x == 0) {  // acq_rel ticket: the release of every consumer's adds (barrier above)
    const bool last = ticket_add(a.ticket, 1u) + 1u == gridDim.x;
    if (last) *a.ticket = 0u;
    flag[0] = last ? 1 : 0;
  }
  consumers_sync();
  if (flag[0]) {  // every load of a thread issued before its stores: one L2 round trip per 9 elements
    __threadfence();
    constexpr int kQ = (kMaxKD + kMaxK + kConsumers - 1) / kConsumers;  // K*(D+1) <= 2304: <= 9 per thread
    double v[kQ];
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
      const int i = threadIdx.x + q * kConsumers;
      v[q] = i < KD1 ? __ldcg(a.acc + i) : 0.0;
    }
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
      const int i = threadIdx.x + q * kConsumers;
      if (i < KD1) {
        __stcg(a.acc + i, 0.0);
        a.out[i] = float(v[q]);
      }
    }
  }
}

cudaError_t launch_kmupdate(const KmUpdateArgs& a, const float* x, const int* keys, int grid, cudaStream_t st) {
  if (a.D % 4 != 0 || a.D < 4 || a.D > 64 || a.K < 1 || a.K > kMaxK || a.K * a.D > kMaxKD)
    return cudaErrorInvalidValue;
  CUtensorMap xmap, amap;
  cudaError_t e = encode_2d(&xmap, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.N, a.D, unsigned(a.D), unsigned(kTP));
  if (e != cudaSuccess) return e;
  if ((e = encode_1d(&amap, keys, CU_TENSOR_MAP_DATA_TYPE_INT32, a.N, unsigned(kTP))) != cudaSuccess) return e;
  if ((e = ensure_smem(npp_kmupdate_kernel, kSmemBytes)) != cudaSuccess) return e;
#if NPP_KU_TP != 96  // measurement variants: the record's ranges are in 96-point tiles
  KmUpdateArgs b = a;
  b.per_block = ((a.N + kTP - 1) / kTP + grid - 1) / grid;
  return launch_pdl(npp_kmupdate_kernel, grid, kThreads, kSmemBytes, st, a.pdl != 0, xmap, amap, b);
#else
  return launch_pdl(npp_kmupdate_kernel, grid, kThreads, kSmemBytes, st, a.pdl != 0, xmap, amap, a);
#endif
}

}  // namespace npp
