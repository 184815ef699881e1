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
// The path is FP32-FMA-bound: 2·N·K·D flops against 4·D bytes of x per point.
#include <cstdint>
#include <mutex>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

constexpr int kMaxStages = 3;
constexpr int kBoxCols = 32;  // 128 B of floats: the 128-B swizzle span
// ping-pong: kSets sets of 8 warps take alternate tiles, so one set's per-tile epilogue (argmin,
// group combine, set barrier) overlaps the other set's FMA stream
#ifndef NPP_KM_SETS
#define NPP_KM_SETS 2
#endif
constexpr int kSets = NPP_KM_SETS;
constexpr int kConsumerWarps = 8;                 // per set
constexpr int kConsumers = kConsumerWarps * 32;   // per set
constexpr int kThreads = kSets * kConsumers;      // no producer warp: see the refill below
constexpr int kSmemHeader = 1024;
constexpr int kMaxStageBytes = 64 * 1024;
constexpr int kSmemLimit = 227 * 1024;
constexpr int kConstFloats = 16384;  // DESIGN.md S8: 32·⌈K/32⌉·D ≤ 16384


// centroids as pairs: km_pairs[(k/2)·D + d] = (c[k & ~1][d], c[k | 1][d]), padded rows zero. One
// packed FFMA2 then advances the dot products of two centroids with one (broadcast) x element, so
// each accumulator half ends as a whole dot product (no final add of even/odd halves).
__constant__ float2 km_pairs[kConstFloats / 2];
__device__ float2 km_pack_buf[kConstFloats / 2];  // staging for the copy into the constant bank

__global__ void npp_kmeans_pack_kernel(const float* __restrict__ c, int K, int Kp, int D) {
  const int n = Kp / 2 * D;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const int k2 = i / D, d = i - k2 * D;
    const int k = 2 * k2;
    km_pack_buf[i] = make_float2(k < K ? c[k * D + d] : 0.f, k + 1 < K ? c[(k + 1) * D + d] : 0.f);
  }
}

__host__ __device__ inline int64_t km_kpad(int64_t K) { return (K + 31) / 32 * 32; }
__host__ __device__ inline int km_boxes(int64_t D) { return int((D + kBoxCols - 1) / kBoxCols); }
__host__ __device__ inline int64_t km_rest_bytes(int64_t K, int tp) {  // everything but the ring
  return 1024 /* alignment pad */ + kSmemHeader + km_kpad(K) * 4 + kSets * 2 * 3 * int64_t(tp) * 8;
}
// ring depth: 3 x 64 KB tiles when they fit (always, with the centroids out of shared memory)
__host__ __device__ inline int km_stages(int64_t K, int tp) {
  return km_rest_bytes(K, tp) + 3 * int64_t(kMaxStageBytes) <= kSmemLimit ? 3 : 2;
}
inline size_t km_smem_bytes(int64_t K, int tp) {
  return size_t(km_rest_bytes(K, tp) + int64_t(km_stages(K, tp)) * kMaxStageBytes);
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

// PPT points per thread, CPT centroids per thread and 32-chunk; G = 32/CPT warp-uniform centroid
// groups; a tile is TP = PPT·256/G points.
template <int PPT, int CPT>
__device__ __forceinline__ void kmeans_body(const CUtensorMap* mapp, const KmeansArgs& a) {
  const CUtensorMap& map = *mapp;
  constexpr int G = 32 / CPT;
  constexpr int LP = kConsumers / G;  // threads (and point lanes) per centroid group
  constexpr int TP = PPT * LP;        // points per tile
  extern __shared__ __align__(1024) unsigned char smem[];
  const int nb = km_boxes(a.D);
  const int stage_bytes = nb * TP * 128;
  const int kStages = km_stages(a.K, TP);  // ring depth (2 or 3)
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kMaxStages;
  // the 128-byte swizzle is a function of smem address bits [7:9]: boxes must be 1 KB aligned
  const unsigned pad = (1024u - (tma::smem_u32(smem) & 1023u)) & 1023u;
  unsigned char* ring = smem + pad + kSmemHeader;
  const int D = int(a.D), K = int(a.K), Kp = int(km_kpad(a.K));
  float* cn = reinterpret_cast<float*>(ring + kStages * kMaxStageBytes);  // [Kp]
  // minima of groups 1..G-1 handed to group 0: [set][2 (tile parity)][G-1 <= 3][TP]
  float* xs_s = cn + Kp;
  int* xs_k = reinterpret_cast<int*>(xs_s + kSets * 2 * 3 * TP);

  // warp index broadcast from lane 0: ptxas then knows the producer/consumer split is warp-
  // uniform and may use the uniform datapath (LDCU) for the centroid reads after it
  const int warp = __shfl_sync(0xffffffffu, int(threadIdx.x >> 5), 0), lane = threadIdx.x & 31;
  const long long bid = blockIdx.x;
  const long long T = (a.N + TP - 1) / TP;
  const long long P = a.per_block;
  const long long r0 = bid * P, r1 = (T < r0 + P) ? T : r0 + P;

  unsigned* released = reinterpret_cast<unsigned*>(empty);  // [kStages] warps done with the slot
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      tma::mbar_init(full + i, 1);
      released[i] = 0;
    }
    tma::mbar_fence_init();
  }
  // ||c_k||² (fp32 FMA chain over d); padded rows (zero) get +inf and are never selected
  for (int k = threadIdx.x; k < Kp; k += kThreads) {
    float s = 0.f;
    if (k < K)
      for (int d = 0; d < D; ++d) s = fmaf(__ldg(a.c + k * D + d), __ldg(a.c + k * D + d), s);
    cn[k] = k < K ? s : __int_as_float(0x7f800000);
  }
  __syncthreads();

  const long long n_tiles = r1 - r0;
  auto issue = [&](long long t, int slot) {  // tile t of the block's range into slot t % kStages
    if (a.trace) {  // white-box schedule trace (npp_execute_traced)
      a.trace[r0 + t] = int(bid);
      atomicAdd(a.trace + T + r0 + t, 1);
    }
    tma::mbar_expect_tx(full + slot, unsigned(stage_bytes));
    for (int bx = 0; bx < nb; ++bx)
      tma::load_2d(ring + slot * kMaxStageBytes + bx * (TP * 128), &map, bx * kBoxCols, int((r0 + t) * TP),
                   full + slot);
  };
  if (threadIdx.x == 0) {
    tma::prefetch_map(&map);
    for (int t = 0; t < kStages && t < n_tiles; ++t) issue(t, t);
  }

  // ------------------------------------------------------------------ consumers
  // centroid group; redux.sync lands in a uniform register, so ptxas treats g as warp-uniform and
  // keeps the centroid reads on the uniform datapath (LDCU)
  const int set = int(__reduce_min_sync(0xffffffffu, unsigned(warp / kConsumerWarps)));
  const int g = int(__reduce_min_sync(0xffffffffu, unsigned((warp % kConsumerWarps) / (kConsumerWarps / G))));
  const int lt = threadIdx.x % LP;  // point lane: points lt + LP·i
  // 128-byte swizzle: 16-byte chunk j of tile row p lives at chunk j ^ (p & 7); LP is a multiple
  // of 8, so every point of the thread has the key lt & 7
  const unsigned key = unsigned(lt & 7);
  const int nd4 = D / 4;
  // slot = t % kStages and round = t / kStages advance incrementally (no 64-bit division per tile)
  int slot = set % kStages;
  unsigned round = unsigned(set / kStages);
  for (long long t = set; t < n_tiles; t += kSets) {
    tma::mbar_wait_warp(full + slot, round & 1u);
    const unsigned char* tile = ring + slot * kMaxStageBytes + lt * 128;
    float bs[PPT];
    int bk[PPT];
#pragma unroll
    for (int i = 0; i < PPT; ++i) bs[i] = __int_as_float(0x7f800000), bk[i] = 0x7fffffff;
    for (int kc = 0; kc < Kp; kc += 32) {
      const int k0 = kc + g * CPT;  // the thread's first centroid of the chunk
      float2 acc[PPT][CPT / 2];  // .x: centroid k0 + 2p, .y: k0 + 2p + 1
#pragma unroll
      for (int i = 0; i < PPT; ++i)
#pragma unroll
        for (int p = 0; p < CPT / 2; ++p) acc[i][p] = make_float2(0.f, 0.f);
      const float2* cq = km_pairs + (k0 >> 1) * D;
#pragma unroll 2
      for (int d4 = 0; d4 < nd4; ++d4) {
        const unsigned char* xb = tile + (d4 >> 3) * (TP * 128) + ((unsigned(d4 & 7) ^ key) << 4);
        float4 xv[PPT];
#pragma unroll
        for (int i = 0; i < PPT; ++i) xv[i] = *reinterpret_cast<const float4*>(xb + LP * 128 * i);
#pragma unroll
        for (int p = 0; p < CPT / 2; ++p) {
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            const float2 cv = cq[p * D + 4 * d4 + q];  // warp-uniform
#pragma unroll
            for (int i = 0; i < PPT; ++i) {
              const float xs = q == 0 ? xv[i].x : q == 1 ? xv[i].y : q == 2 ? xv[i].z : xv[i].w;
              ffma2(acc[i][p], make_float2(xs, xs), cv);
            }
          }
        }
      }
#pragma unroll
      for (int p = 0; p < CPT / 2; ++p) {  // increasing k within the thread: strict < keeps the first
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int k = k0 + 2 * p + h;
          const float nk = cn[k];
#pragma unroll
          for (int i = 0; i < PPT; ++i) {
            const float s = fmaf(-2.f, h ? acc[i][p].y : acc[i][p].x, nk);
            if (s < bs[i]) bs[i] = s, bk[i] = k;
          }
        }
      }
    }
    const long long base = (r0 + t) * TP;
    if (G == 1) {
#pragma unroll
      for (int i = 0; i < PPT; ++i) {
        const long long gi = base + lt + LP * i;
        if (gi < a.N) a.assign[gi] = bk[i];
      }
    } else {  // groups 1.. hand their minima to group 0 (double-buffered by tile parity)
      const int par = int(((t - set) / kSets) & 1);  // kSets is a compile-time constant
      float* ss = xs_s + (set * 2 + par) * 3 * TP;
      int* sk = xs_k + (set * 2 + par) * 3 * TP;
      if (g > 0) {
#pragma unroll
        for (int i = 0; i < PPT; ++i) ss[(g - 1) * TP + lt + LP * i] = bs[i], sk[(g - 1) * TP + lt + LP * i] = bk[i];
      }
      asm volatile("bar.sync %0, %1;" ::"r"(1 + set), "n"(kConsumers) : "memory");  // this set only
      if (g == 0) {
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
          float s = bs[i];
          int k = bk[i];
#pragma unroll
          for (int h = 1; h < G; ++h) {
            const float s2 = ss[(h - 1) * TP + lt + LP * i];
            const int k2 = sk[(h - 1) * TP + lt + LP * i];
            if (s2 < s || (s2 == s && k2 < k)) s = s2, k = k2;
          }
          const long long gi = base + lt + LP * i;
          if (gi < a.N) a.assign[gi] = k;
        }
      }
    }
    // release the slot: the last of the 8 warps to finish with it refills it with tile t+kStages
    // (nobody waits on an "empty" barrier). Every x value the warp read is already consumed, the
    // fences order those reads and the counter before the TMA (async proxy) overwrites the slot.
    __syncwarp();
    if (lane == 0) {
      __threadfence_block();
      if (atomicAdd(released + slot, 1u) == kConsumerWarps - 1) {
        __threadfence_block();
        released[slot] = 0;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        if (t + kStages < n_tiles) issue(t + kStages, slot);
      }
    }
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
__global__ void __maxnreg__(NPP_KM_MAXNREG_D64) npp_kmeans_tma_kernel_d64(const __grid_constant__ CUtensorMap map,
                                                                         KmeansArgs a) {
  kmeans_body<4, 8>(&map, a);  // D <= 64: 256-point tiles
}
__global__ void __maxnreg__(NPP_KM_MAXNREG_D128) npp_kmeans_tma_kernel_d128(
    const __grid_constant__ CUtensorMap map, KmeansArgs a) {
  kmeans_body<2, 8>(&map, a);  // 64 < D <= 128: 128-point tiles
}

namespace {

// The constant bank is one per device and module: KMEANS_ASSIGN launches on different streams are
// ordered by an event so one launch's centroids are never overwritten while another still runs.
// (Inside a stream capture the ordering is the graph's: captured KMEANS_ASSIGN work must not run
// concurrently with other KMEANS_ASSIGN work.)
std::mutex g_km_mutex;
cudaEvent_t g_km_done[64] = {};

cudaError_t launch_tp(void (*kern)(const CUtensorMap, KmeansArgs), const CUtensorMap& map, const KmeansArgs& a,
                      int grid, size_t smem, cudaStream_t st) {
  cudaError_t e = ensure_smem(kern, int(smem));
  if (e != cudaSuccess) return e;
  kern<<<grid, kThreads, smem, st>>>(map, a);
  return cudaGetLastError();
}

}  // namespace

cudaError_t launch_kmeans(const KmeansArgs& a, const float* x, int grid, cudaStream_t st) {
  // tile: 256 points when D <= 64 (4 points x 64 lanes), else 128 (2 points x 64 lanes); both
  // with 4 centroid groups of 8 (S8)
  const bool small = a.D <= 64;
  const int tp = small ? 256 : 128;
  const size_t smem = km_smem_bytes(a.K, tp);
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
  e = launch_tp(small ? npp_kmeans_tma_kernel_d64 : npp_kmeans_tma_kernel_d128, map, a, grid, smem, st);
  if (e != cudaSuccess) return e;
  if (cap == cudaStreamCaptureStatusNone) e = cudaEventRecord(g_km_done[dev], st);
  return e;
}

}  // namespace npp
