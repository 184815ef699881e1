// kern_kmeans.cu — class KM: the three-level k-means assignment nest (BASELINE.json config 4):
//     points mapRows { x_i => (0 until K) argmin { k => Σ_d (x_id − c_kd)² } }     ties -> lowest k
// L0 = points (Map), L1 = centroids (argmin Reduce), L2 = dims (Reduce). The mapping keeps L2 on x
// for coalescing, which the staged access satisfies (§V-B): TP-point tiles of x arrive
// by TMA with the 128-byte swizzle, so the per-point reads of a warp are bank-conflict free, and the
// centroids stay resident in shared memory for the whole launch (reused N/TP times per block).
//   thread t owns points pq + 64i (i < PPT = TP/64) of a tile and centroid quarter q = t / 64 (warp-
//   uniform, so centroid reads are shared-memory broadcasts); it ranks its centroids by
//   s_k = ||c_k||² − 2 x·c_k (the x-independent expansion of the squared distance: same argmin),
//   keeping the first minimum in increasing k; the four quarters meet in shared memory in order.
//   x·c runs on the packed FP32 pipe (Blackwell FFMA2, fma.rn.f32x2): even and odd dims accumulate
//   in the two halves of a float2, which halves the FMA instruction count.
// The path is FP32-FMA-bound: 2·N·K·D flops against 1 KB of x per 4 points.
#include <cstdint>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

constexpr int kStages = 2;
constexpr int kBoxCols = 32;  // 128 B of floats: the 128-B swizzle span
constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kThreads = kConsumers + 32;
constexpr int kSmemHeader = 1024;
constexpr int kMaxStageBytes = 64 * 1024;

__host__ __device__ inline int64_t km_kpad(int64_t K) { return (K + 31) / 32 * 32; }
__host__ __device__ inline int km_boxes(int64_t D) { return int((D + kBoxCols - 1) / kBoxCols); }
inline size_t km_smem_bytes(int64_t D, int64_t K, int tp) {
  return size_t(1024) /* alignment pad */ + size_t(kSmemHeader) + size_t(kStages) * kMaxStageBytes +
         size_t(km_kpad(K)) * size_t(D) * 4 + size_t(km_kpad(K)) * 4 + size_t(4) * tp * 8;
}

// x·c with even/odd dims in the two halves of an f32x2 accumulator
__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

template <int TP>
__device__ __forceinline__ float4 ld_point(const unsigned char* tile, int p, int d4) {
  // 128-byte swizzle: 16-byte chunk j of row p lives at chunk j ^ (p & 7)
  const int box = d4 >> 3, j = d4 & 7;
  return *reinterpret_cast<const float4*>(tile + box * (TP * 128) + p * 128 + ((j ^ (p & 7)) << 4));
}

}  // namespace

template <int PPT>
__global__ void __launch_bounds__(kThreads, 1) npp_kmeans_tma_kernel(const __grid_constant__ CUtensorMap map,
                                                                     KmeansArgs a) {
  constexpr int TP = 64 * PPT;  // points per tile
  extern __shared__ __align__(1024) unsigned char smem[];
  const int nb = km_boxes(a.D);
  const int stage_bytes = nb * TP * 128;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kStages;
  // the 128-byte swizzle is a function of smem address bits [7:9]: boxes must be 1 KB aligned
  const unsigned pad = (1024u - (tma::smem_u32(smem) & 1023u)) & 1023u;
  unsigned char* ring = smem + pad + kSmemHeader;
  const int64_t D = a.D, K = a.K, Kp = km_kpad(K);
  float* cs = reinterpret_cast<float*>(ring + kStages * kMaxStageBytes);  // [Kp][D]
  float* cn = cs + Kp * D;                                                // [Kp]
  float* sb_s = cn + Kp;                                                  // [4][TP]
  int* sb_k = reinterpret_cast<int*>(sb_s + 4 * TP);                      // [4][TP]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x;
  const long long T = (a.N + TP - 1) / TP;
  const long long P = a.per_block;
  const long long r0 = bid * P, r1 = (T < r0 + P) ? T : r0 + P;

  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      tma::mbar_init(full + i, 1);
      tma::mbar_init(empty + i, kConsumerWarps);
    }
    tma::mbar_fence_init();
  }
  // centroids -> shared memory (padded rows are zero, padded norms +inf: never selected)
  for (int64_t i = threadIdx.x; i < Kp * D; i += kThreads) cs[i] = i < K * D ? __ldg(a.c + i) : 0.f;
  __syncthreads();
  for (int64_t k = threadIdx.x; k < Kp; k += kThreads) {
    float s = 0.f;
    for (int64_t d = 0; d < D; ++d) s = fmaf(cs[k * D + d], cs[k * D + d], s);
    cn[k] = k < K ? s : __int_as_float(0x7f800000);
  }
  __syncthreads();

  if (warp == kConsumerWarps) {
    if (lane == 0) {  // ---------------------------------------------- producer
      tma::prefetch_map(&map);
      long long t = 0;
      for (long long cur = r0; cur < r1; ++cur, ++t) {
        const int slot = int(t % kStages);
        if (t >= kStages) tma::mbar_wait(empty + slot, unsigned((t / kStages) & 1) ^ 1u);
        tma::mbar_expect_tx(full + slot, unsigned(stage_bytes));
        for (int bx = 0; bx < nb; ++bx)
          tma::load_2d(ring + slot * kMaxStageBytes + bx * (TP * 128), &map, bx * kBoxCols, int(cur * TP),
                       full + slot);
      }
    }
    return;
  }

  // ------------------------------------------------------------------ consumers
  const int pq = threadIdx.x & 63;
  const int q = threadIdx.x >> 6;  // centroid quarter (warp-uniform)
  const int nd4 = int(D / 4);
  const long long n_tiles = r1 - r0;
  for (long long t = 0; t < n_tiles; ++t) {
    const int slot = int(t % kStages);
    tma::mbar_wait(full + slot, unsigned((t / kStages) & 1));
    const unsigned char* tile = ring + slot * kMaxStageBytes;
    float bs[PPT];
    int bk[PPT];
#pragma unroll
    for (int i = 0; i < PPT; ++i) bs[i] = __int_as_float(0x7f800000), bk[i] = 0x7fffffff;
    for (int64_t kc = 0; kc < Kp; kc += 32) {
      float2 acc[PPT][8];
#pragma unroll
      for (int i = 0; i < PPT; ++i)
#pragma unroll
        for (int c = 0; c < 8; ++c) acc[i][c] = make_float2(0.f, 0.f);
      const float* cq = cs + (kc + q * 8) * D;
#pragma unroll 2
      for (int d4 = 0; d4 < nd4; ++d4) {
        float4 xv[PPT];
#pragma unroll
        for (int i = 0; i < PPT; ++i) xv[i] = ld_point<TP>(tile, pq + 64 * i, d4);
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const float4 cv = *reinterpret_cast<const float4*>(cq + c * D + d4 * 4);
#pragma unroll
          for (int i = 0; i < PPT; ++i) {
            ffma2(acc[i][c], make_float2(xv[i].x, xv[i].y), make_float2(cv.x, cv.y));
            ffma2(acc[i][c], make_float2(xv[i].z, xv[i].w), make_float2(cv.z, cv.w));
          }
        }
      }
#pragma unroll
      for (int c = 0; c < 8; ++c) {  // increasing k within the quarter: strict < keeps the first
        const int k = int(kc) + q * 8 + c;
#pragma unroll
        for (int i = 0; i < PPT; ++i) {
          const float s = fmaf(-2.f, acc[i][c].x + acc[i][c].y, cn[k]);
          if (s < bs[i]) bs[i] = s, bk[i] = k;
        }
      }
    }
    __syncwarp();
    if (lane == 0) tma::mbar_arrive(empty + slot);  // the tile is no longer read
#pragma unroll
    for (int i = 0; i < PPT; ++i) {
      sb_s[q * TP + pq + 64 * i] = bs[i];
      sb_k[q * TP + pq + 64 * i] = bk[i];
    }
    tma::bar_sync_consumers<kConsumers>();
    for (int p = threadIdx.x; p < TP; p += kConsumers) {
      float s = sb_s[p];
      int k = sb_k[p];
#pragma unroll
      for (int qq = 1; qq < 4; ++qq) {
        const float s2 = sb_s[qq * TP + p];
        const int k2 = sb_k[qq * TP + p];
        if (s2 < s || (s2 == s && k2 < k)) s = s2, k = k2;
      }
      const long long i = (r0 + t) * TP + p;
      if (i < a.N) a.assign[i] = k;
    }
    tma::bar_sync_consumers<kConsumers>();
  }
}

cudaError_t launch_kmeans(const KmeansArgs& a, const float* x, int grid, cudaStream_t st) {
  const int tp = a.D <= 64 ? 256 : 128;  // DESIGN.md S8 (KMEANS_ASSIGN)
  const size_t smem = km_smem_bytes(a.D, a.K, tp);
  CUtensorMap map;
  cudaError_t e = tma::encode_2d(&map, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.N, a.D, unsigned(kBoxCols),
                                 unsigned(tp), CU_TENSOR_MAP_SWIZZLE_128B);
  if (e != cudaSuccess) return e;
  if (tp == 256) {
    e = cudaFuncSetAttribute(npp_kmeans_tma_kernel<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
    npp_kmeans_tma_kernel<4><<<grid, kThreads, smem, st>>>(map, a);
  } else {
    e = cudaFuncSetAttribute(npp_kmeans_tma_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
    if (e != cudaSuccess) return e;
    npp_kmeans_tma_kernel<2><<<grid, kThreads, smem, st>>>(map, a);
  }
  return cudaGetLastError();
}

}  // namespace npp
