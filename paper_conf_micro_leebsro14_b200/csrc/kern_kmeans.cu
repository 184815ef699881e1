// kern_kmeans.cu — class KM: the three-level k-means assignment nest (BASELINE.json config 4):
//     points mapRows { x_i => (0 until K) argmin { k => Σ_d (x_id − c_kd)² } }     ties -> lowest k
// L0 = points (Map), L1 = centroids (argmin Reduce), L2 = dims (Reduce). The mapping keeps L2 on x
// for coalescing, which the staged access satisfies (§V-B): 128-point tiles of x arrive
// by TMA with the 128-byte swizzle, so the per-point reads of a warp are bank-conflict free, and the
// centroids stay resident in shared memory for the whole launch (reused N/128 times per block).
//   thread t owns points p = t % 64 and p + 64 of a tile and centroid quarter q = t / 64 (warp-
//   uniform, so centroid reads are shared-memory broadcasts); it ranks its centroids by
//   s_k = ||c_k||² − 2 x·c_k (the x-independent expansion of the squared distance: same argmin),
//   keeping the first minimum in increasing k; the four quarters meet in shared memory in order.
// fp32 arithmetic on CUDA cores (the contraction is 64 x 32 per point: the path is FMA-bound, see
// DESIGN.md §6); blocks stream contiguous tile ranges [bP, bP+P); no workspace.
#include <cstdint>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

constexpr int kTilePts = 128;
constexpr int kBoxBytes = kTilePts * 128;  // one swizzled box: 128 points x 32 floats
constexpr int kRingBytes = 128 * 1024;
constexpr int kMaxStages = 4;
constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kThreads = kConsumers + 32;
constexpr int kSmemHeader = 1024;

__host__ __device__ inline int64_t km_kpad(int64_t K) { return (K + 31) / 32 * 32; }
__host__ __device__ inline int km_boxes(int64_t D) { return int((D + 31) / 32); }
__host__ __device__ inline int km_stages(int64_t D) {
  const int s = kRingBytes / (km_boxes(D) * kBoxBytes);
  return s > kMaxStages ? kMaxStages : s;
}
inline size_t km_smem_bytes(int64_t D, int64_t K) {
  return size_t(1024) /* alignment pad */ + size_t(kSmemHeader) + size_t(kRingBytes) +
         size_t(km_kpad(K)) * size_t(D) * 4 + size_t(km_kpad(K)) * 4 + size_t(4) * kTilePts * 8;
}

__device__ __forceinline__ float4 ld_point(const unsigned char* tile, int p, int d4) {
  // 128-byte swizzle: 16-byte chunk j of row p lives at chunk j ^ (p & 7)
  const int box = d4 >> 3, j = d4 & 7;
  return *reinterpret_cast<const float4*>(tile + box * kBoxBytes + p * 128 + ((j ^ (p & 7)) << 4));
}

}  // namespace

__global__ void __launch_bounds__(kThreads, 1) npp_kmeans_tma_kernel(const __grid_constant__ CUtensorMap map,
                                                                     KmeansArgs a) {
  extern __shared__ __align__(1024) unsigned char smem[];
  const int S = km_stages(a.D);
  const int nb = km_boxes(a.D);
  const int stage_bytes = nb * kBoxBytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kMaxStages;
  // the 128-byte swizzle is a function of smem address bits [7:9]: boxes must be 1 KB aligned
  const unsigned pad = (1024u - (tma::smem_u32(smem) & 1023u)) & 1023u;
  unsigned char* ring = smem + pad + kSmemHeader;
  const int64_t D = a.D, K = a.K, Kp = km_kpad(K);
  float* cs = reinterpret_cast<float*>(ring + kRingBytes);  // [Kp][D]
  float* cn = cs + Kp * D;                                                 // [Kp]
  float* sb_s = cn + Kp;                                                   // [4][128]
  int* sb_k = reinterpret_cast<int*>(sb_s + 4 * kTilePts);                 // [4][128]

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x;
  const long long T = (a.N + kTilePts - 1) / kTilePts;
  const long long P = a.per_block;
  const long long r0 = bid * P, r1 = (T < r0 + P) ? T : r0 + P;

  if (threadIdx.x == 0) {
    for (int i = 0; i < kMaxStages; ++i) {
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
        const int slot = int(t % S);
        if (t >= S) tma::mbar_wait(empty + slot, unsigned((t / S) & 1) ^ 1u);
        tma::mbar_expect_tx(full + slot, unsigned(stage_bytes));
        for (int bx = 0; bx < nb; ++bx)
          tma::load_2d(ring + slot * stage_bytes + bx * kBoxBytes, &map, bx * 32, int(cur * kTilePts), full + slot);
      }
    }
    return;
  }

  // ------------------------------------------------------------------ consumers
  const int p0 = threadIdx.x & 63, p1 = p0 + 64;
  const int q = threadIdx.x >> 6;  // centroid quarter (warp-uniform)
  const int nd4 = int(D / 4);
  const long long n_tiles = r1 - r0;
  for (long long t = 0; t < n_tiles; ++t) {
    const int slot = int(t % S);
    tma::mbar_wait(full + slot, unsigned((t / S) & 1));
    const unsigned char* tile = ring + slot * stage_bytes;
    float bs0 = __int_as_float(0x7f800000), bs1 = bs0;
    int bk0 = 0x7fffffff, bk1 = 0x7fffffff;
    for (int64_t kc = 0; kc < Kp; kc += 32) {
      float acc0[8], acc1[8];
#pragma unroll
      for (int i = 0; i < 8; ++i) acc0[i] = acc1[i] = 0.f;
      const float* cq = cs + (kc + q * 8) * D;
#pragma unroll 2
      for (int d4 = 0; d4 < nd4; ++d4) {
        const float4 xa = ld_point(tile, p0, d4);
        const float4 xb = ld_point(tile, p1, d4);
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float4 cv = *reinterpret_cast<const float4*>(cq + i * D + d4 * 4);
          acc0[i] = fmaf(xa.x, cv.x, acc0[i]);
          acc0[i] = fmaf(xa.y, cv.y, acc0[i]);
          acc0[i] = fmaf(xa.z, cv.z, acc0[i]);
          acc0[i] = fmaf(xa.w, cv.w, acc0[i]);
          acc1[i] = fmaf(xb.x, cv.x, acc1[i]);
          acc1[i] = fmaf(xb.y, cv.y, acc1[i]);
          acc1[i] = fmaf(xb.z, cv.z, acc1[i]);
          acc1[i] = fmaf(xb.w, cv.w, acc1[i]);
        }
      }
#pragma unroll
      for (int i = 0; i < 8; ++i) {  // increasing k within the quarter: strict < keeps the first
        const int k = int(kc) + q * 8 + i;
        const float s0 = fmaf(-2.f, acc0[i], cn[k]);
        const float s1 = fmaf(-2.f, acc1[i], cn[k]);
        if (s0 < bs0) bs0 = s0, bk0 = k;
        if (s1 < bs1) bs1 = s1, bk1 = k;
      }
    }
    __syncwarp();
    if (lane == 0) tma::mbar_arrive(empty + slot);  // the tile is no longer read
    sb_s[q * kTilePts + p0] = bs0, sb_k[q * kTilePts + p0] = bk0;
    sb_s[q * kTilePts + p1] = bs1, sb_k[q * kTilePts + p1] = bk1;
    tma::bar_sync_consumers<kConsumers>();
    if (threadIdx.x < kTilePts) {
      const int p = threadIdx.x;
      float s = sb_s[p];
      int k = sb_k[p];
#pragma unroll
      for (int qq = 1; qq < 4; ++qq) {
        const float s2 = sb_s[qq * kTilePts + p];
        const int k2 = sb_k[qq * kTilePts + p];
        if (s2 < s || (s2 == s && k2 < k)) s = s2, k = k2;
      }
      const long long i = (r0 + t) * kTilePts + p;
      if (i < a.N) a.assign[i] = k;
    }
    tma::bar_sync_consumers<kConsumers>();
  }
}

cudaError_t launch_kmeans(const KmeansArgs& a, const float* x, int grid, cudaStream_t st) {
  const size_t smem = km_smem_bytes(a.D, a.K);
  cudaError_t e = cudaFuncSetAttribute(npp_kmeans_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem));
  if (e != cudaSuccess) return e;
  CUtensorMap map;
  e = tma::encode_2d(&map, x, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, a.N, a.D, 32u, unsigned(kTilePts),
                     CU_TENSOR_MAP_SWIZZLE_128B);
  if (e != cudaSuccess) return e;
  npp_kmeans_tma_kernel<<<grid, kThreads, smem, st>>>(map, a);
  return cudaGetLastError();
}

}  // namespace npp
