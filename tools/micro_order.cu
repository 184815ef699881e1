// micro_order.cu — does the order in which one block walks its 2-D TMA tiles matter on B200?
// [R x C] fp32, tiles of 32 rows x 256 cols (1 KB wide). Each block owns a rectangle of tiles.
//   ORDER 0: column-strip order (a block walks down one 1 KB strip)          — micro_tiles' fast case
//   ORDER 1: band-major order (all column tiles of a 32-row band, then next) — the RX consumer order
//   ORDER 2: band-major, but each block's bands are interleaved with stride = #blocks (cyclic)
// Measurement tool only.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define CK(x)                                                                      \
  do {                                                                             \
    cudaError_t e = (x);                                                           \
    if (e != cudaSuccess) {                                                        \
      std::printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
      std::exit(1);                                                                \
    }                                                                              \
  } while (0)

__device__ __forceinline__ unsigned sa(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(sa(b)), "r"(c));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(b)), "r"(bytes));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(sa(b)));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned ph) {
  asm volatile("{\n .reg .pred p;\n W_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra W_%=;\n}" ::"r"(
                   sa(b)),
               "r"(ph));
}
__device__ __forceinline__ void tma2d(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          sa(dst)),
      "l"(map), "r"(x), "r"(y), "r"(sa(bar))
      : "memory");
}

constexpr int S = 4, TB = 32768;

// block owns bands [b0, b0+nb) (ORDER 0/1) or bands b, b+G, ... (ORDER 2) and column tiles [c0, c0+nc)
template <int ORDER>
__global__ void __launch_bounds__(288, 1) walk(const __grid_constant__ CUtensorMap map, int bands_per_block,
                                               int ctiles_per_block, int nbands, int nct, double* out) {
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + S;
  unsigned char* buf = smem + 1024;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int cgroups = nct / ctiles_per_block;
  const int cg = blockIdx.x % cgroups, bg = blockIdx.x / cgroups;
  const int ntiles = bands_per_block * ctiles_per_block;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, 8);
    }
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  double acc = 0;
  if (warp == 8) {
    if (lane == 0) {
      for (int t = 0; t < ntiles; ++t) {
        const int s = t % S;
        if (t >= S) mbar_wait(empty + s, ((t / S) & 1) ^ 1);
        int band, ct;
        if (ORDER == 0) {
          ct = t / bands_per_block;
          band = t % bands_per_block;
        } else {
          band = t / ctiles_per_block;
          ct = t % ctiles_per_block;
        }
        const int gb = ORDER == 2 ? bg + band * (gridDim.x / cgroups) : bg * bands_per_block + band;
        mbar_expect_tx(full + s, TB);
        tma2d(buf + s * TB, &map, (cg * ctiles_per_block + ct) * 256, (gb % nbands) * 32, full + s);
      }
    }
  } else {
    for (int t = 0; t < ntiles; ++t) {
      const int s = t % S;
      mbar_wait(full + s, (t / S) & 1);
      const float4* f = reinterpret_cast<const float4*>(buf + s * TB);
      float x = 0;
#pragma unroll
      for (int i = threadIdx.x; i < TB / 16; i += 256) {
        float4 r = f[i];
        x += (r.x + r.y) + (r.z + r.w);
      }
      acc += x;
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + s);
    }
  }
  if (acc == 12345.678) out[0] = acc;
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                             const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                             CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  EncodeFn encode = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&encode, cudaEnableDefault, &q));
  const size_t bytes = size_t(256) << 20;
  const int NBUF = 6;
  std::vector<float*> bufs(NBUF);
  for (auto& b : bufs) {
    CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(b, 0, bytes));
  }
  double* out;
  CK(cudaMalloc(&out, 64));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const size_t smem = 1024 + size_t(S) * TB;
  CK(cudaFuncSetAttribute(walk<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  CK(cudaFuncSetAttribute(walk<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  CK(cudaFuncSetAttribute(walk<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  struct Cfg {
    int R, C, bpb, cpb;
  } cfgs[] = {{65536, 1024, 14, 4}, {65536, 1024, 56, 1}, {8192, 8192, 7, 8}, {8192, 8192, 56, 1},
              {8192, 8192, 2, 28}, {1024, 65536, 8, 7}, {1024, 65536, 1, 56}};
  for (auto& c : cfgs) {
    std::vector<CUtensorMap> maps(NBUF);
    for (int i = 0; i < NBUF; ++i) {
      cuuint64_t dims[2] = {(cuuint64_t)c.C, (cuuint64_t)c.R};
      cuuint64_t strides[1] = {(cuuint64_t)c.C * 4};
      cuuint32_t box[2] = {256, 32};
      cuuint32_t es[2] = {1, 1};
      if (encode(&maps[i], CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, bufs[i], dims, strides, box, es,
                 CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                 CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
        std::printf("encode failed\n");
        return 1;
      }
    }
    const int nbands = c.R / 32, nct = c.C / 256;
    const int grid = (nct / c.cpb) * ((nbands + c.bpb - 1) / c.bpb);
    for (int order = 0; order < 3; ++order) {
      auto k = order == 0 ? walk<0> : (order == 1 ? walk<1> : walk<2>);
      for (int w = 0; w < 3; ++w) k<<<grid, 288, smem>>>(maps[w], c.bpb, c.cpb, nbands, nct, out);
      CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(e0));
      for (int it = 0; it < 30; ++it) k<<<grid, 288, smem>>>(maps[it % NBUF], c.bpb, c.cpb, nbands, nct, out);
      CK(cudaEventRecord(e1));
      CK(cudaEventSynchronize(e1));
      CK(cudaGetLastError());
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      const double us = ms * 1e3 / 30;
      std::printf("[%6d,%6d] bands/blk=%3d ctiles/blk=%3d grid=%4d order=%d  %7.2f us %7.1f GB/s\n", c.R, c.C, c.bpb,
                  c.cpb, grid, order, us, bytes / (us * 1e-6) / 1e9);
    }
  }
  return 0;
}
