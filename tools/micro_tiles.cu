// micro_tiles.cu — TMA staging of strided [rows x column-segment] tiles (the sumCols access pattern).
// Measurement tool only.  Each block owns a column tile and a contiguous row range; a stage is a
// 32 KB tile loaded either as per-row 1D bulk copies or as one 2D tensor-map TMA box.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_tiles tools/micro_tiles.cu
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
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(sa(dst)),
               "l"(src), "r"(bytes), "r"(sa(bar))
               : "memory");
}
__device__ __forceinline__ void tma2d(void* dst, const CUtensorMap* map, int x, int y, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          sa(dst)),
      "l"(map), "r"(x), "r"(y), "r"(sa(bar))
      : "memory");
}

// MODE 0: per-row 1D bulk copies of SEGB bytes; MODE 1: 2D TMA box [SEGB/4 cols x ROWS rows]
template <int MODE, int SEGB, int ROWS, int S>
__global__ void __launch_bounds__(288) tiles(const float* __restrict__ a, int R, int C, int tiles_c, int rows_per_block,
                                             const __grid_constant__ CUtensorMap map, double* out) {
  constexpr int STAGE = SEGB * ROWS;
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + S;
  unsigned char* buf = smem + 1024;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ct = blockIdx.x % tiles_c;
  const int rb = blockIdx.x / tiles_c;
  const int r0 = rb * rows_per_block;
  const int r1 = min(R, r0 + rows_per_block);
  const int nst = (r1 - r0 + ROWS - 1) / ROWS;
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
      int s = 0;
      unsigned ph = 0;
      for (int st = 0; st < nst; ++st) {
        if (st >= S) mbar_wait(empty + s, ph ^ 1);
        const int rr = r0 + st * ROWS;
        const int nr = min(ROWS, r1 - rr);
        if (MODE == 0) {
          mbar_expect_tx(full + s, nr * SEGB);
          for (int i = 0; i < nr; ++i)
            bulk_g2s(buf + s * STAGE + i * SEGB, a + size_t(rr + i) * C + size_t(ct) * (SEGB / 4), SEGB, full + s);
        } else {
          mbar_expect_tx(full + s, STAGE);
          tma2d(buf + s * STAGE, &map, ct * (SEGB / 4), rr, full + s);
        }
        if (++s == S) {
          s = 0;
          ph ^= 1;
        }
      }
    }
  } else {
    int s = 0;
    unsigned ph = 0;
    for (int st = 0; st < nst; ++st) {
      mbar_wait(full + s, ph);
      const float4* f = reinterpret_cast<const float4*>(buf + s * STAGE);
      float t = 0;
#pragma unroll
      for (int i = threadIdx.x; i < STAGE / 16; i += 256) {
        float4 r = f[i];
        t += (r.x + r.y) + (r.z + r.w);
      }
      acc += t;
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + s);
      if (++s == S) {
        s = 0;
        ph ^= 1;
      }
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
  int shapes[3][2] = {{65536, 1024}, {8192, 8192}, {1024, 65536}};
  auto make_map = [&](float* p, int R, int C, int boxc, int boxr) {
    CUtensorMap m;
    cuuint64_t dims[2] = {(cuuint64_t)C, (cuuint64_t)R};
    cuuint64_t strides[1] = {(cuuint64_t)C * 4};
    cuuint32_t box[2] = {(cuuint32_t)boxc, (cuuint32_t)boxr};
    cuuint32_t es[2] = {1, 1};
    CUresult r = encode(&m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, p, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
      std::printf("encode failed %d\n", (int)r);
      std::exit(1);
    }
    return m;
  };
  auto run = [&](const char* name, int R, int C, int segb, int rows, int rows_per_block, auto kern) {
    const int tiles_c = C * 4 / segb;
    const int nrb = (R + rows_per_block - 1) / rows_per_block;
    const int grid = tiles_c * nrb;
    const size_t smem = 1024 + size_t(segb * rows > 16384 ? 4 : 8) * segb * rows;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    std::vector<CUtensorMap> maps;
    for (auto b : bufs) maps.push_back(make_map(b, R, C, segb / 4 > 256 ? 256 : segb / 4, rows > 256 ? 256 : rows));
    for (int w = 0; w < 3; ++w) kern<<<grid, 288, smem>>>(bufs[w], R, C, tiles_c, rows_per_block, maps[w], out);
    CK(cudaDeviceSynchronize());
    const int iters = 30;
    CK(cudaEventRecord(e0));
    for (int it = 0; it < iters; ++it)
      kern<<<grid, 288, smem>>>(bufs[it % NBUF], R, C, tiles_c, rows_per_block, maps[it % NBUF], out);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    CK(cudaGetLastError());
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double us = ms * 1e3 / iters;
    std::printf("%-28s [%6d,%6d] grid=%4d  %8.2f us  %8.1f GB/s\n", name, R, C, grid, us, bytes / (us * 1e-6) / 1e9);
  };
  for (auto& sh : shapes) {
    const int R = sh[0], C = sh[1];
    // 1 KB segments x 32 rows: tiles_c = C/256
    {
      const int tc = C / 256;
      int per = 148 / tc;
      if (per < 1) per = 1;
      int rpb = ((R + per - 1) / per + 31) / 32 * 32;
      run("bulk1D 1KBx32", R, C, 1024, 32, rpb, tiles<0, 1024, 32, 4>);
      run("tma2D  1KBx32", R, C, 1024, 32, rpb, tiles<1, 1024, 32, 4>);
    }
    {
      const int tc = C / 1024;
      int per = 148 / tc;
      if (per < 1) per = 1;
      int rpb = ((R + per - 1) / per + 7) / 8 * 8;
      run("bulk1D 4KBx8", R, C, 4096, 8, rpb, tiles<0, 4096, 8, 4>);
    }
    {
      const int tc = C / 256;
      int per = 148 / tc;
      if (per < 1) per = 1;
      int rpb = ((R + per - 1) / per + 15) / 16 * 16;
      run("tma2D  1KBx16 S4", R, C, 1024, 16, rpb, tiles<1, 1024, 16, 4>);
      run("tma2D  1KBx16 S8", R, C, 1024, 16, rpb, tiles<1, 1024, 16, 8>);
    }
    {
      const int tc = C / 512;
      int per = 148 / tc;
      if (per < 1) per = 1;
      int rpb = ((R + per - 1) / per + 15) / 16 * 16;
      run("bulk1D 2KBx16", R, C, 2048, 16, rpb, tiles<0, 2048, 16, 4>);
    }
    {
      const int tc = C / 128;
      int per = 148 / tc;
      if (per < 1) per = 1;
      int rpb = ((R + per - 1) / per + 63) / 64 * 64;
      run("tma2D  512Bx64", R, C, 512, 64, rpb, tiles<1, 512, 64, 4>);
    }
  }
  return 0;
}
