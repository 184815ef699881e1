// micro_gap.cu — where does the per-launch overhead of a 256 MiB streaming pass go when launches run
// back to back (no PDL)? Not part of the library: a measurement tool for the staged sum family.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/micro_gap tools/micro_gap.cu
// One persistent block per SM, a 4-deep ring of 32 KB chunks, static contiguous ranges, 8 consumer
// warps + 1 producer lane (the structure of kern_sum_tma.cu without pool, tags or combine). Modes:
//   bulk        1-D cp.async.bulk of 32 KB contiguous chunks
//   sK/bK RxC   3-D tensor TMA over an [R x C] f32 matrix viewed as {256, C/256, R}, box {256, K, 32/K}
//               (K KB wide x 32/K rows); s: strip-major tile order (a block walks down K-KB column
//               strips, the sumCols order), b: band-major (a block walks across the strips of a band)
// Each mode: 20 launches over 8 distinct 256 MiB buffers captured in a CUDA graph, median of 5 replays;
// per-block globaltimer stamps of launch 10 and 11 give launch gap, ramp (start -> first chunk) and tail.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "../paper_conf_micro_leebsro14_b200/csrc/tma_ring.cuh"

#define CK(x)                                                                      \
  do {                                                                             \
    cudaError_t e = (x);                                                           \
    if (e != cudaSuccess) {                                                        \
      std::printf("CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); \
      std::exit(1);                                                                \
    }                                                                              \
  } while (0)

using namespace npp;

constexpr int NW = 8;
constexpr int S = 4;
constexpr int CH = 32768;

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

struct Args {
  const char* a;
  long long nchunks;
  unsigned long long* times;  // [grid x 4]: start, first chunk, last chunk consumed, exit (or null)
  double* out;
  int mode;  // 0 bulk, 1 tensor
  int nc, rows, band_major;  // tensor: chunks per tile row, rows per tile, tile order
  long long tps, nstrips;    // tiles per strip, strips
};

__global__ void __launch_bounds__((NW + 1) * 32, 1) gap_kernel(const __grid_constant__ CUtensorMap map, Args A) {
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + S;
  unsigned char* buf = smem + 1024;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x, G = gridDim.x;
  const unsigned long long t0 = gtimer();
  const long long c0 = bid * A.nchunks / G, c1 = (bid + 1) * A.nchunks / G;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      tma::mbar_init(full + s, 1);
      tma::mbar_init(empty + s, NW);
    }
    tma::mbar_fence_init();
  }
  __syncthreads();
  double acc = 0;
  if (warp == NW) {
    if (lane == 0) {
      if (A.mode) tma::prefetch_map(&map);
      for (long long c = c0, t = 0; c < c1; ++c, ++t) {
        const int s = int(t % S);
        if (t >= S) tma::mbar_wait(empty + s, unsigned((t / S) & 1) ^ 1u);
        tma::mbar_expect_tx(full + s, CH);
        if (A.mode == 0) {
          asm volatile(
              "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                  tma::smem_u32(buf + s * CH)),
              "l"(A.a + c * CH), "r"(CH), "r"(tma::smem_u32(full + s))
              : "memory");
        } else {
          const long long st = A.band_major ? c % A.nstrips : c / A.tps;
          const long long bd = A.band_major ? c / A.nstrips : c % A.tps;
          tma::load_3d(buf + s * CH, &map, 0, int(st) * A.nc, int(bd) * A.rows, full + s);
        }
      }
    }
  } else {
    unsigned long long tf = 0;
    for (long long c = c0, t = 0; c < c1; ++c, ++t) {
      const int s = int(t % S);
      tma::mbar_wait(full + s, unsigned((t / S) & 1));
      if (t == 0) tf = gtimer();
      const float4* f = reinterpret_cast<const float4*>(buf + s * CH);
      float u = 0;
#pragma unroll 4
      for (int i = threadIdx.x; i < CH / 16; i += NW * 32) {
        float4 r = f[i];
        u += (r.x + r.y) + (r.z + r.w);
      }
      acc += u;
      __syncwarp();
      if (lane == 0) tma::mbar_arrive(empty + s);
    }
    if (A.times && threadIdx.x == 0) {
      A.times[bid * 4 + 1] = tf;
      A.times[bid * 4 + 2] = gtimer();
    }
  }
  if (acc == 12345.678) A.out[0] = acc;
  __syncthreads();
  if (A.times && threadIdx.x == 0) {
    A.times[bid * 4 + 0] = t0;
    A.times[bid * 4 + 3] = gtimer();
  }
}

int main(int argc, char** argv) {
  const int only = argc > 1 ? std::atoi(argv[1]) : -1;  // one config (index) only, stamps off
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const size_t bytes = size_t(256) << 20;
  const int NBUF = 8, NL = 20;
  std::vector<char*> bufs(NBUF);
  for (auto& b : bufs) {
    CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(b, 1, bytes));
  }
  double* out;
  CK(cudaMalloc(&out, 64));
  unsigned long long* times;
  CK(cudaMalloc(&times, size_t(NL) * sms * 32));
  const int smem = 1024 + S * CH;
  CK(cudaFuncSetAttribute(gap_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  struct Cfg {
    const char* name;
    int mode, R, C, nc, band_major;
  };
  const Cfg cfgs[] = {{"bulk          ", 0, 0, 0, 0, 0},      {"s1 [8K,8K]    ", 1, 8192, 8192, 1, 0},
                      {"s2 [8K,8K]    ", 1, 8192, 8192, 2, 0}, {"s4 [8K,8K]    ", 1, 8192, 8192, 4, 0},
                      {"b1 [8K,8K]    ", 1, 8192, 8192, 1, 1}, {"s4 [64K,1K]   ", 1, 65536, 1024, 4, 0},
                      {"s1 [64K,1K]   ", 1, 65536, 1024, 1, 0}, {"s1 [1K,64K]   ", 1, 1024, 65536, 1, 0}};
  for (int ci = 0; ci < int(sizeof(cfgs) / sizeof(cfgs[0])); ++ci) {
    const Cfg& cf = cfgs[ci];
    if (only >= 0 && ci != only) continue;
    const int rows = cf.nc ? 32 / cf.nc : 0;
    const long long nstrips = cf.nc ? cf.C / 256 / cf.nc : 0, tps = cf.nc ? cf.R / rows : 0;
    for (int stamp = 0; stamp < (only >= 0 ? 1 : 2); ++stamp) {
      std::vector<CUtensorMap> maps(NBUF);
      for (int i = 0; i < NBUF; ++i) {
        std::memset(&maps[i], 0, sizeof(CUtensorMap));
        if (cf.mode) {
          const cuuint64_t dims[3] = {256, cuuint64_t(cf.C / 256), cuuint64_t(cf.R)};
          const cuuint64_t strides[2] = {1024, cuuint64_t(cf.C) * 4};
          const cuuint32_t box[3] = {256, cuuint32_t(cf.nc), cuuint32_t(rows)};
          const cuuint32_t estr[3] = {1, 1, 1};
          if (tma::encoder()(&maps[i], CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 3, bufs[i], dims, strides, box, estr,
                             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS) {
            std::printf("encode 3d failed\n");
            return 1;
          }
        }
      }
      cudaGraph_t g;
      cudaGraphExec_t ge;
      CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal));
      for (int i = 0; i < NL; ++i) {
        Args A{bufs[i % NBUF], (long long)(bytes / CH), stamp ? times + size_t(i) * sms * 4 : nullptr, out, cf.mode,
               cf.nc, rows, cf.band_major, tps, nstrips};
        gap_kernel<<<sms, (NW + 1) * 32, smem, st>>>(maps[i % NBUF], A);
      }
      CK(cudaStreamEndCapture(st, &g));
      CK(cudaGraphInstantiate(&ge, g, 0));
      for (int w = 0; w < 3; ++w) CK(cudaGraphLaunch(ge, st));
      CK(cudaStreamSynchronize(st));
      std::vector<float> ts;
      for (int r = 0; r < 5; ++r) {
        CK(cudaEventRecord(e0, st));
        CK(cudaGraphLaunch(ge, st));
        CK(cudaEventRecord(e1, st));
        CK(cudaEventSynchronize(e1));
        float ms;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        ts.push_back(ms * 1e3f / NL);
      }
      std::sort(ts.begin(), ts.end());
      const float us = ts[2];
      std::printf("%s stamps=%d  graph b2b %8.2f us  %7.1f GB/s\n", cf.name, stamp, us, bytes / (us * 1e-6) / 1e9);
      if (stamp) {
        std::vector<unsigned long long> h(size_t(NL) * sms * 4);
        CK(cudaMemcpy(h.data(), times, h.size() * 8, cudaMemcpyDeviceToHost));
        for (int L = 9; L < 12; ++L) {
          const unsigned long long* p = h.data() + size_t(L) * sms * 4;
          const unsigned long long* q = h.data() + size_t(L - 1) * sms * 4;
          unsigned long long s0 = ~0ull, s1 = 0, f0 = ~0ull, f1 = 0, x1 = 0, prev_end = 0;
          std::vector<double> ends;
          for (int b = 0; b < sms; ++b) {
            s0 = std::min(s0, p[b * 4]);
            s1 = std::max(s1, p[b * 4]);
            f0 = std::min(f0, p[b * 4 + 1]);
            f1 = std::max(f1, p[b * 4 + 1]);
            x1 = std::max(x1, p[b * 4 + 3]);
            ends.push_back(double(p[b * 4 + 2]));
            prev_end = std::max(prev_end, q[b * 4 + 3]);
          }
          std::sort(ends.begin(), ends.end());
          std::printf("   launch %2d: gap from prev last exit %.2f | start spread %.2f | first chunk %.2f..%.2f | "
                      "stream end p10 %.2f p50 %.2f max %.2f | last exit %.2f  (us after first start)\n",
                      L, (double(s0) - double(prev_end)) / 1e3, (s1 - s0) / 1e3, (f0 - s0) / 1e3, (f1 - s0) / 1e3,
                      (ends[sms / 10] - s0) / 1e3, (ends[sms / 2] - s0) / 1e3, (ends.back() - s0) / 1e3,
                      (x1 - s0) / 1e3);
        }
      }
      CK(cudaGraphExecDestroy(ge));
      CK(cudaGraphDestroy(g));
    }
  }
  return 0;
}
