// micro_stream.cu — read-bandwidth ceiling experiments on B200 for 256 MiB streaming reductions.
// Not part of the library: a measurement tool to pick the kernel structure for the RX/MX families.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_stream tools/micro_stream.cu
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

__device__ __forceinline__ float4 ldg_nc(const float4* p) {
  float4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w) : "l"(p));
  return r;
}

// B: flat grid-stride / contiguous-per-block LDG streaming; U float4 loads in flight per thread.
template <int U, bool CONTIG>
__global__ void flat_ldg(const float4* __restrict__ a, size_t n4, double* out) {
  double acc = 0;
  const size_t nthreads = size_t(gridDim.x) * blockDim.x;
  if (CONTIG) {
    const size_t per_block = (n4 + gridDim.x - 1) / gridDim.x;
    const size_t b0 = blockIdx.x * per_block;
    const size_t b1 = min(n4, b0 + per_block);
    size_t i = b0 + threadIdx.x;
    for (; i + (U - 1) * blockDim.x < b1; i += U * blockDim.x) {
      float4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) r[u] = ldg_nc(a + i + u * blockDim.x);
      float s = 0;
#pragma unroll
      for (int u = 0; u < U; ++u) s += (r[u].x + r[u].y) + (r[u].z + r[u].w);
      acc += s;
    }
    for (; i < b1; i += blockDim.x) {
      float4 r = ldg_nc(a + i);
      acc += (r.x + r.y) + (r.z + r.w);
    }
  } else {
    size_t i = size_t(blockIdx.x) * blockDim.x + threadIdx.x;
    for (; i + (U - 1) * nthreads < n4; i += U * nthreads) {
      float4 r[U];
#pragma unroll
      for (int u = 0; u < U; ++u) r[u] = ldg_nc(a + i + u * nthreads);
      float s = 0;
#pragma unroll
      for (int u = 0; u < U; ++u) s += (r[u].x + r[u].y) + (r[u].z + r[u].w);
      acc += s;
    }
    for (; i < n4; i += nthreads) {
      float4 r = ldg_nc(a + i);
      acc += (r.x + r.y) + (r.z + r.w);
    }
  }
  if (acc == 12345.678) out[0] = acc;  // keep the loads alive
}

// C: TMA bulk copies (cp.async.bulk) into an S-stage smem ring; one producer warp, NW consumer warps.
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((unsigned)__cvta_generic_to_shared(b)),
               "r"(bytes));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"((unsigned)__cvta_generic_to_shared(b)));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}" ::"r"((unsigned)__cvta_generic_to_shared(b)),
      "r"(parity));
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          (unsigned)__cvta_generic_to_shared(dst)),
      "l"(src), "r"(bytes), "r"((unsigned)__cvta_generic_to_shared(bar))
      : "memory");
}

template <int NW, int S, int CH>
__global__ void __launch_bounds__((NW + 1) * 32) tma_stream(const char* __restrict__ a, size_t nbytes, double* out) {
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + S;
  unsigned char* buf = smem + 128;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const size_t nchunks = nbytes / CH;
  const size_t per_block = (nchunks + gridDim.x - 1) / gridDim.x;
  const size_t c0 = blockIdx.x * per_block;
  const size_t c1 = min(nchunks, c0 + per_block);
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, NW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  double acc = 0;
  if (warp == NW) {  // producer
    if (lane == 0) {
      int s = 0;
      unsigned ph = 0;
      for (size_t c = c0; c < c1; ++c) {
        if (c - c0 >= S) mbar_wait(empty + s, ph ^ 1);
        mbar_expect_tx(full + s, CH);
        bulk_g2s(buf + s * CH, a + c * CH, CH, full + s);
        if (++s == S) {
          s = 0;
          ph ^= 1;
        }
      }
    }
  } else {
    int s = 0;
    unsigned ph = 0;
    for (size_t c = c0; c < c1; ++c) {
      mbar_wait(full + s, ph);
      const float4* f = reinterpret_cast<const float4*>(buf + s * CH);
      float t = 0;
#pragma unroll 4
      for (int i = threadIdx.x; i < CH / 16; i += NW * 32) {
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

int main(int argc, char** argv) {
  const size_t bytes = size_t(256) << 20;
  const int NBUF = 8;
  std::vector<float*> bufs(NBUF);
  for (auto& b : bufs) {
    CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(b, 0, bytes));
  }
  double* out;
  CK(cudaMalloc(&out, 64));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  auto run = [&](const char* name, auto launch) {
    for (int w = 0; w < 4; ++w) launch(bufs[w % NBUF]);
    CK(cudaDeviceSynchronize());
    const int iters = 40;
    CK(cudaEventRecord(e0));
    for (int it = 0; it < iters; ++it) launch(bufs[it % NBUF]);
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    CK(cudaGetLastError());
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double us = ms * 1e3 / iters;
    std::printf("%-48s %8.2f us  %8.1f GB/s\n", name, us, bytes / (us * 1e-6) / 1e9);
  };
  const size_t n4 = bytes / 16;
  char name[128];
  for (int bps : {4, 8}) {
    for (int tpb : {256, 512}) {
      if (bps * tpb > 2048) continue;
      const int grid = sms * bps;
      std::snprintf(name, sizeof name, "flat_ldg U8 contig grid=%d tpb=%d", grid, tpb);
      run(name, [&](float* b) { flat_ldg<8, true><<<grid, tpb>>>((const float4*)b, n4, out); });
      std::snprintf(name, sizeof name, "flat_ldg U8 stride grid=%d tpb=%d", grid, tpb);
      run(name, [&](float* b) { flat_ldg<8, false><<<grid, tpb>>>((const float4*)b, n4, out); });
      std::snprintf(name, sizeof name, "flat_ldg U16 contig grid=%d tpb=%d", grid, tpb);
      run(name, [&](float* b) { flat_ldg<16, true><<<grid, tpb>>>((const float4*)b, n4, out); });
      std::snprintf(name, sizeof name, "flat_ldg U4 contig grid=%d tpb=%d", grid, tpb);
      run(name, [&](float* b) { flat_ldg<4, true><<<grid, tpb>>>((const float4*)b, n4, out); });
    }
  }
  for (int waves : {4, 16}) {
    const int grid = sms * 8 * waves;
    std::snprintf(name, sizeof name, "flat_ldg U8 contig grid=%d tpb=256 (%d waves)", grid, waves);
    run(name, [&](float* b) { flat_ldg<8, true><<<grid, 256>>>((const float4*)b, n4, out); });
  }
  {
    constexpr int NW = 8, S = 4, CH = 32768;
    const size_t smem = 128 + size_t(S) * CH;
    CK(cudaFuncSetAttribute(tma_stream<NW, S, CH>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    for (int bps : {1}) {
      const int grid = sms * bps;
      std::snprintf(name, sizeof name, "tma NW=%d S=%d CH=%d grid=%d", NW, S, CH, grid);
      run(name, [&](float* b) { tma_stream<NW, S, CH><<<grid, (NW + 1) * 32, smem>>>((const char*)b, bytes, out); });
    }
  }
  {
    constexpr int NW = 8, S = 6, CH = 16384;
    const size_t smem = 128 + size_t(S) * CH;
    CK(cudaFuncSetAttribute(tma_stream<NW, S, CH>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    for (int bps : {1, 2}) {
      const int grid = sms * bps;
      std::snprintf(name, sizeof name, "tma NW=%d S=%d CH=%d grid=%d", NW, S, CH, grid);
      run(name, [&](float* b) { tma_stream<NW, S, CH><<<grid, (NW + 1) * 32, smem>>>((const char*)b, bytes, out); });
    }
  }
  {
    constexpr int NW = 4, S = 8, CH = 8192;
    const size_t smem = 128 + size_t(S) * CH;
    CK(cudaFuncSetAttribute(tma_stream<NW, S, CH>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    for (int bps : {2, 3}) {
      const int grid = sms * bps;
      std::snprintf(name, sizeof name, "tma NW=%d S=%d CH=%d grid=%d", NW, S, CH, grid);
      run(name, [&](float* b) { tma_stream<NW, S, CH><<<grid, (NW + 1) * 32, smem>>>((const char*)b, bytes, out); });
    }
  }
  {
    constexpr int NW = 8, S = 3, CH = 65536;
    const size_t smem = 128 + size_t(S) * CH;
    CK(cudaFuncSetAttribute(tma_stream<NW, S, CH>, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    const int grid = sms;
    std::snprintf(name, sizeof name, "tma NW=%d S=%d CH=%d grid=%d", NW, S, CH, grid);
    run(name, [&](float* b) { tma_stream<NW, S, CH><<<grid, (NW + 1) * 32, smem>>>((const char*)b, bytes, out); });
  }
  // plain copy for reference against MEASURED_PEAKS (read+write bytes)
  {
    float* dst;
    CK(cudaMalloc(&dst, bytes));
    for (int w = 0; w < 3; ++w) CK(cudaMemcpyAsync(dst, bufs[w], bytes, cudaMemcpyDeviceToDevice));
    CK(cudaDeviceSynchronize());
    CK(cudaEventRecord(e0));
    for (int it = 0; it < 20; ++it) CK(cudaMemcpyAsync(dst, bufs[it % NBUF], bytes, cudaMemcpyDeviceToDevice));
    CK(cudaEventRecord(e1));
    CK(cudaEventSynchronize(e1));
    float ms;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double us = ms * 1e3 / 20;
    std::printf("%-48s %8.2f us  %8.1f GB/s (r+w)\n", "cudaMemcpy D2D 256MiB", us, 2 * bytes / (us * 1e-6) / 1e9);
  }
  return 0;
}
