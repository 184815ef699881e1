// micro_fma.cu — FP32 FMA throughput on B200: scalar FFMA vs packed FFMA2 (fma.rn.f32x2), by warps/SM.
// Measurement tool only.  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_fma tools/micro_fma.cu
#include <cuda_runtime.h>

#include <cstdio>

__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

template <int CH>
__global__ void k_ffma(float* out, int iters, float a, float b) {
  float acc[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) acc[i] = threadIdx.x * 1e-3f + i;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) acc[i] = fmaf(acc[i], a, b);
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += acc[i];
  if (s == 1.2345f) out[0] = s;
}

template <int CH>
__global__ void k_ffma2(float* out, int iters, float a, float b) {
  float2 acc[CH];
#pragma unroll
  for (int i = 0; i < CH; ++i) acc[i] = make_float2(threadIdx.x * 1e-3f + i, i * 0.5f);
  const float2 av = make_float2(a, a), bv = make_float2(b, b);
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < CH; ++i) ffma2(acc[i], av, bv);
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < CH; ++i) s += acc[i].x + acc[i].y;
  if (s == 1.2345f) out[0] = s;
}

int main() {
  float* out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 20000;
  for (int warps : {4, 8, 16, 32}) {
    const int threads = warps * 32 > 1024 ? 1024 : warps * 32;
    const int blocks = sms * (warps * 32 / threads);
    for (int kind = 0; kind < 2; ++kind) {
      auto launch = [&] {
        if (kind == 0)
          k_ffma<16><<<blocks, threads>>>(out, iters, 0.999f, 0.001f);
        else
          k_ffma2<8><<<blocks, threads>>>(out, iters, 0.999f, 0.001f);
      };
      launch();
      cudaDeviceSynchronize();
      cudaEventRecord(e0);
      launch();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      const double fmas = double(blocks) * threads * iters * 16.0;  // 16 FMAs per iteration either way
      printf("%-6s warps/SM=%2d  %8.3f ms  %7.2f TFLOP/s  %6.1f FMA/clk/SM @1965MHz\n", kind ? "FFMA2" : "FFMA",
             warps, ms, 2 * fmas / (ms * 1e-3) / 1e12, fmas / (ms * 1e-3) / sms / 1.965e9);
    }
  }
  return 0;
}
