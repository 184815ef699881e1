// micro_outer.cu — ceiling of the k-means inner loop shape on B200: a PPT x 4 outer product of
// float4 operands on FFMA2 (two passes .xy/.zw), (a) operands in registers, (b) operands re-read
// from shared memory every step with the kernel's access pattern (4 distinct x rows, 8 c rows per
// warp). Measurement tool only.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_outer tools/micro_outer.cu
#include <cuda_runtime.h>

#include <cstdio>

__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

template <int PPT, bool SMEM, int UNROLL>
__global__ void __launch_bounds__(288, 1) k_outer(float* out, int iters) {
  __shared__ __align__(16) float xs[32 * PPT * 8 * 4 + 64];  // 8 warps x (4*PPT rows x 32 floats)
  __shared__ __align__(16) float cs[32 * 68];
  for (int i = threadIdx.x; i < 32 * PPT * 8 * 4; i += blockDim.x) xs[i] = (i % 97) * 1e-3f;
  for (int i = threadIdx.x; i < 32 * 68; i += blockDim.x) cs[i] = (i % 89) * 1e-3f;
  __syncthreads();
  if (threadIdx.x >= 256) return;  // the idle "producer" warp
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int pg = lane & 3, cg = lane >> 2;
  const float* xb = xs + (warp * 4 * PPT + pg) * 32;
  const float* cq = cs + cg * 68;
  float2 acc[PPT][4];
#pragma unroll
  for (int i = 0; i < PPT; ++i)
#pragma unroll
    for (int m = 0; m < 4; ++m) acc[i][m] = make_float2(0.f, 0.f);
  float4 xv[PPT], cv[4];
#pragma unroll
  for (int i = 0; i < PPT; ++i) xv[i] = *reinterpret_cast<const float4*>(xb + 128 * i + 4 * ((pg + 4 * (i & 1)) & 7));
#pragma unroll
  for (int m = 0; m < 4; ++m) cv[m] = *reinterpret_cast<const float4*>(cq + 8 * m * 68);
#pragma unroll UNROLL
  for (int it = 0; it < iters; ++it) {
    if (SMEM) {
      const int j = it & 7;
#pragma unroll
      for (int i = 0; i < PPT; ++i)
        xv[i] = *reinterpret_cast<const float4*>(xb + 128 * i + 4 * (j ^ ((pg + 4 * (i & 1)) & 7)));
#pragma unroll
      for (int m = 0; m < 4; ++m) cv[m] = *reinterpret_cast<const float4*>(cq + 8 * m * 68 + 4 * j);
    }
#pragma unroll
    for (int m = 0; m < 4; ++m)
#pragma unroll
      for (int i = 0; i < PPT; ++i) ffma2(acc[i][m], make_float2(xv[i].x, xv[i].y), make_float2(cv[m].x, cv[m].y));
#pragma unroll
    for (int m = 0; m < 4; ++m)
#pragma unroll
      for (int i = 0; i < PPT; ++i) ffma2(acc[i][m], make_float2(xv[i].z, xv[i].w), make_float2(cv[m].z, cv[m].w));
  }
  float s = 0;
#pragma unroll
  for (int i = 0; i < PPT; ++i)
#pragma unroll
    for (int m = 0; m < 4; ++m) s += acc[i][m].x + acc[i][m].y;
  if (s == 1.2345f) out[0] = s;
}

template <int PPT, bool SMEM, int UNROLL>
void run(float* out, int sms, const char* name) {
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int iters = 20000;
  k_outer<PPT, SMEM, UNROLL><<<sms, 288>>>(out, iters);
  cudaDeviceSynchronize();
  cudaEventRecord(e0);
  k_outer<PPT, SMEM, UNROLL><<<sms, 288>>>(out, iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double flops = double(sms) * 256 * iters * PPT * 4 * 8;  // PPT*4 pairs x 4 dims x 2
  printf("%-28s %8.3f ms  %7.2f TFLOP/s\n", name, ms, flops / (ms * 1e-3) / 1e12);
}

int main() {
  float* out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run<8, false, 1>(out, sms, "PPT8 regs u1");
  run<8, false, 2>(out, sms, "PPT8 regs u2");
  run<8, true, 1>(out, sms, "PPT8 smem u1");
  run<8, true, 2>(out, sms, "PPT8 smem u2");
  run<8, true, 4>(out, sms, "PPT8 smem u4");
  run<4, false, 1>(out, sms, "PPT4 regs u1");
  run<4, true, 2>(out, sms, "PPT4 smem u2");
  run<4, true, 4>(out, sms, "PPT4 smem u4");
  return 0;
}
