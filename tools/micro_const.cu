// micro_const.cu — throughput of centroid operands served from the constant bank: LDCU (uniform
// datapath, forced by a low register cap) vs LDC (vector registers), in the k-means loop shape
// (x from shared memory, 32 centroids x 64 dims, FFMA2). Measurement tool only.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_const tools/micro_const.cu
#include <cuda_runtime.h>

#include <cstdio>

__constant__ float cf[8192];
__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

template <int PPT>
__device__ __forceinline__ void body(int* out, int D, int Kp, int n_tiles) {
  extern __shared__ __align__(1024) unsigned char smem[];
  const int lt = threadIdx.x;
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = (i % 13) * 0.1f;
  __syncthreads();
  const unsigned key = lt & 7;
  for (int t = 0; t < n_tiles; ++t) {
    const unsigned char* tile = smem + (lt & 127) * 128;
    float bs[PPT];
    int bk[PPT];
    for (int i = 0; i < PPT; ++i) bs[i] = 1e30f, bk[i] = 0;
    for (int kc = 0; kc < Kp; kc += 32 / PPT) {
      float2 acc[PPT][32 / PPT];
      for (int i = 0; i < PPT; ++i)
        for (int m = 0; m < 32 / PPT; ++m) acc[i][m] = make_float2(0, 0);
      const float* cq = cf + kc * D;
#pragma unroll 2
      for (int d4 = 0; d4 < D / 4; ++d4) {
        const unsigned char* xb = tile + (d4 >> 3) * (128 * 128) + ((unsigned(d4 & 7) ^ key) << 4);
        float4 xx[PPT];
#pragma unroll
        for (int i = 0; i < PPT; ++i) xx[i] = *reinterpret_cast<const float4*>(xb + i * 256);
#pragma unroll
        for (int m = 0; m < 32 / PPT; ++m) {
          const float4 c = *reinterpret_cast<const float4*>(cq + m * D + 4 * d4);
#pragma unroll
          for (int i = 0; i < PPT; ++i) {
            ffma2(acc[i][m], make_float2(xx[i].x, xx[i].y), make_float2(c.x, c.y));
            ffma2(acc[i][m], make_float2(xx[i].z, xx[i].w), make_float2(c.z, c.w));
          }
        }
      }
      for (int i = 0; i < PPT; ++i)
        for (int m = 0; m < 32 / PPT; ++m) {
          float s = acc[i][m].x + acc[i][m].y;
          if (s < bs[i]) bs[i] = s, bk[i] = kc + m;
        }
    }
    for (int i = 0; i < PPT; ++i) out[(blockIdx.x * n_tiles + t) * 256 * PPT + i * 256 + threadIdx.x] = bk[i];
  }
}

template <int PPT>
__global__ void __maxnreg__(128) k_ldcu(int* out, int D, int Kp, int n) { body<PPT>(out, D, Kp, n); }
template <int PPT>
__global__ void __maxnreg__(255) k_ldc(int* out, int D, int Kp, int n) { body<PPT>(out, D, Kp, n); }

template <typename F>
void run(F kern, const char* name, int ppt, int sms, int* out) {
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  const int n = 64, Kp = 32, D = 64;
  kern<<<sms, 256, 65536>>>(out, D, Kp, n);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  kern<<<sms, 256, 65536>>>(out, D, Kp, n);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double flops = double(sms) * n * 256 * ppt * 32 * 64 * 2.0;
  printf("%-10s PPT=%d %8.3f ms %7.2f TFLOP/s  (%s)\n", name, ppt, ms, flops / (ms * 1e-3) / 1e12,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int* out;
  cudaMalloc(&out, 148 * 64 * 256 * 4 * 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  run(k_ldcu<1>, "LDCU", 1, sms, out);
  run(k_ldc<1>, "LDC", 1, sms, out);
  run(k_ldcu<2>, "LDCU", 2, sms, out);
  run(k_ldc<2>, "LDC", 2, sms, out);
  run(k_ldcu<4>, "LDCU", 4, sms, out);
  run(k_ldc<4>, "LDC", 4, sms, out);
  return 0;
}
