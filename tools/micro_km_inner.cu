// micro_km_inner.cu — measurement tool only: the k-means dims loop in isolation (x from shared memory
// with the 128-byte swizzle, FFMA2 over pairs of -2c) by thread tile (PPT points x CPT centroids, G = 32/CPT
// warp-uniform centroid groups), warps per SM and centroid source, to see what fraction of the FP32 FMA
// peak the loop itself can reach before any epilogue (profiles/r02/kmeans/micro_inner.log).
//   CSRC 0: constant bank (LDCU.64, one pair per load)   2: shared memory broadcast (LDS.128, two pairs)
//        3: registers only (no centroid loads: the loop's ceiling)   4: half LDS broadcast, half LDCU
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_km_inner tools/micro_km_inner.cu
#include <cuda_runtime.h>

#include <cstdio>

constexpr int D = 64;
__constant__ __align__(16) float2 cp[16 * D];  // 32 centroids as 16 pairs, [pair][d]

__device__ __forceinline__ void ffma2(float2& acc, const float2 a, const float2 b) {
  unsigned long long A = *reinterpret_cast<const unsigned long long*>(&a);
  unsigned long long B = *reinterpret_cast<const unsigned long long*>(&b);
  unsigned long long C = *reinterpret_cast<unsigned long long*>(&acc);
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(C) : "l"(A), "l"(B));
  acc = *reinterpret_cast<float2*>(&C);
}

// XW: x operands per point and load — 4 (one LDS.128 per 4-dim step, the kernel's form) or 1 / 2 (LDS.32 /
// LDS.64 per dim / dim pair, fewer live x registers); MAXR: the register cap (255 = none)
template <int PPT, int CPT, int LP, int WARPS, int CSRC, int UNR, int XW, int MAXR>
__global__ void __maxnreg__(MAXR) k_inner(float* out, int tiles) {
  extern __shared__ __align__(1024) unsigned char smem[];
  constexpr int G = 32 / CPT, NP = CPT / 2, TP = PPT * LP;
  const int warp = __shfl_sync(0xffffffffu, int(threadIdx.x >> 5), 0);
  const int g = int(__reduce_min_sync(0xffffffffu, unsigned((warp * 32 / LP) % G)));
  const int lt = threadIdx.x % LP;
  const unsigned key4 = unsigned(lt & 7) << 4;
  for (int i = threadIdx.x; i < TP * D; i += blockDim.x) reinterpret_cast<float*>(smem)[i] = (i % 97) * 0.01f;
  float2* cs = reinterpret_cast<float2*>(smem + TP * D * 4);  // [D][16 pairs]
  for (int i = threadIdx.x; i < 16 * D; i += blockDim.x) cs[(i % D) * 16 + i / D] = cp[i];
  __syncthreads();
  float2 creg[NP];
#pragma unroll
  for (int p = 0; p < NP; ++p) creg[p] = cp[g * NP + p + 3 * p];
  float best = 0.f;
  for (int t = 0; t < tiles; ++t) {
    float2 acc[PPT][NP];
#pragma unroll
    for (int i = 0; i < PPT; ++i)
#pragma unroll
      for (int p = 0; p < NP; ++p) acc[i][p] = make_float2(0.f, 0.f);
    const float2* cq = cp + (g * NP) * D;
#pragma unroll 1
    for (int bx = 0; bx < 2; ++bx) {
      const unsigned char* tb = smem + bx * (TP * 128) + lt * 128;
#pragma unroll UNR
      for (int j = 0; j < 8; ++j) {
        const int d4 = 8 * bx + j;
        float4 xv[PPT];
        if constexpr (XW == 4) {
#pragma unroll
          for (int i = 0; i < PPT; ++i) xv[i] = *reinterpret_cast<const float4*>(tb + LP * 128 * i + ((unsigned(j) << 4) ^ key4));
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if constexpr (XW == 1) {
#pragma unroll
            for (int i = 0; i < PPT; ++i) {
              const float v = *reinterpret_cast<const float*>(tb + LP * 128 * i + ((unsigned(j) << 4) ^ key4) + 4 * q);
              xv[i] = make_float4(v, v, v, v);
            }
          } else if constexpr (XW == 2) {
            if ((q & 1) == 0) {
#pragma unroll
              for (int i = 0; i < PPT; ++i) {
                const float2 v = *reinterpret_cast<const float2*>(tb + LP * 128 * i + ((unsigned(j) << 4) ^ key4) + 4 * q);
                xv[i] = make_float4(v.x, v.y, v.x, v.y);
              }
            }
          }
          float2 cv[NP];
          if constexpr (CSRC == 0) {
#pragma unroll
            for (int p = 0; p < NP; ++p) cv[p] = cq[p * D + 4 * d4 + q];
          } else if constexpr (CSRC == 2) {
#pragma unroll
            for (int p = 0; p < NP; p += 2) {
              const float4 c4 = *reinterpret_cast<const float4*>(cs + (4 * d4 + q) * 16 + g * NP + p);
              cv[p] = make_float2(c4.x, c4.y), cv[p + 1] = make_float2(c4.z, c4.w);
            }
          } else if constexpr (CSRC == 4) {
#pragma unroll
            for (int p = 0; p < NP / 2; p += 2) {
              const float4 c4 = *reinterpret_cast<const float4*>(cs + (4 * d4 + q) * 16 + g * NP + p);
              cv[p] = make_float2(c4.x, c4.y), cv[p + 1] = make_float2(c4.z, c4.w);
            }
#pragma unroll
            for (int p = NP / 2; p < NP; ++p) cv[p] = cq[p * D + 4 * d4 + q];
          } else {
#pragma unroll
            for (int p = 0; p < NP; ++p) cv[p] = creg[p];
          }
#pragma unroll
          for (int p = 0; p < NP; ++p)
#pragma unroll
            for (int i = 0; i < PPT; ++i) {
              const float xs = q == 0 ? xv[i].x : q == 1 ? xv[i].y : q == 2 ? xv[i].z : xv[i].w;
              ffma2(acc[i][p], make_float2(xs, xs), cv[p]);
            }
        }
      }
    }
#pragma unroll
    for (int i = 0; i < PPT; ++i)
#pragma unroll
      for (int p = 0; p < NP; ++p) best += acc[i][p].x + acc[i][p].y;
  }
  if (best == 1.2345f) out[0] = best;
}

template <int PPT, int CPT, int LP, int WARPS, int CSRC, int UNR = 2, int XW = 4, int MAXR = 255>
void run(float* out, int sms, const char* name) {
  auto kern = k_inner<PPT, CPT, LP, WARPS, CSRC, UNR, XW, MAXR>;
  const int smem = PPT * LP * D * 4 + 16 * D * 8;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, WARPS * 32, smem);
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, kern);
  const int tiles = 400;
  const int grid = sms * per_sm;
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  kern<<<grid, WARPS * 32, smem>>>(out, 10);
  cudaEventRecord(a);
  kern<<<grid, WARPS * 32, smem>>>(out, tiles);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  const double flops = double(grid) * WARPS * 32 * tiles * PPT * double(CPT) * D * 2.0;
  const double peak = sms * 128.0 * 2 * 1.965e9;
  printf("%-34s regs %3d spill %3d blocks/SM %d warps/SM %2d  %.3f ms  %.1f TFLOP/s  frac %.3f  (%s)\n", name,
         fa.numRegs, int(fa.localSizeBytes), per_sm, per_sm * WARPS, ms, flops / ms / 1e9, flops / (ms * 1e-3) / peak,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  float* out;
  cudaMalloc(&out, 4);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  float2 h[16 * D];
  for (int i = 0; i < 16 * D; ++i) h[i] = make_float2(0.001f * (i % 31), -0.002f * (i % 17));
  cudaMemcpyToSymbol(cp, h, sizeof(h));
  for (int rep = 0; rep < 2; ++rep) {
    // run 3 (profiles/r02/kmeans/micro_inner.log): thread tile and centroid source, no register cap
    run<4, 8, 64, 8, 0>(out, sms, "P4 C8 LP64 8w LDCU");
    run<4, 8, 64, 8, 2>(out, sms, "P4 C8 LP64 8w LDS");
    run<4, 8, 64, 8, 4>(out, sms, "P4 C8 LP64 8w hybrid");
    run<4, 8, 64, 8, 3>(out, sms, "P4 C8 LP64 8w regs");
    run<4, 16, 64, 4, 4>(out, sms, "P4 C16 LP64 4w hybrid");
    // runs 4-5: 8 points per thread under a register cap (ptxas keeps LDCU), 24 and 12 warps per SM
    run<4, 8, 64, 8, 0, 2, 4, 80>(out, sms, "P4 C8 LP64 8w LDCU cap80");
    run<8, 8, 32, 8, 0, 2, 2, 80>(out, sms, "P8 C8 LP32 8w LDCU xw2 u2 cap80");
    run<8, 8, 32, 8, 0, 1, 4, 80>(out, sms, "P8 C8 LP32 8w LDCU xw4 u1 cap80");
    run<8, 8, 32, 4, 0, 2, 4, 96>(out, sms, "P8 C8 LP32 4w LDCU xw4 u2 cap96");
    run<8, 8, 32, 4, 0, 4, 4, 128>(out, sms, "P8 C8 LP32 4w LDCU xw4 u4 cap128");
  }
  return 0;
}
