// micro_gather.cu — measurement tool only: the random-gather ceiling PageRank sits under. E 4-byte
// gathers pr[idx[e]] from an L2-resident fp32 vector of N nodes, the indices streamed coalesced from
// HBM (as PageRank's colidx), per-thread sums written once. Reports gathers/s and the L1tex wavefront
// rate for comparison with the kernel's roofline (profiles/r02/pagerank/micro_gather.log).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o micro_gather tools/micro_gather.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t mix(uint64_t x) {  // splitmix64 finaliser, low 32 bits
  x += 0x9e3779b97f4a7c15ull;
  x = (x ^ (x >> 30)) * 0xbf58476d1ce4e5b9ull;
  x = (x ^ (x >> 27)) * 0x94d049bb133111ebull;
  return uint32_t(x ^ (x >> 31));
}

// idx[e]: uniform over [0, N) (SKEW = 0) or a power-law-ish draw (SKEW = 1: min of two uniforms squared
// toward low ids, so a few nodes are hot, as in a power-law in-degree graph)
__global__ void k_fill(uint32_t* idx, float* pr, long long E, uint32_t N, int skew) {
  for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < E; e += (long long)gridDim.x * blockDim.x) {
    uint32_t r = mix(uint64_t(e));
    if (skew) {
      const double u = double(r) / 4294967296.0;
      r = uint32_t(u * u * N);
    } else {
      r %= N;
    }
    idx[e] = r;
  }
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < N; i += (long long)gridDim.x * blockDim.x)
    pr[i] = 1.0f / float(i + 1);
}

template <int UNROLL, bool NC>
__global__ void __launch_bounds__(256) k_gather(const uint32_t* __restrict__ idx, const float* __restrict__ pr,
                                                float* out, long long E) {
  float acc = 0.f;
  const long long stride = (long long)gridDim.x * blockDim.x;
  long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  for (; e + (UNROLL - 1) * stride < E; e += UNROLL * stride) {
    uint32_t j[UNROLL];
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) j[u] = __ldcs(idx + e + u * stride);
#pragma unroll
    for (int u = 0; u < UNROLL; ++u) acc += NC ? __ldg(pr + j[u]) : pr[j[u]];
  }
  for (; e < E; e += stride) acc += pr[__ldcs(idx + e)];
  out[blockIdx.x * (long long)blockDim.x + threadIdx.x] = acc;
}

template <int UNROLL, bool NC>
void run(const uint32_t* idx, const float* pr, float* out, long long E, int grid, const char* name) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  k_gather<UNROLL, NC><<<grid, 256>>>(idx, pr, out, E);
  cudaEventRecord(a);
  const int reps = 5;
  for (int r = 0; r < reps; ++r) k_gather<UNROLL, NC><<<grid, 256>>>(idx, pr, out, E);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  ms /= reps;
  printf("%-34s %8.1f us  %6.1f G gathers/s  (%s)\n", name, ms * 1e3, E / (ms * 1e-3) / 1e9,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  const uint32_t N = 1u << 22;       // 4M nodes: a 16 MB vector, L2-resident
  const long long E = 63LL << 20;    // ~63M edges, as the PageRank workload
  uint32_t* idx;
  float *pr, *out;
  cudaMalloc(&idx, E * 4);
  cudaMalloc(&pr, N * 4ull);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaMalloc(&out, sms * 8 * 256 * 4ull);
  for (int skew = 0; skew < 2; ++skew) {
    k_fill<<<sms * 8, 256>>>(idx, pr, E, N, skew);
    cudaDeviceSynchronize();
    printf("== indices: %s\n", skew ? "skewed (u^2)" : "uniform");
    run<4, false>(idx, pr, out, E, sms * 8, "unroll 4, ld.global");
    run<8, false>(idx, pr, out, E, sms * 8, "unroll 8, ld.global");
    run<8, true>(idx, pr, out, E, sms * 8, "unroll 8, ld.global.nc");
    run<16, true>(idx, pr, out, E, sms * 8, "unroll 16, ld.global.nc");
    run<16, true>(idx, pr, out, E, sms * 4, "unroll 16, ld.global.nc, 4 blk/SM");
  }
  return 0;
}
