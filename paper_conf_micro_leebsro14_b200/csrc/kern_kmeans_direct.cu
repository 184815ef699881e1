// kern_kmeans_direct.cu — the k-means assignment nest (BASELINE.json config 4) under ANY mapping of
// Algorithm 1 whose reduce levels are Span(all): strategy LITERAL and caller-given mappings
// (npp_plan_with_mapping) of KMEANS_ASSIGN, i.e. the three-level nest of PAPER.md L606-610 executed
// exactly as the logical multidimensional mapping says (§IV-A), as the paper's generated
// code would (§IV-E) — the Fig 17 sweep times these against the AUTO family.
//
//   L0 = points (Map): block g covers [g·chunk0, (g+1)·chunk0), its b0 threads take points
//        base + t0 + j·b0 (Span(1) / Span(n) / Span(all) are the chunk the record gives);
//   L1 = centroids (argmin Reduce, Span(all)): thread t1 takes centroids t1 + m·b1;
//   L2 = dims (Reduce, Span(all)): thread t2 takes dims t2 + q·b2; the b2 partial sums of a
//        (point, centroid) meet in shared memory (the Reduce of Fig 9's generated code).
// Each level's thread index comes from the CUDA dim the mapping assigned to it. Split on a reduce
// level is not executed here (npp_plan_with_mapping rejects it).
//
// Results are index-exact (G25): distances are fp64 (products and sums rounded, no FMA) in the
// mapping's order, within γ_{D+b2+3} of the exact distance; a point whose runner-up is not beyond both
// bounds is recomputed by one thread in the oracle's sequential order, the lowest k winning ties.
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.hpp"

namespace npp {

namespace {

__device__ __forceinline__ double sqdiff(float a, float b) {
  const double t = __dsub_rn(double(a), double(b));
  return __dmul_rn(t, t);
}

}  // namespace

__global__ void __launch_bounds__(1024) npp_kmeans_direct_kernel(const KmDirectArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int b0 = a.blk[0], b1 = a.blk[1], b2 = a.blk[2];
  const int nthr = b0 * b1 * b2;
  double* red = reinterpret_cast<double*>(smem_raw);  // [b0][b1][b2] partial distances
  double* bd = red + nthr;                            // [b0][b1] best distance of the (t0, t1) thread
  double* sd = bd + b0 * b1;                          // [b0][b1] its runner-up
  int* bkk = reinterpret_cast<int*>(sd + b0 * b1);    // [b0][b1] its best centroid
  const int tid[3] = {int(threadIdx.x), int(threadIdx.y), int(threadIdx.z)};
  const int t0 = tid[a.dim[0]], t1 = tid[a.dim[1]], t2 = tid[a.dim[2]];
  const int D = a.D, K = a.K;
  const double inf = __longlong_as_double(0x7ff0000000000000ll);
  const long long p_begin = (long long)blockIdx.x * a.chunk0;
  const long long p_end = p_begin + a.chunk0 < a.N ? p_begin + a.chunk0 : a.N;
  const long long iters = (p_end - p_begin + b0 - 1) / b0;  // the same for every thread of the block
  const int mk = (K + b1 - 1) / b1;
  // γ of this order plus γ of the oracle's sequential order (2^-53 units), + slack
  const double rel = double(2 * D + b2 + 8) * 1.1102230246251565e-16 * 1.01;
  for (long long j = 0; j < iters; ++j) {
    const long long p = p_begin + t0 + j * b0;
    const bool valid = p < p_end;
    const float* xp = a.x + (valid ? p : 0) * (long long)D;
    double best = inf, second = inf;
    int bk = 0x7fffffff;
    for (int m = 0; m < mk; ++m) {
      const int k = t1 + m * b1;
      double part = 0.0;
      if (valid && k < K) {
        const float* ck = a.c + (long long)k * D;
        for (int d = t2; d < D; d += b2) part = __dadd_rn(part, sqdiff(__ldg(xp + d), __ldg(ck + d)));
      }
      red[(t0 * b1 + t1) * b2 + t2] = part;
      __syncthreads();
      if (t2 == 0 && valid && k < K) {
        double dist = 0.0;
        for (int q = 0; q < b2; ++q) dist = __dadd_rn(dist, red[(t0 * b1 + t1) * b2 + q]);
        if (dist < best) second = best, best = dist, bk = k;  // k increases: strict < keeps the first
        else if (dist < second) second = dist;
      }
      __syncthreads();
    }
    if (t2 == 0) {
      bd[t0 * b1 + t1] = best;
      sd[t0 * b1 + t1] = second;
      bkk[t0 * b1 + t1] = bk;
    }
    __syncthreads();
    if (t1 == 0 && t2 == 0 && valid) {  // the argmin Reduce across the b1 threads, in t1 order
      double w = inf, s = inf;
      int wk = 0x7fffffff;
      for (int r = 0; r < b1; ++r) {
        const double v = bd[t0 * b1 + r], v2 = sd[t0 * b1 + r];
        const int kv = bkk[t0 * b1 + r];
        if (v < w || (v == w && kv < wk)) {
          s = fmin(s, w);
          w = v, wk = kv;
        } else {
          s = fmin(s, v);
        }
        s = fmin(s, v2);
      }
      // a runner-up within both rounding bounds of the winner may be the fp64-as-written winner: the
      // oracle's sequential distances decide
      if (!(s - w > rel * (s + w))) {
        double w2 = inf;
        int k2 = 0x7fffffff;
        for (int k = 0; k < K; ++k) {
          const float* ck = a.c + (long long)k * D;
          double dist = 0.0;
          for (int d = 0; d < D; ++d) dist = __dadd_rn(dist, sqdiff(__ldg(xp + d), __ldg(ck + d)));
          if (dist < w2) w2 = dist, k2 = k;
        }
        wk = k2;
      }
      a.assign[p] = wk;
    }
    __syncthreads();
  }
}

cudaError_t launch_kmeans_direct(const KmDirectArgs& a, int grid, cudaStream_t st) {
  const int nthr = a.blk[0] * a.blk[1] * a.blk[2];
  const size_t smem = size_t(nthr) * 8 + size_t(a.blk[0]) * a.blk[1] * (8 + 8 + 4);
  cudaError_t e = ensure_smem(npp_kmeans_direct_kernel, int(smem));
  if (e != cudaSuccess) return e;
  dim3 block(1, 1, 1);
  unsigned* bdim[3] = {&block.x, &block.y, &block.z};
  for (int l = 0; l < 3; ++l) *bdim[a.dim[l]] = unsigned(a.blk[l]);
  npp_kmeans_direct_kernel<<<grid, block, smem, st>>>(a);
  return cudaGetLastError();
}

}  // namespace npp
