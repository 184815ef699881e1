// micro_tail.cu — where do the last ~6 us of a 256 MiB streaming pass go on B200?
// Not part of the library: a measurement tool for the staged sum family (launch gap, ramp, tail).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/micro_tail tools/micro_tail.cu
// Variants (one persistent block per SM, 1-D cp.async.bulk chunks through an S-deep smem ring):
//   static   contiguous equal ranges per block (the library's current work split)
//   steal    same ranges, but the last part of each range is claimed through a per-range counter and
//            blocks that finish early steal chunks from the other ranges
//   pdl      static, launched with programmatic stream serialization (next launch's blocks start
//            as SMs free up; kernels are independent so no griddepcontrol.wait is needed)
// Each is timed (a) per launch in isolation (events around one launch, idle GPU before it) and
// (b) back to back in a CUDA graph of 20 launches over 8 distinct buffers.
#include <cuda_runtime.h>

#include <algorithm>
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

__device__ __forceinline__ unsigned su32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* b, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, unsigned parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}" ::"r"(su32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(dst)),
      "l"(src), "r"(bytes), "r"(su32(bar))
      : "memory");
}
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

constexpr int NW = 8;
constexpr int S = 4;
constexpr int CH = 32768;

struct Args {
  const char* a;
  long long nchunks;
  long long per_block;
  long long static_part;         // steal: chunks of each range taken without atomics
  unsigned* next;                // steal: [grid] claim counters (relative to static end), + [grid] done ticket
  unsigned long long* times;     // optional [grid x 2] start/end stamps
  double* out;
  int pdl;
};

// claim the next chunk: own range first (static part, then counter), then steal round-robin
__device__ __forceinline__ long long claim(const Args& A, int bid, long long& own, int& victim, bool steal) {
  const long long r0 = bid * A.per_block;
  const long long r1 = min(A.nchunks, r0 + A.per_block);
  if (!steal) {
    const long long c = r0 + own;
    ++own;
    return c < r1 ? c : -1;
  }
  if (own < A.static_part && r0 + own < r1) return r0 + own++;
  const int G = gridDim.x;
  while (victim < G) {
    const int v = (bid + victim) % G;
    const long long v0 = v * A.per_block;
    const long long v1 = min(A.nchunks, v0 + A.per_block);
    const long long dyn0 = min(v1, v0 + A.static_part);
    if (dyn0 < v1) {
      const unsigned k = atomicAdd(A.next + v, 1u);
      if (dyn0 + k < v1) return dyn0 + k;
    }
    ++victim;
  }
  return -1;
}

template <bool STEAL>
__global__ void __launch_bounds__((NW + 1) * 32, 1) stream_kernel(Args A) {
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + S;
  long long* tag = reinterpret_cast<long long*>(empty + S);
  unsigned char* buf = smem + 1024;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int bid = blockIdx.x;
  if (A.pdl) asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x == 0) {
    if (A.times) A.times[bid * 2] = gtimer();
    for (int s = 0; s < S; ++s) {
      mbar_init(full + s, 1);
      mbar_init(empty + s, NW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  double acc = 0;
  if (warp == NW) {
    if (lane == 0) {
      long long own = 0;
      int victim = STEAL ? 0 : 0;
      long long t = 0;
      for (;; ++t) {
        const long long c = claim(A, bid, own, victim, STEAL);
        const int s = int(t % S);
        if (t >= S) mbar_wait(empty + s, unsigned((t / S) & 1) ^ 1u);
        tag[s] = c;
        if (c < 0) {
          mbar_arrive(full + s);  // end marker (no bytes)
          break;
        }
        mbar_expect_tx(full + s, CH);
        bulk_g2s(buf + s * CH, A.a + c * CH, CH, full + s);
      }
    }
  } else {
    for (long long t = 0;; ++t) {
      const int s = int(t % S);
      mbar_wait(full + s, unsigned((t / S) & 1));
      if (tag[s] < 0) break;
      const float4* f = reinterpret_cast<const float4*>(buf + s * CH);
      float u = 0;
#pragma unroll 4
      for (int i = threadIdx.x; i < CH / 16; i += NW * 32) {
        float4 r = f[i];
        u += (r.x + r.y) + (r.z + r.w);
      }
      acc += u;
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + s);
    }
  }
  if (acc == 12345.678) A.out[0] = acc;
  if (STEAL) {
    __syncthreads();
    if (threadIdx.x == 0) {
      // last block to finish resets the claim counters for the next launch
      __threadfence();
      const unsigned d = atomicAdd(A.next + gridDim.x, 1u);
      if (d + 1 == gridDim.x) {
        for (int v = 0; v < (int)gridDim.x; ++v) A.next[v] = 0;
        A.next[gridDim.x] = 0;
        __threadfence();
      }
    }
  }
  if (A.times && threadIdx.x == 0) A.times[bid * 2 + 1] = gtimer();
}

int main(int argc, char** argv) {
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  const size_t max_bytes = size_t(1) << 30;
  const int NBUF = 8;
  std::vector<char*> bufs(NBUF);
  for (auto& b : bufs) {
    CK(cudaMalloc(&b, max_bytes));
    CK(cudaMemset(b, 1, max_bytes));
  }
  char* flush;
  const size_t flush_bytes = size_t(512) << 20;
  CK(cudaMalloc(&flush, flush_bytes));
  double* out;
  CK(cudaMalloc(&out, 64));
  unsigned* next;
  CK(cudaMalloc(&next, 4096 * 4));
  CK(cudaMemset(next, 0, 4096 * 4));
  unsigned long long* times;
  CK(cudaMalloc(&times, 4096 * 16));
  const int smem = 1024 + S * CH;
  CK(cudaFuncSetAttribute(stream_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  CK(cudaFuncSetAttribute(stream_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));

  auto make_args = [&](const char* a, size_t bytes, bool steal, double static_frac, bool pdl, bool stamp) {
    Args A{};
    A.a = a;
    A.nchunks = (long long)(bytes / CH);
    A.per_block = (A.nchunks + sms - 1) / sms;
    A.static_part = steal ? (long long)(A.per_block * static_frac) : A.per_block;
    A.next = next;
    A.times = stamp ? times : nullptr;
    A.out = out;
    A.pdl = pdl ? 1 : 0;
    return A;
  };
  auto launch = [&](const Args& A, bool steal) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(sms);
    cfg.blockDim = dim3((NW + 1) * 32);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = A.pdl ? 1 : 0;
    if (steal)
      CK(cudaLaunchKernelEx(&cfg, stream_kernel<true>, A));
    else
      CK(cudaLaunchKernelEx(&cfg, stream_kernel<false>, A));
  };
  auto isolated = [&](size_t bytes, bool steal, double frac, int reps, double* spread) {
    std::vector<float> ts;
    double sp = 0;
    for (int r = 0; r < reps; ++r) {
      CK(cudaMemsetAsync(flush, r, flush_bytes, st));  // evict L2, GPU busy -> idle
      CK(cudaStreamSynchronize(st));
      Args A = make_args(bufs[r % NBUF], bytes, steal, frac, false, spread != nullptr);
      CK(cudaEventRecord(e0, st));
      launch(A, steal);
      CK(cudaEventRecord(e1, st));
      CK(cudaEventSynchronize(e1));
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      ts.push_back(ms * 1e3f);
      if (spread) {
        std::vector<unsigned long long> h(sms * 2);
        CK(cudaMemcpy(h.data(), times, sms * 16, cudaMemcpyDeviceToHost));
        unsigned long long s0 = ~0ull, s1 = 0, e0_ = ~0ull, e1_ = 0;
        for (int b = 0; b < sms; ++b) {
          s0 = std::min(s0, h[b * 2]);
          s1 = std::max(s1, h[b * 2]);
          e0_ = std::min(e0_, h[b * 2 + 1]);
          e1_ = std::max(e1_, h[b * 2 + 1]);
        }
        if (r == reps - 1)
          std::printf("    stamps: start spread %.2f us, first end %.2f us, last end %.2f us (after first start)\n",
                      (s1 - s0) / 1e3, (e0_ - s0) / 1e3, (e1_ - s0) / 1e3);
      }
    }
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];
  };
  auto graphed = [&](size_t bytes, bool steal, double frac, bool pdl) {
    const int n = 20;
    cudaGraph_t g;
    cudaGraphExec_t ge;
    CK(cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal));
    for (int i = 0; i < n; ++i) {
      Args A = make_args(bufs[i % NBUF], bytes, steal, frac, pdl, false);
      A.next = next + (i % 8) * 256;  // overlapping (PDL) launches must not share claim counters
      launch(A, steal);
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
      ts.push_back(ms * 1e3f / n);
    }
    CK(cudaGraphExecDestroy(ge));
    CK(cudaGraphDestroy(g));
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];
  };

  std::printf("# size sweep, static split, isolated launches (median of 9)\n");
  for (size_t mb : {32, 64, 128, 256, 512, 1024}) {
    const size_t bytes = mb << 20;
    double sp = 0;
    const float us = isolated(bytes, false, 1.0, 9, &sp);
    std::printf("static   %5zu MiB  isolated %8.2f us  %7.1f GB/s\n", mb, us, bytes / (us * 1e-6) / 1e9);
  }
  const size_t bytes = size_t(256) << 20;
  std::printf("# 256 MiB\n");
  {
    double sp = 0;
    float us = isolated(bytes, false, 1.0, 9, &sp);
    std::printf("static           isolated %8.2f us %7.1f GB/s | graph b2b %8.2f us\n", us,
                bytes / (us * 1e-6) / 1e9, graphed(bytes, false, 1.0, false));
    for (double frac : {0.0, 0.5, 0.75, 0.9}) {
      us = isolated(bytes, true, frac, 9, &sp);
      const float gb = graphed(bytes, true, frac, false);
      std::printf("steal %.2f       isolated %8.2f us %7.1f GB/s | graph b2b %8.2f us %7.1f GB/s\n", frac, us,
                  bytes / (us * 1e-6) / 1e9, gb, bytes / (gb * 1e-6) / 1e9);
    }
    const float gp = graphed(bytes, false, 1.0, true);
    std::printf("pdl static       graph b2b %8.2f us %7.1f GB/s\n", gp, bytes / (gp * 1e-6) / 1e9);
    const float gps = graphed(bytes, true, 0.75, true);
    std::printf("pdl steal 0.75   graph b2b %8.2f us %7.1f GB/s\n", gps, bytes / (gps * 1e-6) / 1e9);
  }
  return 0;
}
