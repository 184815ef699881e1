// kern_sum.cu — kernel families for the 2-level sum nests (sumRows / sumCols and the weighted
// variants), one family per mapping class (§IV-E: "depending on the mapping decision our
// code generator selects the appropriate template"):
//
//   RX  inner Reduce on x   — Fig 9: x-threads stride along the inner pattern, a warp-
//                             synchronous tree (here: shuffles) combines them. With the
//                             inner level on a strided dimension this is also the thread-block/thread
//                             and warp-based mappings of Fig 7 (uncoalesced for sumCols).
//   MX  outer Map on x, inner Reduce on y — the sumCols mapping of P:L596-600: adjacent x-threads own
//                             adjacent columns so every row segment is one coalesced request; y-threads
//                             split the rows and meet in shared memory. With by = 1 this is the 1D
//                             mapping of Fig 2.
//   Split(k) on the inner level (Fig 6c): every block writes its partial to the plan's
//   workspace [gi x O]; the last block of an outer tile (atomic ticket) adds the k partials in order
//   s = 0..k-1 and writes the output — the paper's combiner kernel fused into the same
//   launch, deterministic, and the ticket is reset so the workspace stays reusable.
//
// Index semantics (G11/S9): level block g covers the contiguous range [g*chunk, (g+1)*chunk);
// thread t covers base + t*V + j*b*V (+0..V-1). The grid is linearised: blockIdx.x = s*go + g_outer
// (outer tiles of one inner chunk are adjacent in launch order, so concurrently running blocks read
// neighbouring column segments of the same rows).
//
// Accumulation: fp32 inputs are added in fp32 along a pairwise tree over at most one unrolled batch
// (<= 32 elements per lane) and in fp64 across batches, lanes and blocks; integers in unsigned
// arithmetic of the element width (wraps mod 2^w, G19).
#include <cstdint>

#include "kernels.hpp"

namespace npp {

namespace {

template <typename T> struct AccOf;
template <> struct AccOf<float> { using type = double; };
template <> struct AccOf<int32_t> { using type = unsigned int; };
template <> struct AccOf<int64_t> { using type = unsigned long long; };
template <> struct AccOf<double> { using type = double; };

constexpr int kUnroll = 8;

// ---------------------------------------------------------------- streaming loads (read-only, no L1 allocate)
template <typename T, int V> struct Vec { T v[V]; };

__device__ __forceinline__ void ldg_stream(const float* p, Vec<float, 4>& r) {
  asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]) : "l"(p));
}
__device__ __forceinline__ void ldg_stream(const int32_t* p, Vec<int32_t, 4>& r) {
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]) : "l"(p));
}
__device__ __forceinline__ void ldg_stream(const int64_t* p, Vec<int64_t, 2>& r) {
  long long a, b;
  asm volatile("ld.global.nc.L1::no_allocate.v2.s64 {%0,%1}, [%2];" : "=l"(a), "=l"(b) : "l"(p));
  r.v[0] = a;
  r.v[1] = b;
}
__device__ __forceinline__ void ldg_stream(const double* p, Vec<double, 2>& r) {
  asm volatile("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(r.v[0]), "=d"(r.v[1]) : "l"(p));
}
template <typename T>
__device__ __forceinline__ void ldg_stream(const T* p, Vec<T, 1>& r) { r.v[0] = __ldg(p); }

// ---------------------------------------------------------------- accumulation helpers
template <typename T> struct Ops;

template <> struct Ops<float> {
  using Acc = double;
  using Part = float;  // pairwise fp32 inside one batch
  __device__ static Part mul(float a, float w) { return a * w; }
  __device__ static Part add(Part a, Part b) { return a + b; }
  __device__ static Acc widen(Part p) { return double(p); }
  __device__ static Part from(float x) { return x; }
  __device__ static float finish(Acc a) { return float(a); }
};
template <> struct Ops<double> {
  using Acc = double;
  using Part = double;  // pairwise fp64 inside one batch, fp64 across
  __device__ static Part mul(double a, double w) { return a * w; }
  __device__ static Part add(Part a, Part b) { return a + b; }
  __device__ static Acc widen(Part p) { return p; }
  __device__ static Part from(double x) { return x; }
  __device__ static double finish(Acc a) { return a; }
};
template <> struct Ops<int32_t> {
  using Acc = unsigned int;
  using Part = unsigned int;
  __device__ static Part mul(int32_t a, int32_t w) { return unsigned(a) * unsigned(w); }
  __device__ static Part add(Part a, Part b) { return a + b; }
  __device__ static Acc widen(Part p) { return p; }
  __device__ static Part from(int32_t x) { return unsigned(x); }
  __device__ static int32_t finish(Acc a) { return int32_t(a); }
};
template <> struct Ops<int64_t> {
  using Acc = unsigned long long;
  using Part = unsigned long long;
  __device__ static Part mul(int64_t a, int64_t w) {
    return (unsigned long long)a * (unsigned long long)w;
  }
  __device__ static Part add(Part a, Part b) { return a + b; }
  __device__ static Acc widen(Part p) { return p; }
  __device__ static Part from(int64_t x) { return (unsigned long long)x; }
  __device__ static int64_t finish(Acc a) { return int64_t(a); }
};

// pairwise tree over N values (N a power of two)
template <typename T, int N>
__device__ __forceinline__ typename Ops<T>::Part tree(typename Ops<T>::Part (&p)[N]) {
#pragma unroll
  for (int w = N / 2; w >= 1; w /= 2) {
#pragma unroll
    for (int i = 0; i < w; ++i) p[i] = Ops<T>::add(p[i], p[i + w]);
  }
  return p[0];
}

template <typename T>
__device__ __forceinline__ T ld_any(const T* p) { return __ldg(p); }

// ---------------------------------------------------------------- Split(k) combine (fused combiner)
template <typename T>
__device__ void split_combine(const SumArgs& a, int64_t g_outer, int64_t o_begin, int64_t o_end) {
  using Acc = typename Ops<T>::Acc;
  __shared__ unsigned s_is_last;
  const int tid = threadIdx.y * blockDim.x + threadIdx.x;
  const int nt = blockDim.x * blockDim.y;
  __threadfence();  // publish this block's partials device-wide before taking a ticket
  __syncthreads();
  if (tid == 0) {
    const unsigned t = atomicAdd(a.tickets + g_outer, 1u);
    s_is_last = (t == unsigned(a.gi - 1));
  }
  __syncthreads();
  if (!s_is_last) return;
  __threadfence();
  const Acc* part = static_cast<const Acc*>(a.partials);
  T* out = static_cast<T*>(a.out);
  for (int64_t o = o_begin + tid; o < o_end; o += nt) {
    Acc sum = 0;
    for (int64_t k = 0; k < a.gi; ++k) sum += __ldcg(part + k * a.O + o);  // fixed order s = 0..k-1
    out[o] = Ops<T>::finish(sum);
  }
  if (tid == 0) a.tickets[g_outer] = 0u;  // leave the workspace zeroed for the next execute
}

template <typename T>
__device__ __forceinline__ void emit(const SumArgs& a, int64_t s, int64_t o, typename Ops<T>::Acc acc) {
  using Acc = typename Ops<T>::Acc;
  if (a.gi == 1)
    static_cast<T*>(a.out)[o] = Ops<T>::finish(acc);
  else
    static_cast<Acc*>(a.partials)[s * a.O + o] = acc;
}

}  // namespace

// ====================================================================================== class RX
// block (bi x bo): x = inner (bi threads, V elements each per load), y = outer.
template <typename T, int V, bool W>
__global__ void __launch_bounds__(1024) npp_sum_rx_kernel(SumArgs a) {
  using O_ = Ops<T>;
  using Acc = typename O_::Acc;
  using Part = typename O_::Part;
  extern __shared__ unsigned char smem_raw[];
  Acc* red = reinterpret_cast<Acc*>(smem_raw);  // [bo][bi/32] when bi > 32

  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t bid = blockIdx.x;
  const int64_t g_outer = bid % a.go, s = bid / a.go;
  const int64_t o_begin = g_outer * a.co;
  const int64_t o_end = min(a.O, o_begin + a.co);
  const int64_t i_begin = s * a.ci;
  const int64_t i_end = min(a.I, i_begin + a.ci);
  const T* __restrict__ m = static_cast<const T*>(a.m);
  const T* __restrict__ wv = static_cast<const T*>(a.v);
  const int64_t step = int64_t(a.bi) * V;
  const int nrep = int((a.co + a.bo - 1) / a.bo);
  const int warps_x = (a.bi + 31) / 32;
  // lanes that exist in this thread's warp (blocks smaller than a warp, e.g. TB/T on a 1-wide row)
  const int flat = ty * a.bi + tx;
  const int nthreads = a.bi * a.bo;
  const int lanes = min(32, nthreads - (flat & ~31));
  const unsigned lane_mask = lanes == 32 ? 0xffffffffu : ((1u << lanes) - 1u);

  for (int j = 0; j < nrep; ++j) {
    const int64_t o = o_begin + ty + int64_t(j) * a.bo;
    const bool valid = o < o_end;
    Acc acc = 0;
    if (valid) {
      const T* row = m + o * a.so;
      int64_t i = i_begin + int64_t(tx) * V;
      // full unrolled batches: kUnroll independent loads in flight per lane, then a pairwise tree
      for (; i + (kUnroll - 1) * step < i_end; i += kUnroll * step) {
        Vec<T, V> r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          if constexpr (V > 1)
            ldg_stream(row + (i + u * step), r[u]);
          else
            r[u].v[0] = ld_any(row + (i + u * step) * a.si);
        }
        Part p[kUnroll * V];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
#pragma unroll
          for (int e = 0; e < V; ++e) {
            if constexpr (W)
              p[u * V + e] = O_::mul(r[u].v[e], ld_any(wv + i + u * step + e));
            else
              p[u * V + e] = O_::from(r[u].v[e]);
          }
        }
        acc += O_::widen(tree<T, kUnroll * V>(p));
      }
      for (; i < i_end; i += step) {
        Vec<T, V> r;
        if constexpr (V > 1)
          ldg_stream(row + i, r);
        else
          r.v[0] = ld_any(row + i * a.si);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          if constexpr (W)
            acc += O_::widen(O_::mul(r.v[e], ld_any(wv + i + e)));
          else
            acc += O_::widen(O_::from(r.v[e]));
        }
      }
    }
    // reduce across the bi x-threads of this outer index (warp-synchronous tree)
    const int width = a.bi < 32 ? a.bi : 32;
    for (int off = width / 2; off >= 1; off /= 2) acc += __shfl_xor_sync(lane_mask, acc, off);
    if (warps_x > 1) {
      if ((tx & 31) == 0) red[ty * warps_x + (tx >> 5)] = acc;
      __syncthreads();
      if (tx == 0) {
        acc = red[ty * warps_x];
        for (int w = 1; w < warps_x; ++w) acc += red[ty * warps_x + w];
      }
      __syncthreads();
    }
    if (tx == 0 && valid) emit<T>(a, s, o, acc);
  }
  if (a.gi > 1) split_combine<T>(a, g_outer, o_begin, o_end);
}

// ====================================================================================== class MX
// block (bo x bi): x = outer (bo threads, V adjacent outer indices each), y = inner.
template <typename T, int V, bool W>
__global__ void __launch_bounds__(1024) npp_sum_mx_kernel(SumArgs a) {
  using O_ = Ops<T>;
  using Acc = typename O_::Acc;
  using Part = typename O_::Part;
  extern __shared__ unsigned char smem_raw[];
  Acc* red = reinterpret_cast<Acc*>(smem_raw);  // [bi][bo*V] when bi > 1

  const int tx = threadIdx.x, ty = threadIdx.y;
  const int64_t bid = blockIdx.x;
  const int64_t g_outer = bid % a.go, s = bid / a.go;
  const int64_t o_begin = g_outer * a.co;
  const int64_t o_end = min(a.O, o_begin + a.co);
  const int64_t i_begin = s * a.ci;
  const int64_t i_end = min(a.I, i_begin + a.ci);
  const T* __restrict__ m = static_cast<const T*>(a.m);
  const T* __restrict__ wv = static_cast<const T*>(a.v);
  const int64_t per_rep = int64_t(a.bo) * V;
  const int nrep = int((a.co + per_rep - 1) / per_rep);
  const int ncol = a.bo * V;

  for (int j = 0; j < nrep; ++j) {
    const int64_t o0 = o_begin + int64_t(j) * per_rep + int64_t(tx) * V;
    const bool valid = o0 < o_end;
    Acc acc[V];
#pragma unroll
    for (int e = 0; e < V; ++e) acc[e] = 0;
    if (valid) {
      const T* col = m + o0 * a.so;
      int64_t i = i_begin + ty;
      const int64_t step = a.bi;
      for (; i + (kUnroll - 1) * step < i_end; i += kUnroll * step) {
        Vec<T, V> r[kUnroll];
#pragma unroll
        for (int u = 0; u < kUnroll; ++u) {
          if constexpr (V > 1)
            ldg_stream(col + (i + u * step) * a.si, r[u]);
          else
            r[u].v[0] = ld_any(col + (i + u * step) * a.si);
        }
#pragma unroll
        for (int e = 0; e < V; ++e) {
          Part p[kUnroll];
#pragma unroll
          for (int u = 0; u < kUnroll; ++u) {
            if constexpr (W)
              p[u] = O_::mul(r[u].v[e], ld_any(wv + i + u * step));
            else
              p[u] = O_::from(r[u].v[e]);
          }
          acc[e] += O_::widen(tree<T, kUnroll>(p));
        }
      }
      for (; i < i_end; i += step) {
        Vec<T, V> r;
        if constexpr (V > 1)
          ldg_stream(col + i * a.si, r);
        else
          r.v[0] = ld_any(col + i * a.si);
#pragma unroll
        for (int e = 0; e < V; ++e) {
          if constexpr (W)
            acc[e] += O_::widen(O_::mul(r.v[e], ld_any(wv + i)));
          else
            acc[e] += O_::widen(O_::from(r.v[e]));
        }
      }
    }
    if (a.bi > 1) {  // combine the y-threads through shared memory, in fixed order t = 0..bi-1
#pragma unroll
      for (int e = 0; e < V; ++e) red[ty * ncol + tx * V + e] = acc[e];
      __syncthreads();
      if (ty == 0) {
#pragma unroll
        for (int e = 0; e < V; ++e) {
          Acc sum = red[tx * V + e];
          for (int t = 1; t < a.bi; ++t) sum += red[t * ncol + tx * V + e];
          acc[e] = sum;
        }
      }
      __syncthreads();
    }
    if (ty == 0 && valid) {
#pragma unroll
      for (int e = 0; e < V; ++e)
        if (o0 + e < o_end) emit<T>(a, s, o0 + e, acc[e]);
    }
  }
  if (a.gi > 1) split_combine<T>(a, g_outer, o_begin, o_end);
}

// ====================================================================================== launch
namespace {

template <typename T, int V, bool W>
cudaError_t launch_t(int kclass, const SumArgs& a, dim3 grid, dim3 block, size_t smem, cudaStream_t st) {
  if (kclass == NPP_CLASS_RX)
    npp_sum_rx_kernel<T, V, W><<<grid, block, smem, st>>>(a);
  else
    npp_sum_mx_kernel<T, V, W><<<grid, block, smem, st>>>(a);
  return cudaGetLastError();
}

template <typename T, int V0>
cudaError_t launch_v(int kclass, int vec, bool weighted, const SumArgs& a, dim3 g, dim3 b, size_t smem,
                     cudaStream_t st) {
  if (vec == V0) return weighted ? launch_t<T, V0, true>(kclass, a, g, b, smem, st)
                                 : launch_t<T, V0, false>(kclass, a, g, b, smem, st);
  return weighted ? launch_t<T, 1, true>(kclass, a, g, b, smem, st)
                  : launch_t<T, 1, false>(kclass, a, g, b, smem, st);
}

}  // namespace

cudaError_t launch_sum(int dtype, int kclass, int vec, bool weighted, const SumArgs& a, cudaStream_t st) {
  const int acc = dtype == NPP_I32 ? 4 : 8;
  dim3 grid(unsigned(a.go * a.gi));
  dim3 block;
  size_t smem = 0;
  if (kclass == NPP_CLASS_RX) {
    block = dim3(unsigned(a.bi), unsigned(a.bo));
    if (a.bi > 32) smem = size_t(a.bo) * ((a.bi + 31) / 32) * acc;
  } else {
    block = dim3(unsigned(a.bo), unsigned(a.bi));
    if (a.bi > 1) smem = size_t(a.bi) * a.bo * vec * acc;
  }
  switch (dtype) {
    case NPP_F32: return launch_v<float, 4>(kclass, vec, weighted, a, grid, block, smem, st);
    case NPP_I32: return launch_v<int32_t, 4>(kclass, vec, weighted, a, grid, block, smem, st);
    case NPP_F64: return launch_v<double, 2>(kclass, vec, weighted, a, grid, block, smem, st);
    default: return launch_v<int64_t, 2>(kclass, vec, weighted, a, grid, block, smem, st);
  }
}

// ====================================================================================== S10 temp family
// The weighted sums with their inner zipWith materialised (Fig 15; §V-A):
// phase A writes t(o, i) = m[o, i]·v[i] into the inner allocation, phase B reduces it — the code the
// paper's compiler generates, kept to reproduce Fig 16. MALLOC: one device malloc per outer iteration
// (per block chunk), by the thread with inner index 0, shared through shared memory and freed after
// the reduce; PREALLOC: one [O x I] buffer of the workspace at o*ts_o + i*ts_i (Fig 11a / 11b). The
// block is the record's (RXC: x = inner; else x = outer), scalar accesses (vec = 1), the inner threads
// meet in a shared-memory tree, Split(k) partials combine as in the other families.
template <typename T, bool RXC, bool MALLOC>
__global__ void __launch_bounds__(1024) npp_sum_temp_kernel(SumArgs a) {
  using O_ = Ops<T>;
  using Acc = typename O_::Acc;
  extern __shared__ unsigned char smem_raw[];
  const int to = RXC ? threadIdx.y : threadIdx.x;  // outer-thread index
  const int ti = RXC ? threadIdx.x : threadIdx.y;  // inner-thread index
  const int nbo = a.bo, nbi = a.bi;
  Acc* red = reinterpret_cast<Acc*>(smem_raw);                       // [nbo][nbi]
  T** ptrs = reinterpret_cast<T**>(red + size_t(nbo) * nbi);         // [nbo] (MALLOC)
  const int64_t bid = blockIdx.x;
  const int64_t g_outer = bid % a.go, s = bid / a.go;
  const int64_t o_begin = g_outer * a.co;
  const int64_t o_end = min(a.O, o_begin + a.co);
  const int64_t i_begin = s * a.ci;
  const int64_t i_end = min(a.I, i_begin + a.ci);
  const T* __restrict__ m = static_cast<const T*>(a.m);
  const T* __restrict__ wv = static_cast<const T*>(a.v);
  T* temp = static_cast<T*>(a.temp);
  const int nrep = int((a.co + nbo - 1) / nbo);
  int wtop = 1;
  while (wtop < nbi) wtop <<= 1;
  for (int j = 0; j < nrep; ++j) {
    const int64_t o = o_begin + to + int64_t(j) * nbo;
    const bool valid = o < o_end;
    T* buf = nullptr;
    if constexpr (MALLOC) {
      if (ti == 0) {
        T* p = nullptr;
        if (valid && i_end > i_begin) {
          p = static_cast<T*>(malloc(size_t(i_end - i_begin) * sizeof(T)));
          if (!p) atomicExch(a.err, 1u);
        }
        ptrs[to] = p;
      }
      __syncthreads();
      buf = ptrs[to];
    }
    const bool work = valid && (!MALLOC || buf != nullptr);
    if (work)  // phase A: temp = c zipWith v (the inner Map's allocation)
      for (int64_t i = i_begin + ti; i < i_end; i += nbi) {
        const T x = T(O_::mul(m[o * a.so + i * a.si], __ldg(wv + i)));
        if constexpr (MALLOC)
          buf[i - i_begin] = x;
        else
          temp[o * a.ts_o + i * a.ts_i] = x;
      }
    __syncthreads();
    Acc acc = 0;
    if (work)  // phase B: temp reduce +
      for (int64_t i = i_begin + ti; i < i_end; i += nbi) {
        T x;
        if constexpr (MALLOC)
          x = buf[i - i_begin];
        else
          x = temp[o * a.ts_o + i * a.ts_i];
        acc += O_::widen(O_::from(x));
      }
    red[to * nbi + ti] = acc;
    __syncthreads();
    for (int w = wtop >> 1; w >= 1; w >>= 1) {
      if (ti < w && ti + w < nbi) red[to * nbi + ti] += red[to * nbi + ti + w];
      __syncthreads();
    }
    if (ti == 0 && valid) emit<T>(a, s, o, red[to * nbi]);
    __syncthreads();
    if constexpr (MALLOC) {
      if (ti == 0 && buf) free(buf);
    }
  }
  if (a.gi > 1) split_combine<T>(a, g_outer, o_begin, o_end);
}

template <typename T>
static cudaError_t launch_temp_t(int kclass, bool malloc_mode, const SumArgs& a, dim3 grid, dim3 block, size_t smem,
                                 cudaStream_t st) {
  const bool rx = kclass == NPP_CLASS_RX;
  if (rx && malloc_mode)
    npp_sum_temp_kernel<T, true, true><<<grid, block, smem, st>>>(a);
  else if (rx)
    npp_sum_temp_kernel<T, true, false><<<grid, block, smem, st>>>(a);
  else if (malloc_mode)
    npp_sum_temp_kernel<T, false, true><<<grid, block, smem, st>>>(a);
  else
    npp_sum_temp_kernel<T, false, false><<<grid, block, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_sum_temp(int dtype, int kclass, bool malloc_mode, const SumArgs& a, cudaStream_t st) {
  const int acc = dtype == NPP_I32 ? 4 : 8;
  dim3 grid(unsigned(a.go * a.gi));
  dim3 block = kclass == NPP_CLASS_RX ? dim3(unsigned(a.bi), unsigned(a.bo)) : dim3(unsigned(a.bo), unsigned(a.bi));
  const size_t smem = size_t(a.bo) * a.bi * acc + size_t(a.bo) * sizeof(void*);
  switch (dtype) {
    case NPP_F32: return launch_temp_t<float>(kclass, malloc_mode, a, grid, block, smem, st);
    case NPP_I32: return launch_temp_t<int32_t>(kclass, malloc_mode, a, grid, block, smem, st);
    case NPP_F64: return launch_temp_t<double>(kclass, malloc_mode, a, grid, block, smem, st);
    default: return launch_temp_t<int64_t>(kclass, malloc_mode, a, grid, block, smem, st);
  }
}

template <typename T, int V, bool W>
static void add_attr(int* regs) {
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, npp_sum_rx_kernel<T, V, W>) == cudaSuccess && fa.numRegs > *regs)
    *regs = fa.numRegs;
  if (cudaFuncGetAttributes(&fa, npp_sum_mx_kernel<T, V, W>) == cudaSuccess && fa.numRegs > *regs)
    *regs = fa.numRegs;
}

int sum_kernels_max_regs() {
  int regs = 0;
  add_attr<float, 4, false>(&regs);
  add_attr<float, 1, false>(&regs);
  add_attr<int32_t, 4, false>(&regs);
  add_attr<int32_t, 1, false>(&regs);
  add_attr<int64_t, 2, false>(&regs);
  add_attr<int64_t, 1, false>(&regs);
  add_attr<float, 4, true>(&regs);
  add_attr<float, 1, true>(&regs);
  add_attr<int32_t, 4, true>(&regs);
  add_attr<int32_t, 1, true>(&regs);
  add_attr<int64_t, 2, true>(&regs);
  add_attr<int64_t, 1, true>(&regs);
  add_attr<double, 2, false>(&regs);
  add_attr<double, 1, false>(&regs);
  add_attr<double, 2, true>(&regs);
  add_attr<double, 1, true>(&regs);
  return regs;
}

}  // namespace npp
