// kern_rowscols.cu — sumRows and sumCols of one matrix in ONE pass over it (class RC, S8 "RC").
//
// The Naive Bayes classifier of PAPER.md §VI-E "calculates both the number of words per
// document and the number of documents for each ... word": two nested patterns with different access
// patterns over the same matrix. The paper maps each kernel separately (1D "can only satisfy one of the
// access patterns", MultiDim optimises both). On B200 both outputs are formed from a single HBM read:
// every 32-row x 1 KB tile is staged once (TMA, as the sumRows/sumCols staged family) and reduced in
// both directions out of shared memory, which halves the bytes of the two-kernel schedule.
//
// Work split (S8 RC): the Tr x Tc tile grid is cut into gr x gc rectangular regions of
// cr row bands x cc column tiles; block b of G takes regions [b*nreg/G, (b+1)*nreg/G). Inside a region
// the walk is row-band-major:
//   columns: thread t owns column t of every tile (two row halves for 8-byte types); its per-tile
//            column partial (a pairwise tree over the tile's rows) is added to a shared-memory
//            accumulator slot of the region's columns (<= 32 tiles = 64 KB), flushed at region end;
//   rows:    each warp turns its per-thread row values into per-row partials with one transposing
//            butterfly (lane l ends with row l), keeps them in a register across the band's column
//            tiles, and the eight warps meet in shared memory once per band.
// A row band (column region) covered by several regions is the Split of P:L542-550: contributions meet
// through fp64 / integer atomics and one ticket per row region (column group), taken once at region
// end; the last contributor converts and re-zeroes (the combiner of P:L880-883, fused). gc == 1 rows and gr == 1 columns are
// written directly. Without 16-B row pitch (no tensor map) the same consumers load the tile straight
// from global memory (STAGED = false; the producer warp idles).
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>

#include "kernels.hpp"
#include "tma_ring.cuh"

namespace npp {

namespace {

using namespace tma;

constexpr int kStages = 4;
constexpr int kTileRows = 32;
constexpr int kTileBytes = kTileRows * 1024;
constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kThreads = kConsumers + 32;  // + producer warp
constexpr int kHeader = 1024;
constexpr int kColTilesMax = 32;          // column tiles of one region (select.hpp kRcColTilesMax)
constexpr int kColAccBytes = 64 * 1024;   // [row groups][kColTilesMax * BC] accumulators
constexpr int kRowSumBytes = 2 * kConsumerWarps * 32 * 8;
constexpr int kSmemBytes = kHeader + kStages * kTileBytes + kColAccBytes + kRowSumBytes;

template <typename T> struct RcOps;
template <> struct RcOps<float> {
  using S = float;   // in-tile arithmetic
  using Acc = double;
  __device__ static float finish(double a) { return float(a); }
};
template <> struct RcOps<double> {
  using S = double;
  using Acc = double;
  __device__ static double finish(double a) { return a; }
};
template <> struct RcOps<int32_t> {
  using S = unsigned;
  using Acc = unsigned;
  __device__ static int32_t finish(unsigned a) { return int32_t(a); }
};
template <> struct RcOps<int64_t> {
  using S = unsigned long long;
  using Acc = unsigned long long;
  __device__ static int64_t finish(unsigned long long a) { return int64_t(a); }
};

// N values per lane -> the lane holds Σ over the 32 lanes of value (lane % N): log2 N transposing
// steps (a lane keeps the half its bit selects and receives the partner's copy of it), then plain
// butterfly steps for the lane bits above N. For floats the additions form a pairwise tree.
template <int N, typename S>
__device__ __forceinline__ S transpose_reduce(S (&v)[N], int lane) {
#pragma unroll
  for (int h = N / 2; h >= 1; h /= 2) {
    const bool up = (lane & h) != 0;
#pragma unroll
    for (int i = 0; i < h; ++i) {
      const S send = up ? v[i] : v[i + h];
      const S keep = up ? v[i + h] : v[i];
      v[i] = keep + __shfl_xor_sync(0xffffffffu, send, h);
    }
  }
#pragma unroll
  for (int o = N; o < 32; o *= 2) v[0] += __shfl_xor_sync(0xffffffffu, v[0], o);
  return v[0];
}

template <int N, typename S>
__device__ __forceinline__ S tree_sum(const S (&v)[N]) {
  S t[N / 2];
#pragma unroll
  for (int i = 0; i < N / 2; ++i) t[i] = v[2 * i] + v[2 * i + 1];
#pragma unroll
  for (int w = N / 4; w >= 1; w /= 2)
#pragma unroll
    for (int i = 0; i < w; ++i) t[i] = t[i] + t[i + w];
  return t[0];
}

__device__ __forceinline__ void consumers_sync() { asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory"); }

}  // namespace

template <typename T, bool STAGED>
__global__ void __launch_bounds__(kThreads, 1)
    npp_rowscols_kernel(const __grid_constant__ CUtensorMap map, const RowsColsArgs a) {
  using S = typename RcOps<T>::S;
  using Acc = typename RcOps<T>::Acc;
  constexpr int BC = 1024 / int(sizeof(T));  // columns of a tile
  constexpr int WPG = BC / 32;               // warps across a tile's columns (8 or 4)
  constexpr int NRG = kConsumerWarps / WPG;  // row groups (1 or 2)
  constexpr int RPT = kTileRows / NRG;       // tile rows one thread adds (32 or 16)
  constexpr int CAP = kColTilesMax * BC;     // column accumulators per row group
  static_assert(NRG * CAP * int(sizeof(Acc)) <= kColAccBytes, "column accumulators exceed their region");
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kStages;
  volatile int* flag = reinterpret_cast<volatile int*>(empty + kStages);
  unsigned char* tiles = smem + kHeader;
  Acc* colacc = reinterpret_cast<Acc*>(tiles + kStages * kTileBytes);  // [NRG][CAP]
  Acc* rsum = reinterpret_cast<Acc*>(tiles + kStages * kTileBytes + kColAccBytes);  // [2][8][32]
  Acc* accR = static_cast<Acc*>(a.accR);
  Acc* accC = static_cast<Acc*>(a.accC);
  T* out = static_cast<T*>(a.out);

  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x, G = gridDim.x;
  const long long q0 = bid * a.nreg / G, q1 = (bid + 1) * a.nreg / G;
#ifndef NPP_RC_EARLY_ISSUE
#define NPP_RC_EARLY_ISSUE 1
#endif
  // the producer lane initialises the ring and issues its first kStages tiles before the block barrier,
  // so they load while the consumers zero the column accumulators
  constexpr bool kEarly = STAGED && NPP_RC_EARLY_ISSUE;
  const int init_thread = kEarly ? kConsumers : 0;
  auto tile_rc = [&](long long q, long long* b0, long long* b1, long long* c0, long long* c1) {
    const long long ri = q / a.gc, cj = q - ri * a.gc;
    *b0 = ri * a.cr, *b1 = *b0 + a.cr < a.Tr ? *b0 + a.cr : a.Tr;
    *c0 = cj * a.cc, *c1 = *c0 + a.cc < a.Tc ? *c0 + a.cc : a.Tc;
  };
  long long early = 0;
  if (threadIdx.x == init_thread) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(full + i, 1);
      mbar_init(empty + i, kConsumerWarps);
    }
    mbar_fence_init();
    if (kEarly) {
      prefetch_map(&map);
      if (!a.early_reads) asm volatile("griddepcontrol.wait;" ::: "memory");
      for (long long q = q0; q < q1 && early < kStages; ++q) {
        long long b0, b1, c0, c1;
        tile_rc(q, &b0, &b1, &c0, &c1);
        for (long long br = b0; br < b1 && early < kStages; ++br)
          for (long long ct = c0; ct < c1 && early < kStages; ++ct, ++early) {
            NPP_CHECK(br < a.Tr && ct < a.Tc && q < a.nreg);
            mbar_expect_tx(full + early, kTileBytes);
            load_2d(tiles + early * kTileBytes, &map, int(ct * BC), int(br * kTileRows), full + early);
          }
      }
    }
  }
  if (threadIdx.x < kConsumers)
    for (int i = threadIdx.x; i < NRG * CAP; i += kConsumers) colacc[i] = Acc(0);
  __syncthreads();

  if (warp == kConsumerWarps) {
    // ------------------------------------------------------------ producer: one elected lane
    if (STAGED && lane == 0) {
      if (!kEarly) {
        prefetch_map(&map);
        if (!a.early_reads) asm volatile("griddepcontrol.wait;" ::: "memory");
      }
      long long t = 0;
      for (long long q = q0; q < q1; ++q) {
        long long b0, b1, c0, c1;
        tile_rc(q, &b0, &b1, &c0, &c1);
        for (long long br = b0; br < b1; ++br)
          for (long long ct = c0; ct < c1; ++ct, ++t) {
            if (t < early) continue;  // issued before the block barrier
            const int slot = int(t % kStages);
            if (t >= kStages) mbar_wait(empty + slot, unsigned((t / kStages) & 1) ^ 1u);
            mbar_expect_tx(full + slot, kTileBytes);
            load_2d(tiles + slot * kTileBytes, &map, int(ct * BC), int(br * kTileRows), full + slot);
          }
      }
    }
    return;
  }

  // -------------------------------------------------------------- consumers
  const int rg = warp / WPG;                 // row group: tile rows rg*RPT .. +RPT
  const int col = (warp % WPG) * 32 + lane;  // tile column
  bool waited = false;
  long long t = 0;
  int rb = 0;  // rsum double buffer
  for (long long q = q0; q < q1; ++q) {
    if (a.trace && threadIdx.x == 0) {  // white-box schedule trace: who took region q
      a.trace[q] = int(blockIdx.x);
      atomicAdd(a.trace + a.nreg + q, 1);
    }
    const long long ri = q / a.gc, cj = q - ri * a.gc;
    const long long b0 = ri * a.cr, b1 = b0 + a.cr < a.Tr ? b0 + a.cr : a.Tr;
    const long long c0 = cj * a.cc, c1 = c0 + a.cc < a.Tc ? c0 + a.cc : a.Tc;
    for (long long br = b0; br < b1; ++br) {
      Acc racc = Acc(0);
      for (long long ct = c0; ct < c1; ++ct, ++t) {
        S v[RPT];
        if constexpr (STAGED) {
          const int slot = int(t % kStages);
          mbar_wait(full + slot, unsigned((t / kStages) & 1));
          const T* tile = reinterpret_cast<const T*>(tiles + slot * kTileBytes);
#pragma unroll
          for (int rr = 0; rr < RPT; ++rr) v[rr] = S(tile[(rg * RPT + rr) * BC + col]);
          __syncwarp();
          if (lane == 0) mbar_arrive(empty + slot);
        } else {
          if (!waited) {
            asm volatile("griddepcontrol.wait;" ::: "memory");
            waited = true;
          }
          const long long c = ct * BC + col;
          const long long r0 = br * kTileRows + rg * RPT;
          const T* m = static_cast<const T*>(a.m);
#pragma unroll
          for (int rr = 0; rr < RPT; ++rr)
            v[rr] = (c < a.C && r0 + rr < a.R) ? S(__ldg(m + (r0 + rr) * a.C + c)) : S(0);
        }
        colacc[rg * CAP + (ct - c0) * BC + col] += Acc(tree_sum(v));
        racc += Acc(transpose_reduce(v, lane));  // lane l: row rg*RPT + l % RPT of this band
      }
      // ---- band end: the warps' row partials meet in shared memory
      if (!waited) {  // out / workspace are written only after the previous grid in the stream is done
        asm volatile("griddepcontrol.wait;" ::: "memory");
        waited = true;
      }
      rsum[(rb * kConsumerWarps + warp) * 32 + lane] = racc;
      consumers_sync();
      if (warp == 0) {
        const int g = lane / RPT, li = lane % RPT;
        Acc s = Acc(0);
#pragma unroll
        for (int j = 0; j < WPG; ++j) s += rsum[(rb * kConsumerWarps + g * WPG + j) * 32 + li];
        const long long row = br * kTileRows + lane;
        if (row < a.R) {
#if defined(NPP_RC_NO_COMBINE) || defined(NPP_RC_NO_ROWRED)  // measurement variants (wrong results)
          out[row] = RcOps<T>::finish(s);
#else
          if (a.gc == 1)
            out[row] = RcOps<T>::finish(s);
          else
            atomicAdd(accR + row, s);  // completed by the row-region ticket at region end
#endif
        }
      }
      rb ^= 1;
    }
    // ---- region end: the region's column accumulators
    consumers_sync();
    const long long ncols = (c1 - c0) * BC;
    for (long long c = threadIdx.x; c < ncols; c += kConsumers) {
      Acc s = colacc[c];
      colacc[c] = Acc(0);
      if constexpr (NRG == 2) {
        s += colacc[CAP + c];
        colacc[CAP + c] = Acc(0);
      }
      const long long cg = c0 * BC + c;
      if (cg < a.C) {
#if defined(NPP_RC_NO_COMBINE) || defined(NPP_RC_NO_COLRED)
        out[a.R + cg] = RcOps<T>::finish(s);
#else
        if (a.gr == 1)
          out[a.R + cg] = RcOps<T>::finish(s);
        else
          atomicAdd(accC + cg, s);
#endif
      }
    }
#ifdef NPP_RC_NO_COMBINE
    consumers_sync();
    continue;
#endif
    // Split combine (fused): one fence and one ticket per region and direction. The gc
    // column regions of row region ri add their row partials (band ends above), the gr row regions of
    // column group cj their column partials; the last of each converts and re-zeroes.
    if (a.gr > 1 || a.gc > 1) {
      consumers_sync();
      // acq_rel tickets (the release of every consumer's adds, ordered by the barrier above), the row and
      // the column ticket taken by two warps at once (their round trips overlap)
      if (threadIdx.x == 0) {
        bool last_r = false;
        if (a.gc > 1) {
          last_r = ticket_add(a.tick_r + ri, 1u) + 1u == unsigned(a.gc);
          if (last_r) a.tick_r[ri] = 0u;
        }
        flag[0] = last_r ? 1 : 0;
      } else if (threadIdx.x == 32) {
        bool last_c = false;
        if (a.gr > 1) {
          last_c = ticket_add(a.tick_c + cj, 1u) + 1u == unsigned(a.gr);
          if (last_c) a.tick_c[cj] = 0u;
        }
        flag[1] = last_c ? 1 : 0;
      }
      consumers_sync();
      // no further fence: the ticket atomics were acq_rel (the acquire of every other region's adds) and the
      // barrier above orders this block's threads after them; the reads below go to L2 (ld.cg)
      const bool last_r = flag[0] != 0, last_c = flag[1] != 0;
      // the conversions issue all of a thread's loads before any store: one L2 round trip, not one per
      // element (a region has <= 32 * 256 columns: <= 32 per thread; its rows <= kConsumers per pass)
      // a block may complete both its row region and its column group: both conversions issue their
      // first chunk's loads before any store (one L2 round trip for the pair); further chunks (regions
      // taller than 8 x 256 rows or wider than 8 x 256 columns) follow one round trip each
      const long long rlo = b0 * kTileRows, rhi = b1 * kTileRows < a.R ? b1 * kTileRows : a.R;
      for (long long k = 0;; ++k) {
        const long long r0 = rlo + k * 8 * kConsumers, cb = k * 8 * kConsumers;
        const bool do_r = last_r && r0 < rhi, do_c = last_c && cb < ncols;
        if (!do_r && !do_c) break;
        Acc vr[8], vc[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const long long row = r0 + threadIdx.x + q * kConsumers;
          vr[q] = do_r && row < rhi ? __ldcg(accR + row) : Acc(0);
          const long long c = cb + threadIdx.x + q * kConsumers, cg = c0 * BC + c;
          vc[q] = do_c && c < ncols && cg < a.C ? __ldcg(accC + cg) : Acc(0);
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const long long row = r0 + threadIdx.x + q * kConsumers;
          if (do_r && row < rhi) {
            __stcg(accR + row, Acc(0));
            out[row] = RcOps<T>::finish(vr[q]);
          }
          const long long c = cb + threadIdx.x + q * kConsumers, cg = c0 * BC + c;
          if (do_c && c < ncols && cg < a.C) {
            __stcg(accC + cg, Acc(0));
            out[a.R + cg] = RcOps<T>::finish(vc[q]);
          }
        }
      }
    }
    consumers_sync();  // accumulators re-zeroed and the flags read before the next region
  }
}

// ====================================================================================== host side
namespace {

template <typename T, bool STAGED>
cudaError_t launch_typed(const CUtensorMap& map, const RowsColsArgs& a, int grid, cudaStream_t st) {
  auto kern = npp_rowscols_kernel<T, STAGED>;
  cudaError_t e = ensure_smem(kern, kSmemBytes);
  if (e != cudaSuccess) return e;
  return launch_pdl(kern, grid, kThreads, kSmemBytes, st, a.pdl != 0, map, a);
}

template <typename T>
cudaError_t launch_t(bool staged, const CUtensorMap& map, const RowsColsArgs& a, int grid, cudaStream_t st) {
  return staged ? launch_typed<T, true>(map, a, grid, st) : launch_typed<T, false>(map, a, grid, st);
}

}  // namespace

cudaError_t launch_rowscols(int dtype, bool staged, const RowsColsArgs& a, int grid, cudaStream_t st) {
  CUtensorMap map;
  std::memset(&map, 0, sizeof map);
  const int esz = (dtype == NPP_I64 || dtype == NPP_F64) ? 8 : 4;
  const CUtensorMapDataType dt = dtype == NPP_F32   ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                 : dtype == NPP_I32 ? CU_TENSOR_MAP_DATA_TYPE_INT32
                                 : dtype == NPP_F64 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64
                                                    : CU_TENSOR_MAP_DATA_TYPE_INT64;
  if (staged) {
    cudaError_t e = encode_2d(&map, a.m, dt, esz, a.R, a.C, unsigned(1024 / esz), unsigned(kTileRows));
    if (e != cudaSuccess) return e;
  }
  switch (dtype) {
    case NPP_F32: return launch_t<float>(staged, map, a, grid, st);
    case NPP_I32: return launch_t<int32_t>(staged, map, a, grid, st);
    case NPP_F64: return launch_t<double>(staged, map, a, grid, st);
    default: return launch_t<int64_t>(staged, map, a, grid, st);
  }
}

}  // namespace npp
