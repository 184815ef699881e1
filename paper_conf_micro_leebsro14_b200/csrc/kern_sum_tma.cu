// kern_sum_tma.cu — the staged (TMA) kernel family for sumRows / sumCols (S8, staged).
//
// PAPER.md §V-B: "Multiple threads in one dimension all read a contiguous chunk of the
// data ... and store it in shared memory" so that both nest levels see coalesced memory. On sm_100a
// the chunk is moved by the Tensor Memory Accelerator: one elected producer thread issues 2-D
// cp.async.bulk.tensor copies of 32-row x 1 KB tiles into a 4-deep shared-memory ring (mbarrier
// complete_tx) and eight consumer warps reduce each tile out of shared memory; 128 KB per SM stay in
// flight, which holds HBM3e at its copy ceiling with one persistent block per SM.
//
//   RX (sumRows): warp w owns rows 4w..4w+3 of every 32-row band; a lane reads 2 x 16 B of each row
//                 (conflict-free, contiguous per warp) and accumulates per row; shuffles finish a row.
//   MX (sumCols): thread t owns column t of every 1 KB column tile (two row halves for 8-byte types)
//                 and walks the rows of the band; the Map level stays on x as Fig 1 / P:L596-600 need.
// Out-of-range rows/columns of edge tiles are zero-filled by TMA, which is the identity of +.
//
// Work split: the To x Ti tiles are taken in outer-major order and block b streams the contiguous
// range [b*P, (b+1)*P), P = ceil(To*Ti / G) — every block moves the same bytes (to one tile) and walks
// memory sequentially. Partial sums stay in registers while consecutive tiles share an outer tile.
// An outer tile that lies inside one range is written directly; an outer tile cut by range
// boundaries is the Split(k) of P:L542-550 across the k blocks that share it: each adds its partial
// with one fp64 / integer atomic per output and takes a ticket, and the last of the k converts the
// accumulators to the output type and zeroes them (the combiner of P:L880-883, fused, no second
// launch, no grid barrier). Workspace: tickets [To] + accumulators [O], zero on entry and on exit.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "kernels.hpp"
#include "tma_ring.cuh"

#ifndef NPP_TMA_STAGES
#define NPP_TMA_STAGES 4
#endif

namespace npp {

namespace {

constexpr int kStages = NPP_TMA_STAGES;
constexpr int kTileRows = 32;
constexpr int kTileBytes = kTileRows * 1024;
constexpr int kConsumerWarps = 8;
constexpr int kConsumers = kConsumerWarps * 32;
constexpr int kProducerWarp = kConsumerWarps;      // warp 8: TMA producer (one elected lane)
constexpr int kCombinerWarp = kConsumerWarps + 1;  // warp 9: tickets + conversion of cut outer tiles
constexpr int kThreads = kConsumers + 64;
constexpr int kFlushRing = 8;  // flushes of cut outer tiles in flight between consumers and the combiner
constexpr int kSmemHeader = 1024;          // mbarriers + per-slot tile ids; tiles start 1 KB-aligned
constexpr int kSmemBytes = kSmemHeader + kStages * kTileBytes;
constexpr int kVSlot = 4096;  // weighted sums: the tile's slice of v (<= 4 KB) per ring slot
constexpr int kSmemBytesW = kSmemBytes + kStages * kVSlot;

using tma::mbar_arrive;
using tma::mbar_expect_tx;
using tma::mbar_init;
using tma::mbar_test;
using tma::mbar_wait;
__device__ __forceinline__ void consumers_sync() { tma::bar_sync_consumers<kConsumers>(); }

template <typename T> struct SOps;
template <> struct SOps<float> {
  using Acc = double;
  __device__ static float finish(double a) { return float(a); }
};
template <> struct SOps<double> {
  using Acc = double;
  __device__ static double finish(double a) { return a; }
};
template <> struct SOps<int32_t> {
  using Acc = unsigned int;
  __device__ static int32_t finish(unsigned a) { return int32_t(a); }
};
template <> struct SOps<int64_t> {
  using Acc = unsigned long long;
  __device__ static int64_t finish(unsigned long long a) { return int64_t(a); }
};

// sum of one 16-byte vector: fp32 pairwise for floats, exact unsigned for integers
__device__ __forceinline__ float vsum(const float4& v) { return (v.x + v.y) + (v.z + v.w); }
__device__ __forceinline__ unsigned vsum(const int4& v) {
  return unsigned(v.x) + unsigned(v.y) + unsigned(v.z) + unsigned(v.w);
}
__device__ __forceinline__ unsigned long long vsum(const longlong2& v) {
  return (unsigned long long)v.x + (unsigned long long)v.y;
}
__device__ __forceinline__ double vsum(const double2& v) { return v.x + v.y; }
// weighted: Σ of the 16-byte vector's products with the weights (fp32 pairwise; integers wrap)
__device__ __forceinline__ float vdot(const float4& x, const float4& w) {
  return (x.x * w.x + x.y * w.y) + (x.z * w.z + x.w * w.w);
}
__device__ __forceinline__ unsigned vdot(const int4& x, const int4& w) {
  return unsigned(x.x) * unsigned(w.x) + unsigned(x.y) * unsigned(w.y) + unsigned(x.z) * unsigned(w.z) +
         unsigned(x.w) * unsigned(w.w);
}
__device__ __forceinline__ unsigned long long vdot(const longlong2& x, const longlong2& w) {
  return (unsigned long long)x.x * (unsigned long long)w.x + (unsigned long long)x.y * (unsigned long long)w.y;
}
__device__ __forceinline__ double vdot(const double2& x, const double2& w) { return x.x * w.x + x.y * w.y; }
__device__ __forceinline__ float vmul(float x, float w) { return x * w; }
__device__ __forceinline__ double vmul(double x, double w) { return x * w; }
__device__ __forceinline__ int32_t vmul(int32_t x, int32_t w) { return int32_t(unsigned(x) * unsigned(w)); }
__device__ __forceinline__ int64_t vmul(int64_t x, int64_t w) {
  return int64_t((unsigned long long)x * (unsigned long long)w);
}
template <typename T> struct V16;
template <> struct V16<float> { using type = float4; };
template <> struct V16<int32_t> { using type = int4; };
template <> struct V16<int64_t> { using type = longlong2; };
template <> struct V16<double> { using type = double2; };

template <typename A>
__device__ __forceinline__ A warp_sum(A v) {
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) v += __shfl_xor_sync(0xffffffffu, v, off);
  return v;
}


}  // namespace

#ifdef NPP_SUM_STAMPS  // measurement variant: per-block globaltimer stamps of the last 32 launches
// [launch % 32][block][entry, first tile, consumers' end, combiner's end]; tools/sum_stamps.py reads them
__device__ unsigned long long g_sum_stamps[32][256][4];
__device__ unsigned long long g_sum_blocks;
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#endif

// WT: weighted sums (sumWeightedRows / sumWeightedCols, Fig 15) fused: the zipWith
// product m·v is formed in registers from the staged tile and the tile's slice of v (staged by a 1-D
// TMA box on the same mbarrier), so no inner allocation exists at all (§V-A taken to its limit).
template <typename T, bool ROWS, bool WIDE, bool WT, bool R1>
__global__ void __launch_bounds__(kThreads, 1) npp_sum_tma_kernel(const __grid_constant__ CUtensorMap map,
                                                                  const __grid_constant__ CUtensorMap vmap,
                                                                  StagedArgs a) {
  using Acc = typename SOps<T>::Acc;
  using V = typename V16<T>::type;
  constexpr int BC = 1024 / int(sizeof(T));     // columns of one 1 KB chunk
  // RX: WIDE = 8 rows x 4 KB tiles. MX: WIDE = narrow strips, 128 rows x 256 B (a static split of
  // whole strips then never cuts one: no Split combine at all)
  // RX R1: one-row tiles of 32 KB (a row of 64-256 KB is <= 8 tiles: whole rows balance, no cuts)
  constexpr bool MXN = WIDE && !ROWS;
  constexpr bool ALIGN = MXN || R1;             // static split aligned to whole outer tiles
  constexpr int NCH = R1 ? 32 : ((WIDE && ROWS) ? 4 : 1);  // chunks per tile row: tile = RT rows x NCH KB
  constexpr int RT = MXN ? 128 : (R1 ? 1 : kTileRows / NCH);  // tile rows (32, wide 8, R1 1, MX-narrow 128)
  constexpr int W = MXN ? 256 / int(sizeof(T)) : NCH * BC;  // tile columns
  constexpr int OUT_PER_TILE = ROWS ? RT : W;   // outputs of one outer tile (band / strip)
  extern __shared__ __align__(1024) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem);
  uint64_t* empty = full + kStages;
  uint64_t* fl_full = empty + kStages;        // [kFlushRing] consumer warps -> combiner
  uint64_t* fl_free = fl_full + kFlushRing;   // [kFlushRing] combiner -> consumers
  unsigned* slot_tile = reinterpret_cast<unsigned*>(fl_free + kFlushRing);  // tile | kFlush, kEnd = end
  long long* fl_ot = reinterpret_cast<long long*>(fl_free + kFlushRing) + kStages;  // [kFlushRing] outer tile, -1 = end
  unsigned* fl_cnt = reinterpret_cast<unsigned*>(fl_ot + kFlushRing);  // tiles it contributes
  unsigned char* tiles = smem + kSmemHeader;
  unsigned char* vslots = tiles + kStages * kTileBytes;  // WT only: [kStages][kVSlot]
  Acc* accg = static_cast<Acc*>(a.acc);
  constexpr unsigned kFlush = 1u << 31;  // tile ids < 2^31 - 1 (launch_sum_staged checks)
  constexpr unsigned kEnd = 0xffffffffu;

  // PDL: let the next launch in the stream become resident as SMs free up (its griddepcontrol.wait
  // still orders it after this grid's completion).
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long bid = blockIdx.x, G = gridDim.x;
  const long long total = a.To * a.Ti;
  // static range (MX-narrow: whole strips, so no strip is ever cut)
#ifndef NPP_SUM_FAST_DIV
#define NPP_SUM_FAST_DIV 1
#endif
  // static range (MX-narrow: whole strips, so no strip is ever cut). Tile ids are < 2^31 (the launch
  // checks), so the producer's divisions run in 32 bits, and floor(b·S/G) with b·S < 2^40 in double:
  // exact, since a quotient's fraction is at most 1 − 1/G, far from the 2^-13 rounding error — the 64-bit
  // integer divisions sat in front of the first TMA issue of every launch
  auto fdiv = [](long long num, long long den) -> long long {
    return NPP_SUM_FAST_DIV ? (long long)floor(double(num) / double(den)) : num / den;
  };
  const long long so = NPP_SUM_FAST_DIV ? (long long)(unsigned(a.static_tiles) / unsigned(a.Ti)) : a.static_tiles / a.Ti;
  const long long s0 = ALIGN ? (fdiv(bid * so, G)) * a.Ti : fdiv(bid * a.static_tiles, G);
  const long long s1 = ALIGN ? (fdiv((bid + 1) * so, G)) * a.Ti
                             : fdiv((bid + 1) * a.static_tiles, G);
  const long long U = a.unit;  // pool: units of U tiles from static_tiles on, claimed in order, then single tiles
#ifdef NPP_SUM_STAMPS
  __shared__ unsigned long long* stamp_row;
  if (threadIdx.x == 0) {
    const unsigned long long t0 = gtimer();
    const unsigned long long L = atomicAdd(&g_sum_blocks, 1ull) / (unsigned long long)G;
    stamp_row = g_sum_stamps[L % 32][bid % 256];
    stamp_row[0] = t0;
  }
#endif

  // stream tile cur into ring slot t % kStages (nxt: the block's next tile, -1 = none, for the flush tag)
  auto issue = [&](long long t, long long cur, long long nxt) {
    const unsigned uTi = unsigned(a.Ti);  // tile ids and Ti < 2^31: 32-bit divisions
    const long long ot = NPP_SUM_FAST_DIV ? (long long)(unsigned(cur) / uTi) : cur / a.Ti;
    const bool flush = nxt < 0 || (NPP_SUM_FAST_DIV ? (long long)(unsigned(nxt) / uTi) : nxt / a.Ti) != ot;
    const int slot = int(t % kStages);
    if (t >= kStages) mbar_wait(empty + slot, unsigned((t / kStages) & 1) ^ 1u);
    // the tag travels through shared memory ordered by the slot's mbarriers; it is written and
    // read with (relaxed) shared atomics so compute-sanitizer's racecheck, which does not model
    // mbarrier ordering, sees no plain-access race
    atomicExch(slot_tile + slot, static_cast<unsigned>(cur) | (flush ? kFlush : 0u));
    if (a.trace) {  // white-box schedule trace (npp_execute_traced): who streamed tile cur
      a.trace[cur] = int(bid);
      atomicAdd(a.trace + total + cur, 1);
    }
    constexpr unsigned kVBytes = WT ? (ROWS ? NCH * 1024 : RT * unsigned(sizeof(T))) : 0;
    mbar_expect_tx(full + slot, kTileBytes + kVBytes);
    const long long it = cur - ot * a.Ti;
    NPP_CHECK(cur >= 0 && cur < total && ot < a.To && it >= 0 && it < a.Ti && (nxt < 0 || nxt < total));
    const int ch = int(ROWS ? it * NCH : ot * NCH);  // first 1 KB chunk of the tile's rows
    const int y = int(ROWS ? ot * RT : it * RT);     // first row
    if constexpr (WT) {  // v over the tile's columns (RX) or rows (MX); zero-filled past the end
      if constexpr (ROWS) {
#pragma unroll
        for (int q = 0; q < NCH; ++q)
          tma::load_1d(vslots + slot * kVSlot + q * 1024, &vmap, (ch + q) * BC, full + slot);
      } else {
        tma::load_1d(vslots + slot * kVSlot, &vmap, y, full + slot);
      }
    }
    if constexpr (WIDE && ROWS)  // 3-D map {BC, C/BC, R}: box {BC, 4, 8} = 8 rows x 4 KB
      tma::load_3d(tiles + slot * kTileBytes, &map, 0, ch, y, full + slot);
    else  // 2-D map {C, R}: box {BC, 32} = 32 rows x 1 KB
      tma::load_2d(tiles + slot * kTileBytes, &map, MXN ? int(ot * W) : ch * BC, y, full + slot);
  };
#ifndef NPP_SUM_EARLY_ISSUE
#define NPP_SUM_EARLY_ISSUE 1
#endif
  // the first tiles of the static range are issued by the thread that initialises the barriers, before
  // the block-wide barrier (the producer warp then continues after them): the first loads leave ~a
  // barrier and a warp hand-off earlier
  const long long early = NPP_SUM_EARLY_ISSUE ? (s1 - s0 - 1 < kStages ? (s1 - s0 - 1 > 0 ? s1 - s0 - 1 : 0)
                                                                        : kStages) : 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; ++i) {
      mbar_init(full + i, 1);
      mbar_init(empty + i, kConsumerWarps);
    }
    for (int i = 0; i < kFlushRing; ++i) {
      mbar_init(fl_full + i, kConsumerWarps);
      mbar_init(fl_free + i, 1);
    }
    tma::mbar_fence_init();
    if (early > 0) {
      tma::prefetch_map(&map);
      if (a.early_reads == 0) asm volatile("griddepcontrol.wait;" ::: "memory");
      for (long long j = 0; j < early; ++j) issue(j, s0 + j, s0 + j + 1);  // nxt stays inside the range
    }
  }
  __syncthreads();

  if (warp == kProducerWarp) {
    // ------------------------------------------------------------ producer: one elected lane
    if (lane == 0) {
      tma::prefetch_map(&map);
      if constexpr (WT) tma::prefetch_map(&vmap);
      long long sn = s0, u_cur = 0, u_end = 0;
      // Every launch is a programmatic dependent launch: this block may already be resident while the
      // previous kernel in the stream drains. Unless the caller asserted NPP_EXEC_OVERLAP (inputs not
      // written by earlier stream work), the first read waits for that kernel to complete.
      bool waited = !a.early_reads;
      if (waited) asm volatile("griddepcontrol.wait;" ::: "memory");
      // static range, then pool units in claim order (S8 balance rule)
      auto next_tile = [&]() -> long long {
        if (sn < s1) return sn++;
        if (u_cur < u_end) return u_cur++;
        if (!waited) {  // the pool counter is workspace: touch it only after the previous grid is done
          asm volatile("griddepcontrol.wait;" ::: "memory");
          waited = true;
        }
        const unsigned k = atomicAdd(a.pool, 1u);
        if ((long long)k >= a.claims) {
          // every producer makes exactly one failing claim, so the counter ends at claims + G: the
          // block taking the last value re-arms it for the next launch
          if ((long long)k + 1 == a.claims + G) a.pool[0] = 0u;
          return -1;
        }
        if ((long long)k < a.big_units) {  // units of U tiles, then the tail's single tiles (S8)
          u_cur = a.static_tiles + (long long)k * U;
          u_end = (u_cur + U < a.tail_start) ? u_cur + U : a.tail_start;
        } else {
          u_cur = a.tail_start + ((long long)k - a.big_units);
          u_end = u_cur + 1;
        }
        return u_cur++;
      };
      sn = s0 + early;  // the first `early` tiles of the static range are already in flight
      long long cur = next_tile();
      long long t = early;
      for (; cur >= 0; ++t) {
        const long long nxt = next_tile();  // claimed one ahead: its latency hides behind the slot wait
        issue(t, cur, nxt);
        cur = nxt;
      }
      const int slot = int(t % kStages);  // end marker: an arrival without bytes
      if (t >= kStages) mbar_wait(empty + slot, unsigned((t / kStages) & 1) ^ 1u);
      atomicExch(slot_tile + slot, kEnd);
      mbar_arrive(full + slot);
    }
  } else if (warp == kCombinerWarp) {
    // ------------------------------------------------------------ combiner: the fused Split combine
    // of outer tiles this block only partly covered. Consumers RED their partials into
    // the accumulators and hand the flush over through fl_full (CTA-scope release/acquire); here one
    // gpu-scope fence publishes them (the barrier-then-release pattern), the ticket counts tiles, and
    // whoever completes the Ti tiles of ot converts its outputs — off the consumers' critical path.
    // Flushes are taken in batches: lane j owns the j-th ready entry, so the fences and ticket round
    // trips of up to kFlushRing flushes overlap.
    for (long long k = 0;;) {
      mbar_wait(fl_full + int(k % kFlushRing), unsigned((k / kFlushRing) & 1));
      int nb = 1;
      while (nb < kFlushRing &&
             mbar_test(fl_full + int((k + nb) % kFlushRing), unsigned(((k + nb) / kFlushRing) & 1)))
        ++nb;
      const int i = int((k + lane) % kFlushRing);
      const long long ot = lane < nb ? fl_ot[i] : -1;
      const unsigned cnt = lane < nb ? fl_cnt[i] : 0u;
      const unsigned ends = __ballot_sync(0xffffffffu, lane < nb && ot < 0);
      const int n = ends ? __ffs(ends) - 1 : nb;  // entries before the end marker
      // the ticket add is itself the release (cumulative over the consumers' accumulator adds, which
      // the fl_full mbarrier ordered before it) and the acquire of the contributor that completes
      // the tile; the other lanes read the accumulators after a fence only when some tile completed
      bool last = false;
      if (lane < n) {
        const unsigned prev = tma::ticket_add(a.tickets + ot, cnt);
        last = prev + cnt == unsigned(a.Ti);
        if (last) a.tickets[ot] = 0u;
      }
      // the lane whose acq_rel ticket completed a tile acquired every contributor's adds; __syncwarp orders
      // the other lanes (which read the tile's accumulators from L2 below) after that acquire
      __syncwarp();
      unsigned lasts = __ballot_sync(0xffffffffu, last);
      while (lasts) {  // every contribution to these outer tiles is in: read (L2), convert, re-zero
        const int j = __ffs(lasts) - 1;
        lasts &= lasts - 1;
        const long long o0 = __shfl_sync(0xffffffffu, ot, j) * OUT_PER_TILE;
        const long long oend = ROWS ? a.R : a.C;
        constexpr int J = OUT_PER_TILE >= 256 ? 8 : (OUT_PER_TILE + 31) / 32;  // loads in flight per lane
        for (int base = 0; base < OUT_PER_TILE; base += 32 * J) {
          Acc v[J];
#pragma unroll
          for (int q = 0; q < J; ++q) {
            const long long o = o0 + base + lane + 32 * q;
            v[q] = (base + lane + 32 * q < OUT_PER_TILE && o < oend) ? __ldcg(accg + o) : Acc(0);
          }
#pragma unroll
          for (int q = 0; q < J; ++q) {
            const long long o = o0 + base + lane + 32 * q;
            if (base + lane + 32 * q < OUT_PER_TILE && o < oend) {
              __stcg(accg + o, Acc(0));
              static_cast<T*>(a.out)[o] = SOps<T>::finish(v[q]);
            }
          }
        }
      }
      __syncwarp();
      if (lane < n) mbar_arrive(fl_free + i);
      k += n;
      if (ends) break;
    }
#ifdef NPP_SUM_STAMPS
    if (lane == 0) stamp_row[3] = gtimer();
#endif
  } else {
    // ------------------------------------------------------------ consumers
    constexpr int kGroups = ROWS ? 1 : 256 / W;   // MX row groups (1 / 2 for 4- / 8-byte; MX-narrow 4 / 8)
    constexpr int kRowsPer = RT / kGroups;        // MX rows of a tile one thread adds
    const int col = threadIdx.x % W;
    const int rg = threadIdx.x / W;
    // RX narrow: rows 4w..4w+3; RX wide: acc[0] = row w; MX: acc[k] = column col of chunk k
    Acc acc[4] = {0, 0, 0, 0};
    unsigned n_acc = 0;         // tiles of the current outer tile accumulated since the last flush
    long long nfl = 0;          // flushes handed to the combiner
    bool waited = false;
    for (long long t = 0;; ++t) {
      const int slot = int(t % kStages);
      mbar_wait(full + slot, unsigned((t / kStages) & 1));
#ifdef NPP_SUM_STAMPS
      if (t == 0 && threadIdx.x == 0) stamp_row[1] = gtimer();
#endif
      unsigned tag_u = 0;
      if (lane == 0) tag_u = atomicAdd(slot_tile + slot, 0u);
      tag_u = __shfl_sync(0xffffffffu, tag_u, 0);
      if (tag_u == kEnd) break;
      const long long tag = static_cast<long long>(tag_u);
      const unsigned char* tile = tiles + slot * kTileBytes;
      const unsigned char* vs = vslots + slot * kVSlot;
      if constexpr (ROWS && !WIDE) {
        V w0{}, w1{};
        if constexpr (WT) {
          w0 = *reinterpret_cast<const V*>(vs + lane * 16);
          w1 = *reinterpret_cast<const V*>(vs + 512 + lane * 16);
        }
#pragma unroll
        for (int rr = 0; rr < 4; ++rr) {
          const unsigned char* row = tile + (warp * 4 + rr) * 1024;
          const V v0 = *reinterpret_cast<const V*>(row + lane * 16);
          const V v1 = *reinterpret_cast<const V*>(row + 512 + lane * 16);
          if constexpr (WT)
            acc[rr] += Acc(vdot(v0, w0) + vdot(v1, w1));
          else
            acc[rr] += Acc(vsum(v0) + vsum(v1));
        }
      } else if constexpr (ROWS) {  // wide: warp w adds the 4 KB of row w, 8 x 16 B per lane
        const unsigned char* row = tile + warp * 4096;
        decltype(vsum(V{})) p[8];
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const V x = *reinterpret_cast<const V*>(row + k * 512 + lane * 16);
          if constexpr (WT)
            p[k] = vdot(x, *reinterpret_cast<const V*>(vs + k * 512 + lane * 16));
          else
            p[k] = vsum(x);
        }
#pragma unroll
        for (int w = 4; w >= 1; w /= 2)
#pragma unroll
          for (int i = 0; i < w; ++i) p[i] = p[i] + p[i + w];
        acc[0] += Acc(p[0]);
      } else {
        const T* tt = reinterpret_cast<const T*>(tile);
#pragma unroll
        for (int k = 0; k < NCH; ++k) {
          T v[kRowsPer];
#pragma unroll
          for (int rr = 0; rr < kRowsPer; ++rr) {
            v[rr] = tt[(rg * kRowsPer + rr) * W + k * BC + col];
            if constexpr (WT) v[rr] = vmul(v[rr], reinterpret_cast<const T*>(vs)[rg * kRowsPer + rr]);
          }
          if constexpr (std::is_floating_point<T>::value) {  // floats: pairwise tree inside the tile
#pragma unroll
            for (int w = kRowsPer / 2; w >= 1; w /= 2)
#pragma unroll
              for (int i = 0; i < w; ++i) v[i] = v[i] + v[i + w];
            acc[k] += Acc(v[0]);
          } else {
#pragma unroll
            for (int rr = 0; rr < kRowsPer; ++rr) acc[k] += Acc(v[rr]);
          }
        }
      }
      ++n_acc;
      __syncwarp();
      if (lane == 0) mbar_arrive(empty + slot);
      if (!(tag & kFlush)) continue;

      // ---- flush the partial of outer tile ot (n_acc of its Ti tiles)
      if (!waited) {  // out / accumulators: only after the previous grid in the stream is done
        asm volatile("griddepcontrol.wait;" ::: "memory");
        waited = true;
      }
      const long long ot = NPP_SUM_FAST_DIV ? (long long)((tag & ~kFlush) / unsigned(a.Ti)) : (tag & ~kFlush) / a.Ti;
      const bool whole = n_acc == unsigned(a.Ti);  // this block added every tile of ot
      long long oidx[4];
      Acc val[4];
      bool mine[4];
      if constexpr (ROWS && !WIDE) {
#pragma unroll
        for (int rr = 0; rr < 4; ++rr) {
          val[rr] = warp_sum(acc[rr]);
          oidx[rr] = ot * RT + warp * 4 + rr;
          mine[rr] = lane == rr && oidx[rr] < a.R;
          acc[rr] = 0;
        }
      } else if constexpr (ROWS) {
        val[0] = warp_sum(acc[0]);
        oidx[0] = R1 ? ot : ot * RT + warp;  // R1: every warp holds a piece of the one row
        mine[0] = lane == 0 && oidx[0] < a.R;
        acc[0] = 0;
      } else {
#pragma unroll
        for (int k = 0; k < NCH; ++k) {
          val[k] = acc[k];
          oidx[k] = ot * W + k * BC + col;
          mine[k] = oidx[k] < a.C;
          acc[k] = 0;
        }
      }
      constexpr int NV = ROWS ? (WIDE ? 1 : 4) : NCH;
      const unsigned contributed = n_acc;
      n_acc = 0;
      if (R1 && whole) {  // the eight warps' pieces of a whole row meet in shared memory
        Acc* red = reinterpret_cast<Acc*>(tiles + kStages * kTileBytes);  // [8]
        if (lane == 0) red[warp] = val[0];
        consumers_sync();
        if (threadIdx.x == 0) {
          Acc s = Acc(0);
#pragma unroll
          for (int w = 0; w < kConsumerWarps; ++w) s += red[w];
          if (ot < a.R) static_cast<T*>(a.out)[ot] = SOps<T>::finish(s);
        }
        consumers_sync();
        continue;
      }
      if (MXN && whole) {  // the row groups of a whole strip meet in shared memory, one write per column
        Acc* red = reinterpret_cast<Acc*>(tiles + kStages * kTileBytes);  // [kGroups][W]
        red[rg * W + col] = val[0];
        consumers_sync();
        if (threadIdx.x < W) {
          Acc s = Acc(0);
#pragma unroll
          for (int g = 0; g < kGroups; ++g) s += red[g * W + threadIdx.x];
          if (ot * W + threadIdx.x < a.C) static_cast<T*>(a.out)[ot * W + threadIdx.x] = SOps<T>::finish(s);
        }
        consumers_sync();
        continue;
      }
      if (whole && kGroups == 1 && !R1) {
#pragma unroll
        for (int i = 0; i < NV; ++i)
          if (mine[i]) static_cast<T*>(a.out)[oidx[i]] = SOps<T>::finish(val[i]);
        continue;
      }
#ifdef NPP_SUM_NO_COMBINE  // measurement variant (wrong results): the cost of the fused Split combine
      continue;
#endif
      const int fi = int(nfl % kFlushRing);
      if (nfl >= kFlushRing) mbar_wait(fl_free + fi, unsigned(((nfl / kFlushRing) - 1) & 1));
#pragma unroll
      for (int i = 0; i < NV; ++i)
        if (mine[i]) atomicAdd(accg + oidx[i], val[i]);
      __syncwarp();
      if (lane == 0) {
        if (warp == 0) {
          fl_ot[fi] = ot;
          fl_cnt[fi] = contributed;
        }
        mbar_arrive(fl_full + fi);
      }
      ++nfl;
    }
    // end marker for the combiner
#ifdef NPP_SUM_STAMPS
    if (threadIdx.x == 0) stamp_row[2] = gtimer();
#endif
    const int fi = int(nfl % kFlushRing);
    if (nfl >= kFlushRing) mbar_wait(fl_free + fi, unsigned(((nfl / kFlushRing) - 1) & 1));
    __syncwarp();
    if (lane == 0) {
      if (warp == 0) fl_ot[fi] = -1;
      mbar_arrive(fl_full + fi);
    }
  }
}

#ifdef NPP_SUM_STAMPS
extern "C" __attribute__((visibility("default"))) int npp_debug_sum_stamps(unsigned long long* host) {
  return int(cudaMemcpyFromSymbol(host, g_sum_stamps, sizeof(g_sum_stamps)));  // 32 x 256 x 4 stamps
}
#endif

// ====================================================================================== host side
namespace {

template <typename T, bool ROWS, bool WIDE, bool WT, bool R1 = false>
cudaError_t launch_typed(const CUtensorMap& map, const CUtensorMap& vmap, const StagedArgs& a, int grid,
                         cudaStream_t st) {
  auto kern = npp_sum_tma_kernel<T, ROWS, WIDE, WT, R1>;
  const int smem = (WT ? kSmemBytesW : kSmemBytes) + (((WIDE && !ROWS) || R1) ? 2048 : 0);  // group sums
  cudaError_t e = ensure_smem(kern, smem);
  if (e != cudaSuccess) return e;
  return launch_pdl(kern, grid, kThreads, smem, st, a.pdl != 0, map, vmap, a);
}

template <typename T, bool WT>
cudaError_t launch_w(bool rows, const CUtensorMap& map, const CUtensorMap& vmap, const StagedArgs& a, int grid,
                     cudaStream_t st) {
  // wide tiles are selected for sumRows only (S8); the MX-wide path of the kernel template (4 KB
  // column strips) measured slower than 1 KB strips because of the larger combine per cut strip
  if (rows)
    return a.wide == 2 ? launch_typed<T, true, true, false, true>(map, vmap, a, grid, st)
           : a.wide    ? launch_typed<T, true, true, WT>(map, vmap, a, grid, st)
                       : launch_typed<T, true, false, WT>(map, vmap, a, grid, st);
  return a.wide ? launch_typed<T, false, true, WT>(map, vmap, a, grid, st)
                : launch_typed<T, false, false, WT>(map, vmap, a, grid, st);
}

template <typename T>
cudaError_t launch_dtype(bool rows, const CUtensorMap& map, const CUtensorMap& vmap, const StagedArgs& a, int grid,
                         cudaStream_t st) {
  return a.v ? launch_w<T, true>(rows, map, vmap, a, grid, st) : launch_w<T, false>(rows, map, vmap, a, grid, st);
}

}  // namespace

cudaError_t launch_sum_staged(int dtype, bool rows, const void* m, const StagedArgs& a, int grid, cudaStream_t st) {
  if (a.To * a.Ti >= 0x7fffffffll) return cudaErrorInvalidValue;  // 32-bit slot tags
  const int esz = (dtype == NPP_I64 || dtype == NPP_F64) ? 8 : 4;
  const cuuint64_t bc = cuuint64_t(1024 / esz);
  const CUtensorMapDataType dt = dtype == NPP_F32   ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                 : dtype == NPP_I32 ? CU_TENSOR_MAP_DATA_TYPE_INT32
                                 : dtype == NPP_F64 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64
                                                    : CU_TENSOR_MAP_DATA_TYPE_INT64;
  CUtensorMap map;
  cudaError_t e;
  if (a.wide && !rows) {  // MX-narrow strips: {C, R}, box 128 rows x 256 B
    e = tma::encode_2d(&map, m, dt, esz, a.R, a.C, unsigned(256 / esz), 128u);
  } else if (a.wide) {  // {1 KB chunk, chunks per row, rows}; box 8 rows x 4 KB (or R1: 1 row x 32 KB)
    const cuuint64_t dims[3] = {bc, cuuint64_t(a.C) / bc, cuuint64_t(a.R)};
    const cuuint64_t strides[2] = {1024, cuuint64_t(a.C) * esz};
    const cuuint32_t box[3] = {cuuint32_t(bc), a.wide == 2 ? 32u : 4u, a.wide == 2 ? 1u : cuuint32_t(kTileRows / 4)};
    e = tma::encode_nd(&map, m, dt, 3, dims, strides, box);
  } else {  // {C, R}; box 32 rows x 1 KB
    e = tma::encode_2d(&map, m, dt, esz, a.R, a.C, unsigned(bc), unsigned(kTileRows));
  }
  if (e != cudaSuccess) return e;
  CUtensorMap vmap;  // weighted: 1-D map over v (C elements for sumRows, R for sumCols)
  std::memset(&vmap, 0, sizeof vmap);
  if (a.v && (e = tma::encode_1d(&vmap, a.v, dt, rows ? a.C : a.R, unsigned(rows ? bc : kTileRows))) != cudaSuccess)
    return e;
  switch (dtype) {
    case NPP_F32: return launch_dtype<float>(rows, map, vmap, a, grid, st);
    case NPP_I32: return launch_dtype<int32_t>(rows, map, vmap, a, grid, st);
    case NPP_F64: return launch_dtype<double>(rows, map, vmap, a, grid, st);
    default: return launch_dtype<int64_t>(rows, map, vmap, a, grid, st);
  }
}

}  // namespace npp
