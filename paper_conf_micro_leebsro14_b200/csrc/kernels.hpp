// kernels.hpp — launch interface between the C-ABI layer (api.cu) and the kernel families.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>
#include <utility>

#include "npp.h"

// Device-side bounds checks (measurement / validation builds only: -DNPP_DEVICE_CHECKS). A failed check
// traps the kernel, so a parity run against such a build proves the checked indices stayed in range —
// the stand-in for compute-sanitizer where the pool has it closed (profiles/r02/device_checks/).
#ifdef NPP_DEVICE_CHECKS
#define NPP_CHECK(cond) \
  do {                  \
    if (!(cond)) __trap(); \
  } while (0)
#else
#define NPP_CHECK(cond) \
  do {                  \
  } while (0)
#endif

namespace npp {

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) is per device: set it once per (kernel, device) under a
// lock (the first launch on each device of a process that drives several GPUs sets its own).
cudaError_t ensure_smem_attr(const void* func, int smem_bytes);
template <typename... Params>
cudaError_t ensure_smem(void (*kern)(Params...), int smem_bytes) {
  return ensure_smem_attr(reinterpret_cast<const void*>(kern), smem_bytes);
}

// Launch `kern` on `st`; with `overlap` as a programmatic dependent launch (PDL): its blocks may become
// resident while the previous kernel in the stream drains; the kernel orders itself after that kernel
// with `griddepcontrol.wait` (before its first read, or — NPP_EXEC_OVERLAP — before its first write).
template <typename... Params, typename... Args>
cudaError_t launch_pdl(void (*kern)(Params...), int grid, int threads, int smem, cudaStream_t st, bool overlap,
                       Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(unsigned(grid));
  cfg.blockDim = dim3(unsigned(threads));
  cfg.dynamicSmemBytes = size_t(smem);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = overlap ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

// Arguments of one 2-level sum launch (S9). Element (o, i) of the nest lives at
// m[o*so + i*si]; level o is split into go blocks of co indices, level i into gi blocks of ci.
struct SumArgs {
  const void* m;
  const void* v;       // weight vector indexed by the inner index (weighted patterns), else NULL
  void* out;
  void* partials;      // [gi x O] accumulator type, Split(k) only
  unsigned* tickets;   // [go], Split(k) only, zero on entry and on exit
  int64_t O, I;        // outer / inner sizes
  int64_t so, si;      // element strides of the outer / inner index
  int bo, bi;          // threads along the outer / inner level
  int64_t co, ci;      // chunk (indices per block) of the outer / inner level
  int64_t go, gi;      // blocks along the outer / inner level
  void* temp;          // S10 PREALLOC: the [O x I] zipWith buffer (weighted sums), else NULL
  int64_t ts_o, ts_i;  // its element strides along the outer / inner index (Fig 11)
  unsigned* err;       // S10 MALLOC: set to 1 when a device malloc returns NULL
};

cudaError_t launch_sum(int dtype, int kclass, int vec, bool weighted, const SumArgs& a, cudaStream_t st);
// S10: weighted sums with the inner allocation materialised (MALLOC or PREALLOC), vec = 1
cudaError_t launch_sum_temp(int dtype, int kclass, bool malloc_mode, const SumArgs& a, cudaStream_t st);
int sum_kernels_max_regs();

// Arguments of one staged (TMA) sum launch (S8 staged): the matrix is [R x C]; tiles are
// 32 rows x 1 KB (or 8 rows x 4 KB, `wide`), To x Ti of them in outer-major order. Block b of G streams the static range
// [b*Ts/G, (b+1)*Ts/G), then claims units of `unit` tiles of the pool [Ts, To*Ti) (S8).
struct StagedArgs {
  void* out;
  const void* v;        // weighted sums: v [C] (sumWeightedRows) or [R] (sumWeightedCols), else NULL
  void* acc;           // [O] accumulators (fp64 / u32 / u64), zero on entry and on exit
  unsigned* pool;      // [2]: pool claim counter, blocks-done ticket (zero on entry and on exit)
  unsigned* tickets;   // [To] tiles contributed per outer tile (partial contributors), zero on entry/exit
  int64_t O;           // outputs: R (sumRows) or C (sumCols)
  int64_t R, C;
  int64_t To, Ti;      // tiles along the outer / inner level
  int64_t static_tiles; // Ts
  int64_t unit;         // U: pool claim unit (tiles)
  int64_t tail_start;   // T - F: the pool's last F tiles are claimed one at a time (S8)
  int64_t big_units;    // claims of U tiles before the tail: ceil((tail_start - Ts) / U)
  int64_t claims;       // big_units + F
  int early_reads;      // NPP_EXEC_OVERLAP: stream the inputs before the previous kernel completes
  int wide;             // 1: tiles of 8 rows x 4 KB (RX) / 128 rows x 256 B (MX-narrow); 2: RX one-row 32 KB tiles
  int pdl;              // launch as a programmatic dependent launch (npp_execute_ex without NPP_EXEC_NO_PDL)
  int* trace;           // npp_execute_traced: [2 x To*Ti] block of each tile, loads per tile (else NULL)
};

cudaError_t launch_sum_staged(int dtype, bool rows, const void* m, const StagedArgs& a, int grid, cudaStream_t st);

// Batched logistic-regression gradient (class LR, S8): x [B*Rb x C] row-major fp32.
struct LogregArgs {
  const float* y;      // [B*Rb]
  const float* w;      // [C]
  float* g;            // [B x C] output
  double* acc;         // [B x C] fp64 accumulators of batches cut by range boundaries (zero on entry/exit)
  unsigned* tickets;   // [B] (zero on entry/exit)
  int64_t B, Rb, C;
  int64_t Ti;          // 32-row tiles per batch
  int64_t per_block;   // P: block b streams tiles [b*P, (b+1)*P) of the batch-major order
  int* trace;          // npp_execute_traced: [2 x B*Ti] block of each tile, loads per tile (else NULL)
};
cudaError_t launch_logreg(const LogregArgs& a, const float* x, int grid, cudaStream_t st);

// k-means assignment (class KM, S8): x [N x D], c [K x D] fp32 -> a [N] int32.
struct KmeansArgs {
  const float* x;      // [N x D] (near-tie rechecks read it from global memory)
  const float* c;      // [K x D]
  int* assign;         // [N]
  int64_t N, D, K;
  int64_t per_block;   // P: block b handles TP-point tiles [b*P, (b+1)*P)
  int sets;            // warp sets of 256 threads taking the block's tiles round robin (record L0 block / 64)
  int* trace;          // npp_execute_traced: [2 x T] block of each tile, loads per tile (else NULL)
};
cudaError_t launch_kmeans(const KmeansArgs& a, const float* x, int grid, cudaStream_t st);

// k-means assignment under a LITERAL / caller-given mapping with Span(all) reduce levels (class KM,
// staged = 0; kern_kmeans_direct.cu): per level l = 0 (points), 1 (centroids), 2 (dims) the CUDA dim and
// threads of the record; level 0's chunk (points per block); grid = ceil(N / chunk0) blocks.
struct KmDirectArgs {
  const float* x;      // [N x D]
  const float* c;      // [K x D]
  int* assign;         // [N]
  int64_t N;
  int D, K;
  int dim[3];
  int blk[3];
  int64_t chunk0;
};
cudaError_t launch_kmeans_direct(const KmDirectArgs& a, int grid, cudaStream_t st);

// sumRows + sumCols of one matrix in one pass (class RC, S8 RC): the ceil(R/32) x ceil(C/BC)
// tile grid is cut into regions of cr row bands x cc column tiles, gr x gc of them in row-region-major
// order; block b of G takes regions [b*nreg/G, (b+1)*nreg/G). out = [R row sums | C column sums].
struct RowsColsArgs {
  const void* m;       // [R x C]
  void* out;           // [R + C]
  void* accR;          // [R] accumulators (fp64 / u32 / u64) of row bands cut by column regions
  void* accC;          // [C] accumulators of columns cut by row regions
  unsigned* tick_r;    // [gr] column regions done per row region (zero on entry and on exit)
  unsigned* tick_c;    // [gc] row regions done per column group (zero on entry and on exit)
  int64_t R, C;
  int64_t Tr, Tc;      // 32-row bands, BC-column tiles
  int64_t cr, cc;      // bands / column tiles per region
  int64_t gr, gc;      // regions along rows / columns
  int64_t nreg;        // gr * gc
  int early_reads;     // NPP_EXEC_OVERLAP
  int pdl;             // programmatic dependent launch (not NPP_EXEC_NO_PDL)
  int* trace;          // npp_execute_traced: [2 x nreg] block of each region, visits per region (else NULL)
};
cudaError_t launch_rowscols(int dtype, bool staged, const RowsColsArgs& a, int grid, cudaStream_t st);

// k-means centroid update (class KU, S8 KU): x [N x D] fp32, keys [N] int32 ->
// out [K x (D+1)] fp32 = per group (Σ x, count). Block b takes 96-point tiles [b*P, (b+1)*P) (S8 KU).
struct KmUpdateArgs {
  float* out;          // [K x (D+1)]
  double* acc;         // [K x (D+1)] fp64 accumulators (zero on entry and on exit)
  unsigned* ticket;    // blocks done (zero on entry and on exit)
  int64_t N, D, K;
  int64_t per_block;   // P
  int early_reads;     // NPP_EXEC_OVERLAP
  int pdl;             // programmatic dependent launch (not NPP_EXEC_NO_PDL)
  int* trace;          // npp_execute_traced: [2 x T] block of each 96-point tile, loads per tile (else NULL)
};
cudaError_t launch_kmupdate(const KmUpdateArgs& a, const float* x, const int* keys, int grid, cudaStream_t st);

// One PageRank step over the CSR of in-neighbours (class PR, S8 PR, Fig 5).
struct PagerankArgs {
  const long long* rowptr;  // [N+1]
  const int* colidx;        // [E] in-neighbour ids
  const float* pr;          // [N] previous PageRank
  const int* outdeg;        // [N] out-degrees (>= 1 for every id that occurs in colidx)
  float* out;               // [N]
  unsigned* pool;           // row-chunk claim counter (zero on entry and on exit)
  float* contrib;           // [N] workspace: prevPR(w) / w.degree (Fig 5's inner map, once per node)
  int64_t N;        // rows computed (a shard's rows, or all nodes)
  int64_t Nnodes;   // nodes of the graph: length of pr / outdeg / contrib, and the N of (1-damp)/N
  float damp;
};
// V: lanes per row (row-group mapping); seg_rows > 0: the segmented mapping with that many rows per claim
cudaError_t launch_pagerank(const PagerankArgs& a, int V, int seg_rows, int grid, cudaStream_t st);

}  // namespace npp
