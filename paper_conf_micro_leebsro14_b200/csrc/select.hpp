// select.hpp — internal interface of the CUDA-free mapping selector.
#pragma once

#include <cstdint>
#include <string>

#include "npp.h"

namespace npp {

constexpr int kMaxLevels = 3;
constexpr int kMaxAccesses = 6;

// S1: one nest = levels (size, sync) + accesses (contiguous level, execution-count mask).
struct Access {
  int contig;     // level whose index is stride-1 for this array (-1: none)
  unsigned mask;  // bit l set: N_l multiplies the execution count (Fig 8)
};

struct Nest {
  int pattern = 0;
  int L = 0;
  int64_t N[kMaxLevels] = {0, 0, 0};  // -1 = unknown size (G17)
  bool sync[kMaxLevels] = {false, false, false};
  int nacc = 0;
  Access acc[kMaxAccesses];
  int64_t cols = 0;  // matrix columns (sums), for the vector-width rule of R2
  int64_t K = 0;     // KMEANS_UPDATE: number of groups (the groupBy key range, not a nest level)
  int64_t E = 0;     // PAGERANK: number of edges (the inner level is sized by the average ceil(E/N))
};

struct Choice {  // one point of the candidate space plus its ControlDOP/R2 refinements
  int dims[kMaxLevels] = {0, 0, 0};
  int blocks[kMaxLevels] = {1, 1, 1};
  int spans[kMaxLevels] = {NPP_SPAN_ONE, NPP_SPAN_ONE, NPP_SPAN_ONE};
  int64_t factors[kMaxLevels] = {1, 1, 1};
  int64_t chunks[kMaxLevels] = {0, 0, 0};  // 0 = derive from span/factor (S9)
  int vec = 1;
  int staged = 0;  // 1: TMA-staged tile family (S8)
  int64_t persistent_grid = 0;  // staged: blocks launched (0: product of the level grids)
  int64_t claim_tiles = 0;      // staged: tiles per dynamic claim
  int64_t static_tiles = 0;     // staged sums: tiles split statically before the claim pool (Ts)
  int temp = NPP_TEMP_NONE;     // weighted sums: inner allocation (S10)
  int64_t temp_stride[2] = {0, 0};
};

// S10 (§V-A, Fig 11): the preallocated [outer x inner] buffer of a weighted sum is laid out
// for the mapping — outer level on x: offset m, stride M (Fig 11b); otherwise offset m*N, stride 1.
void temp_layout(const struct Nest& n, Choice* c);

constexpr int kStageRows = 32;  // BR of the staged family (S8): tiles of 32 rows x 1 KB
constexpr int64_t kStageRowsNarrowMx = 128;  // BR of the MX-narrow strips (S8): tiles of 128 rows x 256 B
constexpr int64_t kPoolDiv = 8;       // S8 balance rule: about 1/kPoolDiv of the tiles form the shared pool
constexpr int64_t kPoolUnit = 4;      // S8 balance rule: pool claim unit when outer tiles are long
constexpr int64_t kPoolUnitShort = 8;  // S8 balance rule: pool claim unit when outer tiles are 9-512 tiles
constexpr int64_t kPoolUnitShortTiMax = 512;
constexpr int64_t kWholeUnitMax = 8;  // S8 balance rule: outer tiles of <= 8 tiles are claimed whole

// S8 staged-family tiling shared with the kernels: a tile is BR rows x W columns (32 KB) made of
// 1 KB chunks of BC elements. Narrow: 32 rows x 1 KB; wide (SUM_ROWS with a row pitch that is a
// multiple of 4 KB): 8 rows x 4 KB.
struct StagedTiling {
  int64_t BR, BC, W;  // tile rows, chunk columns, tile columns
  int64_t To, Ti;     // tiles along the outer / inner level
  bool wide;
  bool r1 = false;    // SUM_ROWS one-row tiles of 32 KB (row pitch 64-256 KB, a multiple of 32 KB)
};
StagedTiling staged_tiling(int pattern, int64_t R, int64_t C, int dtype);
struct StagedBalance {
  int64_t G, U, Ts;  // persistent blocks, pool claim unit, statically split tiles
};
StagedBalance staged_balance(int64_t To, int64_t Ti, int sm_count);

// S8 RC (SUM_ROWS_COLS): the Tr x Tc grid of 32-row x 1 KB tiles is cut into gr x gc regions of cr row
// bands x cc column tiles (cc <= kRcColTilesMax: a region's column accumulators fit shared memory);
// G = min(SMs, nreg) blocks take contiguous region ranges.
constexpr int64_t kRcColTilesMax = 32;
struct RcTiling {
  int64_t BC, Tr, Tc, cr, cc, gr, gc, nreg, G;
};
RcTiling rc_tiling(int64_t R, int64_t C, int dtype, int sm_count);

// thread-local error message shared with the API layer
void set_error(const std::string& msg);

int dtype_size(int dtype);
bool is_sum_pattern(int pattern);
bool is_rows_pattern(int pattern);  // SUM_ROWS / SUM_WEIGHTED_ROWS
int build_nest(int pattern, const int64_t* shape, int ndim, Nest* out);
int check_limits(const npp_limits* lim);
bool hard_ok(const Nest& n, int dtype, const npp_limits& lim, const Choice& c);
int64_t score(const Nest& n, const npp_limits& lim, const Choice& c);
// full pipeline (S2..S9) into a record
int select_mapping(const Nest& n, int dtype, const npp_limits& lim, int strategy, npp_mapping* out);
// S9 for a caller-provided choice (npp_plan_with_mapping): validates and fills the record
int record_from_choice(const Nest& n, int dtype, const npp_limits& lim, Choice c, int64_t score_value,
                       npp_mapping* out);

}  // namespace npp
