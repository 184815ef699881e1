// api.cu — the C ABI of include/npp.h: limits query, plans, execution.
//
// npp_plan runs the CUDA-free selector (select.cpp: nest -> constraints -> Algorithm 1 -> ControlDOP
// -> R2) once per (pattern, shape, dtype, strategy) and freezes the mapping record; npp_execute only
// translates that record into one kernel launch of the matching family (§IV-E) — the
// paper's split between a static decision and launch-time parameters.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <mutex>
#include <map>
#include <string>
#include <utility>

#include "kernels.hpp"
#include "select.hpp"

namespace npp {
extern thread_local std::string g_error;

cudaError_t ensure_smem_attr(const void* func, int smem_bytes) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return e;
  // the attribute is an upper bound: keep the largest value set so far per (kernel, device), raise it
  // when a launch needs more (a smaller later value would break launches that need the larger one)
  static std::mutex mu;
  static std::map<std::pair<const void*, int>, int> cur;
  std::lock_guard<std::mutex> lock(mu);
  int& have = cur[std::make_pair(func, dev)];
  if (have >= smem_bytes) return cudaSuccess;
  e = cudaFuncSetAttribute(func, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_bytes);
  if (e == cudaSuccess) have = smem_bytes;
  return e;
}
}  // namespace npp

struct npp_plan_s {
  int pattern = 0;
  int dtype = 0;
  int strategy = 0;
  int ndim = 0;
  int64_t shape[3] = {0, 0, 0};
  bool empty = false;
  npp_mapping map{};
  npp_limits lim{};
};

namespace {

using npp::set_error;

int cuda_fail(const char* what, cudaError_t e) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, cudaGetErrorString(e));
  set_error(buf);
  return NPP_ERR_CUDA;
}

int n_inputs(int pattern) {
  switch (pattern) {
    case NPP_SUM_ROWS:
    case NPP_SUM_COLS:
    case NPP_SUM_ROWS_COLS: return 1;
    case NPP_SUM_WEIGHTED_ROWS:
    case NPP_SUM_WEIGHTED_COLS:
    case NPP_KMEANS_ASSIGN:
    case NPP_KMEANS_UPDATE: return 2;
    case NPP_LOGREG_GRAD: return 3;
    case NPP_PAGERANK: return 4;
    default: return -1;
  }
}

// bytes of input k and of the output, for npp_execute_host
int64_t input_bytes(const npp_plan_s* p, int k) {
  const int64_t es = npp::dtype_size(p->dtype);
  const int64_t* s = p->shape;
  switch (p->pattern) {
    case NPP_SUM_ROWS:
    case NPP_SUM_COLS:
    case NPP_SUM_ROWS_COLS: return s[0] * s[1] * es;
    case NPP_SUM_WEIGHTED_ROWS: return k == 0 ? s[0] * s[1] * es : s[1] * es;
    case NPP_SUM_WEIGHTED_COLS: return k == 0 ? s[0] * s[1] * es : s[0] * es;
    case NPP_KMEANS_ASSIGN: return k == 0 ? s[0] * s[1] * 4 : s[2] * s[1] * 4;
    case NPP_KMEANS_UPDATE: return k == 0 ? s[0] * s[1] * 4 : s[0] * 4;
    case NPP_PAGERANK: return k == 0 ? (s[0] + 1) * 8 : (k == 1 ? s[1] * 4 : (p->ndim == 3 ? s[2] : s[0]) * 4);
    case NPP_LOGREG_GRAD: return k == 0 ? s[0] * s[1] * s[2] * 4 : (k == 1 ? s[0] * s[1] * 4 : s[2] * 4);
    default: return 0;
  }
}

int64_t output_bytes(const npp_plan_s* p) {
  const int64_t es = npp::dtype_size(p->dtype);
  const int64_t* s = p->shape;
  switch (p->pattern) {
    case NPP_SUM_ROWS:
    case NPP_SUM_WEIGHTED_ROWS: return s[0] * es;
    case NPP_SUM_COLS:
    case NPP_SUM_WEIGHTED_COLS: return s[1] * es;
    case NPP_SUM_ROWS_COLS: return (s[0] + s[1]) * es;
    case NPP_KMEANS_ASSIGN: return s[0] * 4;
    case NPP_KMEANS_UPDATE: return s[2] * (s[1] + 1) * 4;
    case NPP_PAGERANK: return s[0] * 4;
    case NPP_LOGREG_GRAD: return s[0] * s[2] * 4;
    default: return 0;
  }
}

int validate_request(int pattern, const int64_t* shape, int ndim, int dtype, bool* empty) {
  if (!shape || ndim < 1 || ndim > 3) {
    set_error("shape must hold 2 or 3 sizes");
    return NPP_ERR_INVALID_ARG;
  }
  if (dtype < NPP_F32 || dtype > NPP_F64) {
    set_error("unknown dtype");
    return NPP_ERR_INVALID_ARG;
  }
  if (n_inputs(pattern) < 0) {
    set_error("unknown pattern");
    return NPP_ERR_INVALID_ARG;
  }
  if ((pattern == NPP_KMEANS_ASSIGN || pattern == NPP_LOGREG_GRAD || pattern == NPP_KMEANS_UPDATE ||
       pattern == NPP_PAGERANK) &&
      dtype != NPP_F32) {
    set_error("k-means, logreg and PageRank are defined for f32");
    return NPP_ERR_UNSUPPORTED;
  }
  *empty = false;
  for (int d = 0; d < ndim; ++d) {
    if (shape[d] < 0) {
      set_error("npp_plan needs known, non-negative sizes");
      return NPP_ERR_INVALID_ARG;
    }
    // a PageRank step over N > 0 nodes without edges still writes (1 - damp) / N: only N = 0 is empty
    if (shape[d] == 0 && !(pattern == NPP_PAGERANK && d == 1)) *empty = true;
  }
  return NPP_OK;
}

int get_limits(const npp_limits* limits, npp_limits* out) {
  if (limits) {
    *out = *limits;
    return npp::check_limits(out);
  }
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail("cudaGetDevice", e);
  return npp_limits_query(dev, out);
}

inline bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

}  // namespace

extern "C" {

int npp_version(void) { return NPP_VERSION; }

const char* npp_last_error(void) { return npp::g_error.c_str(); }

int npp_limits_query(int device, npp_limits* out) {
  if (!out) {
    set_error("out is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  cudaDeviceProp prop;
  cudaError_t e = cudaGetDeviceProperties(&prop, device);
  if (e != cudaSuccess) return cuda_fail("cudaGetDeviceProperties", e);
  npp_limits l{};
  l.sm_count = prop.multiProcessorCount;
  l.max_threads_per_sm = prop.maxThreadsPerMultiProcessor;
  l.max_threads_per_block = prop.maxThreadsPerBlock;
  l.max_block_dim[0] = prop.maxThreadsDim[0];
  l.max_block_dim[1] = prop.maxThreadsDim[1];
  l.max_block_dim[2] = prop.maxThreadsDim[2];
  l.warp_size = prop.warpSize;
  l.max_blocks_per_sm = prop.maxBlocksPerMultiProcessor;
  l.regs_per_sm = prop.regsPerMultiprocessor;
  l.regs_per_block = prop.regsPerBlock;
  l.smem_per_block = int64_t(prop.sharedMemPerBlockOptin);
  int regs = npp::sum_kernels_max_regs();
  l.regs_per_thread = regs > 0 ? regs : 1;
  *out = l;
  return NPP_OK;
}

int npp_plan(int pattern, const int64_t* shape, int ndim, int dtype, int strategy, const npp_limits* limits,
             npp_plan_t* out) {
  if (!out) {
    set_error("out is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  *out = nullptr;
  bool empty = false;
  int st = validate_request(pattern, shape, ndim, dtype, &empty);
  if (st) return st;
  npp_plan_s* p = new npp_plan_s();
  p->pattern = pattern;
  p->dtype = dtype;
  p->strategy = strategy;
  p->ndim = ndim;
  for (int d = 0; d < ndim; ++d) p->shape[d] = shape[d];
  p->empty = empty;
  if (empty) {
    p->map = npp_mapping{};
    p->map.kernel_class = NPP_CLASS_EMPTY;
    *out = p;
    return NPP_OK;
  }
  if (pattern == NPP_SUM_ROWS_COLS && strategy != NPP_MAP_AUTO) {
    delete p;
    set_error("SUM_ROWS_COLS executes with strategy AUTO only (the one-pass family); the paper's two-kernel "
              "schedule is a SUM_ROWS plan plus a SUM_COLS plan");
    return NPP_ERR_UNSUPPORTED;
  }
  if (pattern == NPP_KMEANS_UPDATE && strategy != NPP_MAP_AUTO) {
    delete p;
    set_error("KMEANS_UPDATE executes with strategy AUTO only (class KU)");
    return NPP_ERR_UNSUPPORTED;
  }
  if (pattern == NPP_PAGERANK && strategy != NPP_MAP_AUTO) {
    delete p;
    set_error("PAGERANK executes with strategy AUTO only (class PR)");
    return NPP_ERR_UNSUPPORTED;
  }
  if (pattern == NPP_PAGERANK && ndim >= 2 && shape[1] >= (int64_t(1) << 31)) {
    delete p;
    set_error("PAGERANK plans need E < 2^31 edges (the kernel keeps 32-bit edge offsets inside a row chunk)");
    return NPP_ERR_UNSUPPORTED;
  }
  st = get_limits(limits, &p->lim);
  if (!st) st = npp_select(pattern, shape, ndim, dtype, &p->lim, strategy, &p->map);
  if (st) {
    delete p;
    return st;
  }
  if (p->map.kernel_class == NPP_CLASS_LOGREG && !p->map.staged) {
    delete p;
    set_error("LOGREG_GRAD executes through its staged (AUTO) kernel family only");
    return NPP_ERR_UNSUPPORTED;
  }
  if (p->map.kernel_class == NPP_CLASS_KMEANS && !p->map.staged) {  // direct executor: no Split
    for (int l = 0; l < p->map.nlevels; ++l)
      if (p->map.level[l].span == NPP_SPLIT_K) {
        delete p;
        set_error("KMEANS_ASSIGN mappings with Split(k) on a reduce level are not executable (AUTO or a mapping "
                  "without Split)");
        return NPP_ERR_UNSUPPORTED;
      }
  }
  if (pattern == NPP_SUM_ROWS_COLS && strategy != NPP_MAP_AUTO) {  // (also checked before selection)
    delete p;
    set_error("SUM_ROWS_COLS executes with strategy AUTO only (the one-pass family); the paper's two-kernel "
              "schedule is a SUM_ROWS plan plus a SUM_COLS plan");
    return NPP_ERR_UNSUPPORTED;
  }
  *out = p;
  return NPP_OK;
}

int npp_plan_with_mapping(int pattern, const int64_t* shape, int ndim, int dtype, const npp_mapping* forced,
                          const npp_limits* limits, npp_plan_t* out) {
  if (!out || !forced) {
    set_error("out/forced is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  *out = nullptr;
  bool empty = false;
  int st = validate_request(pattern, shape, ndim, dtype, &empty);
  if (st) return st;
  if (empty) {
    set_error("npp_plan_with_mapping needs non-empty sizes");
    return NPP_ERR_INVALID_ARG;
  }
  npp_limits lim{};
  st = get_limits(limits, &lim);
  if (st) return st;
  npp::Nest nest;
  st = npp::build_nest(pattern, shape, ndim, &nest);
  if (st) return st;
  if (forced->nlevels != nest.L) {
    set_error("forced mapping has the wrong number of levels");
    return NPP_ERR_INVALID_ARG;
  }
  npp::Choice c;
  bool seen[3] = {false, false, false};
  for (int l = 0; l < nest.L; ++l) {
    const npp_level& lv = forced->level[l];
    if (lv.dim < 0 || lv.dim >= nest.L || seen[lv.dim] || lv.span < 0 || lv.span > 3 || lv.block < 1 ||
        lv.factor < 1) {
      set_error("forced mapping: dims must be an injective assignment of the first L dims; spans 0..3;"
                " blocks and factors >= 1");
      return NPP_ERR_INVALID_ARG;
    }
    seen[lv.dim] = true;
    c.dims[l] = lv.dim;
    c.blocks[l] = lv.block;
    c.spans[l] = lv.span;
    c.factors[l] = lv.factor;
    if (lv.span == NPP_SPLIT_K && !nest.sync[l]) {
      set_error("Split(k) applies only where Span(all) was forced by a Reduce (P:L545-546)");
      return NPP_ERR_NO_FEASIBLE_MAPPING;
    }
  }
  if (!npp::hard_ok(nest, dtype, lim, c)) {
    set_error("forced mapping violates a hard constraint (Table II / device limits)");
    return NPP_ERR_NO_FEASIBLE_MAPPING;
  }
  if (pattern == NPP_KMEANS_ASSIGN) {  // the direct 3-level executor (kern_kmeans_direct.cu): no Split, no vec
    for (int l = 0; l < nest.L; ++l)
      if (c.spans[l] == NPP_SPLIT_K) {
        set_error("KMEANS_ASSIGN mappings with Split(k) on a reduce level are not executable");
        return NPP_ERR_UNSUPPORTED;
      }
    if (forced->vec > 1 || forced->temp != NPP_TEMP_NONE) {
      set_error("KMEANS_ASSIGN mappings take vec = 1 and no temp");
      return NPP_ERR_UNSUPPORTED;
    }
    npp_plan_s* p = new npp_plan_s();
    p->pattern = pattern;
    p->dtype = dtype;
    p->strategy = -1;
    p->ndim = ndim;
    for (int d = 0; d < ndim; ++d) p->shape[d] = shape[d];
    p->lim = lim;
    c.vec = 1;
    npp::record_from_choice(nest, dtype, lim, c, npp::score(nest, lim, c), &p->map);
    *out = p;
    return NPP_OK;
  }
  if (!npp::is_sum_pattern(pattern)) {
    set_error("explicit mappings are executable for the 2-level sum families and KMEANS_ASSIGN only");
    return NPP_ERR_UNSUPPORTED;
  }
  // class RX (inner Reduce on x) finishes a row with xor-shuffles over min(b_x, 32) lanes: the x block must
  // be a power of two <= 32 or a multiple of 32, or two rows would share (or lose) lanes of one warp
  if (c.dims[1] == NPP_DIM_X) {
    const int bx = c.blocks[1];
    if (!((bx <= 32 && (bx & (bx - 1)) == 0) || bx % 32 == 0)) {
      set_error("explicit RX mapping: the x-level block must be a power of two <= 32 or a multiple of 32");
      return NPP_ERR_UNSUPPORTED;
    }
  }
  // vector width: only on the x level when it is the stride-1 level of m and C % vec == 0
  const int v0 = 16 / npp::dtype_size(dtype);
  const bool rows = pattern == NPP_SUM_ROWS || pattern == NPP_SUM_WEIGHTED_ROWS;
  const int x_level = c.dims[0] == NPP_DIM_X ? 0 : 1;
  c.vec = forced->vec <= 1 ? 1 : forced->vec;
  if (c.vec != 1 && (c.vec != v0 || x_level != (rows ? 1 : 0) || nest.cols % v0 != 0)) {
    set_error("vec must be 1, or 16/sizeof(dtype) on the stride-1 x level with C % vec == 0");
    return NPP_ERR_UNSUPPORTED;
  }
  // S10: the inner allocation of a weighted sum (NONE, MALLOC, or PREALLOC with a Fig 11 layout)
  const bool weighted_pat = pattern == NPP_SUM_WEIGHTED_ROWS || pattern == NPP_SUM_WEIGHTED_COLS;
  c.temp = forced->temp;
  if (c.temp != NPP_TEMP_NONE) {
    const int64_t M = nest.N[0], N = nest.N[1];
    if (!weighted_pat || c.vec != 1 || (c.temp != NPP_TEMP_MALLOC && c.temp != NPP_TEMP_PREALLOC)) {
      set_error("temp (S10) applies to the weighted sums with vec = 1 (NONE, MALLOC or PREALLOC)");
      return NPP_ERR_UNSUPPORTED;
    }
    if (c.temp == NPP_TEMP_PREALLOC) {
      const int64_t so = forced->temp_stride[0], si = forced->temp_stride[1];
      if (!((so == N && si == 1) || (so == 1 && si == M))) {
        set_error("PREALLOC temp strides must be (inner, 1) (Fig 11a) or (1, outer) (Fig 11b)");
        return NPP_ERR_INVALID_ARG;
      }
      c.temp_stride[0] = so;
      c.temp_stride[1] = si;
    } else {
      c.temp_stride[0] = 0;
      c.temp_stride[1] = 1;
      // device-side malloc draws from the context's heap; it can only be sized before the first
      // kernel that uses it, so the first MALLOC plan reserves max(1 GiB, 1.25 x the nest's bytes)
      const size_t need = size_t(double(M) * double(N) * npp::dtype_size(dtype) * 1.25) + (64u << 20);
      size_t cur = 0;
      if (cudaDeviceGetLimit(&cur, cudaLimitMallocHeapSize) != cudaSuccess) cur = 0;
      if (cur < need) {
        const size_t want = need > (size_t(1) << 30) ? need : (size_t(1) << 30);
        if (cudaDeviceSetLimit(cudaLimitMallocHeapSize, want) != cudaSuccess) {
          cudaGetLastError();
          set_error("MALLOC temp: the device malloc heap is already fixed below this nest's size");
          return NPP_ERR_UNSUPPORTED;
        }
      }
    }
  }
  npp_plan_s* p = new npp_plan_s();
  p->pattern = pattern;
  p->dtype = dtype;
  p->strategy = -1;
  p->ndim = ndim;
  for (int d = 0; d < ndim; ++d) p->shape[d] = shape[d];
  p->lim = lim;
  npp::record_from_choice(nest, dtype, lim, c, npp::score(nest, lim, c), &p->map);
  *out = p;
  return NPP_OK;
}

int npp_plan_mapping(npp_plan_t plan, npp_mapping* out) {
  if (!plan || !out) {
    set_error("plan/out is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  *out = plan->map;
  return NPP_OK;
}

int64_t npp_plan_workspace_bytes(npp_plan_t plan) { return plan ? plan->map.workspace_bytes : 0; }

int npp_plan_launches(npp_plan_t plan) {
  if (!plan) return 0;
  if (plan->empty) return output_bytes(plan) > 0 ? 1 : 0;
  // k-means (staged): centroid pack + assignment; PageRank: per-node contribution + the CSR kernel
  return ((plan->pattern == NPP_KMEANS_ASSIGN && plan->map.staged) || plan->pattern == NPP_PAGERANK) ? 2 : 1;
}

void npp_plan_destroy(npp_plan_t plan) { delete plan; }

}  // extern "C"

namespace {

// npp_execute_ex / npp_execute_traced: `trace` (device, may be NULL) receives the tile schedule
int execute_impl(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace, void* stream,
                 unsigned flags, int* trace) {
  if (flags & ~(NPP_EXEC_OVERLAP | NPP_EXEC_NO_PDL)) {
    set_error("unknown npp_execute_ex flag bits");
    return NPP_ERR_INVALID_ARG;
  }
  if ((flags & NPP_EXEC_OVERLAP) && (flags & NPP_EXEC_NO_PDL)) {
    set_error("NPP_EXEC_OVERLAP needs a programmatic dependent launch (not NPP_EXEC_NO_PDL)");
    return NPP_ERR_INVALID_ARG;
  }
  const bool overlap = (flags & NPP_EXEC_OVERLAP) != 0;
  const int pdl = (flags & NPP_EXEC_NO_PDL) ? 0 : 1;
  if (!plan) {
    set_error("plan is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (plan->empty) {
    const int64_t ob = output_bytes(plan);
    if (ob > 0) {
      if (!out) {
        set_error("out is NULL");
        return NPP_ERR_INVALID_ARG;
      }
      cudaError_t e = cudaMemsetAsync(out, 0, size_t(ob), st);
      if (e != cudaSuccess) return cuda_fail("cudaMemsetAsync", e);
    }
    return NPP_OK;
  }
  const int need = n_inputs(plan->pattern);
  if (!ins || n_in != need || !out) {
    set_error("wrong number of inputs or NULL pointer");
    return NPP_ERR_INVALID_ARG;
  }
  for (int k = 0; k < need; ++k)
    if (!ins[k] && !(plan->pattern == NPP_PAGERANK && k == 1 && plan->shape[1] == 0)) {  // E = 0: no colidx
      set_error("input pointer is NULL");
      return NPP_ERR_INVALID_ARG;
    }
  const npp_mapping& m = plan->map;
  if (m.workspace_bytes > 0 && !workspace) {
    set_error("this plan needs a workspace (npp_plan_workspace_bytes)");
    return NPP_ERR_WORKSPACE;
  }
  if (m.vec > 1 || m.staged) {
    for (int k = 0; k < need; ++k)
      if (!aligned16(ins[k])) {
        set_error("vectorised / TMA-staged plan: inputs must be 16-byte aligned");
        return NPP_ERR_ALIGNMENT;
      }
  }
  if (plan->pattern == NPP_LOGREG_GRAD) {  // class LR (S8)
    npp::LogregArgs g{};
    g.y = static_cast<const float*>(ins[1]);
    g.w = static_cast<const float*>(ins[2]);
    g.g = static_cast<float*>(out);
    g.B = plan->shape[0];
    g.Rb = plan->shape[1];
    g.C = plan->shape[2];
    g.Ti = (g.Rb + 31) / 32;
    g.per_block = m.claim_tiles;
    g.tickets = static_cast<unsigned*>(workspace);
    g.acc = reinterpret_cast<double*>(static_cast<char*>(workspace) + ((4 * g.B + 255) / 256) * 256);
    g.trace = trace;
    cudaError_t e = npp::launch_logreg(g, static_cast<const float*>(ins[0]), int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("logreg kernel launch", e);
    return NPP_OK;
  }
  if (plan->pattern == NPP_KMEANS_ASSIGN && !m.staged) {  // class KM, direct executor (LITERAL / explicit)
    npp::KmDirectArgs k{};
    k.x = static_cast<const float*>(ins[0]);
    k.c = static_cast<const float*>(ins[1]);
    k.assign = static_cast<int*>(out);
    k.N = plan->shape[0];
    k.D = int(plan->shape[1]);
    k.K = int(plan->shape[2]);
    for (int l = 0; l < 3; ++l) {
      k.dim[l] = m.level[l].dim;
      k.blk[l] = m.level[l].block;
    }
    k.chunk0 = m.level[0].chunk;
    cudaError_t e = npp::launch_kmeans_direct(k, int(m.level[0].grid), st);
    if (e != cudaSuccess) return cuda_fail("kmeans direct kernel launch", e);
    return NPP_OK;
  }
  if (plan->pattern == NPP_KMEANS_ASSIGN) {  // class KM (S8)
    npp::KmeansArgs k{};
    k.c = static_cast<const float*>(ins[1]);
    k.assign = static_cast<int*>(out);
    k.N = plan->shape[0];
    k.D = plan->shape[1];
    k.K = plan->shape[2];
    k.per_block = m.claim_tiles;
    k.sets = m.level[0].block / 64;
    k.trace = trace;
    cudaError_t e = npp::launch_kmeans(k, static_cast<const float*>(ins[0]), int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("kmeans kernel launch", e);
    return NPP_OK;
  }
  if (plan->pattern == NPP_PAGERANK) {  // class PR (S8 PR)
    npp::PagerankArgs r{};
    r.rowptr = static_cast<const long long*>(ins[0]);
    r.colidx = static_cast<const int*>(ins[1]);
    r.pr = static_cast<const float*>(ins[2]);
    r.outdeg = static_cast<const int*>(ins[3]);
    r.out = static_cast<float*>(out);
    r.pool = static_cast<unsigned*>(workspace);
    r.contrib = reinterpret_cast<float*>(static_cast<char*>(workspace) + 256);
    r.N = plan->shape[0];
    r.Nnodes = plan->ndim == 3 ? plan->shape[2] : plan->shape[0];
    r.damp = 0.85f;
    const int seg = m.level[1].span == NPP_SPLIT_K ? int(m.claim_tiles) : 0;  // S8 PR: segmented or row groups
    cudaError_t e = npp::launch_pagerank(r, m.level[1].block, seg, int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("PageRank kernel launch", e);
    return NPP_OK;
  }
  if (plan->pattern == NPP_KMEANS_UPDATE) {  // class KU (S8 KU)
    npp::KmUpdateArgs u{};
    u.out = static_cast<float*>(out);
    u.ticket = static_cast<unsigned*>(workspace);
    u.acc = reinterpret_cast<double*>(static_cast<char*>(workspace) + 256);
    u.N = plan->shape[0];
    u.D = plan->shape[1];
    u.K = plan->shape[2];
    u.per_block = m.claim_tiles;
    u.early_reads = overlap ? 1 : 0;
    u.pdl = pdl;
    u.trace = trace;
    cudaError_t e = npp::launch_kmupdate(u, static_cast<const float*>(ins[0]), static_cast<const int*>(ins[1]),
                                         int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("k-means update kernel launch", e);
    return NPP_OK;
  }
  if (plan->pattern == NPP_SUM_ROWS_COLS) {  // class RC (S8 RC): one pass, both outputs
    const npp::RcTiling t = npp::rc_tiling(plan->shape[0], plan->shape[1], plan->dtype, plan->lim.sm_count);
    const int64_t ab = plan->dtype == NPP_I32 ? 4 : 8;
    char* ws = static_cast<char*>(workspace);
    npp::RowsColsArgs r{};
    r.m = ins[0];
    r.out = out;
    r.R = plan->shape[0];
    r.C = plan->shape[1];
    r.Tr = t.Tr, r.Tc = t.Tc, r.cr = t.cr, r.cc = t.cc, r.gr = t.gr, r.gc = t.gc, r.nreg = t.nreg;
    const int64_t o_tc = ((4 * t.gr + 255) / 256) * 256;
    const int64_t o_ar = o_tc + ((4 * t.gc + 255) / 256) * 256;
    const int64_t o_ac = o_ar + ((r.R * ab + 255) / 256) * 256;
    r.tick_r = reinterpret_cast<unsigned*>(ws);
    r.tick_c = reinterpret_cast<unsigned*>(ws + o_tc);
    r.accR = ws + o_ar;
    r.accC = ws + o_ac;
    r.early_reads = overlap ? 1 : 0;
    r.pdl = pdl;
    r.trace = trace;
    cudaError_t e = npp::launch_rowscols(plan->dtype, m.staged != 0, r, int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("rows+cols kernel launch", e);
    return NPP_OK;
  }
  if (!npp::is_sum_pattern(plan->pattern)) {
    set_error("pattern not executable in this build");
    return NPP_ERR_UNSUPPORTED;
  }
  const bool rows = plan->pattern == NPP_SUM_ROWS || plan->pattern == NPP_SUM_WEIGHTED_ROWS;
  const bool weighted = plan->pattern == NPP_SUM_WEIGHTED_ROWS || plan->pattern == NPP_SUM_WEIGHTED_COLS;
  const int64_t R = plan->shape[0], C = plan->shape[1];
  if (m.staged) {  // TMA tile family (S8 staged)
    const npp::StagedTiling t = npp::staged_tiling(plan->pattern, R, C, plan->dtype);
    npp::StagedArgs s{};
    s.out = out;
    s.v = weighted ? ins[1] : nullptr;
    s.R = R;
    s.C = C;
    s.O = rows ? R : C;
    s.To = t.To;
    s.Ti = t.Ti;
    const npp::StagedBalance bal = npp::staged_balance(t.To, t.Ti, plan->lim.sm_count);
    s.static_tiles = bal.Ts;
    s.unit = bal.U;
    {  // S8 claim order: units of U, then the last F = min(G, T - Ts) tiles singly when U < Ti
      const int64_t T = t.To * t.Ti, G = m.grid;
      const int64_t F = bal.U < t.Ti ? std::min<int64_t>(G, T - bal.Ts) : 0;
      s.tail_start = T - F;
      s.big_units = (s.tail_start - bal.Ts + bal.U - 1) / bal.U;
      s.claims = s.big_units + F;
    }
    s.early_reads = overlap ? 1 : 0;
    s.pdl = pdl;
    s.trace = trace;
    s.wide = t.r1 ? 2 : (t.wide ? 1 : 0);
    s.pool = static_cast<unsigned*>(workspace);  // S9 staged workspace: [256 B pool][tickets][acc]
    s.tickets = reinterpret_cast<unsigned*>(static_cast<char*>(workspace) + 256);
    s.acc = static_cast<char*>(workspace) + 256 + ((t.To * 4 + 255) / 256) * 256;
    cudaError_t e = npp::launch_sum_staged(plan->dtype, rows, ins[0], s, int(m.grid), st);
    if (e != cudaSuccess) return cuda_fail("staged kernel launch", e);
    return NPP_OK;
  }
  npp::SumArgs a{};
  a.m = ins[0];
  a.v = weighted ? ins[1] : nullptr;
  a.out = out;
  a.O = rows ? R : C;
  a.I = rows ? C : R;
  a.so = rows ? C : 1;
  a.si = rows ? 1 : C;
  const npp_level& lo = m.level[0];
  const npp_level& li = m.level[1];
  a.bo = lo.block;
  a.bi = li.block;
  a.co = lo.chunk;
  a.ci = li.chunk;
  a.go = lo.grid;
  a.gi = li.grid;
  int64_t ws_used = 0;  // S9 workspace: [partials][tickets] (Split), then the S10 temp region
  if (a.gi > 1) {
    const int acc = plan->dtype == NPP_I32 ? 4 : 8;
    const int64_t part = ((a.gi * a.O * acc + 255) / 256) * 256;
    a.partials = workspace;
    a.tickets = reinterpret_cast<unsigned*>(static_cast<char*>(workspace) + part);
    ws_used = part + ((a.go * 4 + 255) / 256) * 256;
  }
  if (m.temp != NPP_TEMP_NONE) {  // S10: the weighted sum with its zipWith materialised
    if (m.temp == NPP_TEMP_PREALLOC) {
      a.temp = static_cast<char*>(workspace) + ws_used;
      a.ts_o = m.temp_stride[0];
      a.ts_i = m.temp_stride[1];
    } else {
      a.err = reinterpret_cast<unsigned*>(static_cast<char*>(workspace) + ws_used);
    }
    cudaError_t e = npp::launch_sum_temp(plan->dtype, m.kernel_class, m.temp == NPP_TEMP_MALLOC, a, st);
    if (e != cudaSuccess) return cuda_fail("temp kernel launch", e);
    return NPP_OK;
  }
  cudaError_t e = npp::launch_sum(plan->dtype, m.kernel_class, m.vec, weighted, a, st);
  if (e != cudaSuccess) return cuda_fail("kernel launch", e);
  return NPP_OK;
}

}  // namespace

extern "C" {

int npp_execute(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace, void* stream) {
  return execute_impl(plan, ins, n_in, out, workspace, stream, 0u, nullptr);
}

int npp_execute_ex(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace, void* stream,
                   unsigned flags) {
  return execute_impl(plan, ins, n_in, out, workspace, stream, flags, nullptr);
}

int64_t npp_plan_tiles(npp_plan_t plan) {
  if (!plan || plan->empty) return 0;
  const npp_mapping& m = plan->map;
  const int64_t* s = plan->shape;
  switch (m.kernel_class) {
    case NPP_CLASS_RX:
    case NPP_CLASS_MX:
      if (!m.staged) return 0;
      return m.level[0].grid * m.level[1].grid;  // To x Ti (S9: chunk = one tile per level)
    case NPP_CLASS_LOGREG: return s[0] * ((s[1] + 31) / 32);
    case NPP_CLASS_KMEANS:
      if (!m.staged) return 0;
      return (s[0] + (s[1] <= 64 ? 255 : 127)) / (s[1] <= 64 ? 256 : 128);
    case NPP_CLASS_KMUPDATE: return (s[0] + 95) / 96;  // S8 KU tiles
    case NPP_CLASS_RC: return m.level[0].grid * m.level[1].grid;
    default: return 0;
  }
}

int npp_execute_traced(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace, void* stream,
                       int32_t* trace) {
  if (!trace) {
    set_error("trace is NULL");
    return NPP_ERR_INVALID_ARG;
  }
  if (npp_plan_tiles(plan) <= 0) {
    set_error("npp_execute_traced: the plan has no tile schedule (staged families only)");
    return NPP_ERR_UNSUPPORTED;
  }
  return execute_impl(plan, ins, n_in, out, workspace, stream, 0u, trace);
}

int npp_execute_host(npp_plan_t plan, const void* const* host_ins, int n_in, void* host_out,
                     void* const* dev_ins, void* dev_out, void* workspace, void* stream) {
  if (!plan || !host_out || !dev_out || (n_in > 0 && (!host_ins || !dev_ins))) {
    set_error("NULL argument");
    return NPP_ERR_INVALID_ARG;
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!plan->empty) {
    if (n_in != n_inputs(plan->pattern)) {
      set_error("wrong number of inputs");
      return NPP_ERR_INVALID_ARG;
    }
    for (int k = 0; k < n_in; ++k) {
      cudaError_t e = cudaMemcpyAsync(dev_ins[k], host_ins[k], size_t(input_bytes(plan, k)),
                                      cudaMemcpyHostToDevice, st);
      if (e != cudaSuccess) return cuda_fail("cudaMemcpyAsync H2D", e);
    }
  }
  int rc = npp_execute(plan, const_cast<const void* const*>(reinterpret_cast<void* const*>(dev_ins)), n_in,
                       dev_out, workspace, stream);
  if (rc) return rc;
  cudaError_t e = cudaMemcpyAsync(host_out, dev_out, size_t(output_bytes(plan)), cudaMemcpyDeviceToHost, st);
  if (e != cudaSuccess) return cuda_fail("cudaMemcpyAsync D2H", e);
  e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return cuda_fail("cudaStreamSynchronize", e);
  return NPP_OK;
}

}  // extern "C"
