/*
 * npp.h — C ABI of the B200-native nested-parallel-pattern library (libnpp.so).
 *
 * Implements the data-parallel hot path of Lee et al., "Locality-Aware Mapping of Nested Parallel
 * Patterns on GPUs" (MICRO'14; /root/reference/PAPER.md, cited P:L<line>): a nested pattern is mapped
 * onto a logical multidimensional thread domain — per nest level a dimension, a block size and a
 * span (Span(1) / Span(n) / Span(all) / Split(k), §IV-A) — chosen by Algorithm 1
 * (§IV-D) and executed by one hand-written sm_100a kernel family per mapping class
 * (§IV-E).  The exact selection rules are DESIGN.md §3.
 *
 * Conventions for every entry point
 *   - Plain C types only. Device pointers are raw CUDA device addresses; `stream` is a cudaStream_t
 *     passed as void* (NULL = legacy default stream).
 *   - Return value: NPP_OK (0) or a negative npp_status. On error a thread-local message is
 *     available from npp_last_error(). No C++ exception crosses this boundary.
 *   - The library never allocates device memory and never allocates inside kernels (§V-A):
 *     the caller owns inputs, outputs and the workspace (size from npp_plan_workspace_bytes).
 *   - Layout: dense row-major, leading dimension = number of columns; no padding, no views.
 *   - Results: output dtype = input dtype. Integer sums wrap modulo 2^32 / 2^64 (accumulated as
 *     unsigned). fp32 sums accumulate in fp64 (fp32 only inside one 16-byte vector), so each output is
 *     within 1e-5 * Σ|terms| of the exact sum.
 */
#ifndef NPP_H_
#define NPP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define NPP_VERSION 4  /* 3: SUM_ROWS_COLS, KMEANS_UPDATE, PAGERANK; 4: static_tiles, NPP_EXEC_NO_PDL, traces, F64 */

#if defined(__GNUC__)
#define NPP_API __attribute__((visibility("default")))
#else
#define NPP_API
#endif
#define NPP_MAX_LEVELS 4

typedef enum {
  NPP_OK = 0,
  NPP_ERR_INVALID_ARG = -1,          /* bad pattern/dtype/shape/pointer/strategy */
  NPP_ERR_UNSUPPORTED = -2,          /* valid request this build does not implement */
  NPP_ERR_ALIGNMENT = -3,            /* plan uses 16-byte vector loads; a pointer is not 16-B aligned */
  NPP_ERR_WORKSPACE = -4,            /* workspace NULL or too small for the plan */
  NPP_ERR_NO_FEASIBLE_MAPPING = -5,  /* no candidate satisfies the hard constraints (Table II) */
  NPP_ERR_CUDA = -6                  /* a CUDA runtime call or kernel launch failed */
} npp_status;

/* F64: the sums in double (the fp64 of Fig 9's generated kernel), accumulated in fp64 */
typedef enum { NPP_F32 = 0, NPP_I32 = 1, NPP_I64 = 2, NPP_F64 = 3 } npp_dtype;

/* Patterns (shape, inputs, output) — Fig 1, Fig 15, BASELINE.json configs 4-5.
 *   SUM_ROWS           {R,C}   ins={m[R*C]}                  out[R]  = Σ_c m[r,c]
 *   SUM_COLS           {R,C}   ins={m[R*C]}                  out[C]  = Σ_r m[r,c]
 *   KMEANS_ASSIGN      {N,D,K} ins={x[N*D] f32, c[K*D] f32}  out[N] int32 = argmin_k Σ_d (x-c)^2, ties→lowest k
 *   LOGREG_GRAD        {B,Rb,C} ins={x[B*Rb*C] f32, y[B*Rb] f32, w[C] f32}
 *                                                            out[B*C] f32 = Σ_{i in batch b} x_ij(σ(x_i·w)-y_i)
 *   SUM_WEIGHTED_ROWS  {R,C}   ins={m[R*C], v[C]}            out[R]  = Σ_c m[r,c]·v[c]
 *   SUM_WEIGHTED_COLS  {R,C}   ins={m[R*C], v[R]}            out[C]  = Σ_r m[r,c]·v[r]
 *   SUM_ROWS_COLS      {R,C}   ins={m[R*C]}                  out[R+C] = [Σ_c m[r,c] (r<R) | Σ_r m[r,c] (c<C)]
 *                      both outputs of the Naive Bayes counts (§VI-E) from ONE read of m;
 *                      executable with strategy AUTO (npp_select/npp_enumerate give every strategy's
 *                      record for analysis; the paper's two-kernel schedule = a SUM_ROWS and a SUM_COLS plan)
 *   KMEANS_UPDATE      {N,D,K} ins={x[N*D] f32, a[N] int32}  out[K*(D+1)] f32: row k = (Σ_{i: a_i=k} x_i, count_k)
 *                      the centroid update after an assignment: Table I groupBy + Reduce per group;
 *                      keys outside [0,K) belong to no group; counts exact below 2^24. AUTO only.
 *   PAGERANK           {N,E}   ins={rowptr[N+1] int64, colidx[E] int32, pr[N] f32, outdeg[N] int32}
 *                      out[N] f32 = (1-0.85)/N + 0.85 * Σ_{j=rowptr[n]}^{rowptr[n+1]-1} pr[w_j]/outdeg[w_j], w_j = colidx[j]
 *                      one PageRank step (Fig 5) over the CSR of IN-neighbours; the caller
 *                      guarantees 0 <= rowptr[n] <= rowptr[n+1] <= E, 0 <= colidx < N and outdeg >= 1 for
 *                      every id in colidx (no device-side checks). AUTO only; E < 2^31. The record's inner
 *                      level is Split (segmented: warps claim 31 rows, their edges over 32 lanes) when
 *                      ceil(E/N) >= 8, else Span(all) over V lanes per row (S8 PR). */
typedef enum {
  NPP_SUM_ROWS = 0,
  NPP_SUM_COLS = 1,
  NPP_KMEANS_ASSIGN = 2,
  NPP_LOGREG_GRAD = 3,
  NPP_SUM_WEIGHTED_ROWS = 4,
  NPP_SUM_WEIGHTED_COLS = 5,
  NPP_SUM_ROWS_COLS = 6,
  NPP_KMEANS_UPDATE = 7,
  NPP_PAGERANK = 8
} npp_pattern;

/* AUTO     = Algorithm 1 + ControlDOP + the runtime step R2 (L810-817; S8)
 * LITERAL  = Algorithm 1 + ControlDOP exactly as the paper states them (S2-S6)
 * 1D, TB_THREAD, WARP = the prior-work mappings of Fig 2 and Fig 7 (S7; 2-level only) */
typedef enum {
  NPP_MAP_AUTO = 0,
  NPP_MAP_LITERAL = 1,
  NPP_MAP_1D = 2,
  NPP_MAP_TB_THREAD = 3,
  NPP_MAP_WARP = 4
} npp_strategy;

typedef enum { NPP_SPAN_ONE = 0, NPP_SPAN_ALL = 1, NPP_SPAN_N = 2, NPP_SPLIT_K = 3 } npp_span;
typedef enum { NPP_DIM_X = 0, NPP_DIM_Y = 1, NPP_DIM_Z = 2 } npp_dim;
/* Where the inner zipWith of the weighted sums (Fig 15) keeps its per-outer-iteration
 * result (§V-A, Fig 16): NONE = not materialised (the product is reduced in registers;
 * AUTO); MALLOC = a device malloc per outer iteration (the unoptimised code of Fig 16);
 * PREALLOC = one [outer x inner] buffer in the plan's workspace, addressed
 * o*temp_stride[0] + i*temp_stride[1] — (inner, 1) is Fig 11a (offset m*N, stride 1), (1, outer) is
 * Fig 11b (offset m, stride M). */
typedef enum { NPP_TEMP_NONE = 0, NPP_TEMP_MALLOC = 1, NPP_TEMP_PREALLOC = 2 } npp_temp;
typedef enum {
  NPP_CLASS_RX = 0,      /* inner Reduce on x (sumRows family; TB/T and warp baselines)   */
  NPP_CLASS_MX = 1,      /* outer Map on x, inner Reduce on y (sumCols family; 1D)        */
  NPP_CLASS_KMEANS = 2,  /* 3-level: Map points / argmin centroids / Reduce dims          */
  NPP_CLASS_LOGREG = 3,  /* 3-level: Map batches / Reduce rows / Map+Reduce columns       */
  NPP_CLASS_EMPTY = 4,   /* a zero-sized level: output zero-filled (or nothing to do)     */
  NPP_CLASS_RC = 5,      /* 2-level, both levels Reduce: row and column sums in one pass  */
  NPP_CLASS_KMUPDATE = 6,/* groupBy + Reduce: per-centroid sums and counts                */
  NPP_CLASS_PAGERANK = 7 /* irregular inner Map+Reduce over CSR rows (Fig 5)              */
} npp_kernel_class;

/* One nest level of a mapping (§IV-A). dim: npp_dim; span: npp_span; factor: n of Span(n) or k of
 * Split(k) (1 otherwise); chunk: indices of this level one thread block covers (S9);
 * grid: blocks along this level = ceil(N/chunk). */
typedef struct {
  int32_t dim;
  int32_t block;
  int32_t span;
  int32_t reserved;
  int64_t factor;
  int64_t chunk;
  int64_t grid;
} npp_level;

/* The mapping record (S9). Level 0 is the outermost pattern. `vec` = elements per thread
 * per 16-byte load on the x level (1 = scalar). `score` = soft-constraint score of the static
 * decision (S4); `dop` = Alg 1 DOP of the record's spans (G7); `threads` = grid * Π block.
 * block[d] = threads along CUDA dim d. The grid is launched linearised (grid blocks along x). */
typedef struct {
  int32_t nlevels;
  int32_t kernel_class;
  int32_t vec;
  int32_t staged;  /* 1: TMA-staged tile family (S8, §V-B prefetch); 0: direct-load family */
  npp_level level[NPP_MAX_LEVELS];
  int64_t score;
  int64_t dop;
  int64_t threads;
  int64_t grid;
  int32_t block[3];
  int32_t smem_bytes;
  int64_t workspace_bytes;
  int64_t claim_tiles; /* staged plans: tiles a persistent block claims at a time (dynamic Span) */
  int32_t temp;           /* npp_temp: the weighted sums' inner allocation (S10) */
  int32_t reserved2;
  int64_t temp_stride[2]; /* PREALLOC: element strides of the temp buffer along (outer, inner) */
  int64_t static_tiles;   /* staged sums: the first Ts tiles (outer-major order) are split statically over the
                             grid, the rest form the claim pool of units of claim_tiles (S8); else 0 */
} npp_mapping;

/* Hardware limits the selector's hard constraints and ControlDOP read (L658-662, L799-803).
 * regs_per_thread = the largest register count of this library's kernels (cudaFuncGetAttributes). */
typedef struct {
  int32_t sm_count;
  int32_t max_threads_per_sm;
  int32_t max_threads_per_block;
  int32_t max_block_dim[3];
  int32_t warp_size;
  int32_t max_blocks_per_sm;
  int32_t regs_per_sm;
  int32_t regs_per_block;
  int32_t regs_per_thread;
  int32_t reserved;
  int64_t smem_per_block;
} npp_limits;

typedef struct npp_plan_s* npp_plan_t;

/* Library version (NPP_VERSION). */
NPP_API int npp_version(void);

/* Thread-local description of the last error on this thread ("" if none). Never NULL. */
NPP_API const char* npp_last_error(void);

/* Fill `out` from cudaGetDeviceProperties(device) and the kernels' register counts.
 * Errors: NPP_ERR_INVALID_ARG (out NULL), NPP_ERR_CUDA (no such device / no driver). */
NPP_API int npp_limits_query(int device, npp_limits* out);

/* Pure, CUDA-free mapping selection (a1-a5: nest, constraints, Algorithm 1, ControlDOP, R2) for
 * `pattern` with `ndim` sizes in `shape` (each >= 1, or -1 = unknown size, LITERAL only, G17) under
 * `limits`. Writes the mapping record to `out`. Deterministic: equal inputs give equal records.
 * Errors: INVALID_ARG, UNSUPPORTED (e.g. forced strategy on a 3-level nest),
 *         NO_FEASIBLE_MAPPING. */
NPP_API int npp_select(int pattern, const int64_t* shape, int ndim, int dtype, const npp_limits* limits,
               int strategy, npp_mapping* out);

/* Algorithm 1's search space (S2, Alg 1): every candidate that passes the hard
 * constraints (S3), in enumeration order (dims permutations lexicographic, then block sizes with
 * level 0 most significant, then spans ONE < ALL), each with ControlDOP (S6) applied and recorded as
 * strategy LITERAL records it (S9; score = its S4 soft score). Pure and CUDA-free like npp_select.
 * Writes the first min(cap, count) records to `out` (caller-owned array; NULL allowed with cap 0)
 * and returns count (>= 0), or a negative npp_status. Used for the score-vs-performance sweep of
 * P:L1358-1415 (Fig 17); every record is executable through npp_plan_with_mapping (2-level sums). */
NPP_API int64_t npp_enumerate(int pattern, const int64_t* shape, int ndim, int dtype, const npp_limits* limits,
                              npp_mapping* out, int64_t cap);

/* Build an immutable plan for (pattern, shape, dtype, strategy). limits == NULL queries the current
 * device. Sizes may be 0 (the plan then zero-fills the output). The plan is a host object owned by
 * the caller (npp_plan_destroy). Errors: as npp_select, plus NPP_ERR_CUDA from the limits query. */
NPP_API int npp_plan(int pattern, const int64_t* shape, int ndim, int dtype, int strategy,
             const npp_limits* limits, npp_plan_t* out);

/* Build a plan from a caller-given mapping (dims, blocks, spans, factors, vec of `forced`; the other
 * fields are recomputed). Rejects mappings that violate a hard constraint (S3) or cannot be executed
 * by a kernel family (NPP_ERR_NO_FEASIBLE_MAPPING / NPP_ERR_UNSUPPORTED) — e.g. Fig 9's 64x32 block. */
NPP_API int npp_plan_with_mapping(int pattern, const int64_t* shape, int ndim, int dtype,
                          const npp_mapping* forced, const npp_limits* limits, npp_plan_t* out);

/* Copy the plan's mapping record. */
NPP_API int npp_plan_mapping(npp_plan_t plan, npp_mapping* out);

/* Workspace bytes npp_execute needs (0 if none). The workspace must be zero-filled before its first
 * use with a plan; every successful execute leaves its counters, tickets and accumulators zero-filled
 * again (Split tickets reset). The S10 temp region of a PREALLOC weighted plan (the last
 * outer*inner*sizeof(dtype) bytes rounded up to 256) is scratch: written before it is read, left
 * holding the zipWith products. */
NPP_API int64_t npp_plan_workspace_bytes(npp_plan_t plan);

/* Enqueue the plan's kernel(s) on `stream` (async; no host sync; one kernel launch for every sum and
 * logreg pattern, Split combine fused; KMEANS_ASSIGN adds a small centroid-pack kernel). `ins` holds `n_in` device pointers in the order of the pattern table above;
 * `out` is the device output. Vector plans (mapping.vec > 1) need 16-byte aligned pointers.
 * Errors: INVALID_ARG, ALIGNMENT, WORKSPACE, CUDA (launch error; async faults surface at the
 * caller's next synchronisation). Concurrent executes of one plan need distinct workspaces.
 * KMEANS_ASSIGN first packs the centroids as pairs (a 64 KB module buffer) and copies them
 * device-to-device into the library's constant bank (one per device) before its kernel; executes of KMEANS_ASSIGN plans on
 * different streams are ordered by an internal event so they never overwrite each other's
 * centroids. Inside a stream capture that ordering is the caller's: captured KMEANS_ASSIGN work
 * must not run concurrently with other KMEANS_ASSIGN work on the same device. */
NPP_API int npp_execute(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace,
                void* stream);

/* Execution flags of npp_execute_ex. */
#define NPP_EXEC_OVERLAP 1u
#define NPP_EXEC_NO_PDL 2u
/* npp_execute with flags. NPP_EXEC_OVERLAP: the caller asserts that no work enqueued earlier on
 * `stream` writes this call's inputs (e.g. inputs resident before the preceding kernel started); the
 * staged (TMA) kernels are then launched as programmatic dependent launches (sm_90+ PDL): their blocks
 * start streaming the inputs while the previous kernel on the stream drains, and they write `out` and
 * the workspace only after that kernel has completed (griddepcontrol.wait). Other plans ignore the
 * flag. NPP_EXEC_NO_PDL: launch every kernel as a plain stream-ordered launch (no programmatic dependent
 * launch attribute at all: the kernel's blocks become resident only after the previous kernel completed;
 * used to time one kernel in isolation). OVERLAP together with NO_PDL, or unknown flag bits:
 * NPP_ERR_INVALID_ARG. Otherwise identical to npp_execute. */
NPP_API int npp_execute_ex(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace,
                           void* stream, unsigned flags);

/* End-to-end call with HOST buffers: copies `host_ins` (pinned or pageable host memory, same order
 * and sizes as npp_execute) into the caller's device buffers `dev_ins`, executes, copies the result
 * into `host_out` and synchronises `stream` before returning. */
NPP_API int npp_execute_host(npp_plan_t plan, const void* const* host_ins, int n_in, void* host_out,
                     void* const* dev_ins, void* dev_out, void* workspace, void* stream);

/* Tiles of the plan's schedule (white-box tests of the runtime rule, S8): To*Ti for a staged
 * sum (outer-major tile order), B*ceil(Rb/32) for LOGREG_GRAD, ceil(N/TP) for KMEANS_ASSIGN (TP = 256 if
 * D <= 64 else 128), ceil(N/96) for KMEANS_UPDATE, the number of regions for SUM_ROWS_COLS; 0 for plans
 * without a tile schedule (direct-load families, PAGERANK, empty plans). */
NPP_API int64_t npp_plan_tiles(npp_plan_t plan);

/* npp_execute that also records the schedule: `trace` is a caller-owned DEVICE int32 array of
 * 2*npp_plan_tiles(plan) entries, the second half zero-filled by the caller. For every tile t the kernel
 * writes trace[t] = index of the block that loaded it and adds 1 to trace[n + t] per load (so a correct
 * schedule leaves every trace[n + t] == 1). Enqueue only, like npp_execute; the trace costs one store and
 * one atomic per tile. Errors: as npp_execute; NPP_ERR_UNSUPPORTED if the plan has no tile schedule;
 * NPP_ERR_INVALID_ARG if trace is NULL. */
NPP_API int npp_execute_traced(npp_plan_t plan, const void* const* ins, int n_in, void* out, void* workspace,
                               void* stream, int32_t* trace);

/* Number of kernel launches one npp_execute of this plan enqueues (0 for an empty plan). */
NPP_API int npp_plan_launches(npp_plan_t plan);

/* Destroy a plan (NULL is ignored). */
NPP_API void npp_plan_destroy(npp_plan_t plan);

#ifdef __cplusplus
}
#endif

#endif /* NPP_H_ */
