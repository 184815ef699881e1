// kernels.hpp — launch interface between the C-ABI layer (api.cu) and the kernel families.
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "npp.h"

namespace npp {

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
};

cudaError_t launch_sum(int dtype, int kclass, int vec, bool weighted, const SumArgs& a, cudaStream_t st);
int sum_kernels_max_regs();

}  // namespace npp
