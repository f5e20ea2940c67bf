// sgr_topo.cuh — topology-driven mapping of the same method: the
// paper's Algorithm 4 ("T-base"), Jacobi reading (DESIGN.md
// §3 C1). Every iteration visits ALL n vertices, one thread per vertex ("maps each
// vertex to a thread, ... the thread stays idle or is responsible to process the vertex
// depending on whether the corresponding vertex has been processed or not"):
//   assign  (Alg. 4 l.4-13): v with colored[v] = false takes the first fit against the
//           snapshot X of the iteration's start, written to T (others copy X[v]);
//   detect  (Alg. 4 l.15-21): every v in V with a neighbour w, T[w] = T[v], lose(v, w)
//           becomes uncolored again; `changed` (l.3, l.12, l.22) is the count of those.
// colored[v] = false is stored as a round stamp, flag[v] == r, so no flag array is ever
// cleared. The result (colors, rounds, |W_r|) is identical to the data-driven path and to
// the oracle's O2: detection over V equals detection over W (DESIGN.md §3 proof (ii)).
// This is the comparison mapping the paper measured against Algorithm 5, not the hot path.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "sgr_common.cuh"

namespace sgr {

// First fit of v against snapshot X, one thread, any degree: 64-color windows [base+1,
// base+64], rescanning the row per window (first fit <= deg + 1).
__device__ __forceinline__ int32_t thread_first_fit(const int32_t* __restrict__ col_idx,
                                                    const int32_t* __restrict__ X, int32_t v,
                                                    int64_t s, int64_t e) {
  for (int32_t base = 0;; base += 64) {
    uint64_t m = 0;
    for (int64_t j = s; j < e; ++j) {
      const int32_t w = ld_ro(col_idx + j);
      if (w == v) continue;  // a self-loop never forbids (reading C7)
      const uint32_t idx = (uint32_t)(__ldg(X + w) - base - 1);
      if (idx < 64u) m |= 1ull << idx;
    }
    if (~m) return base + __ffsll((long long)~m);
  }
}

// Alg. 4 l.4-13 for iteration r: T[v] = colored[v] ? X[v] : first fit against X.
static __global__ void __launch_bounds__(1024) k_topo_assign(const int64_t* __restrict__ row_ptr,
                                                            const int32_t* __restrict__ col_idx,
                                                            int64_t n, int32_t r,
                                                            const int32_t* __restrict__ flag,
                                                            const int32_t* __restrict__ X,
                                                            int32_t* __restrict__ T,
                                                            unsigned long long* edges) {
  unsigned long long my = 0;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    if (__ldg(flag + v) == r) {  // colored[v] = false
      const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
      T[v] = thread_first_fit(col_idx, X, (int32_t)v, s, e);
      my += (unsigned long long)(e - s);
    } else {
      T[v] = __ldg(X + v);
    }
  }
  block_add(my, edges);
}

// Alg. 4 l.15-21 for iteration r over every vertex: a conflict makes v uncolored for
// iteration r + 1 (flag[v] = r + 1) and counts towards `changed`.
template <int TB>
__global__ void __launch_bounds__(1024) k_topo_detect(const int64_t* __restrict__ row_ptr,
                                                     const int32_t* __restrict__ col_idx,
                                                     int64_t n, int32_t r,
                                                     const int32_t* __restrict__ T,
                                                     int32_t* __restrict__ flag,
                                                     int32_t* __restrict__ changed) {
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = base + threadIdx.x;
    bool c = false;
    if (v < n) {
      const int32_t tv = __ldg(T + v);
      const int64_t e = ld_ro(row_ptr + v + 1);
      for (int64_t j = ld_ro(row_ptr + v); j < e && !c; ++j) {
        const int32_t w = ld_ro(col_idx + j);
        c = lose<TB>((int32_t)v, w) && __ldg(T + w) == tv;
      }
      if (c) flag[v] = r + 1;
    }
    const unsigned m = __ballot_sync(0xffffffffu, c);
    if ((threadIdx.x & 31) == 0 && m) atomicAdd(changed, __popc(m));
  }
}

static __global__ void k_topo_init(int64_t n, int32_t* __restrict__ flag, int32_t* __restrict__ X) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    flag[v] = 1;  // every vertex uncolored in iteration 1
    X[v] = 0;     // 0 = no color yet
  }
}

}  // namespace sgr
