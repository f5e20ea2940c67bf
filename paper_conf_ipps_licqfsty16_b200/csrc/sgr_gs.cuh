// sgr_gs.cuh — reduced-round variants of the method (DESIGN.md §3
// reading C20; sgr_color_gs in include/sgr.h). Not the hot path.
//
// K-sub-step Gauss-Seidel rounds: the paper's kernels write color[v] in place inside the
// parallel assignment loop (Alg. 5 l.4-10), so threads may read colors that
// other threads of the same round already changed. Here that becomes
// deterministic: a round's worklist is split by a fixed id partition into K sub-steps run
// in order; sub-step j assigns its members against the colors left by sub-steps < j
// (Jacobi within the sub-step: k_gs_assign reads C, k_gs_commit writes it afterwards).
// Detection and compaction after the K sub-steps reuse the step kernels (Alg. 5 l.12-15).
// Partition 2 is the paper-faithful nondeterministic mode: one in-place sub-step whose
// first fits read C while other warps write it (only properness and color counts are
// checkable).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "sgr_common.cuh"

namespace sgr {

// Sub-step of v: strided (v mod K) or blocked (floor(v K / n)).
__device__ __forceinline__ int64_t gs_part(int64_t v, int64_t n, int64_t K, int partition) {
  return partition == 1 ? (int64_t)(((unsigned __int128)v * (unsigned long long)K) / (unsigned long long)n)
                        : v % K;
}

// Sub-step j of a round: T[i] = first fit of wl[i] against C for the members of part j
// (one warp per listed vertex; C is not written while this kernel runs). Sum of degrees of
// the members into *edges (one atomic per block).
static __global__ void __launch_bounds__(1024) k_gs_assign(const int64_t* __restrict__ row_ptr,
                                                           const int32_t* __restrict__ col_idx,
                                                           const int32_t* __restrict__ wl, int64_t len,
                                                           int64_t n, int64_t K, int partition,
                                                           int64_t j, const int32_t* __restrict__ C,
                                                           int32_t* __restrict__ T,
                                                           unsigned long long* edges) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  unsigned long long my = 0;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    if (gs_part(v, n, K, partition) != j) continue;  // warp-uniform
    const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
    const int32_t t = warp_first_fit_from<false>(col_idx, C, s, e, 0, lane);
    if (lane == 0) {
      T[i] = t;
      my += (unsigned long long)(e - s);
    }
  }
  block_add(my, edges);
}

// Sub-step j's writes become visible to the next sub-step: C[wl[i]] = T[i] for part j.
static __global__ void k_gs_commit(const int32_t* __restrict__ wl, int64_t len, int64_t n, int64_t K,
                                   int partition, int64_t j, const int32_t* __restrict__ T,
                                   int32_t* __restrict__ C) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = wl[i];
    if (gs_part(v, n, K, partition) == j) C[v] = T[i];
  }
}

// Paper-faithful in-place assignment (nondeterministic): one warp per listed vertex reads
// its neighbours' colors from L2 (ld.global.cg: other warps' writes of this launch may or
// may not be seen) and writes its first fit straight into C.
static __global__ void __launch_bounds__(1024) k_gs_inplace(const int64_t* __restrict__ row_ptr,
                                                            const int32_t* __restrict__ col_idx,
                                                            const int32_t* __restrict__ wl, int64_t len,
                                                            int32_t* C, unsigned long long* edges) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  unsigned long long my = 0;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
    const int32_t t = warp_first_fit_from<true>(col_idx, C, s, e, 0, lane);
    if (lane == 0) {
      __stcg(C + v, t);
      my += (unsigned long long)(e - s);
    }
  }
  block_add(my, edges);
}

static __global__ void k_gs_init(int64_t n, int32_t* __restrict__ wl, int32_t* __restrict__ C) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    wl[v] = (int32_t)v;  // W_1 = V
    C[v] = 0;            // 0 = not yet colored
  }
}

}  // namespace sgr
