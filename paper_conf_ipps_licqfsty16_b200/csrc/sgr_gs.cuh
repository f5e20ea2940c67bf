// sgr_gs.cuh — reduced-round variants of the method (DESIGN.md §3
// reading C20; sgr_color_gs in include/sgr.h). Not the hot path.
//
// K-sub-step Gauss-Seidel rounds: the paper's kernels write color[v] in place inside the
// parallel assignment loop (Alg. 5 l.4-10), so threads may read colors that
// other threads of the same round already changed. Here that becomes
// deterministic: a round's worklist is split by a fixed id partition into K sub-steps run
// in order; sub-step j assigns its members against the colors left by sub-steps < j
// (Jacobi within the sub-step: k_gs_assign_seg reads C, k_gs_commit_seg writes it after).
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

// ---- bucketed sub-steps: each round's worklist is split once into its K sub-step
// segments (a histogram, an exclusive scan and a scatter), so a sub-step touches only its
// own members; low-degree members take their first fit one thread each, the others one warp.
static __global__ void k_gs_hist(const int32_t* __restrict__ wl, int64_t len, int64_t n, int64_t K,
                                 int partition, int32_t* __restrict__ cnt) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len;
       i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + gs_part(wl[i], n, K, partition), 1);
}

// Exclusive scan of the K counts (one block; K <= a few thousand), cnt -> off[0..K], and
// the scatter cursors reset to the offsets.
static __global__ void k_gs_scan(const int32_t* __restrict__ cnt, int64_t K, int32_t* __restrict__ off,
                                 int32_t* __restrict__ cur) {
  if (threadIdx.x == 0) {
    int32_t run = 0;
    for (int64_t j = 0; j < K; ++j) {
      off[j] = run;
      cur[j] = run;
      run += cnt[j];
    }
    off[K] = run;
  }
}

static __global__ void k_gs_scatter(const int32_t* __restrict__ wl, int64_t len, int64_t n, int64_t K,
                                    int partition, int32_t* __restrict__ cur, int32_t* __restrict__ seg) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = wl[i];
    seg[atomicAdd(cur + gs_part(v, n, K, partition), 1)] = v;
  }
}

// Sub-step j over its segment seg[off[j] .. off[j+1]): T[i] = first fit against C. Lane L of
// a warp takes entry 32 w + L; a member of degree <= 64 is done by its own thread (64-color
// register windows, rescanning the row per window); larger ones are appended to big[] (one
// atomic per warp) for k_gs_assign_big, one warp each.
static __global__ void __launch_bounds__(1024) k_gs_assign_seg(const int64_t* __restrict__ row_ptr,
                                                               const int32_t* __restrict__ col_idx,
                                                               const int32_t* __restrict__ seg,
                                                               const int32_t* __restrict__ off, int64_t j,
                                                               const int32_t* __restrict__ C,
                                                               int32_t* __restrict__ T,
                                                               int32_t* __restrict__ big,
                                                               int32_t* __restrict__ nbig,
                                                               unsigned long long* edges) {
  const int lane = threadIdx.x & 31;
  const int64_t b = __ldg(off + j), e_ = __ldg(off + j + 1);
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  unsigned long long my = 0;
  for (int64_t base = b + (((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) << 5); base < e_;
       base += nw << 5) {
    const int64_t i = base + lane;
    const bool ok = i < e_;
    const int32_t v = ok ? __ldg(seg + i) : 0;
    const int64_t s = ok ? ld_ro(row_ptr + v) : 0, e = ok ? ld_ro(row_ptr + v + 1) : 0;
    const bool small = ok && e - s <= 64;
    if (small) {
      int32_t t = 0;
      for (int32_t wb = 0; t == 0; wb += 64) {  // colors (wb, wb + 64]
        uint64_t m = 0;
        for (int64_t q = s; q < e; ++q) {
          const uint32_t idx = (uint32_t)(__ldg(C + ld_ro(col_idx + q)) - wb - 1);
          if (idx < 64u) m |= 1ull << idx;
        }
        if (~m) t = wb + __ffsll((long long)~m);
      }
      T[i] = t;
      my += (unsigned long long)(e - s);
    }
    const unsigned bm = __ballot_sync(0xffffffffu, ok && !small);
    if (bm) {
      int o = 0;
      if (lane == 0) o = atomicAdd(nbig, __popc(bm));
      o = __shfl_sync(0xffffffffu, o, 0);
      if (ok && !small) big[o + __popc(bm & ((1u << lane) - 1u))] = (int32_t)i;
    }
  }
  block_add(my, edges);
}

// The sub-step's members of degree > 64 (positions in seg), one warp each.
static __global__ void __launch_bounds__(1024) k_gs_assign_big(const int64_t* __restrict__ row_ptr,
                                                               const int32_t* __restrict__ col_idx,
                                                               const int32_t* __restrict__ seg,
                                                               const int32_t* __restrict__ big,
                                                               const int32_t* __restrict__ nbig,
                                                               const int32_t* __restrict__ C,
                                                               int32_t* __restrict__ T,
                                                               unsigned long long* edges) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  const int64_t cnt = __ldg(nbig);
  unsigned long long my = 0;
  for (int64_t q = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); q < cnt; q += (int64_t)gridDim.x * wpb) {
    const int32_t i = __ldg(big + q);
    const int32_t v = __ldg(seg + i);
    const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
    const int32_t t = warp_first_fit_from<false>(col_idx, C, s, e, 0, lane);
    if (lane == 0) {
      T[i] = t;
      my += (unsigned long long)(e - s);
    }
  }
  block_add(my, edges);
}

static __global__ void k_gs_commit_seg(const int32_t* __restrict__ seg, const int32_t* __restrict__ off,
                                       int64_t j, const int32_t* __restrict__ T, int32_t* __restrict__ C) {
  const int64_t b = __ldg(off + j), e = __ldg(off + j + 1);
  for (int64_t i = b + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < e;
       i += (int64_t)gridDim.x * blockDim.x)
    C[seg[i]] = T[i];
}

static __global__ void k_gs_init(int64_t n, int32_t* __restrict__ wl, int32_t* __restrict__ C) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    wl[v] = (int32_t)v;  // W_1 = V
    C[v] = 0;            // 0 = not yet colored
  }
}

}  // namespace sgr
