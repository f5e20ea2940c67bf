// sgr_step.cuh — step entry points (Algorithm 5 split line by line), order-preserving
// compaction, CSR validation and the final max-color reduction. Not on the fused hot path.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "sgr_common.cuh"

namespace sgr {

static __global__ void k_max_color(const int32_t* __restrict__ c, int64_t n, int32_t* out) {
  int32_t m = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, __ldg(c + i));
  m = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)m);
  if ((threadIdx.x & 31) == 0 && m) atomicMax(out, m);
}

// ---------------------------------------------------------------------------------------
// Step entry points (Algorithm 5 split line by line; not on the fused hot path).

// Alg. 5 l.4-10: warp per listed vertex, exact for any degree.
static __global__ void __launch_bounds__(1024) k_assign_step(const int64_t* __restrict__ row_ptr,
                                                     const int32_t* __restrict__ col_idx,
                                                     const int32_t* __restrict__ wl, int64_t len,
                                                     const int32_t* __restrict__ X,
                                                     int32_t* __restrict__ tent) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    const int32_t t =
        warp_first_fit_from<false>(col_idx, X, ld_ro(row_ptr + v), ld_ro(row_ptr + v + 1), 0, lane);
    if (lane == 0) tent[i] = t;
  }
}

// Alg. 5 l.9: colors[wl[i]] = tent[i].
static __global__ void k_commit_step(const int32_t* __restrict__ wl, const int32_t* __restrict__ tent,
                              int64_t len, int32_t* __restrict__ colors) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len;
       i += (int64_t)gridDim.x * blockDim.x)
    colors[wl[i]] = tent[i];
}

// Alg. 5 l.13-14: warp per listed vertex.
template <int TB>
__global__ void __launch_bounds__(1024) k_detect_step(const int64_t* __restrict__ row_ptr,
                                                     const int32_t* __restrict__ col_idx,
                                                     const int32_t* __restrict__ wl, int64_t len,
                                                     const int32_t* __restrict__ C,
                                                     uint8_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    const int32_t cv = __ldg(C + v);
    bool c = false;
    for (int64_t j = ld_ro(row_ptr + v) + lane; j < ld_ro(row_ptr + v + 1) && !c; j += 32) {
      const int32_t w = ld_ro(col_idx + j);
      c = (__ldg(C + w) == cv) && lose<TB>(v, w);
    }
    c = __any_sync(0xffffffffu, c);
    if (lane == 0) out[i] = c ? 1 : 0;
  }
}

// Order-preserving compaction (Fig. 5): tile counts -> scan -> scatter.
constexpr int kCompactTile = 1024;  // elements per tile (256 threads x 4)

static __global__ void __launch_bounds__(256) k_compact_count(const uint8_t* __restrict__ flags,
                                                       int64_t len, int32_t* __restrict__ tile_cnt) {
  const int64_t t0 = (int64_t)blockIdx.x * kCompactTile;
  int c = 0;
  for (int u = 0; u < 4; ++u) {
    const int64_t i = t0 + u * 256 + threadIdx.x;
    c += (i < len && flags[i]) ? 1 : 0;
  }
  c = __reduce_add_sync(0xffffffffu, c);
  __shared__ int red[8];
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = c;
  __syncthreads();
  if (threadIdx.x == 0) {
    int s = 0;
    for (int q = 0; q < 8; ++q) s += red[q];
    tile_cnt[blockIdx.x] = s;
  }
}

// Exclusive scan of tile counts by one block (tiles <= a few million: sequential chunks).
static __global__ void __launch_bounds__(1024) k_compact_scan(int32_t* __restrict__ tile_cnt, int64_t tiles,
                                                       int64_t* __restrict__ total) {
  __shared__ int64_t carry_s;
  __shared__ int64_t warp_s[32];
  if (threadIdx.x == 0) carry_s = 0;
  __syncthreads();
  for (int64_t b = 0; b < tiles; b += blockDim.x) {
    const int64_t i = b + threadIdx.x;
    int64_t x = i < tiles ? tile_cnt[i] : 0;
    // inclusive warp scan
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    int64_t y = x;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int64_t t = __shfl_up_sync(0xffffffffu, y, o);
      if (lane >= o) y += t;
    }
    if (lane == 31) warp_s[wid] = y;
    __syncthreads();
    if (wid == 0) {
      int64_t z = warp_s[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        int64_t t = __shfl_up_sync(0xffffffffu, z, o);
        if (lane >= o) z += t;
      }
      warp_s[lane] = z;
    }
    __syncthreads();
    const int64_t incl = y + (wid ? warp_s[wid - 1] : 0) + carry_s;
    if (i < tiles) tile_cnt[i] = (int32_t)(incl - x);
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry_s = incl;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry_s;
}

static __global__ void __launch_bounds__(256) k_compact_scatter(const int32_t* __restrict__ wl,
                                                         const uint8_t* __restrict__ flags,
                                                         int64_t len,
                                                         const int32_t* __restrict__ tile_off,
                                                         int32_t* __restrict__ out) {
  __shared__ int warp_tot[8 * 4];
  const int64_t t0 = (int64_t)blockIdx.x * kCompactTile;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  // element order inside the tile: chunk u (0..3) of 256, then thread
  bool f[4];
  unsigned m[4];
  for (int u = 0; u < 4; ++u) {
    const int64_t i = t0 + u * 256 + threadIdx.x;
    f[u] = i < len && flags[i];
    m[u] = __ballot_sync(0xffffffffu, f[u]);
    if (lane == 0) warp_tot[u * 8 + wid] = __popc(m[u]);
  }
  __syncthreads();
  if (threadIdx.x == 0) {  // exclusive scan over 32 (chunk, warp) slots in element order
    int s = 0;
    for (int q = 0; q < 32; ++q) {
      const int t = warp_tot[q];
      warp_tot[q] = s;
      s += t;
    }
  }
  __syncthreads();
  const int64_t base = tile_off[blockIdx.x];
  for (int u = 0; u < 4; ++u) {
    if (f[u]) {
      const int64_t i = t0 + u * 256 + threadIdx.x;
      out[base + warp_tot[u * 8 + wid] + __popc(m[u] & ((1u << lane) - 1u))] = wl[i];
    }
  }
}

// Device CSR validation: 1 offsets, 2 range, 4 unsorted.
static __global__ void k_validate(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                           int64_t n, int64_t nnz, int32_t* violations) {
  int viol = 0;
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x) {
    const int64_t s = row_ptr[v], e = row_ptr[v + 1];
    if (e < s || s < 0 || e > nnz) {
      viol |= 1;
      continue;
    }
    for (int64_t j = s; j < e; ++j) {
      const int32_t w = col_idx[j];
      if (w < 0 || w >= n) viol |= 2;
      if (j > s && col_idx[j - 1] > w) viol |= 4;
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0 && (row_ptr[0] != 0 || row_ptr[n] != nnz)) viol |= 1;
  if (viol) atomicOr(violations, viol);
}

}  // namespace sgr
