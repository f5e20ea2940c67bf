// sgr_common.cuh — device helpers shared by the round kernels and the step entry points.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sgr {

template <int TB>
__device__ __forceinline__ bool lose(int32_t v, int32_t w) {
  // Which endpoint of a monochromatic edge (v, w) returns to the worklist:
  // TB 1 = PAPER, Alg. 5 l.14: v < w -> v;  TB 0 = LOWID_KEEPS: v > w -> v.
  // Both are false for w == v: a self-loop never conflicts (DESIGN.md §3 reading C7).
  if constexpr (TB == 1) return v < w;
  else return v > w;
}

// Loads of the read-only CSR arrays R (row_ptr) and C (col_idx). SGR_LDG = 1 (default):
// through the read-only data path, __ldg / ld.global.nc — the paper's D-ldg / T-ldg
// optimization (Fig. 4). SGR_LDG = 0: the normal load path, ld.global.ca — the
// paper's D-base / T-base (the ablation of P:236; tools/ldg_ablation.py).
#ifndef SGR_LDG
#define SGR_LDG 1
#endif
template <class T>
__device__ __forceinline__ T ld_ro(const T* p) {
#if SGR_LDG
  return __ldg(p);
#else
  return __ldca(p);
#endif
}
__device__ __forceinline__ int32_t ldg_i32(const int32_t* p) { return ld_ro(p); }
__device__ __forceinline__ int64_t ldg_i64(const int64_t* p) { return ld_ro(p); }

// Read-only load of col_idx (the CSR never changes during a coloring). Measured on B200
// (tools/gather_bench.cu): ld.global.nc.L1::no_allocate is up to 3.5x slower than plain
// ld.global.nc for this access mix, so the plain read-only path is used.
__device__ __forceinline__ int32_t ld_stream(const int32_t* p) { return ld_ro(p); }

// Color loads. A persistent kernel writes the color buffers while it runs, so it must not
// read them through the non-coherent path: Persist loads go to L2 (ld.global.cg); the
// per-round kernels (buffers read-only for their lifetime) use the read-only path.
template <bool Persist>
__device__ __forceinline__ int32_t ld_color(const int32_t* p) {
  if constexpr (Persist) return __ldcg(p);
  else return __ldg(p);
}

// Warp-aggregated push: lanes with `pred` append `v`; one atomicAdd per warp (the paper's
// "globally shared worklist is only atomically updated once for each thread block",
// P:230, at warp granularity). All 32 lanes must call it.
__device__ __forceinline__ void warp_push(bool pred, int32_t v, int32_t* list, int32_t* count) {
  const unsigned m = __ballot_sync(0xffffffffu, pred);
  if (m == 0) return;
  const int lane = threadIdx.x & 31;
  int base = 0;
  const int leader = __ffs(m) - 1;
  if (lane == leader) base = atomicAdd(count, __popc(m));
  base = __shfl_sync(0xffffffffu, base, leader);
  if (pred) list[base + __popc(m & ((1u << lane) - 1u))] = v;
}

__device__ __forceinline__ uint64_t warp_or64(uint64_t x) {
  const uint32_t lo = __reduce_or_sync(0xffffffffu, (uint32_t)x);
  const uint32_t hi = __reduce_or_sync(0xffffffffu, (uint32_t)(x >> 32));
  return ((uint64_t)hi << 32) | lo;
}

// Exact warp-cooperative first fit over the window [base, base + 256) and beyond: the
// caller guarantees every color in [1, base) is forbidden (base = 0: none). Used by the
// step entry point and as the rare fallback when a first-fit exceeds the table size.
// All 32 lanes must call it with the same arguments; returns the same value on all lanes.
template <bool Persist>
__device__ __forceinline__ int32_t warp_first_fit_from(const int32_t* __restrict__ col_idx,
                                                       const int32_t* X, int64_t s, int64_t e,
                                                       int32_t base, int lane) {
  for (;;) {
    uint64_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
    if (base == 0) m0 = 1;  // color 0 is never a candidate
    for (int64_t j = s + lane; j < e; j += 32) {
      const uint32_t idx = (uint32_t)(ld_color<Persist>(X + ld_stream(col_idx + j)) - base);
      if (idx < 256u) {
        const uint64_t bit = 1ull << (idx & 63);
        const uint32_t q = idx >> 6;
        m0 |= q == 0 ? bit : 0ull;
        m1 |= q == 1 ? bit : 0ull;
        m2 |= q == 2 ? bit : 0ull;
        m3 |= q == 3 ? bit : 0ull;
      }
    }
    m0 = warp_or64(m0);
    m1 = warp_or64(m1);
    m2 = warp_or64(m2);
    m3 = warp_or64(m3);
    if (~m0) return base + __ffsll((long long)~m0) - 1;
    if (~m1) return base + 64 + __ffsll((long long)~m1) - 1;
    if (~m2) return base + 128 + __ffsll((long long)~m2) - 1;
    if (~m3) return base + 192 + __ffsll((long long)~m3) - 1;
    base += 256;
  }
}

// Block-level sum of a per-thread counter, one atomicAdd per block. All threads must call.
__device__ __forceinline__ void block_add(unsigned long long x, unsigned long long* dst) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  __shared__ unsigned long long red[32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  __syncthreads();
  if (lane == 0) red[wid] = x;
  __syncthreads();
  if (wid == 0) {
    x = lane < (int)(blockDim.x >> 5) ? red[lane] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (lane == 0 && x) atomicAdd(dst, x);
  }
}

}  // namespace sgr
