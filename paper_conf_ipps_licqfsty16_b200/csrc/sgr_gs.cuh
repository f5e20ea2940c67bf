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


// =======================================================================================
// Persistent K-sub-step rounds (one cooperative launch, one grid barrier per sub-step).
//
// Two color buffers alternate per sub-step: sub-step j reads Cur and writes its members'
// new colors into Nxt, which before that equals the colors of one sub-step earlier — so the
// same sub-step also copies the previous sub-step's members (the only vertices that changed
// since) from Cur into Nxt. Nobody reads Nxt during the sub-step, so after the barrier Nxt
// is exactly the colors every later sub-step must see (Jacobi inside a sub-step, the
// earlier sub-steps' colors across them: reading C20).
// Sub-step 0 of round R also detects the conflicts of round R-1 (Alg. 5 l.12-15) over all
// of W_{R-1} against Cur (round R-1's final colors; Nxt is not read), pushing the losers
// into round R's per-part lists, and assigns the part-0 members at once (same snapshot).
// Lists: region j of a list array holds part j's members, low-degree ones from the front
// (thread per vertex), the others from the back (warp per vertex), counts per part.
namespace gsp {

// Members of each part among all n vertices (the list regions' sizes).
static __global__ void k_part_hist(int64_t n, int64_t K, int partition, int32_t* __restrict__ cnt) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n;
       v += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(cnt + gs_part(v, n, K, partition), 1);
}

constexpr int kSmallDeg = 64;  // thread-per-vertex first fit / detection up to this degree

struct Ctrl {
  uint32_t bar_count;
  int32_t rounds;        // R: assignment rounds run
  int32_t status;        // 1: max_rounds reached with W non-empty
  int32_t final_buf;     // index of the color buffer holding the result
  unsigned long long edges[2];  // per round parity: sum deg(W_R) (pushed members)
  unsigned long long verts_total, edges_total;  // sum over rounds of |W_R|, sum deg(W_R)
};

struct Args {
  const int64_t* row_ptr;
  const int32_t* col_idx;
  int32_t* C[2];
  int32_t* L[2];
  const int32_t* poff;   // K + 1 region offsets
  int32_t* cnt;          // [2][K][2]: per list parity, part: small count, big count
  Ctrl* ctrl;
  int32_t* round_sizes;
  int64_t* round_edges;
  int64_t n;
  int64_t K;
  int32_t partition;
  int32_t max_rounds;
  int32_t round_cap;
  int32_t tiebreak;
};

__device__ __forceinline__ int32_t* cnt_of(const Args& a, int par, int64_t j, int big) {
  return a.cnt + ((int64_t)par * a.K + j) * 2 + big;
}

__device__ __forceinline__ void gsync(Ctrl* c, uint32_t& epoch) {
  __syncthreads();
  ++epoch;
  if (threadIdx.x == 0) {
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(&c->bar_count) : "memory");
    const uint32_t target = epoch * gridDim.x;
    uint32_t v;
    do {
      asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&c->bar_count) : "memory");
      if ((int32_t)(v - target) < 0) __nanosleep(32);
    } while ((int32_t)(v - target) < 0);
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(&c->bar_count) : "memory");
  }
  __syncthreads();
}

// 8-lane group per low-degree vertex (v < 0: idle group): lane gl gathers entries gl + 8u
// (u < 8: all 64 at once); the group ORs its 64-bit color masks (bit c - 1 = color c; a
// degree <= 64 row leaves a free color <= 65) and, with want_conf, ORs the conflict test.
// Every listed entry counts, self-loops included (Alg. 5 l.5-6 literally, as O3).
// All 32 lanes of the warp must call it. Returns the first fit.
template <int TB>
__device__ __forceinline__ int32_t group_scan(const Args& a, const int32_t* Cur, int32_t v, int64_t s,
                                              int64_t e, int gl, unsigned gmask, bool want_conf,
                                              bool& conf) {
  const int32_t d = v >= 0 ? (int32_t)(e - s) : 0;
  int32_t w[8], c[8];
#pragma unroll
  for (int u = 0; u < 8; ++u) w[u] = gl + 8 * u < d ? ld_ro(a.col_idx + s + gl + 8 * u) : -1;
#pragma unroll
  for (int u = 0; u < 8; ++u) c[u] = w[u] >= 0 ? __ldcg(Cur + w[u]) : 0;
  const int32_t cv = (want_conf && v >= 0) ? __ldcg(Cur + v) : -1;
  uint64_t m = 0;
  bool cf = false;
#pragma unroll
  for (int u = 0; u < 8; ++u) {
    const uint32_t ci = (uint32_t)(c[u] - 1);
    m |= ci < 64u ? (1ull << ci) : 0ull;
    cf |= w[u] >= 0 && c[u] == cv && lose<TB>(v, w[u]);
  }
#pragma unroll
  for (int o = 4; o > 0; o >>= 1) m |= __shfl_xor_sync(0xffffffffu, m, o);
  conf = (__ballot_sync(0xffffffffu, cf) & gmask) != 0u;
  return ~m ? __ffsll((long long)~m) : 65;
}

// One warp per high-degree vertex: 8 entries per lane per batch (ids first, then all 8
// gathers), so a long row keeps 256 loads in flight instead of one chain per lane.
template <int TB>
__device__ __forceinline__ bool warp_conflict(const Args& a, const int32_t* Cur, int32_t v, int64_t s,
                                              int64_t e, int lane) {
  const int32_t cv = __ldcg(Cur + v);
  bool c = false;
  for (int64_t q0 = s; q0 < e; q0 += 256) {
    int32_t w[8], col[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t q = q0 + 32 * u + lane;
      w[u] = q < e ? ld_ro(a.col_idx + q) : -1;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) col[u] = w[u] >= 0 ? __ldcg(Cur + w[u]) : -1;
#pragma unroll
    for (int u = 0; u < 8; ++u) c |= w[u] >= 0 && col[u] == cv && lose<TB>(v, w[u]);
  }
  return __any_sync(0xffffffffu, c);
}

// First fit of a high-degree vertex against Cur, one warp: 256-color windows (bit i of the
// window word = color base + i + 1), rescanning the row per window, batches of 8 per lane.
__device__ __forceinline__ int32_t warp_fit(const Args& a, const int32_t* Cur, int64_t s, int64_t e,
                                           int lane) {
  for (int32_t base = 0;; base += 256) {
    uint64_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
    for (int64_t q0 = s; q0 < e; q0 += 256) {
      int32_t w[8], c[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int64_t q = q0 + 32 * u + lane;
        w[u] = q < e ? ld_ro(a.col_idx + q) : -1;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) c[u] = w[u] >= 0 ? __ldcg(Cur + w[u]) : 0;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t idx = (uint32_t)(c[u] - base - 1);
        const uint64_t bit = 1ull << (idx & 63u);
        m0 |= idx < 64u ? bit : 0ull;
        m1 |= idx - 64u < 64u ? bit : 0ull;
        m2 |= idx - 128u < 64u ? bit : 0ull;
        m3 |= idx - 192u < 64u ? bit : 0ull;
      }
    }
    m0 = warp_or64(m0);
    m1 = warp_or64(m1);
    m2 = warp_or64(m2);
    m3 = warp_or64(m3);
    if (~m0) return base + __ffsll((long long)~m0);
    if (~m1) return base + 64 + __ffsll((long long)~m1);
    if (~m2) return base + 128 + __ffsll((long long)~m2);
    if (~m3) return base + 192 + __ffsll((long long)~m3);
  }
}

// Huge members (degree > SGR_GS_HUGE): one BLOCK each — its warps take the row's 256-entry
// tiles in turn (warp w: tiles w, w + nwb, ...), so a hub row is scanned by every warp of a
// block instead of one (the sub-steps whose part holds a hub used to wait for one warp's
// serial walk of it). Block-uniform; all threads of the block must call.
#ifndef SGR_GS_HUGE
#define SGR_GS_HUGE 2048
#endif
template <int TB>
__device__ __forceinline__ bool block_conflict(const Args& a, const int32_t* Cur, int32_t v, int64_t s,
                                               int64_t e) {
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5, nwb = blockDim.x >> 5;
  const int32_t cv = __ldcg(Cur + v);
  bool c = false;
  for (int64_t q0 = s + 256 * (int64_t)wi; q0 < e; q0 += 256 * (int64_t)nwb) {
    int32_t w[8], col[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int64_t q = q0 + 32 * u + lane;
      w[u] = q < e ? ld_ro(a.col_idx + q) : -1;
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) col[u] = w[u] >= 0 ? __ldcg(Cur + w[u]) : -1;
#pragma unroll
    for (int u = 0; u < 8; ++u) c |= w[u] >= 0 && col[u] == cv && lose<TB>(v, w[u]);
  }
  return __syncthreads_or(c) != 0;
}
// First fit of a huge member, one block: 256-color windows as warp_fit, the warps' window
// masks merged in shared memory (sm: 4 words, zero on entry and on return).
__device__ __forceinline__ int32_t block_fit(const int32_t* __restrict__ col_idx, const int32_t* Cur,
                                            int64_t s, int64_t e, unsigned long long* sm) {
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5, nwb = blockDim.x >> 5;
  for (int32_t base = 0;; base += 256) {
    uint64_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
    for (int64_t q0 = s + 256 * (int64_t)wi; q0 < e; q0 += 256 * (int64_t)nwb) {
      int32_t w[8], c[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int64_t q = q0 + 32 * u + lane;
        w[u] = q < e ? ld_ro(col_idx + q) : -1;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) c[u] = w[u] >= 0 ? __ldcg(Cur + w[u]) : 0;
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t idx = (uint32_t)(c[u] - base - 1);
        const uint64_t bit = 1ull << (idx & 63u);
        m0 |= idx < 64u ? bit : 0ull;
        m1 |= idx - 64u < 64u ? bit : 0ull;
        m2 |= idx - 128u < 64u ? bit : 0ull;
        m3 |= idx - 192u < 64u ? bit : 0ull;
      }
    }
    m0 = warp_or64(m0);
    m1 = warp_or64(m1);
    m2 = warp_or64(m2);
    m3 = warp_or64(m3);
    if (lane == 0) {
      if (m0) atomicOr(sm + 0, (unsigned long long)m0);
      if (m1) atomicOr(sm + 1, (unsigned long long)m1);
      if (m2) atomicOr(sm + 2, (unsigned long long)m2);
      if (m3) atomicOr(sm + 3, (unsigned long long)m3);
    }
    __syncthreads();
    const uint64_t t0 = sm[0], t1 = sm[1], t2 = sm[2], t3 = sm[3];
    __syncthreads();  // every thread has read the merged masks before they are cleared
    if (threadIdx.x < 4) sm[threadIdx.x] = 0ull;
    __syncthreads();
    if (~t0) return base + __ffsll((long long)~t0);
    if (~t1) return base + 64 + __ffsll((long long)~t1);
    if (~t2) return base + 128 + __ffsll((long long)~t2);
    if (~t3) return base + 192 + __ffsll((long long)~t3);
  }
}

// Paper-faithful in-place assignment (nondeterministic): one warp per listed vertex reads
// its neighbours' colors from L2 (ld.global.cg: other warps' writes of this launch may or
// may not be seen) and writes its first fit straight into C; vertices of degree
// > SGR_GS_HUGE take a whole block (block_fit), as in the sub-step kernel.
// Any row longer than SGR_GS_HUGE (selects the in-place kernel's instantiation once per call).
static __global__ void k_any_huge(const int64_t* __restrict__ row_ptr, int64_t n, int32_t* flag) {
  for (int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += (int64_t)gridDim.x * blockDim.x)
    if (ld_ro(row_ptr + v + 1) - ld_ro(row_ptr + v) > SGR_GS_HUGE) *flag = 1;
}

template <bool Huge>
static __global__ void __launch_bounds__(1024) k_gs_inplace(const int64_t* __restrict__ row_ptr,
                                                            const int32_t* __restrict__ col_idx,
                                                            const int32_t* __restrict__ wl, int64_t len,
                                                            int32_t* C, unsigned long long* edges) {
  if constexpr (!Huge) {  // no row above SGR_GS_HUGE: warps only, no block-level pass
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
    return;
  }
  __shared__ unsigned long long sm[4];
  __shared__ int32_t huge[64];  // this block's huge vertices (list positions)
  __shared__ int32_t nhuge;
  if (threadIdx.x < 4) sm[threadIdx.x] = 0ull;
  if (threadIdx.x == 0) nhuge = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  unsigned long long my = 0;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
    if (e - s > SGR_GS_HUGE) {  // deferred to the whole block (up to 64 per block)
      int slot = 0;
      if (lane == 0) slot = atomicAdd(&nhuge, 1);
      slot = __shfl_sync(0xffffffffu, slot, 0);
      if (slot < 64) {
        if (lane == 0) huge[slot] = (int32_t)i;
        continue;
      }
    }
    const int32_t t = warp_first_fit_from<true>(col_idx, C, s, e, 0, lane);
    if (lane == 0) {
      __stcg(C + v, t);
      my += (unsigned long long)(e - s);
    }
  }
  __syncthreads();
  const int32_t nh = min(nhuge, 64);
  for (int32_t h = 0; h < nh; ++h) {  // huge vertices: the whole block each (block_fit)
    const int32_t v = __ldg(wl + huge[h]);
    const int64_t s = ld_ro(row_ptr + v), e = ld_ro(row_ptr + v + 1);
    const int32_t t = block_fit(col_idx, C, s, e, sm);
    if (threadIdx.x == 0) {
      __stcg(C + v, t);
      my += (unsigned long long)(e - s);
    }
  }
  block_add(my, edges);
}

// Push v (degree d) into round list `par`, region of its part j: low-degree members from
// the front, the others from the back. Warp-collective (all 32 lanes call; `pred` selects
// the pushing lanes): lanes with the same (part, kind) share one atomicAdd (the callers
// iterate parts in order, so a warp's lanes usually share both). Lists are unordered.
__device__ __forceinline__ void push_warp(const Args& a, int par, int32_t v, int64_t d, bool pred) {
  const int64_t j = pred ? gs_part(v, a.n, a.K, a.partition) : -1;
  const int big = d > kSmallDeg ? 1 : 0;
  const long long key = pred ? (long long)(2 * j + big) : -1ll;
  const unsigned grp = __match_any_sync(0xffffffffu, key);
  const int lane = threadIdx.x & 31;
  const int lead = __ffs(grp) - 1;
  int32_t o = 0;
  if (pred && lane == lead) o = atomicAdd(cnt_of(a, par, j, big), __popc(grp));
  o = __shfl_sync(0xffffffffu, o, lead) + __popc(grp & ((1u << lane) - 1u));
  if (pred) {
    if (!big) (par ? a.L[1] : a.L[0])[__ldg(a.poff + j) + o] = v;
    else (par ? a.L[1] : a.L[0])[__ldg(a.poff + j + 1) - 1 - o] = v;
  }
}

// The vertex at position p of the part-major order (part 0's vertices, then part 1's, ...):
// blocked parts are contiguous id ranges, so p itself; strided part j holds j, j + K, ...
__device__ __forceinline__ int32_t vertex_at(const Args& a, int64_t p) {
  if (a.partition == 1) return (int32_t)p;
  int64_t lo = 0, hi = a.K;  // largest j with poff[j] <= p
  while (hi - lo > 1) {
    const int64_t mid = (lo + hi) >> 1;
    if (__ldg(a.poff + mid) <= p) lo = mid;
    else hi = mid;
  }
  return (int32_t)(lo + a.K * (p - __ldg(a.poff + lo)));
}

template <int TB>
__global__ void __launch_bounds__(256, 3) k_gs_persistent(Args a) {
  __shared__ unsigned long long gs_sm[4];  // block_fit's merged window masks
  if (threadIdx.x < 4) gs_sm[threadIdx.x] = 0ull;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t nthr = (int64_t)gridDim.x * blockDim.x;
  const int64_t gw = tid >> 5, nw = nthr >> 5;
  Ctrl* ctrl = a.ctrl;
  const bool leader = blockIdx.x == 0 && threadIdx.x == 0;
  uint32_t epoch = 0;
  int cb = 0;   // Cur = C[cb]
  int par = 0;  // W_{R-1}'s lists in L[par]; round R's are pushed into L[par ^ 1]
  unsigned long long my_edges = 0;
  for (int R = 1;; ++R) {
    // ---------------- sub-step 0: detect round R-1 over W_{R-1}, assign part 0 ----------
    const int32_t* Cur = (cb ? a.C[1] : a.C[0]);
    int32_t* Nxt = (cb ? a.C[0] : a.C[1]);
    const int np = par ^ 1;  // round R's lists
    const int g = lane >> 3, gl = lane & 7;
    const unsigned gmask = 0xffu << (g * 8);
    if (R == 1) {  // W_0 = V, everything "conflicts": round 1 starts with every vertex,
                   // visited in part-major order so a warp's pushes share one atomic
      for (int64_t b0 = tid - lane; b0 < a.n; b0 += nthr) {
        const int64_t p = b0 + lane;
        const bool ok = p < a.n;
        const int32_t v = ok ? vertex_at(a, p) : 0;
        const int64_t s = ok ? ld_ro(a.row_ptr + v) : 0, e = ok ? ld_ro(a.row_ptr + v + 1) : 0;
        push_warp(a, np, v, e - s, ok);
        my_edges += (unsigned long long)(e - s);
      }
    } else {
      // small members of every part of W_{R-1}: an 8-lane group each; detection against
      // Cur, the losers pushed, part-0 losers take their first fit from the same scan
      for (int64_t j = 0; j < a.K; ++j) {
        const int32_t base = __ldg(a.poff + j);
        const int32_t ns = __ldcg(cnt_of(a, par, j, 0));
        for (int64_t b0 = gw * 4; b0 < ns; b0 += nw * 4) {
          const int64_t i = b0 + g;
          const int32_t v = i < ns ? __ldcg(&(par ? a.L[1] : a.L[0])[base + i]) : -1;
          const int64_t s = v >= 0 ? ld_ro(a.row_ptr + v) : 0, e = v >= 0 ? ld_ro(a.row_ptr + v + 1) : 0;
          bool conf = false;
          const int32_t tent = group_scan<TB>(a, Cur, v, s, e, gl, gmask, true, conf);
          const bool lead = v >= 0 && gl == 0;
          push_warp(a, np, v, e - s, lead && conf);
          if (lead) {
            if (!conf) {
              if (a.K == 1) Nxt[v] = __ldcg(Cur + v);  // K = 1: W_{R-1} is the previous sub-step
            } else {
              my_edges += (unsigned long long)(e - s);
              if (j == 0) Nxt[v] = tent;
            }
          }
        }
      }
    }
    // huge members: block per vertex (detection; part-0 ones also take their first fit)
    for (int64_t j = 0; j < a.K; ++j) {
      const int32_t top = __ldg(a.poff + j + 1);
      const int32_t nbg = R == 1 ? 0 : __ldcg(cnt_of(a, par, j, 1));
      for (int64_t i = blockIdx.x; i < nbg; i += gridDim.x) {
        const int32_t v = __ldcg(&(par ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s <= SGR_GS_HUGE) continue;  // block-uniform
        if (!block_conflict<TB>(a, Cur, v, s, e)) {
          if (a.K == 1 && threadIdx.x == 0) Nxt[v] = __ldcg(Cur + v);
          continue;
        }
        if (threadIdx.x < 32) push_warp(a, np, v, e - s, lane == 0);
        if (threadIdx.x == 0) my_edges += (unsigned long long)(e - s);
        if (j == 0) {
          const int32_t t = block_fit(a.col_idx, Cur, s, e, gs_sm);
          if (threadIdx.x == 0) Nxt[v] = t;
        }
      }
    }
    // big members: warp per vertex (detection; part-0 ones also take their first fit)
    for (int64_t j = 0; j < a.K; ++j) {
      const int32_t top = __ldg(a.poff + j + 1);
      const int32_t nbg = R == 1 ? 0 : __ldcg(cnt_of(a, par, j, 1));
      for (int64_t i = gw; i < nbg; i += nw) {
        const int32_t v = __ldcg(&(par ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s > SGR_GS_HUGE) continue;  // the blocks took it
        if (!warp_conflict<TB>(a, Cur, v, s, e, lane)) {
          if (a.K == 1 && lane == 0) Nxt[v] = __ldcg(Cur + v);
          continue;
        }
        push_warp(a, np, v, e - s, lane == 0);
        if (lane == 0) my_edges += (unsigned long long)(e - s);
        if (j == 0) {
          const int32_t t = warp_fit(a, Cur, s, e, lane);
          if (lane == 0) Nxt[v] = t;
        }
      }
    }
    // copy: the previous sub-step's members (W_{R-1} ∩ part K-1) into Nxt (K = 1: done above,
    // where each member either takes its new color or keeps its old one)
    if (R > 1 && a.K > 1) {
      const int64_t j = a.K - 1;
      const int32_t base = __ldg(a.poff + j), top = __ldg(a.poff + j + 1);
      const int32_t ns = __ldcg(cnt_of(a, par, j, 0)), nbg = __ldcg(cnt_of(a, par, j, 1));
      for (int64_t i = tid; i < ns + nbg; i += nthr) {
        const int32_t u = i < ns ? __ldcg(&(par ? a.L[1] : a.L[0])[base + i]) : __ldcg(&(par ? a.L[1] : a.L[0])[top - 1 - (i - ns)]);
        Nxt[u] = __ldcg(Cur + u);
      }
    }
    block_add(my_edges, &ctrl->edges[np]);
    my_edges = 0;
    gsync(ctrl, epoch);
    if (R == 1) {  // part-0 members of round 1 (all vertices conflict): their first fits
      const int32_t base0 = __ldg(a.poff);
      const int32_t ns0 = __ldcg(cnt_of(a, np, 0, 0));
      for (int64_t b0 = gw * 4; b0 < ns0; b0 += nw * 4) {
        const int64_t i = b0 + g;
        const int32_t v = i < ns0 ? __ldcg(&(np ? a.L[1] : a.L[0])[base0 + i]) : -1;
        const int64_t s = v >= 0 ? ld_ro(a.row_ptr + v) : 0, e = v >= 0 ? ld_ro(a.row_ptr + v + 1) : 0;
        bool conf;
        const int32_t tent = group_scan<TB>(a, Cur, v, s, e, gl, gmask, false, conf);
        if (v >= 0 && gl == 0) Nxt[v] = tent;
      }
      const int32_t top = __ldg(a.poff + 1);
      const int32_t nbg = __ldcg(cnt_of(a, np, 0, 1));
      for (int64_t i = blockIdx.x; i < nbg; i += gridDim.x) {  // huge: block per vertex
        const int32_t v = __ldcg(&(np ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s <= SGR_GS_HUGE) continue;
        const int32_t t = block_fit(a.col_idx, Cur, s, e, gs_sm);
        if (threadIdx.x == 0) Nxt[v] = t;
      }
      for (int64_t i = gw; i < nbg; i += nw) {
        const int32_t v = __ldcg(&(np ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s > SGR_GS_HUGE) continue;
        const int32_t t = warp_fit(a, Cur, s, e, lane);
        if (lane == 0) Nxt[v] = t;
      }
      gsync(ctrl, epoch);
    }
    // |W_R| and its edges; the previous parity's counts can be cleared for round R+1
    int64_t wsz = 0;
    for (int64_t j = 0; j < a.K; ++j) wsz += (int64_t)__ldcg(cnt_of(a, np, j, 0)) + __ldcg(cnt_of(a, np, j, 1));
    if (wsz == 0) {  // W_R empty: round R-1 was the last; its final colors are in Cur
      if (leader) {
        ctrl->rounds = R - 1;
        ctrl->final_buf = cb;
      }
      return;
    }
    if (R > a.max_rounds) {
      if (leader) {
        ctrl->rounds = R - 1;
        ctrl->final_buf = cb;
        ctrl->status = 1;
      }
      return;
    }
    if (leader) {
      const unsigned long long ed = __ldcg(&ctrl->edges[np]);
      ctrl->verts_total += (unsigned long long)wsz;
      ctrl->edges_total += ed;
      if (R - 1 < a.round_cap) {
        if (a.round_sizes) a.round_sizes[R - 1] = (int32_t)wsz;
        if (a.round_edges) a.round_edges[R - 1] = (int64_t)ed;
      }
    }
    cb ^= 1;
    // ---------------- sub-steps 1 .. K-1: assign part j, copy part j-1 ---------------
    for (int64_t j = 1; j < a.K; ++j) {
      const int32_t* Cj = (cb ? a.C[1] : a.C[0]);
      int32_t* Nj = (cb ? a.C[0] : a.C[1]);
      const int32_t base = __ldg(a.poff + j), top = __ldg(a.poff + j + 1);
      const int32_t ns = __ldcg(cnt_of(a, np, j, 0)), nbg = __ldcg(cnt_of(a, np, j, 1));
      for (int64_t b0 = gw * 4; b0 < ns; b0 += nw * 4) {
        const int64_t i = b0 + g;
        const int32_t v = i < ns ? __ldcg(&(np ? a.L[1] : a.L[0])[base + i]) : -1;
        const int64_t s = v >= 0 ? ld_ro(a.row_ptr + v) : 0, e = v >= 0 ? ld_ro(a.row_ptr + v + 1) : 0;
        bool conf;
        const int32_t tent = group_scan<TB>(a, Cj, v, s, e, gl, gmask, false, conf);
        if (v >= 0 && gl == 0) Nj[v] = tent;
      }
      for (int64_t i = blockIdx.x; i < nbg; i += gridDim.x) {  // huge: block per vertex
        const int32_t v = __ldcg(&(np ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s <= SGR_GS_HUGE) continue;
        const int32_t t = block_fit(a.col_idx, Cj, s, e, gs_sm);
        if (threadIdx.x == 0) Nj[v] = t;
      }
      for (int64_t i = gw; i < nbg; i += nw) {
        const int32_t v = __ldcg(&(np ? a.L[1] : a.L[0])[top - 1 - i]);
        const int64_t s = ld_ro(a.row_ptr + v), e = ld_ro(a.row_ptr + v + 1);
        if (e - s > SGR_GS_HUGE) continue;
        const int32_t t = warp_fit(a, Cj, s, e, lane);
        if (lane == 0) Nj[v] = t;
      }
      {  // copy part j-1's members (changed in the previous sub-step) into Nj
        const int32_t pb = __ldg(a.poff + j - 1), pt = __ldg(a.poff + j);
        const int32_t ps = __ldcg(cnt_of(a, np, j - 1, 0)), pg = __ldcg(cnt_of(a, np, j - 1, 1));
        for (int64_t i = tid; i < ps + pg; i += nthr) {
          const int32_t u = i < ps ? __ldcg(&(np ? a.L[1] : a.L[0])[pb + i]) : __ldcg(&(np ? a.L[1] : a.L[0])[pt - 1 - (i - ps)]);
          Nj[u] = __ldcg(Cj + u);
        }
      }
      gsync(ctrl, epoch);
      cb ^= 1;
    }
    // round R's lists become W_R; clear the parity round R+1 pushes into, and its edges
    if (tid < 2 * a.K) a.cnt[(int64_t)par * a.K * 2 + tid] = 0;
    if (leader) ctrl->edges[par] = 0ull;
    gsync(ctrl, epoch);
    par = np;
  }
}

}  // namespace gsp
}  // namespace sgr
