// sgr_kernels.cuh — sm_100a kernels of the deterministic SGR round.
//
// One fused pass F_k per round k >= 2 computes, for every v in W_k (Alg. 5):
//   conflict(v) = exists w in adj(v): X[w] == X[v] and lose(v, w)       (Alg. 5 l.12-15)
//   tent(v)     = min{c > 0 : c not in {X[w] : w in adj(v)}}              (Alg. 5 l.4-8)
//   Y[v]        = conflict(v) ? tent(v) : X[v];  W_{k+1} gets v iff conflict(v)
// where X = C_k is the color snapshot of round k and Y the ping-pong buffer (it holds
// C_{k-1}, which differs from C_{k+1} only inside W_k — DESIGN.md §3 proof (iv)). The
// detection of round k and the assignment of round k+1 read the same snapshot, so one
// adjacency scan serves both. F_1 (round 1 = "every vertex takes color 1") needs no
// color gathers at all: conflict(v) depends only on the smallest / largest neighbour id.
//
// Work is binned statically by degree (a vertex's degree never changes, and W only
// shrinks): thread per vertex (d <= small), warp per vertex (d <= med), CTA per vertex.
// Worklist pushes use warp ballot + popc + one atomicAdd per warp ("one atomic
// per thread block", here per warp), or one atomic per pushed vertex in the warp/CTA bins.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace sgr {

constexpr int kBins = 3;  // 0 = thread, 1 = warp, 2 = CTA per vertex
constexpr int kWinWords = 4;  // forbidden-color window: 4 x 64 bits = colors [base, base+256)
constexpr int kWinBits = 64 * kWinWords;

// Device-resident loop state (lives in the workspace).
struct Ctrl {
  int32_t k;           // index of the next fused pass F_k (k = 2 after F_1)
  int32_t active;      // 1 while W_k is non-empty
  int32_t status;      // 0 ok, 1 = max_rounds reached with W non-empty
  int32_t max_rounds;
  int32_t cnt[2][kBins];          // |W| per parity (k & 1) and bin
  int32_t round_cap;
  int32_t pad0;
  unsigned long long edges_acc[kBins];  // scanned CSR entries of the running pass, per bin
  unsigned long long verts_total[kBins + 1];   // sum |W_r| per bin (+ F_1 at [kBins])
  unsigned long long edges_total[kBins + 1];   // sum deg(W_r) per bin (+ round 1)
  unsigned long long pushes_total[kBins + 1];  // sum |W_{r+1}| produced per bin (+ F_1)
  int32_t* round_sizes;  // optional trace (device)
  int64_t* round_edges;
  int32_t max_color;     // filled by k_max_color
  int32_t violations;    // filled by k_validate
};

struct RoundArgs {
  const int64_t* __restrict__ row_ptr;
  const int32_t* __restrict__ col_idx;
  int32_t* col[2];             // color ping-pong buffers: C_k lives in col[(k-1) & 1]
  int32_t* wl[2][kBins];       // worklists: W_k^bin lives in wl[k & 1][bin]
  Ctrl* ctrl;
  int32_t n;
  int32_t small_max;           // thread-bin degree bound (<= 62)
  int32_t med_max;             // warp-bin degree bound
};

// Select without dynamic indexing into the kernel-parameter struct (that would copy the
// whole struct to local memory).
__device__ __forceinline__ int32_t* sel_col(const RoundArgs& a, int par) {
  return par ? a.col[1] : a.col[0];
}
__device__ __forceinline__ int32_t* sel_wl(const RoundArgs& a, int par, int bin) {
  return par ? a.wl[1][bin] : a.wl[0][bin];
}

template <int TB>
__device__ __forceinline__ bool lose(int32_t v, int32_t w) {
  // TB 0 = LOWID_KEEPS (v > w recolors), 1 = PAPER (Alg. 5 l.14: v < w recolors)
  if constexpr (TB == 1) return v < w;
  else return v > w;
}

__device__ __forceinline__ int32_t ldg_i32(const int32_t* p) { return __ldg(p); }
__device__ __forceinline__ int64_t ldg_i64(const int64_t* p) { return __ldg(p); }

// Read-only streaming load for col_idx (no L1 allocation: each entry is used once).
__device__ __forceinline__ int32_t ld_stream(const int32_t* p) {
  int32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

__device__ __forceinline__ int bin_of(int64_t d, int small_max, int med_max) {
  return d <= small_max ? 0 : (d <= med_max ? 1 : 2);
}

// Warp-aggregated push: every lane with `pred` appends `v` to list/count; one atomic per
// warp. Must be called by all 32 lanes (convergent).
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

// Set bit (c - base) of a kWinWords-word window held in registers.
__device__ __forceinline__ void win_set(uint64_t (&m)[kWinWords], int32_t c, int32_t base) {
  const uint32_t idx = (uint32_t)(c - base);
  if (idx < (uint32_t)kWinBits) {
    const uint64_t bit = 1ull << (idx & 63);
    const uint32_t word = idx >> 6;
#pragma unroll
    for (int q = 0; q < kWinWords; ++q) m[q] |= (word == (uint32_t)q) ? bit : 0ull;
  }
}

// First zero bit of the window (bit 0 of window base 0 stands for color 0 and is preset).
// Returns -1 if all kWinBits bits are set.
__device__ __forceinline__ int win_first_zero(const uint64_t (&m)[kWinWords]) {
#pragma unroll
  for (int q = 0; q < kWinWords; ++q)
    if (~m[q]) return q * 64 + __ffsll((long long)~m[q]) - 1;
  return -1;
}

__device__ __forceinline__ uint64_t warp_or64(uint64_t x) {
  const uint32_t lo = __reduce_or_sync(0xffffffffu, (uint32_t)x);
  const uint32_t hi = __reduce_or_sync(0xffffffffu, (uint32_t)(x >> 32));
  return ((uint64_t)hi << 32) | lo;
}

// ---------------------------------------------------------------------------------------
// Exact warp-cooperative first fit for any degree (used by the warp bin, the CTA bin's
// rescans and the step entry points): windows of kWinBits colors until a free one shows.
// All 32 lanes must call it with the same arguments; returns the same value on all lanes.
__device__ __forceinline__ int32_t warp_first_fit_from(const int32_t* __restrict__ col_idx,
                                                       const int32_t* __restrict__ X,
                                                       int64_t s, int64_t e, int32_t base,
                                                       int lane) {
  for (;;) {
    uint64_t m[kWinWords] = {};
    if (base == 0) m[0] = 1;  // color 0 is never a candidate
    for (int64_t j = s + lane; j < e; j += 32) win_set(m, ldg_i32(X + ld_stream(col_idx + j)), base);
#pragma unroll
    for (int q = 0; q < kWinWords; ++q) m[q] = warp_or64(m[q]);
    const int z = win_first_zero(m);
    if (z >= 0) return base + z;
    base += kWinBits;
  }
}

// ---------------------------------------------------------------------------------------
// F_1: round-1 detection + round-2 assignment without color gathers. Every color is 1
// after round 1 (Alg. 5 l.4-9 with an all-zero snapshot), so
//   LOWID: conflict(v) <=> min adj(v) < v ;  PAPER: conflict(v) <=> max adj(v) > v
// (rows are sorted ascending, so these are the first / last entry; self-loops can never
// satisfy the strict inequality). tent(v) = mex({1}) = 2.
// Writes col[0] = C_1 (all 1) and col[1] = C_2, and W_2 split into bins in wl[0][*].
template <int TB>
__global__ void __launch_bounds__(256) k_first(RoundArgs a) {
  Ctrl* ctrl = a.ctrl;
  int32_t* __restrict__ X = a.col[0];
  int32_t* __restrict__ Y = a.col[1];
  unsigned long long pushes = 0;
  const int64_t n = a.n;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t vi = base + threadIdx.x;
    bool conflict = false;
    int b = 0;
    if (vi < n) {
      const int32_t v = (int32_t)vi;
      const int64_t s = ldg_i64(a.row_ptr + v), e = ldg_i64(a.row_ptr + v + 1);
      if (e > s) {
        if constexpr (TB == 1) conflict = ldg_i32(a.col_idx + e - 1) > v;
        else conflict = ldg_i32(a.col_idx + s) < v;
      }
      b = bin_of(e - s, a.small_max, a.med_max);
      X[v] = 1;
      Y[v] = conflict ? 2 : 1;
    }
#pragma unroll
    for (int q = 0; q < kBins; ++q)
      warp_push(conflict && b == q, (int32_t)vi, a.wl[0][q], &ctrl->cnt[0][q]);
    pushes += conflict;
  }
  (void)pushes;
}

// Generic F_1 for rows that are NOT sorted: scan the whole row for min / max.
template <int TB>
__global__ void __launch_bounds__(256) k_first_unsorted(RoundArgs a) {
  Ctrl* ctrl = a.ctrl;
  int32_t* __restrict__ X = a.col[0];
  int32_t* __restrict__ Y = a.col[1];
  const int64_t n = a.n;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t vi = base + threadIdx.x;
    bool conflict = false;
    int b = 0;
    if (vi < n) {
      const int32_t v = (int32_t)vi;
      const int64_t s = ldg_i64(a.row_ptr + v), e = ldg_i64(a.row_ptr + v + 1);
      for (int64_t j = s; j < e && !conflict; ++j) conflict = lose<TB>(v, ldg_i32(a.col_idx + j));
      b = bin_of(e - s, a.small_max, a.med_max);
      X[v] = 1;
      Y[v] = conflict ? 2 : 1;
    }
#pragma unroll
    for (int q = 0; q < kBins; ++q)
      warp_push(conflict && b == q, (int32_t)vi, a.wl[0][q], &ctrl->cnt[0][q]);
  }
}

// Block-level sum of a per-thread counter, one atomicAdd per block.
__device__ __forceinline__ void block_add(unsigned long long x, unsigned long long* dst) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  __shared__ unsigned long long red[32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (lane == 0) red[wid] = x;
  __syncthreads();
  if (wid == 0) {
    x = lane < (int)(blockDim.x >> 5) ? red[lane] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (lane == 0 && x) atomicAdd(dst, x);
  }
}

// ---------------------------------------------------------------------------------------
// F_k, thread bin (deg <= small_max <= 62): one thread per vertex, forbidden set in one
// u64 register (mex <= deg+1 <= 63, so colors >= 64 can be ignored exactly).
template <int TB>
__global__ void __launch_bounds__(256) k_round_thread(RoundArgs a) {
  Ctrl* ctrl = a.ctrl;
  const int k = ctrl->k;
  const int p = k & 1;
  const int cnt = ctrl->cnt[p][0];
  const int32_t* __restrict__ X = sel_col(a, (k - 1) & 1);
  int32_t* __restrict__ Y = sel_col(a, k & 1);
  const int32_t* __restrict__ W = sel_wl(a, p, 0);
  int32_t* Wn = sel_wl(a, p ^ 1, 0);
  int32_t* outcnt = &ctrl->cnt[p ^ 1][0];
  unsigned long long edges = 0;
  for (int base = blockIdx.x * blockDim.x; base < cnt; base += gridDim.x * blockDim.x) {
    const int i = base + threadIdx.x;
    bool conflict = false;
    int32_t v = 0;
    if (i < cnt) {
      v = ldg_i32(W + i);
      const int64_t s = ldg_i64(a.row_ptr + v), e = ldg_i64(a.row_ptr + v + 1);
      const int32_t xv = ldg_i32(X + v);
      uint64_t mask = 1ull;
      for (int64_t j = s; j < e; j += 4) {
        int32_t w[4], c[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) w[u] = (j + u < e) ? ld_stream(a.col_idx + j + u) : v;
#pragma unroll
        for (int u = 0; u < 4; ++u) c[u] = ldg_i32(X + w[u]);
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          mask |= (c[u] < 64) ? (1ull << (c[u] & 63)) : 0ull;
          conflict |= (c[u] == xv) & lose<TB>(v, w[u]);
        }
      }
      // padded slots read X[v] = xv, harmless: xv's bit is only needed if v conflicts,
      // in which case a neighbour already carries xv (DESIGN.md §3 proof (v)).
      const int32_t tent = __ffsll((long long)~mask) - 1;
      Y[v] = conflict ? tent : xv;
      edges += (unsigned long long)(e - s);
    }
    warp_push(conflict, v, Wn, outcnt);
  }
  block_add(edges, &ctrl->edges_acc[0]);
}

// F_k, warp bin: one warp per vertex, lanes stride the row; 256-color register window
// per lane, OR-reduced across the warp; windows slide only when the first is full.
template <int TB>
__global__ void __launch_bounds__(256) k_round_warp(RoundArgs a) {
  Ctrl* ctrl = a.ctrl;
  const int k = ctrl->k;
  const int p = k & 1;
  const int cnt = ctrl->cnt[p][1];
  const int32_t* __restrict__ X = sel_col(a, (k - 1) & 1);
  int32_t* __restrict__ Y = sel_col(a, k & 1);
  const int32_t* __restrict__ W = sel_wl(a, p, 1);
  int32_t* Wn = sel_wl(a, p ^ 1, 1);
  int32_t* outcnt = &ctrl->cnt[p ^ 1][1];
  const int lane = threadIdx.x & 31;
  const int warps_per_block = blockDim.x >> 5;
  unsigned long long edges = 0;
  for (int i = blockIdx.x * warps_per_block + (threadIdx.x >> 5); i < cnt;
       i += gridDim.x * warps_per_block) {
    const int32_t v = ldg_i32(W + i);
    const int64_t s = ldg_i64(a.row_ptr + v), e = ldg_i64(a.row_ptr + v + 1);
    const int32_t xv = ldg_i32(X + v);
    uint64_t m[kWinWords] = {1ull, 0ull, 0ull, 0ull};
    bool conflict = false;
    int64_t j = s + lane;
    for (; j + 32 < e; j += 64) {  // two independent gathers in flight per lane
      const int32_t w0 = ld_stream(a.col_idx + j), w1 = ld_stream(a.col_idx + j + 32);
      const int32_t c0 = ldg_i32(X + w0), c1 = ldg_i32(X + w1);
      win_set(m, c0, 0);
      win_set(m, c1, 0);
      conflict |= ((c0 == xv) & lose<TB>(v, w0)) | ((c1 == xv) & lose<TB>(v, w1));
    }
    if (j < e) {
      const int32_t w0 = ld_stream(a.col_idx + j);
      const int32_t c0 = ldg_i32(X + w0);
      win_set(m, c0, 0);
      conflict |= (c0 == xv) & lose<TB>(v, w0);
    }
    conflict = __any_sync(0xffffffffu, conflict);
    if (conflict) {
#pragma unroll
      for (int q = 0; q < kWinWords; ++q) m[q] = warp_or64(m[q]);
      int32_t tent = win_first_zero(m);
      if (tent < 0) tent = warp_first_fit_from(a.col_idx, X, s, e, kWinBits, lane);
      if (lane == 0) {
        Y[v] = tent;
        Wn[atomicAdd(outcnt, 1)] = v;
      }
    } else if (lane == 0) {
      Y[v] = xv;
    }
    if (lane == 0) edges += (unsigned long long)(e - s);
  }
  block_add(edges, &ctrl->edges_acc[1]);
}

// F_k, CTA bin: one CTA per vertex (hubs). Same window scheme, reduced across the CTA.
template <int TB>
__global__ void __launch_bounds__(512) k_round_cta(RoundArgs a) {
  Ctrl* ctrl = a.ctrl;
  const int k = ctrl->k;
  const int p = k & 1;
  const int cnt = ctrl->cnt[p][2];
  const int32_t* __restrict__ X = sel_col(a, (k - 1) & 1);
  int32_t* __restrict__ Y = sel_col(a, k & 1);
  const int32_t* __restrict__ W = sel_wl(a, p, 2);
  int32_t* Wn = sel_wl(a, p ^ 1, 2);
  int32_t* outcnt = &ctrl->cnt[p ^ 1][2];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  __shared__ uint64_t smask[32][kWinWords];
  __shared__ int sconf[32];
  __shared__ int32_t s_tent;
  unsigned long long edges = 0;
  for (int i = blockIdx.x; i < cnt; i += gridDim.x) {
    const int32_t v = ldg_i32(W + i);
    const int64_t s = ldg_i64(a.row_ptr + v), e = ldg_i64(a.row_ptr + v + 1);
    const int32_t xv = ldg_i32(X + v);
    uint64_t m[kWinWords] = {1ull, 0ull, 0ull, 0ull};
    bool conflict = false;
    const int64_t stride = blockDim.x;
    int64_t j = s + threadIdx.x;
    for (; j + 3 * stride < e; j += 4 * stride) {
      int32_t w[4], c[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) w[u] = ld_stream(a.col_idx + j + u * stride);
#pragma unroll
      for (int u = 0; u < 4; ++u) c[u] = ldg_i32(X + w[u]);
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        win_set(m, c[u], 0);
        conflict |= (c[u] == xv) & lose<TB>(v, w[u]);
      }
    }
    for (; j < e; j += stride) {
      const int32_t w0 = ld_stream(a.col_idx + j);
      const int32_t c0 = ldg_i32(X + w0);
      win_set(m, c0, 0);
      conflict |= (c0 == xv) & lose<TB>(v, w0);
    }
    const int wconf = __any_sync(0xffffffffu, conflict);
#pragma unroll
    for (int q = 0; q < kWinWords; ++q) m[q] = warp_or64(m[q]);
    if (lane == 0) {
      sconf[wid] = wconf;
#pragma unroll
      for (int q = 0; q < kWinWords; ++q) smask[wid][q] = m[q];
    }
    __syncthreads();
    if (wid == 0) {
      int c = lane < nw ? sconf[lane] : 0;
      c = __any_sync(0xffffffffu, c);
      uint64_t mm[kWinWords];
#pragma unroll
      for (int q = 0; q < kWinWords; ++q) mm[q] = warp_or64(lane < nw ? smask[lane][q] : 0ull);
      int32_t tent = -1;
      if (c) {
        tent = win_first_zero(mm);
        if (tent < 0) tent = warp_first_fit_from(a.col_idx, X, s, e, kWinBits, lane);
      }
      if (lane == 0) {
        Y[v] = c ? tent : xv;
        if (c) Wn[atomicAdd(outcnt, 1)] = v;
        edges += (unsigned long long)(e - s);
      }
    }
    __syncthreads();
  }
  (void)s_tent;
  block_add(edges, &ctrl->edges_acc[2]);
}

// End of pass F_k (one thread): fold the pass's counters into totals / the trace, consume
// W_k, advance k, and decide whether W_{k+1} is non-empty. A pass that found W_k empty
// changes nothing, so surplus passes issued before the host sees `active == 0` are no-ops.
__global__ void k_advance(Ctrl* ctrl, int first) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  if (first) {  // after F_1: round 1 scanned every row once conceptually (|W_1| = n)
    const int p = 0;
    int tot = 0;
    for (int q = 0; q < kBins; ++q) {
      tot += ctrl->cnt[p][q];
      ctrl->pushes_total[kBins] += (unsigned long long)ctrl->cnt[p][q];
    }
    ctrl->k = 2;
    ctrl->active = tot > 0;
    if (ctrl->active && ctrl->max_rounds < 2) {
      ctrl->status = 1;
      ctrl->active = 0;
    }
    return;
  }
  const int k = ctrl->k;
  const int p = k & 1;
  int tot_in = 0;
  for (int q = 0; q < kBins; ++q) tot_in += ctrl->cnt[p][q];
  if (tot_in == 0) {
    ctrl->active = 0;
    return;
  }
  unsigned long long e_all = 0;
  int tot_out = 0;
  for (int q = 0; q < kBins; ++q) {
    ctrl->verts_total[q] += (unsigned long long)ctrl->cnt[p][q];
    ctrl->edges_total[q] += ctrl->edges_acc[q];
    ctrl->pushes_total[q] += (unsigned long long)ctrl->cnt[p ^ 1][q];
    e_all += ctrl->edges_acc[q];
    ctrl->edges_acc[q] = 0;
    ctrl->cnt[p][q] = 0;
    tot_out += ctrl->cnt[p ^ 1][q];
  }
  if (k - 1 < ctrl->round_cap) {
    if (ctrl->round_sizes) ctrl->round_sizes[k - 1] = tot_in;
    if (ctrl->round_edges) ctrl->round_edges[k - 1] = (int64_t)e_all;
  }
  ctrl->k = k + 1;
  ctrl->active = tot_out > 0;
  if (ctrl->active && k + 1 > ctrl->max_rounds) {  // W_{k+1} non-empty beyond the cap
    ctrl->status = 1;
    ctrl->active = 0;
    for (int q = 0; q < kBins; ++q) ctrl->cnt[p ^ 1][q] = 0;
  }
}

__global__ void k_max_color(const int32_t* __restrict__ c, int64_t n, Ctrl* ctrl) {
  int32_t m = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    m = max(m, __ldg(c + i));
  m = __reduce_max_sync(0xffffffffu, (unsigned)m);
  if ((threadIdx.x & 31) == 0 && m) atomicMax(&ctrl->max_color, m);
}

// ---------------------------------------------------------------------------------------
// Step entry points (Algorithm 5 split line by line; not on the fused hot path).

// Alg. 5 l.4-10: warp per listed vertex, exact for any degree.
__global__ void __launch_bounds__(256) k_assign_step(const int64_t* __restrict__ row_ptr,
                                                     const int32_t* __restrict__ col_idx,
                                                     const int32_t* __restrict__ wl, int64_t len,
                                                     const int32_t* __restrict__ X,
                                                     int32_t* __restrict__ tent) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  for (int64_t i = (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); i < len;
       i += (int64_t)gridDim.x * wpb) {
    const int32_t v = __ldg(wl + i);
    const int32_t t = warp_first_fit_from(col_idx, X, __ldg(row_ptr + v), __ldg(row_ptr + v + 1), 0, lane);
    if (lane == 0) tent[i] = t;
  }
}

// Alg. 5 l.9: colors[wl[i]] = tent[i].
__global__ void k_commit_step(const int32_t* __restrict__ wl, const int32_t* __restrict__ tent,
                              int64_t len, int32_t* __restrict__ colors) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len;
       i += (int64_t)gridDim.x * blockDim.x)
    colors[wl[i]] = tent[i];
}

// Alg. 5 l.13-14: warp per listed vertex.
template <int TB>
__global__ void __launch_bounds__(256) k_detect_step(const int64_t* __restrict__ row_ptr,
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
    for (int64_t j = __ldg(row_ptr + v) + lane; j < __ldg(row_ptr + v + 1) && !c; j += 32) {
      const int32_t w = __ldg(col_idx + j);
      c = (__ldg(C + w) == cv) && lose<TB>(v, w);
    }
    c = __any_sync(0xffffffffu, c);
    if (lane == 0) out[i] = c ? 1 : 0;
  }
}

// Order-preserving compaction (Fig. 5): tile counts -> scan -> scatter.
constexpr int kCompactTile = 1024;  // elements per tile (256 threads x 4)

__global__ void __launch_bounds__(256) k_compact_count(const uint8_t* __restrict__ flags,
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
__global__ void __launch_bounds__(1024) k_compact_scan(int32_t* __restrict__ tile_cnt, int64_t tiles,
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

__global__ void __launch_bounds__(256) k_compact_scatter(const int32_t* __restrict__ wl,
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
__global__ void k_validate(const int64_t* __restrict__ row_ptr, const int32_t* __restrict__ col_idx,
                           int64_t n, int64_t nnz, Ctrl* ctrl) {
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
  if (viol) atomicOr(&ctrl->violations, viol);
}

}  // namespace sgr
