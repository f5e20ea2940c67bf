// sgr_host.cuh — host-side helpers shared by sgr.cu (single GPU) and sgr_dist.cu
// (multi-GPU): workspace layout, kernel-argument construction, grid sizing.
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <cstdlib>
#include <cstring>

#include "sgr_internal.h"
#include "sgr_round.cuh"

namespace sgr {

inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// Workspace layout (bytes, each piece 256-aligned):
//   Ctrl | colors: 2 x n words (u16 packed / i32) | wl_t: 2 x n i32 | wl_m: 2 x cap_m i32 | wl_c: 2 x cap_c i64 |
//   big_id: n i32 | acc_bits: cap_big x 32 u32 | acc_cnt: cap_big u64 |
//   (packed mode) fixed: cap_big x 32 u32 | len: 2 x n i32 | adj: 2 x (nnz + 16) i32
// 32-bit mode: the caller's colors_out is one of the two ping-pong buffers. Packed mode
// (12-bit color + round mod 16, trimming) uses two workspace buffers and unpacks at the end.
struct Layout {
  bool packed;
  int64_t cap_m, cap_c, cap_big;
  size_t off_col, off_t, off_m, off_c, off_big, off_accb, off_accc, off_fixed, off_len, off_adj,
      off_fin, off_bm;
  size_t zero_begin, zero_end, total;
};

inline Layout layout(int64_t n, int64_t nnz, const Resolved& r) {
  Layout L;
  L.packed = r.color_bits == 16;
  L.cap_m = std::min<int64_t>(n, nnz / (r.small_max + 1) + 1);
  // each bin-2 vertex (deg > med_max) has <= deg / kChunk + 1 chunks
  L.cap_c = nnz / kChunk + nnz / (r.med_max + 1) + 2;
  L.cap_big = nnz / (r.med_max + 1) + 1;
  const size_t nb = align_up((size_t)n * 4, 256);
  size_t o = align_up(sizeof(Ctrl), 256);
  L.off_col = o;
  o += 2 * align_up((size_t)n * (L.packed ? sizeof(Packed) : 4), 256);
  L.off_t = o;
  o += 2 * nb;
  L.off_m = o;
  o += 2 * align_up((size_t)L.cap_m * 4, 256);
  L.off_c = o;
  o += 2 * align_up((size_t)L.cap_c * 8, 256);
  L.off_big = o;
  o += nb;
  L.off_accb = o;
  L.zero_begin = o;
  o += align_up((size_t)L.cap_big * 128, 256);
  L.off_accc = o;
  o += align_up((size_t)L.cap_big * 8, 256);
  L.off_fixed = L.off_len = L.off_adj = o;
  if (L.packed) {
    L.off_fixed = o;
    o += align_up((size_t)L.cap_big * 128, 256);
    L.off_len = o;
    o += 2 * nb;
  }
  L.zero_end = o;  // accumulators, fixed sets and list lengths start at zero
  L.off_fin = o;
  o += align_up((size_t)L.cap_big * 8, 256);
  // worklist membership bitmaps (dense passes of the flat build): 2 x ceil(n / 32) words
  L.off_bm = o;
  o += 2 * align_up((size_t)((n + 31) / 32) * 4, 256);
  if (L.packed) {
    L.off_adj = o;
    o += 2 * align_up((size_t)(nnz + 16) * 4, 256);
  }
  L.total = o;
  return L;
}


// The dense passes' bitmaps (single-GPU colorings only: F_1 writes W_2's when set).
template <class C>
inline void set_bitmaps(RoundArgs<C>& a, void* ws, const Layout& L, int64_t n) {
  char* b = (char*)ws;
  const size_t bmb = align_up((size_t)((n + 31) / 32) * 4, 256);
  a.bm[0] = (uint32_t*)(b + L.off_bm);
  a.bm[1] = (uint32_t*)(b + L.off_bm + bmb);
  if constexpr (packed<C>()) a.dcol = (int16_t*)a.adj[0];  // unused by the flat build
}

template <class C>
inline void build_args(RoundArgs<C>& a, const sgr_csr* csr, int64_t n, int64_t nnz,
                       int32_t* colors, void* ws, const Layout& L, const Resolved& r) {
  memset(&a, 0, sizeof(a));
  char* b = (char*)ws;
  const size_t nb = align_up((size_t)n * 4, 256);
  a.row_ptr = csr->row_ptr;
  a.col_idx = csr->col_idx;
  if constexpr (packed<C>()) {
    a.col[0] = (C*)(b + L.off_col);
    a.col[1] = (C*)(b + L.off_col + align_up((size_t)n * sizeof(C), 256));
    a.fixed = (uint32_t*)(b + L.off_fixed);
    a.fin = (int64_t*)(b + L.off_fin);
    a.len[0] = (int32_t*)(b + L.off_len);
    a.len[1] = (int32_t*)(b + L.off_len + nb);
    const size_t ab = align_up((size_t)(nnz + 16) * 4, 256);
    a.adj[0] = (int32_t*)(b + L.off_adj);
    a.adj[1] = (int32_t*)(b + L.off_adj + ab);
  } else {
    a.col[0] = (C*)colors;
    a.col[1] = (C*)(b + L.off_col);
  }
  a.wl_t[0] = (int32_t*)(b + L.off_t);
  a.wl_t[1] = (int32_t*)(b + L.off_t + nb);
  const size_t sm = align_up((size_t)L.cap_m * 4, 256);
  a.wl_m[0] = (int32_t*)(b + L.off_m);
  a.wl_m[1] = (int32_t*)(b + L.off_m + sm);
  const size_t sc = align_up((size_t)L.cap_c * 8, 256);
  a.wl_c[0] = (int64_t*)(b + L.off_c);
  a.wl_c[1] = (int64_t*)(b + L.off_c + sc);
  a.big_id = (int32_t*)(b + L.off_big);
  a.acc_bits = (uint32_t*)(b + L.off_accb);
  a.acc_cnt = (unsigned long long*)(b + L.off_accc);
  a.ctrl = (Ctrl*)b;
  a.n = (int32_t)n;
  a.nnz = nnz;
  a.v_begin = 0;
  a.v_end = (int32_t)n;
  a.small_max = r.small_max;
  a.med_max = r.med_max;
  a.color_cap = r.color_cap;
  a.flat_bin0 = r.flat_bin0;
}

// Streaming per-vertex kernels (F_1, unpack, max): one thread per vertex up to 64 blocks
// per SM, so the dependent row_ptr -> col_idx loads of many vertices are in flight.
// (B = threads per block; the caps keep 64 x 256 / 8 x 256 threads per SM for any B.)
inline int first_grid(int64_t n, int B = 256) {
  return (int)std::max<int64_t>(1, std::min<int64_t>((n + B - 1) / B, (int64_t)num_sms() * 64 * 256 / B));
}
// Per-vertex kernels that end in one atomic per warp (unpack + max): 8 blocks per SM.
inline int reduce_grid(int64_t n, int B = 256) {
  return (int)std::max<int64_t>(1, std::min<int64_t>((n + B - 1) / B, std::max<int64_t>(num_sms(), (int64_t)num_sms() * 8 * 256 / B)));
}

// Dynamic shared memory of a round-kernel block of `B` threads (per-warp slices).
template <class C, bool Hub = true>
constexpr size_t round_smem(int B = kBlock) { return (size_t)(B / 32) * WarpSmem<C, Hub>::kBytes; }
// Largest block the round kernels of this build accept (their launch bounds).
template <class C, bool Hub = true>
constexpr int round_max_block() { return kMaxThreads<C, Hub>; }

// Blocks of the round kernels: as many as are co-resident (persistent: required).
template <int TB, class C, bool Hub = true, bool T0 = false>
inline int round_grid(bool persistent, int B = kBlock) {
  // The > 48 KB dynamic shared memory opt-in is a per-device function attribute: one bit
  // per device (setting it twice from racing threads is harmless; the bit only skips the
  // call once it has succeeded on that device).
  static std::atomic<uint64_t> attr_set{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = (dev >= 0 && dev < 64) ? (1ull << dev) : 0ull;
  if (!bit || !(attr_set.load(std::memory_order_acquire) & bit)) {
    // the opt-in covers the largest block the build accepts
    const int smax = (int)round_smem<C, Hub>(round_max_block<C, Hub>());
    const cudaError_t e1 = cudaFuncSetAttribute(
        k_persistent<TB, C, Hub, T0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smax);
    const cudaError_t e2 = cudaFuncSetAttribute(
        k_round<TB, C, Hub>, cudaFuncAttributeMaxDynamicSharedMemorySize, smax);
    if (e1 == cudaSuccess && e2 == cudaSuccess && bit) attr_set.fetch_or(bit, std::memory_order_acq_rel);
    if (e1 != cudaSuccess || e2 != cudaSuccess) cudaGetLastError();  // do not leak into later checks
  }
  int per_sm = 0;
  cudaError_t e = persistent
      ? cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_persistent<TB, C, Hub, T0>, B,
                                                      round_smem<C, Hub>(B))
      : cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_round<TB, C, Hub>, B,
                                                      round_smem<C, Hub>(B));
  if (e != cudaSuccess || per_sm <= 0) per_sm = 1;
  if (const char* env = getenv("SGR_BLOCKS_PER_SM")) {  // experiments: shrink the grid
    const int lim = atoi(env);
    if (lim > 0 && lim < per_sm) per_sm = lim;
  }
  return per_sm * num_sms();
}

// Blocks of k_dense (its own register allocation; the flat build's shared memory).
template <int TB, class C>
inline int dense_grid(int B = kBlock) {
  static std::atomic<uint64_t> attr_set{0};
  int dev = 0;
  cudaGetDevice(&dev);
  const uint64_t bit = (dev >= 0 && dev < 64) ? (1ull << dev) : 0ull;
  if (!bit || !(attr_set.load(std::memory_order_acquire) & bit)) {
    const cudaError_t e1 = cudaFuncSetAttribute(k_dense<TB, C>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                (int)round_smem<C, false>(round_max_block<C, false>()));
    if (e1 == cudaSuccess && bit) attr_set.fetch_or(bit, std::memory_order_acq_rel);
    if (e1 != cudaSuccess) cudaGetLastError();
  }
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_dense<TB, C>, B, round_smem<C, false>(B)) !=
          cudaSuccess ||
      per_sm <= 0)
    per_sm = 1;
  return per_sm * num_sms();
}

}  // namespace sgr
