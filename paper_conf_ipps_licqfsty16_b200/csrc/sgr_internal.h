// sgr_internal.h — declarations shared by sgr.cu and sgr_dist.cu (not part of the ABI).
#pragma once
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "sgr.h"

namespace sgr {

struct Ctrl;

struct Resolved {
  int tiebreak;
  int32_t max_rounds;
  int loop_mode;
  int color_bits;
  int small_max;
  int med_max;
  cudaStream_t stream;
  int32_t* round_sizes;
  int64_t* round_edges;
  int32_t round_cap;
  int validate;
  int batch;
  int profile;
  float* round_ms;
  int32_t color_cap;
  int64_t* round_ns;
  int block;      // threads per block (opts->block_size; 0 -> 256)
  int sorted;     // rows sorted ascending (F_1 reads one entry per row); 0: whole rows
  int flat_bin0;  // opts->flat_bin0 test hook: 0 auto, 1 groups, 2 thread per vertex
};

// Threads-per-block limits (opts->block_size): per-vertex kernels, and the fused round
// kernels (register budget fixed by their launch bounds: hub build 512, others 768).
constexpr int kMaxBlockAny = 1024;

void set_error(const char* fmt, ...);
sgr_status cuda_fail(cudaError_t e, const char* what, int line);
int num_sms();
void keep_pool_memory();
Resolved resolve_opts(const sgr_opts* o, int64_t n);
bool block_ok(int B, int lo, int hi);
size_t ws_bytes(int64_t n, int64_t nnz, const Resolved& r);
void fill_stats(const Ctrl& c, int64_t n, int64_t nnz, sgr_stats* st, int cb);

}  // namespace sgr
