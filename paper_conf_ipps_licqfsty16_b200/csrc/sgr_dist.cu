// sgr_dist.cu — multi-GPU layer: nnz-balanced contiguous vertex ranges.
#include <cuda_runtime.h>

#include <cstring>

#include "sgr.h"
#include "sgr_internal.h"

using namespace sgr;

extern "C" {

sgr_status sgr_partition(const int64_t* row_ptr, int64_t n, int32_t P, int64_t* ranges) {
  if (!row_ptr || n < 0 || P < 1 || !ranges) return SGR_EINVAL;
  const int64_t nnz = row_ptr[n];
  ranges[0] = 0;
  for (int32_t p = 1; p < P; ++p) {
    // target = ceil(p * nnz / P) without overflow for nnz < 2^62 / P
    const int64_t target = (int64_t)(((__int128)p * nnz + P - 1) / P);
    ranges[p] = std::lower_bound(row_ptr, row_ptr + n + 1, target) - row_ptr;
    if (ranges[p] > n) ranges[p] = n;
    if (ranges[p] < ranges[p - 1]) ranges[p] = ranges[p - 1];
  }
  ranges[P] = n;
  return SGR_OK;
}

sgr_status sgr_nccl_unique_id(void* id_out) {
  (void)id_out;
  set_error("sgr_nccl_unique_id: not built yet");
  return SGR_EUNSUPPORTED;
}

sgr_status sgr_comm_init(void** comm, int32_t rank, int32_t world, const void* id, int32_t device) {
  (void)comm; (void)rank; (void)world; (void)id; (void)device;
  set_error("sgr_comm_init: not built yet");
  return SGR_EUNSUPPORTED;
}

sgr_status sgr_comm_destroy(void* comm) {
  (void)comm;
  return SGR_OK;
}

sgr_status sgr_color_dist(void* comm, const sgr_csr* local, int64_t n_global, int64_t v_begin,
                          int64_t v_end, int64_t nnz_local, int32_t* colors_out, sgr_stats* stats,
                          const sgr_opts* opts) {
  (void)comm; (void)local; (void)n_global; (void)v_begin; (void)v_end; (void)nnz_local;
  (void)colors_out; (void)stats; (void)opts;
  set_error("sgr_color_dist: not built yet");
  return SGR_EUNSUPPORTED;
}

sgr_status sgr_color_partitioned(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t P,
                                 const int64_t* ranges, int32_t* colors_out, sgr_stats* stats,
                                 const sgr_opts* opts) {
  (void)csr; (void)n; (void)nnz; (void)P; (void)ranges; (void)colors_out; (void)stats; (void)opts;
  set_error("sgr_color_partitioned: not built yet");
  return SGR_EUNSUPPORTED;
}

}  // extern "C"
