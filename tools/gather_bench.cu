// gather_bench.cu — microbenchmark: throughput of random 4-byte / 2-byte gathers on sm_100a
// through the different load paths (default, .cg, .nc, .nc.L1::no_allocate, texture).
// Standalone tool (not part of libsgr): nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdlib>
#include <algorithm>
#include <vector>

#define CK(x)                                                                    \
  do {                                                                           \
    cudaError_t e = (x);                                                         \
    if (e != cudaSuccess) {                                                      \
      printf("CUDA %s at %d: %s\n", #x, __LINE__, cudaGetErrorString(e));        \
      exit(1);                                                                   \
    }                                                                            \
  } while (0)

template <int MODE>
__device__ __forceinline__ int ld(const int* p) {
  int r;
  if constexpr (MODE == 0) r = *p;
  else if constexpr (MODE == 1) r = __ldcg(p);
  else if constexpr (MODE == 2) r = __ldg(p);
  else asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}

template <int MODE, int U>
__global__ void k_gather(const int* __restrict__ idx, long long m, const int* __restrict__ x,
                         unsigned long long* out) {
  unsigned long long acc = 0;
  const long long stride = (long long)gridDim.x * blockDim.x * U;
  for (long long j = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; j < m; j += stride) {
    int w[U];
#pragma unroll
    for (int u = 0; u < U; ++u) w[u] = (j + u * blockDim.x < m) ? __ldg(idx + j + u * blockDim.x) : 0;
#pragma unroll
    for (int u = 0; u < U; ++u) acc += ld<MODE>(x + w[u]);
  }
  if (acc == 0x1234567) *out = acc;
}

template <int U>
__global__ void k_gather_tex(const int* __restrict__ idx, long long m, cudaTextureObject_t t,
                             unsigned long long* out) {
  unsigned long long acc = 0;
  const long long stride = (long long)gridDim.x * blockDim.x * U;
  for (long long j = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; j < m; j += stride) {
    int w[U];
#pragma unroll
    for (int u = 0; u < U; ++u) w[u] = (j + u * blockDim.x < m) ? __ldg(idx + j + u * blockDim.x) : 0;
#pragma unroll
    for (int u = 0; u < U; ++u) acc += tex1Dfetch<int>(t, w[u]);
  }
  if (acc == 0x1234567) *out = acc;
}

template <int U>
__global__ void k_gather16(const int* __restrict__ idx, long long m, const unsigned short* __restrict__ x,
                           unsigned long long* out) {
  unsigned long long acc = 0;
  const long long stride = (long long)gridDim.x * blockDim.x * U;
  for (long long j = (long long)blockIdx.x * blockDim.x * U + threadIdx.x; j < m; j += stride) {
    int w[U];
#pragma unroll
    for (int u = 0; u < U; ++u) w[u] = (j + u * blockDim.x < m) ? __ldg(idx + j + u * blockDim.x) : 0;
#pragma unroll
    for (int u = 0; u < U; ++u) acc += __ldg(x + w[u]);
  }
  if (acc == 0x1234567) *out = acc;
}

// Streaming read (baseline for the index stream alone).
__global__ void k_stream(const int* __restrict__ idx, long long m, unsigned long long* out) {
  unsigned long long acc = 0;
  for (long long j = (long long)blockIdx.x * blockDim.x + threadIdx.x; j < m;
       j += (long long)gridDim.x * blockDim.x)
    acc += __ldg(idx + j);
  if (acc == 0x1234567) *out = acc;
}

int main(int argc, char** argv) {
  const long long n = argc > 1 ? atoll(argv[1]) : (1 << 24);     // color array length
  const long long m = argc > 2 ? atoll(argv[2]) : (256ll << 20);  // gathers
  const int locality = argc > 3 ? atoi(argv[3]) : 0;  // 0 random, k>0: sorted runs of 32 within windows of k
  int dev = 0, sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  std::vector<int> h(m);
  unsigned long long s = 88172645463325252ull;
  for (long long i = 0; i < m; ++i) {
    s ^= s << 13; s ^= s >> 7; s ^= s << 17;
    h[i] = (int)(s % (unsigned long long)n);
  }
  if (locality > 0) {  // groups of 32 consecutive entries drawn sorted from a window of `locality`
    for (long long i = 0; i + 32 <= m; i += 32) {
      long long base = h[i] % (n - locality > 0 ? n - locality : 1);
      std::vector<int> g(32);
      for (int k = 0; k < 32; ++k) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; g[k] = (int)(base + s % locality); }
      std::sort(g.begin(), g.end());
      for (int k = 0; k < 32; ++k) h[i + k] = g[k];
    }
  }
  int *d_idx, *d_x;
  unsigned short* d_x16;
  unsigned long long* d_out;
  CK(cudaMalloc(&d_idx, m * 4));
  CK(cudaMalloc(&d_x, n * 4));
  CK(cudaMalloc(&d_x16, n * 2));
  CK(cudaMalloc(&d_out, 8));
  CK(cudaMemcpy(d_idx, h.data(), m * 4, cudaMemcpyHostToDevice));
  CK(cudaMemset(d_x, 1, n * 4));
  CK(cudaMemset(d_x16, 1, n * 2));
  cudaTextureObject_t tex = 0;
  {
    cudaResourceDesc rd = {};
    rd.resType = cudaResourceTypeLinear;
    rd.res.linear.devPtr = d_x;
    rd.res.linear.desc = cudaCreateChannelDesc<int>();
    rd.res.linear.sizeInBytes = n * 4;
    cudaTextureDesc td = {};
    td.readMode = cudaReadModeElementType;
    if (cudaCreateTextureObject(&tex, &rd, &td, nullptr) != cudaSuccess) tex = 0;
  }
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto timeit = [&](const char* name, auto launch) {
    launch();
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0);
    for (int r = 0; r < 5; ++r) launch();
    cudaEventRecord(e1);
    CK(cudaEventSynchronize(e1));
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    ms /= 5;
    printf("%-34s %8.3f ms  %7.1f G gathers/s  (%.2f per SM-cycle @1.9GHz)\n", name, ms,
           m / ms / 1e6, m / (ms * 1e-3) / sms / 1.9e9);
  };
  const int bps = argc > 4 ? atoi(argv[4]) : 8;  // blocks of 256 threads per SM
  const int grid = sms * bps, blk = 256;
  printf("n=%lld m=%lld locality=%d sms=%d blocks/SM=%d\n", n, m, locality, sms, bps);
  timeit("stream idx only", [&] { k_stream<<<grid, blk>>>(d_idx, m, d_out); });
  timeit("default ld (U=8)", [&] { k_gather<0, 8><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ld.cg (U=8)", [&] { k_gather<1, 8><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ld.nc/ldg (U=8)", [&] { k_gather<2, 8><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ld.nc.L1::no_allocate (U=8)", [&] { k_gather<3, 8><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ldg (U=2)", [&] { k_gather<2, 2><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ldg (U=16)", [&] { k_gather<2, 16><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ldg (U=32)", [&] { k_gather<2, 32><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  timeit("ld.cg (U=16)", [&] { k_gather<1, 16><<<grid, blk>>>(d_idx, m, d_x, d_out); });
  if (tex) timeit("tex1Dfetch (U=8)", [&] { k_gather_tex<8><<<grid, blk>>>(d_idx, m, tex, d_out); });
  timeit("u16 ldg (U=8)", [&] { k_gather16<8><<<grid, blk>>>(d_idx, m, d_x16, d_out); });
  return 0;
}
