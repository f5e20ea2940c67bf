// sgr.cu — host side of libsgr.so: the C ABI of include/sgr.h (single GPU + step entry
// points). Multi-GPU lives in sgr_dist.cu. DESIGN.md §5 describes the round loop.
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <vector>

#include "sgr.h"
#include "sgr_internal.h"
#include "sgr_host.cuh"
#include "sgr_round.cuh"
#include "sgr_step.cuh"
#include "sgr_topo.cuh"
#include "sgr_gs.cuh"

namespace sgr {

static thread_local char g_err[512] = "";

void set_error(const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
}

sgr_status cuda_fail(cudaError_t e, const char* what, int line) {
  set_error("%s (line %d): %s", what, line, cudaGetErrorString(e));
  return SGR_ECUDA;
}

// Keep freed stream-ordered allocations in the device's default pool (the default release
// threshold of 0 hands GB-sized workspaces back to the driver at every synchronize, and
// the next call pays for fresh allocations).
void keep_pool_memory() {
  static bool done[64] = {false};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64 || done[dev]) return;
  cudaMemPool_t pool;
  if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  }
  done[dev] = true;
}

int num_sms() {
  static int sms[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 148;
  if (sms[dev] == 0) {
    int v = 0;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0)
      v = 148;
    sms[dev] = v;
  }
  return sms[dev];
}

Resolved resolve_opts(const sgr_opts* o, int64_t n) {
  Resolved r;
  sgr_opts d;
  sgr_opts_default(&d);
  if (!o) o = &d;
  r.tiebreak = o->tiebreak == SGR_TIEBREAK_PAPER ? 1 : 0;
  r.max_rounds = o->max_rounds > 0 ? o->max_rounds : (int32_t)std::min<int64_t>(n + 1, INT32_MAX);
  r.loop_mode = (o->loop_mode == SGR_LOOP_HOST || o->loop_mode == SGR_LOOP_GRAPH)
                    ? o->loop_mode : SGR_LOOP_PERSISTENT;
  r.color_bits = o->color_bits == 32 ? 32 : 16;
  r.small_max = o->bin_small_max > 0 ? std::min(o->bin_small_max, kMaxSmall) : kMaxSmall;
  // default med_max: 256, or 128 on graphs of <= 2^20 vertices, where the shorter rows
  // trimmed as bin-2 lists pay (profiles/r02_ncu_summary.md: R-MAT s16 -6.6 %, rmat-g s20
  // -2.5 %; R-MAT s24 +0.2 % with 128, so large graphs keep 256)
  r.med_max = o->bin_med_max > 0 ? std::min(o->bin_med_max, kMaxMed)
                                 : (n <= (int64_t(1) << 20) ? 128 : kMaxMed);
  r.med_max = std::max(r.med_max, r.small_max);
  r.stream = (cudaStream_t)o->stream;
  r.round_sizes = o->round_sizes;
  r.round_edges = o->round_edges;
  r.round_ns = o->round_ns;
  r.round_cap = (o->round_sizes || o->round_edges || o->round_ns) ? o->round_cap : 0;
  r.validate = o->validate;
  r.batch = o->rounds_per_batch > 0 ? o->rounds_per_batch : 8;
  r.profile = o->profile;
  r.round_ms = o->round_ms;
  r.color_cap = (o->color_cap > 0 && o->color_cap < (int32_t)kColorMask) ? o->color_cap
                                                                         : (int32_t)kColorMask;
  r.block = o->block_size > 0 ? o->block_size : kBlock;
  r.sorted = o->unsorted_rows ? 0 : 1;
  r.flat_bin0 = (o->flat_bin0 >= 0 && o->flat_bin0 <= 2) ? o->flat_bin0 : 0;
  return r;
}

// Bytes of the L2 persisting carve-out for the color buffers (0: off). Experiment switch
// SGR_L2PERSIST=1, read once per process; sets the device's persisting-L2 limit once.
static size_t l2_persist_bytes() {
  static size_t bytes = [] {
    const char* e = getenv("SGR_L2PERSIST");
    if (!(e && e[0] == '1')) return (size_t)0;
    int dev = 0, mx = 0, win = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&mx, cudaDevAttrMaxPersistingL2CacheSize, dev);
    cudaDeviceGetAttribute(&win, cudaDevAttrMaxAccessPolicyWindowSize, dev);
    if (mx <= 0 || win <= 0) return (size_t)0;
    cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, (size_t)mx);
    return (size_t)std::min(mx, win);
  }();
  return bytes;
}

// opts->block_size: a multiple of 32 within [lo, hi] (sgr.h).
bool block_ok(int B, int lo, int hi) { return B % 32 == 0 && B >= lo && B <= hi; }

// Pinned host slots for termination flags (reused across calls on this thread).
static int32_t* pinned_flags() {
  static thread_local int32_t* p = nullptr;
  if (!p && cudaMallocHost(&p, 64 * sizeof(int32_t)) != cudaSuccess) p = nullptr;
  return p;
}

size_t ws_bytes(int64_t n, int64_t nnz, const Resolved& r) { return layout(n, nnz, r).total; }

// ----- CUDA-graph cache: one graph = `batch` round passes -----------------------------------
struct GraphKey {
  unsigned char args[sizeof(RoundArgs<int32_t>)];
  int tiebreak, bits, batch, dev, grid, block;
  bool operator==(const GraphKey& o) const { return memcmp(this, &o, sizeof(GraphKey)) == 0; }
};

static std::mutex g_graph_mu;
static std::vector<std::pair<GraphKey, cudaGraphExec_t>> g_graphs;

template <int TB, class C>
static sgr_status get_graph(const RoundArgs<C>& a, int grid, int B, int batch, cudaGraphExec_t* out) {
  GraphKey key;
  memset(&key, 0, sizeof(key));
  static_assert(sizeof(RoundArgs<C>) <= sizeof(key.args), "graph key");
  memcpy(key.args, &a, sizeof(a));
  key.tiebreak = TB;
  key.bits = packed<C>() ? 16 : 32;
  key.batch = batch;
  key.grid = grid;
  key.block = B;
  cudaGetDevice(&key.dev);
  std::lock_guard<std::mutex> lk(g_graph_mu);
  for (auto& e : g_graphs)
    if (e.first == key) {
      *out = e.second;
      return SGR_OK;
    }
  cudaStream_t cs;
  cudaError_t err = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
  if (err != cudaSuccess) return cuda_fail(err, "cudaStreamCreate", __LINE__);
  err = cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal);
  if (err != cudaSuccess) {
    cudaStreamDestroy(cs);
    return cuda_fail(err, "cudaStreamBeginCapture", __LINE__);
  }
  for (int b = 0; b < batch; ++b) {
    k_round<TB, C><<<grid, B, round_smem<C>(B), cs>>>(a);
    if constexpr (packed<C>()) k_finalize<TB, C><<<grid, kBlock, 0, cs>>>(a);
    k_advance<<<1, 32, 0, cs>>>(a.ctrl, 0);
  }
  cudaGraph_t graph;
  err = cudaStreamEndCapture(cs, &graph);
  cudaStreamDestroy(cs);
  if (err != cudaSuccess) return cuda_fail(err, "cudaStreamEndCapture", __LINE__);
  cudaGraphExec_t exec;
  err = cudaGraphInstantiate(&exec, graph, 0);
  cudaGraphDestroy(graph);
  if (err != cudaSuccess) return cuda_fail(err, "cudaGraphInstantiate", __LINE__);
  if (g_graphs.size() >= 8) {
    cudaGraphExecDestroy(g_graphs.front().second);
    g_graphs.erase(g_graphs.begin());
  }
  g_graphs.push_back({key, exec});
  *out = exec;
  return SGR_OK;
}

// NVTX range for the scope (balanced on every exit path).
struct NvtxRange {
  bool open = true;
  explicit NvtxRange(const char* m) { nvtxRangePushA(m); }
  void end() {
    if (open) nvtxRangePop();
    open = false;
  }
  ~NvtxRange() { end(); }
};

// ----- profiling (opts->profile): CUDA events around launches ------------------------------
struct Prof {
  bool on = false;
  std::vector<cudaEvent_t> pool;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> marks;
  size_t used = 0;
  cudaEvent_t get() {
    if (used == pool.size()) {
      cudaEvent_t e;
      cudaEventCreate(&e);
      pool.push_back(e);
    }
    return pool[used++];
  }
  template <class F>
  void timed(int cls, cudaStream_t s, F&& fn) {
    if (!on) {
      fn();
      return;
    }
    cudaEvent_t e0 = get(), e1 = get();
    cudaEventRecord(e0, s);
    fn();
    cudaEventRecord(e1, s);
    marks.push_back({cls, {e0, e1}});
  }
  void reset() {
    used = 0;
    marks.clear();
  }
  ~Prof() {
    for (auto e : pool) cudaEventDestroy(e);
  }
};

// Byte model and counters from the final Ctrl.
void fill_stats(const Ctrl& c, int64_t n, int64_t nnz, sgr_stats* st, int cb) {
  int64_t vpass = 0, epass = 0, b_round = 0;
  for (int q = 0; q < kBins; ++q) {
    vpass += (int64_t)c.verts_total[q];
    epass += (int64_t)c.edges_total[q];
    st->bin_vertices[q] = (int64_t)c.verts_total[q];
    st->bin_edges[q] = (int64_t)c.edges_total[q];
    // per worklist vertex: 4 B id + 16 B row pair + X[v] + Y[v] words; per adjacency entry
    // actually read: 4 B list entry + an X[w] word (cb = 2 packed, 4 plain); 4 B per vertex
    // pushed to W_{k+1}; 4 B per compacted list entry written (below)
    b_round += (20 + 2 * cb) * (int64_t)c.verts_total[q] + (4 + cb) * (int64_t)c.entries_total[q] +
               4 * (int64_t)c.pushes_total[q];
    st->entries_read += (int64_t)c.entries_total[q];
  }
  st->chunk_items = (int64_t)c.items_total;
  st->entries_written = (int64_t)c.list_writes_total;
  b_round += 4 * (int64_t)c.list_writes_total;
  for (int q = 0; q < kBins; ++q) st->bin_warp_cycles[q] = (int64_t)c.bin_cycles[q];
#if SGR_PHASE_CYCLES
  if (getenv("SGR_PHASES")) {  // experiments: bin-2 phase breakdown
    fprintf(stderr, "sgr phases (warp-cycles): issue %llu wait %llu gather %llu post %llu | barrier %llu finalize %llu counters %llu\n",
            c.phase_cycles[0], c.phase_cycles[1], c.phase_cycles[2], c.phase_cycles[3],
            c.phase_cycles[4], c.phase_cycles[5], c.phase_cycles[6]);
  }
#endif
  st->rounds = c.k - 1;
  st->num_colors = c.max_color;
  st->vertices_processed = n + vpass;
  st->edges_scanned = nnz + epass;
  // F_1 per vertex: 8 B row offset + 4 B first/last entry + two color-word writes; 4 B/push.
  // Final: packed, read a word + write int32 (max fused); plain, the max-color read.
  const int64_t b_first = (12 + 2 * cb) * n + 4 * (int64_t)c.pushes_total[kBins];
  const int64_t b_final = (cb == 2 ? 6 : 4) * n;
  st->bytes_algorithmic = b_first + b_round + b_final;
  st->kernel_bytes[SGR_K_FIRST] = b_first;
  st->kernel_bytes[SGR_K_ROUND] = b_round;
  st->kernel_bytes[SGR_K_CTRL] = 0;
  st->kernel_bytes[SGR_K_FINAL] = b_final;
}

// One complete coloring with working color type C. *overflow_out = 1 if a u16 first fit
// exceeded 65535 (the caller then reruns with 32-bit colors).
template <int TB, class C>
static sgr_status run_color(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                            sgr_stats* stats, const Resolved& r, void* ws, const Layout& L,
                            int* overflow_out) {
  cudaStream_t s = r.stream;
  RoundArgs<C> a;
  build_args<C>(a, csr, n, nnz, colors_out, ws, L, r);
  if (r.loop_mode == SGR_LOOP_PERSISTENT) set_bitmaps<C>(a, ws, L, n);  // dense flat passes
  Prof prof;
  prof.on = r.profile != 0;
  int32_t launches = 0;
  const bool persistent = r.loop_mode == SGR_LOOP_PERSISTENT;
  const int B = r.block;
  // the block size must suit the build the coloring runs (hub: <= 512 threads when packed);
  // the persistent path enqueues both builds, so both must accept it
  if (!block_ok(B, 64, round_max_block<C, true>()) ||
      (persistent && !block_ok(B, 64, round_max_block<C, false>()))) {
    set_error("sgr_color: block_size %d not supported by the round kernels (64..%d, multiple of 32)",
              B, round_max_block<C, true>());
    return SGR_EINVAL;
  }
  const int grid = round_grid<TB, C>(persistent, B);
  const int grid_flat = persistent ? round_grid<TB, C, false>(true, B) : grid;
  const int grid_flat_t0 = persistent ? round_grid<TB, C, false, true>(true, B) : grid;
  const int grid_dense = persistent && a.bm[0] ? dense_grid<TB, C>(B) : 0;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  sgr_status status = SGR_OK;
  do {
    Ctrl hc;
    memset(&hc, 0, sizeof(hc));
    hc.k = 1;
    hc.max_rounds = r.max_rounds;
    hc.round_cap = r.round_cap;
    hc.round_sizes = r.round_sizes;
    hc.round_edges = r.round_edges;
    hc.round_ns = r.round_ns;
    cudaError_t le = cudaMemcpyAsync(a.ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s);
    if (le == cudaSuccess)
      le = cudaMemsetAsync((char*)ws + L.zero_begin, 0, L.zero_end - L.zero_begin, s);
    if (le != cudaSuccess) {
      status = cuda_fail(le, "workspace init", __LINE__);
      break;
    }
    if (r.round_cap > 0) {  // round 1: |W_1| = n, sum of degrees = nnz
      int32_t n32 = (int32_t)n;
      int64_t nz = nnz;
      if (r.round_sizes) cudaMemcpyAsync(r.round_sizes, &n32, 4, cudaMemcpyHostToDevice, s);
      if (r.round_edges) cudaMemcpyAsync(r.round_edges, &nz, 8, cudaMemcpyHostToDevice, s);
    }
    cudaEventCreate(&ev0);
    cudaEventCreate(&ev1);
    cudaEventRecord(ev0, s);

    // NVTX ranges (SURVEY §5 tracing): host-side enqueue phases, visible to ncu
    // (--nvtx --nvtx-include) and nsys; one range per round batch in the host/graph loops
    {
      NvtxRange nr("sgr F1");
      prof.timed(SGR_K_FIRST, s, [&] { k_first<TB, C><<<first_grid(n, B), B, 0, s>>>(a, r.sorted); });
      prof.timed(SGR_K_CTRL, s, [&] { k_advance<<<1, 32, 0, s>>>(a.ctrl, 1); });
    }
    launches += 2;
    le = cudaGetLastError();
    if (le != cudaSuccess) {
      status = cuda_fail(le, "launch F_1", __LINE__);
      break;
    }

    NvtxRange nr_rounds(persistent ? "sgr rounds (persistent)" : "sgr rounds (host loop)");
    if (persistent) {
      // both builds are enqueued; the one that does not match F_1's bins returns at once
      prof.timed(SGR_K_ROUND, s, [&] {
        // cooperative launches; optionally with an L2 persisting window over the two color
        // buffers (SGR_L2PERSIST=1, experiment: the gathers' working set kept resident
        // against the streaming lists)
        cudaLaunchAttribute at[2];
        at[0].id = cudaLaunchAttributeCooperative;
        at[0].val.cooperative = 1;
        int nat = 1;
        // packed: both color buffers are adjacent in the workspace; plain: the workspace one
        const size_t colb = packed<C>() ? 2 * align_up((size_t)n * sizeof(C), 256) : (size_t)n * 4;
        if (l2_persist_bytes() > 0) {
          at[1].id = cudaLaunchAttributeAccessPolicyWindow;
          at[1].val.accessPolicyWindow.base_ptr = (void*)a.col[packed<C>() ? 0 : 1];
          at[1].val.accessPolicyWindow.num_bytes = std::min(colb, l2_persist_bytes());
          at[1].val.accessPolicyWindow.hitRatio = 1.0f;
          at[1].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
          at[1].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
          nat = 2;
        }
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(B);
        cfg.dynamicSmemBytes = round_smem<C, true>(B);
        cfg.stream = s;
        cfg.attrs = at;
        cfg.numAttrs = nat;
        le = cudaLaunchKernelEx(&cfg, k_persistent<TB, C, true>, a);
        if (le == cudaSuccess && grid_dense > 0) {  // dense passes (flat build, meshes)
          cfg.gridDim = dim3(grid_dense);
          cfg.dynamicSmemBytes = round_smem<C, false>(B);
          le = cudaLaunchKernelEx(&cfg, k_dense<TB, C>, a);
          if (le == cudaSuccess)  // k_persistent's grid barrier starts from zero again
            le = cudaMemsetAsync(&a.ctrl->bar_count, 0, sizeof(uint32_t), s);
        }
        if (le == cudaSuccess) {
          cfg.gridDim = dim3(grid_flat);
          cfg.dynamicSmemBytes = round_smem<C, false>(B);
          le = cudaLaunchKernelEx(&cfg, k_persistent<TB, C, false>, a);
        }
        if (le == cudaSuccess) {  // flat build, thread-per-vertex bin 0 (flat_thread_bin0)
          cfg.gridDim = dim3(grid_flat_t0);
          le = cudaLaunchKernelEx(&cfg, k_persistent<TB, C, false, true>, a);
        }
      });
      launches += grid_dense > 0 ? 4 : 3;
      if (le != cudaSuccess) {
        status = cuda_fail(le, "cooperative launch of k_persistent", __LINE__);
        break;
      }
    } else {
      int32_t* flags = pinned_flags();
      if (!flags) {
        status = cuda_fail(cudaErrorMemoryAllocation, "cudaMallocHost", __LINE__);
        break;
      }
      cudaEvent_t done_ev[2];
      cudaEventCreateWithFlags(&done_ev[0], cudaEventDisableTiming);
      cudaEventCreateWithFlags(&done_ev[1], cudaEventDisableTiming);
      const bool use_graph = r.loop_mode == SGR_LOOP_GRAPH && !prof.on;
      cudaGraphExec_t gexec = nullptr;
      if (use_graph) status = get_graph<TB, C>(a, grid, B, r.batch, &gexec);
      // Pipelined termination test: batch b's `active` flag is read after batch b+1 is
      // enqueued, so the GPU never waits for the host; surplus passes are no-ops.
      int64_t batches = 0;
      bool finished = status != SGR_OK;
      while (!finished) {
        NvtxRange nr_batch("sgr round batch");
        if (use_graph) {
          le = cudaGraphLaunch(gexec, s);
        } else {
          for (int b = 0; b < r.batch; ++b) {
            prof.timed(SGR_K_ROUND, s, [&] {
              k_round<TB, C><<<grid, B, round_smem<C>(B), s>>>(a);
              if constexpr (packed<C>()) k_finalize<TB, C><<<grid, kBlock, 0, s>>>(a);
            });
            prof.timed(SGR_K_CTRL, s, [&] { k_advance<<<1, 32, 0, s>>>(a.ctrl, 0); });
          }
          le = cudaGetLastError();
        }
        launches += 2 * r.batch;
        if (le != cudaSuccess) {
          status = cuda_fail(le, "launch round batch", __LINE__);
          break;
        }
        const int slot = (int)(batches & 1);
        cudaMemcpyAsync(&flags[slot], &a.ctrl->active, 4, cudaMemcpyDeviceToHost, s);
        cudaEventRecord(done_ev[slot], s);
        if (batches > 0) {
          cudaEventSynchronize(done_ev[slot ^ 1]);
          if (flags[slot ^ 1] == 0) finished = true;
        }
        ++batches;
      }
      cudaEventDestroy(done_ev[0]);
      cudaEventDestroy(done_ev[1]);
      if (status != SGR_OK) break;
    }

    nr_rounds.end();
    prof.timed(SGR_K_FINAL, s, [&] {
      if constexpr (packed<C>())
        k_unpack<<<reduce_grid(n, B), B, 0, s>>>(a.col[0], colors_out, n, &a.ctrl->max_color);
      else
        k_max_color<<<reduce_grid(n, B), B, 0, s>>>(colors_out, n, &a.ctrl->max_color);
    });
    launches += 1;
    cudaEventRecord(ev1, s);
    Ctrl fin;
    cudaMemcpyAsync(&fin, a.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s);
    le = cudaStreamSynchronize(s);
    if (le != cudaSuccess) {
      status = cuda_fail(le, "sgr_color", __LINE__);
      break;
    }
    *overflow_out = fin.overflow;
    if (stats) {
      fill_stats(fin, n, nnz, stats, (int)sizeof(C));
      cudaEventElapsedTime(&stats->elapsed_ms, ev0, ev1);
      stats->launches = launches;
      stats->grid_blocks = fin.big_count ? grid : grid_flat;
      stats->color_bits = packed<C>() ? 16 : 32;
      int32_t ri = 0;
      for (auto& m : prof.marks) {
        float ms = 0.f;
        cudaEventElapsedTime(&ms, m.second.first, m.second.second);
        stats->kernel_ms[m.first] += ms;
        stats->kernel_launches[m.first] += 1;
        if (m.first == SGR_K_ROUND && r.round_ms && ri < r.round_cap) r.round_ms[ri++] = ms;
      }
    }
    if (fin.status == 1 && !fin.overflow) {
      set_error("sgr_color: max_rounds (%d) reached", r.max_rounds);
      status = SGR_ENOCONV;
    }
  } while (0);
  if (ev0) cudaEventDestroy(ev0);
  if (ev1) cudaEventDestroy(ev1);
  return status;
}

template <int TB>
static sgr_status run_any(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                          sgr_stats* stats, const Resolved& r, void* ws, const Layout& L) {
  int overflow = 0;
  if (r.color_bits == 16) {
    const sgr_status st = run_color<TB, Packed>(csr, n, nnz, colors_out, stats, r, ws, L, &overflow);
    if (st != SGR_OK || !overflow) return st;
    // a color exceeded 12 bits (4095): the packed run is discarded and redone
    // with plain 32-bit colors (no trimming)
  }
  Resolved r32 = r;
  r32.color_bits = 32;
  const Layout L32 = layout(n, nnz, r32);
  const sgr_status st = run_color<TB, int32_t>(csr, n, nnz, colors_out, stats, r32, ws, L32, &overflow);
  if (st == SGR_OK && overflow) {
    set_error("sgr_color: 32-bit color overflow");
    return SGR_EUNSUPPORTED;
  }
  return st;
}

#define CK(call)                                                  \
  do {                                                            \
    cudaError_t e_ = (call);                                      \
    if (e_ != cudaSuccess) return cuda_fail(e_, #call, __LINE__); \
  } while (0)

// K sub-steps per round in one cooperative launch (gsp::k_gs_persistent, a grid barrier per
// sub-step); partitions 0 (strided) and 1 (blocked).
template <int TB>
static sgr_status color_gs_persistent(const sgr_csr* csr, int64_t n, int64_t nnz, int64_t K,
                                      int32_t partition, int32_t* colors_out, sgr_stats* stats,
                                      const Resolved& r) {
  cudaStream_t s = r.stream;
  const size_t nb = align_up((size_t)n * 4, 256);
  const size_t kb = align_up((size_t)(K + 1) * 4, 256);
  const size_t cb2 = align_up((size_t)4 * K * 4, 256);
  char* ws = nullptr;
  CK(cudaMallocAsync((void**)&ws, 3 * nb + cb2 + 2 * kb + 256, s));
  gsp::Args a;
  memset(&a, 0, sizeof(a));
  a.row_ptr = csr->row_ptr;
  a.col_idx = csr->col_idx;
  a.C[0] = colors_out;
  a.C[1] = (int32_t*)ws;
  a.L[0] = (int32_t*)(ws + nb);
  a.L[1] = (int32_t*)(ws + 2 * nb);
  a.cnt = (int32_t*)(ws + 3 * nb);
  int32_t* poff = (int32_t*)(ws + 3 * nb + cb2);
  int32_t* pcur = (int32_t*)(ws + 3 * nb + cb2 + kb);
  a.poff = poff;
  a.ctrl = (gsp::Ctrl*)(ws + 3 * nb + cb2 + 2 * kb);
  a.n = n;
  a.K = K;
  a.partition = partition;
  a.max_rounds = r.max_rounds;
  a.round_sizes = r.round_sizes;
  a.round_edges = r.round_edges;
  a.round_cap = r.round_cap;
  a.tiebreak = TB;
  CK(cudaMemsetAsync(a.C[0], 0, (size_t)n * 4, s));  // 0 = not yet colored
  CK(cudaMemsetAsync(a.C[1], 0, (size_t)n * 4, s));
  CK(cudaMemsetAsync(a.cnt, 0, cb2, s));
  CK(cudaMemsetAsync(a.ctrl, 0, sizeof(gsp::Ctrl), s));
  // list regions: part j's members, counted and scanned
  int32_t* hist = a.cnt;  // scratch for the histogram (re-zeroed below)
  gsp::k_part_hist<<<std::max(1, (int)std::min<int64_t>((n + 255) / 256, num_sms() * 8)), 256, 0, s>>>(
      n, K, partition, hist);
  k_gs_scan<<<1, 32, 0, s>>>(hist, K, poff, pcur);
  CK(cudaMemsetAsync(a.cnt, 0, cb2, s));
  int per_sm = 0;
  const void* fn = (const void*)gsp::k_gs_persistent<TB>;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gsp::k_gs_persistent<TB>, 256, 0) != cudaSuccess ||
      per_sm <= 0)
    per_sm = 1;
  const int grid = per_sm * num_sms();
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventRecord(e0, s));
  void* args[] = {(void*)&a};
  cudaError_t le = cudaLaunchCooperativeKernel(fn, grid, 256, args, 0, s);
  if (le != cudaSuccess) {
    cudaFreeAsync(ws, s);
    return cuda_fail(le, "cooperative launch of k_gs_persistent", __LINE__);
  }
  CK(cudaEventRecord(e1, s));
  gsp::Ctrl fin;
  CK(cudaMemcpyAsync(&fin, a.ctrl, sizeof(fin), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  if (fin.final_buf == 1)
    CK(cudaMemcpyAsync(colors_out, a.C[1], (size_t)n * 4, cudaMemcpyDeviceToDevice, s));
  int32_t* dmax = (int32_t*)(ws + 3 * nb);  // reuse the counters
  CK(cudaMemsetAsync(dmax, 0, 4, s));
  k_max_color<<<reduce_grid(n), 256, 0, s>>>(colors_out, n, dmax);
  int32_t mx = 0;
  CK(cudaMemcpyAsync(&mx, dmax, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  sgr_status status = SGR_OK;
  if (fin.status == 1) {
    set_error("sgr_color_gs: max_rounds (%d) reached", r.max_rounds);
    status = SGR_ENOCONV;
  }
  if (stats) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    stats->rounds = fin.rounds;
    stats->num_colors = mx;
    stats->vertices_processed = (int64_t)fin.verts_total;
    stats->edges_scanned = (int64_t)fin.edges_total;
    stats->entries_read = (int64_t)fin.edges_total;
    stats->elapsed_ms = ms;
    stats->launches = 4;
    stats->color_bits = 32;
    stats->grid_blocks = grid;
    // per round: detection re-reads W's rows (id + color per entry), the first fits read
    // them again; per member its id (list), row pair, two color words; the copies
    stats->bytes_algorithmic = (int64_t)fin.edges_total * 16 + (int64_t)fin.verts_total * 40;
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFreeAsync(ws, s);
  cudaStreamSynchronize(s);
  return status;
}
}  // namespace sgr

using namespace sgr;


extern "C" {

void sgr_opts_default(sgr_opts* o) {
  if (!o) return;
  memset(o, 0, sizeof(*o));
  o->tiebreak = SGR_TIEBREAK_LOWID_KEEPS;
  o->loop_mode = SGR_LOOP_AUTO;
}

size_t sgr_workspace_bytes(int64_t n, int64_t nnz, const sgr_opts* opts) {
  if (n <= 0) return 0;
  return ws_bytes(n, nnz, resolve_opts(opts, n));
}

const char* sgr_strerror(sgr_status s) {
  switch (s) {
    case SGR_OK: return "ok";
    case SGR_EINVAL: return "invalid argument";
    case SGR_ENOMEM: return "out of memory";
    case SGR_ECUDA: return "CUDA error";
    case SGR_ENCCL: return "NCCL error";
    case SGR_ENOCONV: return "max_rounds reached";
    case SGR_EUNSUPPORTED: return "unsupported";
  }
  return "unknown";
}

const char* sgr_last_error(void) { return g_err; }
const char* sgr_version(void) { return "sgr-b200 0.2 (sm_100a)"; }

static sgr_status run_validate(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* dviol,
                               cudaStream_t s, int32_t* viol_out) {
  CK(cudaMemsetAsync(dviol, 0, sizeof(int32_t), s));
  k_validate<<<num_sms() * 4, 256, 0, s>>>(csr->row_ptr, csr->col_idx, n, nnz, dviol);
  CK(cudaGetLastError());
  int32_t v = 0;
  CK(cudaMemcpyAsync(&v, dviol, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  *viol_out = v;
  return SGR_OK;
}

sgr_status sgr_validate_csr(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* violations,
                            void* stream) {
  if (!csr || !csr->row_ptr || n < 0 || nnz < 0 || !violations || (nnz > 0 && !csr->col_idx))
    return SGR_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  int32_t* d;
  CK(cudaMallocAsync((void**)&d, sizeof(int32_t), s));
  sgr_status st = run_validate(csr, n, nnz, d, s, violations);
  cudaFreeAsync(d, s);
  cudaStreamSynchronize(s);
  return st;
}

sgr_status sgr_color_ex(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                        sgr_stats* stats, const sgr_opts* opts, void* workspace,
                        size_t workspace_bytes) {
  if (!csr || n < 0 || nnz < 0 || n >= ((int64_t)1 << 31)) {
    set_error("sgr_color: invalid sizes or csr");
    return SGR_EINVAL;
  }
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n == 0) return SGR_OK;
  if (!csr->row_ptr || !colors_out || (nnz > 0 && !csr->col_idx)) {
    set_error("sgr_color: null pointer");
    return SGR_EINVAL;
  }
  if (((uintptr_t)csr->col_idx & 15u) != 0) {
    set_error("sgr_color: col_idx must be 16-byte aligned");
    return SGR_EINVAL;
  }
  const Resolved r = resolve_opts(opts, n);
  cudaStream_t s = r.stream;
  keep_pool_memory();
  const Layout L = layout(n, nnz, r);
  void* ws = workspace;
  bool own = false;
  if (!ws || workspace_bytes < L.total) {
    CK(cudaMallocAsync(&ws, L.total, s));
    own = true;
  }
  sgr_status status = SGR_OK;
  if (r.validate) {
    int32_t viol = 0;
    status = run_validate(csr, n, nnz, &((Ctrl*)ws)->violations, s, &viol);
    if (!r.sorted) viol &= ~4;  // any row order is accepted with opts->unsorted_rows
    if (status == SGR_OK && viol) {
      set_error("sgr_color: invalid CSR (violation mask %d)", viol);
      status = SGR_EINVAL;
    }
  }
  if (status == SGR_OK)
    status = r.tiebreak ? run_any<1>(csr, n, nnz, colors_out, stats, r, ws, L)
                        : run_any<0>(csr, n, nnz, colors_out, stats, r, ws, L);
  if (own) {
    cudaFreeAsync(ws, s);
    cudaStreamSynchronize(s);
  }
  return status;
}

sgr_status sgr_color(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                     sgr_stats* stats) {
  return sgr_color_ex(csr, n, nnz, colors_out, stats, nullptr, nullptr, 0);
}

sgr_status sgr_color_host(const int64_t* row_ptr, const int32_t* col_idx, int64_t n,
                          int64_t nnz, int32_t* colors_out, sgr_stats* stats,
                          const sgr_opts* opts) {
  if (n < 0 || nnz < 0 || !row_ptr || (n > 0 && !colors_out) || (nnz > 0 && !col_idx))
    return SGR_EINVAL;
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n == 0) return SGR_OK;
  const Resolved r = resolve_opts(opts, n);
  cudaStream_t s = r.stream;
  keep_pool_memory();
  int64_t* d_rp = nullptr;
  int32_t* d_ci = nullptr;
  int32_t* d_col = nullptr;
  CK(cudaMallocAsync((void**)&d_rp, (size_t)(n + 1) * 8, s));
  CK(cudaMallocAsync((void**)&d_ci, (size_t)std::max<int64_t>(nnz, 1) * 4, s));
  CK(cudaMallocAsync((void**)&d_col, (size_t)n * 4, s));
  CK(cudaMemcpyAsync(d_rp, row_ptr, (size_t)(n + 1) * 8, cudaMemcpyHostToDevice, s));
  if (nnz > 0) CK(cudaMemcpyAsync(d_ci, col_idx, (size_t)nnz * 4, cudaMemcpyHostToDevice, s));
  sgr_csr csr{d_rp, d_ci};
  sgr_status st = sgr_color_ex(&csr, n, nnz, d_col, stats, opts, nullptr, 0);
  if (st == SGR_OK) CK(cudaMemcpyAsync(colors_out, d_col, (size_t)n * 4, cudaMemcpyDeviceToHost, s));
  cudaFreeAsync(d_rp, s);
  cudaFreeAsync(d_ci, s);
  cudaFreeAsync(d_col, s);
  CK(cudaStreamSynchronize(s));
  return st;
}

// Pipelined end to end over a batch of host graphs: graph i+1's upload (stream `up`) and
// graph i-1's download (stream `down`) run on the copy engines while graph i is colored on
// the caller's stream. Two device buffer sets; the input set of graph i+1 was last read
// by coloring i-1, which sgr_color_ex finished (it synchronizes) before the upload is
// issued; the colors set of graph i waits for the download of graph i-2 (event).
sgr_status sgr_color_host_batch(const int64_t* const* row_ptr, const int32_t* const* col_idx,
                                const int64_t* n, const int64_t* nnz, int32_t* const* colors_out,
                                int32_t count, sgr_stats* stats, const sgr_opts* opts) {
  if (count < 0 || (count > 0 && (!row_ptr || !col_idx || !n || !nnz || !colors_out)))
    return SGR_EINVAL;
  int64_t max_n = 0, max_nnz = 1;
  for (int32_t i = 0; i < count; ++i) {
    if (n[i] < 0 || nnz[i] < 0 || n[i] >= ((int64_t)1 << 31) || !row_ptr[i] ||
        (n[i] > 0 && !colors_out[i]) || (nnz[i] > 0 && !col_idx[i])) {
      set_error("sgr_color_host_batch: graph %d: invalid sizes or null pointer", i);
      return SGR_EINVAL;
    }
    max_n = std::max(max_n, n[i]);
    max_nnz = std::max(max_nnz, nnz[i]);
  }
  if (stats) memset(stats, 0, sizeof(sgr_stats) * (size_t)count);
  if (count == 0 || max_n == 0) return SGR_OK;
  const Resolved r = resolve_opts(opts, max_n);
  cudaStream_t s = r.stream, up = nullptr, down = nullptr;
  keep_pool_memory();
  CK(cudaStreamCreateWithFlags(&up, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&down, cudaStreamNonBlocking));
  cudaEvent_t ev_alloc, ev_up[2], ev_down[2];
  CK(cudaEventCreateWithFlags(&ev_alloc, cudaEventDisableTiming));
  for (int b = 0; b < 2; ++b) {
    CK(cudaEventCreateWithFlags(&ev_up[b], cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&ev_down[b], cudaEventDisableTiming));
  }
  int64_t* d_rp[2] = {nullptr, nullptr};
  int32_t* d_ci[2] = {nullptr, nullptr};
  int32_t* d_col[2] = {nullptr, nullptr};
  for (int b = 0; b < 2 && b < count; ++b) {
    CK(cudaMallocAsync((void**)&d_rp[b], (size_t)(max_n + 1) * 8, s));
    CK(cudaMallocAsync((void**)&d_ci[b], (size_t)max_nnz * 4, s));
    CK(cudaMallocAsync((void**)&d_col[b], (size_t)max_n * 4, s));
  }
  CK(cudaEventRecord(ev_alloc, s));
  CK(cudaStreamWaitEvent(up, ev_alloc, 0));
  CK(cudaStreamWaitEvent(down, ev_alloc, 0));
  auto upload = [&](int32_t i) -> sgr_status {
    const int b = i & 1;
    CK(cudaMemcpyAsync(d_rp[b], row_ptr[i], (size_t)(n[i] + 1) * 8, cudaMemcpyHostToDevice, up));
    if (nnz[i] > 0)
      CK(cudaMemcpyAsync(d_ci[b], col_idx[i], (size_t)nnz[i] * 4, cudaMemcpyHostToDevice, up));
    CK(cudaEventRecord(ev_up[b], up));
    return SGR_OK;
  };
  sgr_status st = upload(0);
  for (int32_t i = 0; i < count && st == SGR_OK; ++i) {
    const int b = i & 1;
    if (i + 1 < count && (st = upload(i + 1)) != SGR_OK) break;
    if (n[i] == 0) continue;
    CK(cudaStreamWaitEvent(s, ev_up[b], 0));
    if (i >= 2) CK(cudaStreamWaitEvent(s, ev_down[b], 0));  // graph i-2's colors are out
    sgr_csr csr{d_rp[b], d_ci[b]};
    st = sgr_color_ex(&csr, n[i], nnz[i], d_col[b], stats ? &stats[i] : nullptr, opts, nullptr, 0);
    if (st != SGR_OK) break;
    CK(cudaMemcpyAsync(colors_out[i], d_col[b], (size_t)n[i] * 4, cudaMemcpyDeviceToHost, down));
    CK(cudaEventRecord(ev_down[b], down));
  }
  CK(cudaStreamSynchronize(up));
  CK(cudaStreamSynchronize(down));
  for (int b = 0; b < 2; ++b) {
    if (d_rp[b]) cudaFreeAsync(d_rp[b], s);
    if (d_ci[b]) cudaFreeAsync(d_ci[b], s);
    if (d_col[b]) cudaFreeAsync(d_col[b], s);
  }
  CK(cudaStreamSynchronize(s));
  cudaEventDestroy(ev_alloc);
  for (int b = 0; b < 2; ++b) {
    cudaEventDestroy(ev_up[b]);
    cudaEventDestroy(ev_down[b]);
  }
  cudaStreamDestroy(up);
  cudaStreamDestroy(down);
  return st;
}

// ----- topology-driven mapping (Algorithm 4; sgr_topo.cuh) -------------------
sgr_status sgr_color_topo(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                          sgr_stats* stats, const sgr_opts* opts) {
  if (!csr || n < 0 || nnz < 0 || n >= ((int64_t)1 << 31)) {
    set_error("sgr_color_topo: invalid sizes or csr");
    return SGR_EINVAL;
  }
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n == 0) return SGR_OK;
  if (!csr->row_ptr || !colors_out || (nnz > 0 && !csr->col_idx)) {
    set_error("sgr_color_topo: null pointer");
    return SGR_EINVAL;
  }
  const Resolved r = resolve_opts(opts, n);
  cudaStream_t s = r.stream;
  keep_pool_memory();
  // workspace: flag[n] | T[n] | changed | edges
  const size_t nb = align_up((size_t)n * 4, 256);
  char* ws = nullptr;
  CK(cudaMallocAsync((void**)&ws, 2 * nb + 256, s));
  int32_t* flag = (int32_t*)ws;
  int32_t* buf[2] = {colors_out, (int32_t*)(ws + nb)};
  int32_t* changed = (int32_t*)(ws + 2 * nb);
  unsigned long long* edges = (unsigned long long*)(ws + 2 * nb + 64);
  int32_t* hcnt = nullptr;
  CK(cudaMallocHost((void**)&hcnt, sizeof(int32_t)));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int B = r.block;
  if (!block_ok(B, 32, kMaxBlockAny)) {
    set_error("sgr_color_topo: block_size %d (32..1024, multiple of 32)", B);
    return SGR_EINVAL;
  }
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((n + B - 1) / B, (int64_t)num_sms() * 16 * 256 / B));
  std::vector<int32_t> sizes;
  sgr_status status = SGR_OK;
  int launches = 0;
  CK(cudaMemsetAsync(edges, 0, 8, s));
  CK(cudaEventRecord(e0, s));
  k_topo_init<<<grid, B, 0, s>>>(n, flag, buf[0]);
  ++launches;
  int32_t cnt = (int32_t)n;  // |W_1| = n
  int32_t rr = 1;
  int cur = 0;
  while (cnt > 0) {
    if (rr > r.max_rounds) {
      status = SGR_ENOCONV;
      set_error("sgr_color_topo: max_rounds reached");
      break;
    }
    sizes.push_back(cnt);
    k_topo_assign<<<grid, B, 0, s>>>(csr->row_ptr, csr->col_idx, n, rr, flag, buf[cur],
                                       buf[cur ^ 1], edges);
    CK(cudaMemsetAsync(changed, 0, 4, s));
    if (r.tiebreak)
      k_topo_detect<1><<<grid, B, 0, s>>>(csr->row_ptr, csr->col_idx, n, rr, buf[cur ^ 1], flag, changed);
    else
      k_topo_detect<0><<<grid, B, 0, s>>>(csr->row_ptr, csr->col_idx, n, rr, buf[cur ^ 1], flag, changed);
    launches += 2;
    CK(cudaGetLastError());
    // the host reads `changed` every iteration (Alg. 4 l.22)
    CK(cudaMemcpyAsync(hcnt, changed, 4, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    cnt = *hcnt;
    cur ^= 1;
    ++rr;
  }
  if (cur == 1)
    CK(cudaMemcpyAsync(colors_out, buf[1], (size_t)n * 4, cudaMemcpyDeviceToDevice, s));
  int32_t* dmax = changed;
  CK(cudaMemsetAsync(dmax, 0, 4, s));
  k_max_color<<<grid, B, 0, s>>>(colors_out, n, dmax);
  launches += 1;
  CK(cudaEventRecord(e1, s));
  int32_t mx = 0;
  unsigned long long ed = 0;
  CK(cudaMemcpyAsync(&mx, dmax, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaMemcpyAsync(&ed, edges, 8, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  const int32_t R = (int32_t)sizes.size();
  if (r.round_sizes && r.round_cap > 0)
    CK(cudaMemcpy(r.round_sizes, sizes.data(), (size_t)std::min(R, r.round_cap) * 4,
                  cudaMemcpyHostToDevice));
  if (stats) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    stats->rounds = R;
    stats->num_colors = mx;
    int64_t vp = 0;
    for (int32_t x : sizes) vp += x;
    stats->vertices_processed = vp;
    stats->edges_scanned = (int64_t)ed;
    stats->entries_read = (int64_t)ed;
    stats->elapsed_ms = ms;
    stats->launches = launches;
    stats->color_bits = 32;
    // per iteration: every vertex's flag and X/T word, plus the detection pass over V
    // (row pair, own color, every row entry and its color); the assignment of W_r reads
    // its rows and their colors
    stats->bytes_algorithmic = (int64_t)R * ((int64_t)n * (4 + 4 + 4 + 16 + 4) + nnz * 8) +
                               (int64_t)ed * 8;
    stats->grid_blocks = grid;
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFreeHost(hcnt);
  cudaFreeAsync(ws, s);
  cudaStreamSynchronize(s);
  return status;
}

static int grid_for(int64_t items, int per_block, int B = 256) {
  const int64_t b = (items + per_block - 1) / per_block;
  return (int)std::max<int64_t>(1, std::min<int64_t>(b, (int64_t)num_sms() * 16 * 256 / B));
}

// ----- reduced-round variants (sgr_gs.cuh) --------------------------
sgr_status sgr_color_gs(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t substeps,
                        int32_t partition, int32_t* colors_out, sgr_stats* stats,
                        const sgr_opts* opts) {
  if (!csr || n < 0 || nnz < 0 || n >= ((int64_t)1 << 31) || substeps < 1 || partition < 0 ||
      partition > 2) {
    set_error("sgr_color_gs: invalid sizes, csr, substeps or partition");
    return SGR_EINVAL;
  }
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n == 0) return SGR_OK;
  if (!csr->row_ptr || !colors_out || (nnz > 0 && !csr->col_idx)) {
    set_error("sgr_color_gs: null pointer");
    return SGR_EINVAL;
  }
  const Resolved r = resolve_opts(opts, n);
  const int B = r.block;
  if (!block_ok(B, 32, kMaxBlockAny)) {
    set_error("sgr_color_gs: block_size %d (32..1024, multiple of 32)", B);
    return SGR_EINVAL;
  }
  const int64_t K = partition == 2 ? 1 : substeps;
  cudaStream_t s = r.stream;
  keep_pool_memory();
  const char* hl = getenv("SGR_GS_HOSTLOOP");
  if (partition != 2 && !(hl && hl[0] == '1'))
    return r.tiebreak ? color_gs_persistent<1>(csr, n, nnz, K, partition, colors_out, stats, r)
                      : color_gs_persistent<0>(csr, n, nnz, K, partition, colors_out, stats, r);
  // host-driven rounds (the in-place mode; SGR_GS_HOSTLOOP=1 for the sub-step modes)
  // workspace: W[2] | T | flags | seg | tiles | counters | K counts / offsets / cursors
  const size_t nb = align_up((size_t)n * 4, 256);
  const int64_t tiles = (n + kCompactTile - 1) / kCompactTile;
  const size_t kb = align_up((size_t)(K + 1) * 4, 256);
  char* ws = nullptr;
  CK(cudaMallocAsync((void**)&ws, 6 * nb + align_up((size_t)tiles * 4, 256) + 256 + 4 * kb, s));
  int32_t* W[2] = {(int32_t*)ws, (int32_t*)(ws + nb)};
  int32_t* T = (int32_t*)(ws + 2 * nb);
  uint8_t* flags = (uint8_t*)(ws + 3 * nb);
  int32_t* tile = (int32_t*)(ws + 4 * nb);
  char* tail = ws + 4 * nb + align_up((size_t)tiles * 4, 256);
  int64_t* dcount = (int64_t*)tail;
  unsigned long long* edges = (unsigned long long*)(tail + 64);
  int32_t* seg = (int32_t*)(tail + 256);
  int32_t* kcnt = (int32_t*)(tail + 256 + nb);
  int32_t* koff = (int32_t*)(tail + 256 + nb + kb);
  int32_t* kcur = (int32_t*)(tail + 256 + nb + 2 * kb);
  int32_t* kbig = (int32_t*)(tail + 256 + nb + 3 * kb);  // per sub-step: members of degree > 64
  int32_t* bigl = (int32_t*)(tail + 256 + nb + 4 * kb);
  int64_t* hcnt = nullptr;
  CK(cudaMallocHost((void**)&hcnt, sizeof(int64_t)));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  const int grid_v = (int)std::max<int64_t>(1, std::min<int64_t>((n + B - 1) / B, (int64_t)num_sms() * 16 * 256 / B));
  std::vector<int32_t> sizes;
  std::vector<int64_t> round_edges;
  sgr_status status = SGR_OK;
  int launches = 0;
  unsigned long long edges_prev = 0;
  CK(cudaMemsetAsync(edges, 0, 8, s));
  CK(cudaEventRecord(e0, s));
  k_gs_init<<<grid_v, B, 0, s>>>(n, W[0], colors_out);
  ++launches;
  int64_t len = n;
  int cur = 0;
  int huge = -1;  // in-place mode: any row above SGR_GS_HUGE (unknown yet)
  while (len > 0) {
    if ((int64_t)sizes.size() >= r.max_rounds) {
      status = SGR_ENOCONV;
      set_error("sgr_color_gs: max_rounds reached");
      break;
    }
    sizes.push_back((int32_t)len);
    const int gw = grid_for(len, B / 32, B);
    if (partition == 2) {
      if (huge < 0) {  // once per call: is any row long enough for the block-level pass?
        CK(cudaMemsetAsync(kcnt, 0, 4, s));
        gsp::k_any_huge<<<grid_v, B, 0, s>>>(csr->row_ptr, n, kcnt);
        int32_t h = 0;
        CK(cudaMemcpyAsync(&h, kcnt, 4, cudaMemcpyDeviceToHost, s));
        CK(cudaStreamSynchronize(s));
        huge = h;
        ++launches;
      }
      if (huge)
        gsp::k_gs_inplace<true><<<gw, B, 0, s>>>(csr->row_ptr, csr->col_idx, W[cur], len, colors_out, edges);
      else
        gsp::k_gs_inplace<false><<<gw, B, 0, s>>>(csr->row_ptr, csr->col_idx, W[cur], len, colors_out, edges);
      ++launches;
    } else {
      // the round's members split once into K contiguous sub-step segments
      const int gl = grid_for(len, B, B);
      CK(cudaMemsetAsync(kcnt, 0, (size_t)K * 4, s));
      CK(cudaMemsetAsync(kbig, 0, (size_t)K * 4, s));
      k_gs_hist<<<gl, B, 0, s>>>(W[cur], len, n, K, partition, kcnt);
      k_gs_scan<<<1, 32, 0, s>>>(kcnt, K, koff, kcur);
      k_gs_scatter<<<gl, B, 0, s>>>(W[cur], len, n, K, partition, kcur, seg);
      launches += 3;
      // a sub-step's share is unknown on the host: size for the whole round (blocks past
      // the segment exit at once); the big members get one warp each, at least a wave
      const int gseg = std::max(grid_for(len, B, B), num_sms());
      const int gbig = num_sms() * 8 * 256 / B;
      for (int64_t j = 0; j < K; ++j) {  // sub-steps in order (Alg. 5 l.4-10 split K ways)
        k_gs_assign_seg<<<gseg, B, 0, s>>>(csr->row_ptr, csr->col_idx, seg, koff, j, colors_out, T,
                                           bigl, kbig + j, edges);
        k_gs_assign_big<<<gbig, B, 0, s>>>(csr->row_ptr, csr->col_idx, seg, bigl, kbig + j, colors_out,
                                           T, edges);
        k_gs_commit_seg<<<gseg, B, 0, s>>>(seg, koff, j, T, colors_out);
        launches += 3;
      }
    }
    // Alg. 5 l.12-15 over W_r, then the order-preserving compaction
    if (r.tiebreak)
      k_detect_step<1><<<gw, B, 0, s>>>(csr->row_ptr, csr->col_idx, W[cur], len, colors_out, flags);
    else
      k_detect_step<0><<<gw, B, 0, s>>>(csr->row_ptr, csr->col_idx, W[cur], len, colors_out, flags);
    const int64_t tl = (len + kCompactTile - 1) / kCompactTile;
    k_compact_count<<<(unsigned)tl, 256, 0, s>>>(flags, len, tile);
    k_compact_scan<<<1, 1024, 0, s>>>(tile, tl, dcount);
    k_compact_scatter<<<(unsigned)tl, 256, 0, s>>>(W[cur], flags, len, tile, W[cur ^ 1]);
    launches += 4;
    CK(cudaGetLastError());
    unsigned long long ed = 0;
    CK(cudaMemcpyAsync(hcnt, dcount, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    CK(cudaMemcpyAsync(&ed, edges, 8, cudaMemcpyDeviceToHost, s));
    CK(cudaStreamSynchronize(s));
    round_edges.push_back((int64_t)(ed - edges_prev));
    edges_prev = ed;
    len = *hcnt;
    cur ^= 1;
  }
  int32_t* dmax = (int32_t*)(tail + 128);
  CK(cudaMemsetAsync(dmax, 0, 4, s));
  k_max_color<<<grid_v, B, 0, s>>>(colors_out, n, dmax);
  ++launches;
  CK(cudaEventRecord(e1, s));
  int32_t mx = 0;
  CK(cudaMemcpyAsync(&mx, dmax, 4, cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  const int32_t R = (int32_t)sizes.size();
  if (r.round_cap > 0) {
    const int32_t m = std::min(R, r.round_cap);
    if (r.round_sizes) CK(cudaMemcpy(r.round_sizes, sizes.data(), (size_t)m * 4, cudaMemcpyHostToDevice));
    if (r.round_edges) CK(cudaMemcpy(r.round_edges, round_edges.data(), (size_t)m * 8, cudaMemcpyHostToDevice));
  }
  if (stats) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    stats->rounds = R;
    stats->num_colors = mx;
    int64_t vp = 0;
    for (int32_t x : sizes) vp += x;
    stats->vertices_processed = vp;
    stats->edges_scanned = (int64_t)edges_prev;
    stats->entries_read = (int64_t)edges_prev;
    stats->elapsed_ms = ms;
    stats->launches = launches;
    stats->color_bits = 32;
    stats->grid_blocks = grid_v;
    // per worklist vertex and sub-step: the id; per member: row pair, the first-fit scan of
    // its row (id + color per entry), T write + commit; detection re-reads the row
    stats->bytes_algorithmic = vp * (4 * K + 16 + 12) + (int64_t)edges_prev * 16;
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFreeHost(hcnt);
  cudaFreeAsync(ws, s);
  cudaStreamSynchronize(s);
  return status;
}

// ----- step entry points ------------------------------------------------------------------

sgr_status sgr_assign(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors_in, int32_t* tent_out, const sgr_opts* opts) {
  if (!csr || n < 0 || wl_len < 0) return SGR_EINVAL;
  if (wl_len == 0) return SGR_OK;
  if (!csr->row_ptr || !wl || !colors_in || !tent_out ||
      (const void*)colors_in == (const void*)tent_out) {
    set_error("sgr_assign: null or aliased pointer");
    return SGR_EINVAL;
  }
  const Resolved r = resolve_opts(opts, n);
  if (!block_ok(r.block, 32, kMaxBlockAny)) return SGR_EINVAL;
  k_assign_step<<<grid_for(wl_len, r.block / 32, r.block), r.block, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl, wl_len,
                                                           colors_in, tent_out);
  CK(cudaGetLastError());
  return SGR_OK;
}

sgr_status sgr_commit(const int32_t* wl, const int32_t* tent, int64_t wl_len, int32_t* colors,
                      const sgr_opts* opts) {
  if (wl_len < 0) return SGR_EINVAL;
  if (wl_len == 0) return SGR_OK;
  if (!wl || !tent || !colors) return SGR_EINVAL;
  const Resolved r = resolve_opts(opts, 0);
  if (!block_ok(r.block, 32, kMaxBlockAny)) return SGR_EINVAL;
  k_commit_step<<<grid_for(wl_len, r.block, r.block), r.block, 0, r.stream>>>(wl, tent, wl_len, colors);
  CK(cudaGetLastError());
  return SGR_OK;
}

sgr_status sgr_detect(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors, uint8_t* conflict_out, const sgr_opts* opts) {
  if (!csr || n < 0 || wl_len < 0) return SGR_EINVAL;
  if (wl_len == 0) return SGR_OK;
  if (!csr->row_ptr || !wl || !colors || !conflict_out) return SGR_EINVAL;
  const Resolved r = resolve_opts(opts, n);
  if (!block_ok(r.block, 32, kMaxBlockAny)) return SGR_EINVAL;
  const int g = grid_for(wl_len, r.block / 32, r.block);
  if (r.tiebreak)
    k_detect_step<1><<<g, r.block, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl, wl_len, colors,
                                                  conflict_out);
  else
    k_detect_step<0><<<g, r.block, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl, wl_len, colors,
                                                  conflict_out);
  CK(cudaGetLastError());
  return SGR_OK;
}

sgr_status sgr_compact(const int32_t* wl, const uint8_t* flags, int64_t len, int32_t* wl_out,
                       int64_t* count_out, const sgr_opts* opts) {
  if (len < 0 || !count_out) return SGR_EINVAL;
  const Resolved r = resolve_opts(opts, 0);
  cudaStream_t s = r.stream;
  if (len == 0) {
    CK(cudaMemsetAsync(count_out, 0, sizeof(int64_t), s));
    return SGR_OK;
  }
  if (!wl || !flags || !wl_out) return SGR_EINVAL;
  const int64_t tiles = (len + kCompactTile - 1) / kCompactTile;
  int32_t* tile = nullptr;
  CK(cudaMallocAsync((void**)&tile, (size_t)tiles * 4, s));
  k_compact_count<<<(unsigned)tiles, 256, 0, s>>>(flags, len, tile);
  k_compact_scan<<<1, 1024, 0, s>>>(tile, tiles, count_out);
  k_compact_scatter<<<(unsigned)tiles, 256, 0, s>>>(wl, flags, len, tile, wl_out);
  cudaError_t e = cudaGetLastError();
  cudaFreeAsync(tile, s);
  if (e != cudaSuccess) return cuda_fail(e, "sgr_compact", __LINE__);
  return SGR_OK;
}

}  // extern "C"
