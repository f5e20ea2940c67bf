// sgr.cu — host side of libsgr.so: the C ABI of include/sgr.h (single GPU + step entry
// points). Multi-GPU lives in sgr_dist.cu. See DESIGN.md §5 for the round loop.
#include <cuda_runtime.h>

#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <vector>

#include "sgr.h"
#include "sgr_internal.h"
#include "sgr_kernels.cuh"

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

int num_sms() {
  static int sms[64] = {0};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 148;
  if (dev < 0 || dev >= 64) return 148;
  if (sms[dev] == 0) {
    int v = 0;
    if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0)
      v = 148;
    sms[dev] = v;
  }
  return sms[dev];
}

static size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

Resolved resolve_opts(const sgr_opts* o, int64_t n) {
  Resolved r;
  sgr_opts d;
  sgr_opts_default(&d);
  if (!o) o = &d;
  r.tiebreak = o->tiebreak == SGR_TIEBREAK_PAPER ? 1 : 0;
  r.max_rounds = o->max_rounds > 0 ? o->max_rounds : (int32_t)std::min<int64_t>(n + 1, INT32_MAX);
  r.loop_mode = o->loop_mode == SGR_LOOP_HOST ? SGR_LOOP_HOST : SGR_LOOP_GRAPH;
  r.block = o->block_size > 0 ? o->block_size : 256;
  r.block = std::max(32, std::min(1024, r.block / 32 * 32));
  r.small_max = o->bin_small_max > 0 ? std::min(o->bin_small_max, 62) : 32;
  r.med_max = o->bin_med_max > 0 ? std::max(o->bin_med_max, r.small_max) : 4096;
  r.stream = (cudaStream_t)o->stream;
  r.round_sizes = o->round_sizes;
  r.round_edges = o->round_edges;
  r.round_cap = (o->round_sizes || o->round_edges) ? o->round_cap : 0;
  r.validate = o->validate;
  r.batch = o->rounds_per_batch > 0 ? o->rounds_per_batch : 8;
  r.profile = o->profile;
  return r;
}

// Workspace layout: [Ctrl][Y: n int32][wl: 2 x kBins x n int32]
size_t ws_bytes(int64_t n) {
  size_t b = align_up(sizeof(Ctrl), 256);
  b += align_up((size_t)n * 4, 256);
  b += (size_t)2 * kBins * align_up((size_t)n * 4, 256);
  return b;
}

struct Workspace {
  Ctrl* ctrl;
  int32_t* y;
  int32_t* wl[2][kBins];
};

static Workspace carve(void* base, int64_t n) {
  Workspace w;
  char* p = (char*)base;
  w.ctrl = (Ctrl*)p;
  p += align_up(sizeof(Ctrl), 256);
  w.y = (int32_t*)p;
  p += align_up((size_t)n * 4, 256);
  for (int par = 0; par < 2; ++par)
    for (int q = 0; q < kBins; ++q) {
      w.wl[par][q] = (int32_t*)p;
      p += align_up((size_t)n * 4, 256);
    }
  return w;
}

// Pinned host slots for termination flags (reused across calls on this thread).
static int32_t* pinned_flags() {
  static thread_local int32_t* p = nullptr;
  if (!p) {
    if (cudaMallocHost(&p, 64 * sizeof(int32_t)) != cudaSuccess) p = nullptr;
  }
  return p;
}

// ----- per-launch grids ------------------------------------------------------------------
struct Grids {
  int first, thread_b, warp_b, cta_b, block, cta_threads;
};

static Grids make_grids(int64_t n, const Resolved& r) {
  Grids g;
  const int sms = num_sms();
  g.block = r.block;
  const int per_sm = std::max(1, 2048 / g.block);
  g.first = (int)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, (int64_t)sms * 8));
  g.thread_b = (int)std::max<int64_t>(1, std::min<int64_t>((n + g.block - 1) / g.block, (int64_t)sms * per_sm));
  g.warp_b = (int)std::max<int64_t>(1, std::min<int64_t>((n * 32 + g.block - 1) / g.block, (int64_t)sms * per_sm));
  g.cta_threads = 512;
  g.cta_b = sms * 4;
  return g;
}

// ----- the round-pass launcher (shared by the host loop, graph capture and dist) --------
template <int TB>
static void launch_pass(const RoundArgs& a, const Grids& g, cudaStream_t s) {
  k_round_cta<TB><<<g.cta_b, g.cta_threads, 0, s>>>(a);
  k_round_warp<TB><<<g.warp_b, g.block, 0, s>>>(a);
  k_round_thread<TB><<<g.thread_b, g.block, 0, s>>>(a);
  k_advance<<<1, 32, 0, s>>>(a.ctrl, 0);
}

void launch_first(const RoundArgs& a, int tiebreak, bool sorted, int grid, cudaStream_t s) {
  if (sorted) {
    if (tiebreak) k_first<1><<<grid, 256, 0, s>>>(a);
    else k_first<0><<<grid, 256, 0, s>>>(a);
  } else {
    if (tiebreak) k_first_unsorted<1><<<grid, 256, 0, s>>>(a);
    else k_first_unsorted<0><<<grid, 256, 0, s>>>(a);
  }
}

void launch_round_pass(const RoundArgs& a, int tiebreak, int64_t n, const Resolved& r,
                       cudaStream_t s) {
  Grids g = make_grids(n, r);
  if (tiebreak) launch_pass<1>(a, g, s);
  else launch_pass<0>(a, g, s);
}

// ----- CUDA-graph cache: one graph = `batch` fused passes ----------------------------------
struct GraphKey {
  RoundArgs a;
  Grids g;
  int tiebreak, batch, dev;
  bool operator==(const GraphKey& o) const { return memcmp(this, &o, sizeof(GraphKey)) == 0; }
};

struct GraphEntry {
  GraphKey key;
  cudaGraphExec_t exec;
};

static std::mutex g_graph_mu;
static std::vector<GraphEntry> g_graphs;

static sgr_status get_graph(const GraphKey& key, cudaGraphExec_t* out) {
  std::lock_guard<std::mutex> lk(g_graph_mu);
  for (auto& e : g_graphs)
    if (e.key == key) {
      *out = e.exec;
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
  for (int b = 0; b < key.batch; ++b) {
    if (key.tiebreak) launch_pass<1>(key.a, key.g, cs);
    else launch_pass<0>(key.a, key.g, cs);
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
    cudaGraphExecDestroy(g_graphs.front().exec);
    g_graphs.erase(g_graphs.begin());
  }
  g_graphs.push_back({key, exec});
  *out = exec;
  return SGR_OK;
}

// ----- profiling (opts->profile): CUDA events around every launch -----------------------
struct Prof {
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
  ~Prof() {
    for (auto e : pool) cudaEventDestroy(e);
  }
};

template <int TB>
static void launch_pass_prof(const RoundArgs& a, const Grids& g, cudaStream_t s, Prof& pr) {
  auto timed = [&](int cls, auto&& fn) {
    cudaEvent_t e0 = pr.get(), e1 = pr.get();
    cudaEventRecord(e0, s);
    fn();
    cudaEventRecord(e1, s);
    pr.marks.push_back({cls, {e0, e1}});
  };
  timed(SGR_K_HUB, [&] { k_round_cta<TB><<<g.cta_b, g.cta_threads, 0, s>>>(a); });
  timed(SGR_K_MED, [&] { k_round_warp<TB><<<g.warp_b, g.block, 0, s>>>(a); });
  timed(SGR_K_SMALL, [&] { k_round_thread<TB><<<g.thread_b, g.block, 0, s>>>(a); });
  timed(SGR_K_CTRL, [&] { k_advance<<<1, 32, 0, s>>>(a.ctrl, 0); });
}

// Fill the byte model and counters from the final Ctrl.
void fill_stats(const Ctrl& c, int64_t n, int64_t nnz, sgr_stats* st) {
  const int64_t vpass = (int64_t)(c.verts_total[0] + c.verts_total[1] + c.verts_total[2]);
  const int64_t epass = (int64_t)(c.edges_total[0] + c.edges_total[1] + c.edges_total[2]);
  st->rounds = c.k - 1;
  st->num_colors = c.max_color;
  st->vertices_processed = (n > 0 ? n : 0) + vpass;
  st->edges_scanned = (n > 0 ? nnz : 0) + epass;
  // F_1: 8 B row offset + 4 B first/last col entry + 8 B two color writes per vertex,
  //      + 4 B per pushed vertex.
  const int64_t b_first = 20 * n + 4 * (int64_t)c.pushes_total[kBins];
  int64_t b_bins[kBins];
  for (int q = 0; q < kBins; ++q)  // per vertex: 4 B id + 16 B row pair + 4 B X[v] + 4 B Y[v]
    b_bins[q] = 28 * (int64_t)c.verts_total[q] + 8 * (int64_t)c.edges_total[q] +
                4 * (int64_t)c.pushes_total[q];
  st->bytes_algorithmic = b_first + b_bins[0] + b_bins[1] + b_bins[2];
  st->kernel_bytes[SGR_K_FIRST] = b_first;
  st->kernel_bytes[SGR_K_SMALL] = b_bins[0];
  st->kernel_bytes[SGR_K_MED] = b_bins[1];
  st->kernel_bytes[SGR_K_HUB] = b_bins[2];
  st->kernel_bytes[SGR_K_CTRL] = 0;
}

}  // namespace sgr

using namespace sgr;

#define CK(call)                                                         \
  do {                                                                   \
    cudaError_t e_ = (call);                                             \
    if (e_ != cudaSuccess) return cuda_fail(e_, #call, __LINE__);        \
  } while (0)

extern "C" {

void sgr_opts_default(sgr_opts* o) {
  if (!o) return;
  memset(o, 0, sizeof(*o));
  o->tiebreak = SGR_TIEBREAK_LOWID_KEEPS;
  o->loop_mode = SGR_LOOP_AUTO;
}

size_t sgr_workspace_bytes(int64_t n, int64_t nnz, const sgr_opts* opts) {
  (void)nnz;
  (void)opts;
  return n > 0 ? ws_bytes(n) : 0;
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
const char* sgr_version(void) { return "sgr-b200 0.1 (sm_100a)"; }

static sgr_status run_validate(const sgr_csr* csr, int64_t n, int64_t nnz, Ctrl* ctrl,
                               cudaStream_t s, int32_t* viol_out) {
  CK(cudaMemsetAsync(&ctrl->violations, 0, sizeof(int32_t), s));
  k_validate<<<num_sms() * 4, 256, 0, s>>>(csr->row_ptr, csr->col_idx, n, nnz, ctrl);
  CK(cudaGetLastError());
  int32_t v = 0;
  CK(cudaMemcpyAsync(&v, &ctrl->violations, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  CK(cudaStreamSynchronize(s));
  *viol_out = v;
  return SGR_OK;
}

sgr_status sgr_validate_csr(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* violations,
                            void* stream) {
  if (!csr || !csr->row_ptr || n < 0 || nnz < 0 || !violations || (nnz > 0 && !csr->col_idx))
    return SGR_EINVAL;
  cudaStream_t s = (cudaStream_t)stream;
  Ctrl* ctrl;
  CK(cudaMallocAsync((void**)&ctrl, sizeof(Ctrl), s));
  sgr_status st = run_validate(csr, n, nnz, ctrl, s, violations);
  cudaFreeAsync(ctrl, s);
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
  const Resolved r = resolve_opts(opts, n);
  cudaStream_t s = r.stream;
  const size_t need = ws_bytes(n);
  void* ws = workspace;
  bool own = false;
  if (!ws || workspace_bytes < need) {
    CK(cudaMallocAsync(&ws, need, s));
    own = true;
  }
  Workspace w = carve(ws, n);
  sgr_status status = SGR_OK;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr;
  Prof prof;
  int32_t launches = 0;
  do {
    if (r.validate) {
      int32_t viol = 0;
      status = run_validate(csr, n, nnz, w.ctrl, s, &viol);
      if (status != SGR_OK) break;
      if (viol) {
        set_error("sgr_color: CSR contract violated (mask %d)", viol);
        status = SGR_EINVAL;
        break;
      }
    }
    // Ctrl init (host image -> device)
    Ctrl hc;
    memset(&hc, 0, sizeof(hc));
    hc.k = 1;
    hc.max_rounds = r.max_rounds;
    hc.round_cap = r.round_cap;
    hc.round_sizes = r.round_sizes;
    hc.round_edges = r.round_edges;
    if (cudaMemcpyAsync(w.ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s) != cudaSuccess) {
      status = cuda_fail(cudaGetLastError(), "ctrl init", __LINE__);
      break;
    }
    if (r.round_cap > 0) {  // round 1: |W_1| = n, sum deg = nnz
      int32_t n32 = (int32_t)n;
      int64_t nz = nnz;
      if (r.round_sizes) cudaMemcpyAsync(r.round_sizes, &n32, 4, cudaMemcpyHostToDevice, s);
      if (r.round_edges) cudaMemcpyAsync(r.round_edges, &nz, 8, cudaMemcpyHostToDevice, s);
    }
    cudaEventCreate(&ev0);
    cudaEventCreate(&ev1);
    cudaEventRecord(ev0, s);

    RoundArgs a;
    memset(&a, 0, sizeof(a));
    a.row_ptr = csr->row_ptr;
    a.col_idx = csr->col_idx;
    a.col[0] = colors_out;
    a.col[1] = w.y;
    for (int par = 0; par < 2; ++par)
      for (int q = 0; q < kBins; ++q) a.wl[par][q] = w.wl[par][q];
    a.ctrl = w.ctrl;
    a.n = (int32_t)n;
    a.small_max = r.small_max;
    a.med_max = r.med_max;
    const Grids g = make_grids(n, r);

    cudaEvent_t pf0 = nullptr, pf1 = nullptr;
    if (r.profile) {
      pf0 = prof.get();
      pf1 = prof.get();
      cudaEventRecord(pf0, s);
    }
    launch_first(a, r.tiebreak, true, g.first, s);
    if (r.profile) {
      cudaEventRecord(pf1, s);
      prof.marks.push_back({SGR_K_FIRST, {pf0, pf1}});
    }
    k_advance<<<1, 32, 0, s>>>(w.ctrl, 1);
    launches += 2;
    cudaError_t le = cudaGetLastError();
    if (le != cudaSuccess) {
      status = cuda_fail(le, "launch F_1", __LINE__);
      break;
    }

    int32_t* flags = pinned_flags();
    if (!flags) {
      status = cuda_fail(cudaErrorMemoryAllocation, "cudaMallocHost", __LINE__);
      break;
    }
    cudaEvent_t done_ev[2];
    cudaEventCreateWithFlags(&done_ev[0], cudaEventDisableTiming);
    cudaEventCreateWithFlags(&done_ev[1], cudaEventDisableTiming);
    const bool use_graph = r.loop_mode == SGR_LOOP_GRAPH && !r.profile;
    cudaGraphExec_t gexec = nullptr;
    if (use_graph) {
      GraphKey key;
      memset(&key, 0, sizeof(key));
      key.a = a;
      key.g = g;
      key.tiebreak = r.tiebreak;
      key.batch = r.batch;
      cudaGetDevice(&key.dev);
      status = get_graph(key, &gexec);
      if (status != SGR_OK) break;
    }
    // Pipelined termination test: batch b's `active` flag is read only after batch b+1 is
    // enqueued, so the GPU never idles waiting for the host; surplus passes are no-ops.
    int64_t batches = 0;
    bool finished = false;
    while (!finished) {
      if (use_graph) {
        le = cudaGraphLaunch(gexec, s);
        launches += 4 * r.batch;
      } else {
        for (int b = 0; b < r.batch; ++b) {
          if (r.profile) {
            if (r.tiebreak) launch_pass_prof<1>(a, g, s, prof);
            else launch_pass_prof<0>(a, g, s, prof);
          } else {
            if (r.tiebreak) launch_pass<1>(a, g, s);
            else launch_pass<0>(a, g, s);
          }
        }
        launches += 4 * r.batch;
        le = cudaGetLastError();
      }
      if (le != cudaSuccess) {
        status = cuda_fail(le, "launch round batch", __LINE__);
        break;
      }
      const int slot = (int)(batches & 1);
      cudaMemcpyAsync(&flags[slot], &w.ctrl->active, 4, cudaMemcpyDeviceToHost, s);
      cudaEventRecord(done_ev[slot], s);
      if (batches > 0) {
        cudaEventSynchronize(done_ev[slot ^ 1]);
        if (flags[slot ^ 1] == 0) finished = true;
      }
      ++batches;
      if (batches > ((int64_t)r.max_rounds / r.batch) + 4) {  // defensive: cannot happen
        cudaEventSynchronize(done_ev[slot]);
        if (flags[slot] == 0) finished = true;
      }
    }
    cudaEventDestroy(done_ev[0]);
    cudaEventDestroy(done_ev[1]);
    if (status != SGR_OK) break;

    k_max_color<<<g.first, 256, 0, s>>>(colors_out, n, w.ctrl);
    launches += 1;
    cudaEventRecord(ev1, s);
    Ctrl fin;
    cudaMemcpyAsync(&fin, w.ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s);
    le = cudaStreamSynchronize(s);
    if (le != cudaSuccess) {
      status = cuda_fail(le, "sgr_color", __LINE__);
      break;
    }
    if (stats) {
      fill_stats(fin, n, nnz, stats);
      cudaEventElapsedTime(&stats->elapsed_ms, ev0, ev1);
      stats->launches = launches;
      if (r.profile) {
        for (auto& m : prof.marks) {
          float ms = 0.f;
          cudaEventElapsedTime(&ms, m.second.first, m.second.second);
          stats->kernel_ms[m.first] += ms;
          stats->kernel_launches[m.first] += 1;
        }
      }
    }
    if (fin.status == 1) {
      set_error("sgr_color: max_rounds (%d) reached", r.max_rounds);
      status = SGR_ENOCONV;
    }
  } while (0);
  if (ev0) cudaEventDestroy(ev0);
  if (ev1) cudaEventDestroy(ev1);
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
  if (st == SGR_OK) {
    CK(cudaMemcpyAsync(colors_out, d_col, (size_t)n * 4, cudaMemcpyDeviceToHost, s));
  }
  cudaFreeAsync(d_rp, s);
  cudaFreeAsync(d_ci, s);
  cudaFreeAsync(d_col, s);
  CK(cudaStreamSynchronize(s));
  return st;
}

// ----- step entry points ------------------------------------------------------------------
static int grid_for(int64_t items, int per_block) {
  const int64_t b = (items + per_block - 1) / per_block;
  return (int)std::max<int64_t>(1, std::min<int64_t>(b, (int64_t)num_sms() * 16));
}

sgr_status sgr_assign(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors_in, int32_t* tent_out, const sgr_opts* opts) {
  if (!csr || n < 0 || wl_len < 0) return SGR_EINVAL;
  if (wl_len == 0) return SGR_OK;
  if (!csr->row_ptr || !csr->col_idx || !wl || !colors_in || !tent_out ||
      (const void*)colors_in == (const void*)tent_out) {
    set_error("sgr_assign: null or aliased pointer");
    return SGR_EINVAL;
  }
  const Resolved r = resolve_opts(opts, n);
  k_assign_step<<<grid_for(wl_len, 8), 256, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl, wl_len,
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
  k_commit_step<<<grid_for(wl_len, 256), 256, 0, r.stream>>>(wl, tent, wl_len, colors);
  CK(cudaGetLastError());
  return SGR_OK;
}

sgr_status sgr_detect(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors, uint8_t* conflict_out, const sgr_opts* opts) {
  if (!csr || n < 0 || wl_len < 0) return SGR_EINVAL;
  if (wl_len == 0) return SGR_OK;
  if (!csr->row_ptr || !csr->col_idx || !wl || !colors || !conflict_out) return SGR_EINVAL;
  const Resolved r = resolve_opts(opts, n);
  if (r.tiebreak)
    k_detect_step<1><<<grid_for(wl_len, 8), 256, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl,
                                                               wl_len, colors, conflict_out);
  else
    k_detect_step<0><<<grid_for(wl_len, 8), 256, 0, r.stream>>>(csr->row_ptr, csr->col_idx, wl,
                                                               wl_len, colors, conflict_out);
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
