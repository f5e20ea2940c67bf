// sgr_dist.cu — multi-GPU layer.
//
// The graph is split into contiguous vertex ranges balanced by nnz (sgr_partition). Every
// partition owns the rows of its range (local row offsets, GLOBAL column ids) and keeps a
// full replica of the color array. A round is:
//   1. the fused pass F_k over the partition's owned worklists (the same kernels as one GPU;
//      row_ptr is shifted by -v_begin so global ids index the local offsets),
//   2. k_pack: the partition's part of W_{k+1} as (v, new color word) records,
//   3. an all-gather of the records (NCCL over NVLink between ranks, or device copies
//      between partitions that share one GPU),
//   4. k_apply: every replica writes the other partitions' records into both ping-pong
//      buffers (a remote vertex is never written by the local pass); the same launch
//      advances the round (lockstep) and re-arms the send count.
// Round k's records are a subset of W_k, so the largest count of the previous exchange is
// a valid capacity for the padded all-gather: one collective per round (plus one counts
// gather before the first). The result is bit-identical to one GPU: the passes read the
// same snapshot values, only the owner computes each vertex.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <cstdlib>
#include <functional>
#include <map>
#include <vector>

#include "sgr.h"
#include "sgr_host.cuh"
#include "sgr_internal.h"
#include "sgr_round.cuh"
#include "sgr_step.cuh"

#if SGR_HAVE_NCCL
#include <nccl.h>
#endif

namespace sgr {

struct DistComm {
#if SGR_HAVE_NCCL
  ncclComm_t comm = nullptr;
#endif
  int rank = 0, world = 1, device = 0;
};

struct Part {
  int64_t lo = 0, hi = 0, nnz = 0;
  sgr_csr csr{};        // owned rows: row_ptr (hi - lo + 1 local offsets), col_idx (global ids)
  void* ws = nullptr;   // workspace (layout(n_global, nnz_local))
  int32_t* colors = nullptr;  // plain mode ping-pong partner / final output
  uint2* send = nullptr;
  bool own_colors = false;
};

using Gather = std::function<sgr_status(std::vector<Part>& parts, uint2* recv, int32_t cap,
                                        cudaStream_t s)>;

#define DCK(call)                                                            \
  do {                                                                       \
    cudaError_t e_ = (call);                                                 \
    if (e_ != cudaSuccess) return cuda_fail(e_, #call, __LINE__);           \
  } while (0)

// Runs the rounds for every partition in `parts` (all on the current device, one stream).
// `me0` is the index of parts[0] among all `world` partitions (NCCL: the rank).
template <int TB, class C>
static sgr_status run_parts(std::vector<Part>& parts, int world, int me0, int64_t n,
                            int32_t* colors_out, sgr_stats* stats, const Gather& gather,
                            int64_t cap_hint, const Resolved& r, int* overflow_out) {
  cudaStream_t s = r.stream;
  const int B = r.block;
  if (!block_ok(B, 64, round_max_block<C, true>())) {
    set_error("sgr_color_dist: block_size %d not supported by the round kernels", B);
    return SGR_EINVAL;
  }
  keep_pool_memory();
  const int P = (int)parts.size();
  std::vector<Layout> Ls;
  std::vector<RoundArgs<C>> args(P);
  // a record count never exceeds its owner's range: size by the largest range anywhere
  int64_t cap_max = std::max<int64_t>(1, cap_hint);
  for (int i = 0; i < P; ++i) cap_max = std::max(cap_max, parts[i].hi - parts[i].lo);
  for (int i = 0; i < P; ++i) {
    Part& pt = parts[i];
    Ls.push_back(layout(n, pt.nnz, r));
    DCK(cudaMallocAsync(&pt.ws, Ls[i].total, s));
    DCK(cudaMallocAsync((void**)&pt.send, (size_t)(cap_max + 1) * sizeof(uint2), s));
    // the padded all-gather copies whole slots; records past a rank's count are never
    // read, but start them defined (compute-sanitizer initcheck)
    DCK(cudaMemsetAsync(pt.send, 0, (size_t)(cap_max + 1) * sizeof(uint2), s));
    if (!packed<C>() && (i > 0 || !colors_out)) {
      DCK(cudaMallocAsync((void**)&pt.colors, (size_t)n * 4, s));
      pt.own_colors = true;
    } else {
      pt.colors = colors_out;
    }
    sgr_csr shifted{pt.csr.row_ptr - pt.lo, pt.csr.col_idx};
    build_args<C>(args[i], &shifted, n, pt.nnz, pt.colors, pt.ws, Ls[i], r);
    args[i].v_begin = (int32_t)pt.lo;
    args[i].v_end = (int32_t)pt.hi;
    Ctrl hc;
    memset(&hc, 0, sizeof(hc));
    hc.k = 1;
    hc.max_rounds = INT32_MAX;
    DCK(cudaMemcpyAsync(args[i].ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
    DCK(cudaMemsetAsync((char*)pt.ws + Ls[i].zero_begin, 0, Ls[i].zero_end - Ls[i].zero_begin, s));
    k_fill_c1<C><<<first_grid(n), 256, 0, s>>>(args[i]);
    k_first<TB, C><<<first_grid(pt.hi - pt.lo), 256, 0, s>>>(args[i], r.sorted);
    k_advance<<<1, 32, 0, s>>>(args[i].ctrl, 1, 0);
  }
  DCK(cudaGetLastError());
  const int grid = round_grid<TB, C>(false, B);
  const int grid_flat = round_grid<TB, C, false>(false, B);
  std::vector<int32_t> big(P, 0);  // per part: F_1's bin-2 slots (0: flat build)
  uint2* recv = nullptr;
  DCK(cudaMallocAsync((void**)&recv, (size_t)world * (cap_max + 1) * sizeof(uint2), s));
  std::vector<uint2> hdr(world);
  int32_t* counts_host = nullptr;  // per part: (record count, overflow flag)
  DCK(cudaMallocHost(&counts_host, 2 * sizeof(int32_t) * world));
  bool overflow_seen = false;

  // one exchange: pack -> all-gather with capacity cap -> apply; returns per-part counts
  auto exchange = [&](int32_t cap, std::vector<int32_t>& cnt) -> sgr_status {
    for (int i = 0; i < P; ++i) {
      DCK(cudaMemsetAsync(parts[i].send, 0, sizeof(uint2), s));
      k_pack<C><<<first_grid(parts[i].hi - parts[i].lo + 1), 256, 0, s>>>(args[i], parts[i].send, cap);
    }
    DCK(cudaGetLastError());
    sgr_status st = gather(parts, recv, cap, s);
    if (st != SGR_OK) return st;
    for (int i = 0; i < P; ++i)
      k_apply<C><<<first_grid(cap), 256, 0, s>>>(args[i], recv, world, cap + 1, me0 + i,
                                                 parts[i].send, 0);
    DCK(cudaGetLastError());
    DCK(cudaMemcpy2DAsync(counts_host, sizeof(uint2), recv, (size_t)(cap + 1) * sizeof(uint2),
                          sizeof(uint2), world, cudaMemcpyDeviceToHost, s));
    DCK(cudaStreamSynchronize(s));
    cnt.resize(world);
    for (int q = 0; q < world; ++q) {
      cnt[q] = counts_host[2 * q];
      if (counts_host[2 * q + 1]) overflow_seen = true;
    }
    if (overflow_seen) std::fill(cnt.begin(), cnt.end(), 0);  // stop; rerun with int32 words
    return SGR_OK;
  };

  sgr_status status = SGR_OK;
  cudaEvent_t ev0, ev1;
  cudaEventCreate(&ev0);
  cudaEventCreate(&ev1);
  std::vector<int32_t> cnt;
  // W_2: a counts-only round first, so the data gather is sized by the real maximum
  {
    for (int i = 0; i < P; ++i) DCK(cudaMemsetAsync(parts[i].send, 0, sizeof(uint2), s));
    for (int i = 0; i < P; ++i)
      k_pack<C><<<first_grid(parts[i].hi - parts[i].lo + 1), 256, 0, s>>>(args[i], parts[i].send, 0);
    status = gather(parts, recv, 0, s);
    for (int i = 0; i < P && status == SGR_OK; ++i)
      DCK(cudaMemcpyAsync(&big[i], &args[i].ctrl->big_count, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    if (status == SGR_OK) {
      DCK(cudaMemcpy2DAsync(counts_host, sizeof(uint2), recv, sizeof(uint2), sizeof(uint2),
                            world, cudaMemcpyDeviceToHost, s));
      DCK(cudaStreamSynchronize(s));
    }
  }
  cudaEventRecord(ev0, s);
  int32_t cap = 0;
  for (int q = 0; q < world && status == SGR_OK; ++q) {
    cap = std::max(cap, counts_host[2 * q]);
    if (counts_host[2 * q + 1]) overflow_seen = true;
  }
  if (overflow_seen) cap = 0;
  int64_t vertices = n, rounds = 1;
  if (status == SGR_OK) status = exchange(cap, cnt);  // W_2 records
  int64_t total = 0;
  for (int32_t c : cnt) total += c;
  if (total > 0) rounds = 2;
  vertices += total;
  // Passes k = 2, 3, ...: the host reads the per-rank counts of W_{k+1} with a lag of
  // kLag passes (pinned slots + events) instead of blocking after every exchange. The
  // all-gather capacity comes from the newest counts read so far: they bound every later
  // round's counts because W only shrinks. Once some W_j is read to be empty no further
  // passes are issued; the <= kLag already in flight run on empty worklists (no-ops), and
  // R is taken from the counts, not from the passes issued.
  constexpr int kLag = 2;
  int32_t* slots = nullptr;  // [kLag + 1][world][2]
  cudaEvent_t sev[kLag + 1];
  for (int q = 0; q <= kLag; ++q) cudaEventCreateWithFlags(&sev[q], cudaEventDisableTiming);
  if (status == SGR_OK) DCK(cudaMallocHost(&slots, sizeof(int32_t) * 2 * world * (kLag + 1)));
  int32_t known_cap = status == SGR_OK ? *std::max_element(cnt.begin(), cnt.end()) : 0;
  bool done = status != SGR_OK || total == 0 || overflow_seen;
  int64_t issued = 0, consumed = 0;  // passes issued / whose counts were read
  // One pass = per partition: fused round, finalize, advance, pack; the exchange; apply.
  auto enqueue_pass = [&](int32_t cap_k, cudaStream_t st) -> sgr_status {
    for (int i = 0; i < P; ++i) {
      // the build the persistent kernel would pick: the flat one (more L1, no finalize
      // phase) when F_1 put no vertex of this part into bin 2 (world-1 cfg2 31.3 -> 26.5 ms)
      if (big[i] == 0) {
        k_round<TB, C, false><<<grid_flat, B, round_smem<C, false>(B), st>>>(args[i]);
      } else {
        k_round<TB, C><<<grid, B, round_smem<C>(B), st>>>(args[i]);
        if constexpr (packed<C>()) k_finalize<TB, C><<<grid, kBlock, 0, st>>>(args[i]);
      }
      // W_{k+1} is bounded by cap_k: size the grid by it, not by the range (a thin
      // round's pack was ~9.5K blocks that found nothing to do). The pack runs before the
      // advance (pre = 1), which k_apply carries, with the send-count reset.
      k_pack<C><<<first_grid(std::min<int64_t>(cap_k, parts[i].hi - parts[i].lo) + 1), 256, 0, st>>>(
          args[i], parts[i].send, cap_k, 1);
    }
    DCK(cudaGetLastError());
    const sgr_status gst = gather(parts, recv, cap_k, st);
    if (gst != SGR_OK) return gst;
    for (int i = 0; i < P; ++i)
      k_apply<C><<<first_grid(cap_k), 256, 0, st>>>(args[i], recv, world, cap_k + 1, me0 + i,
                                                    parts[i].send, 1);
    DCK(cudaGetLastError());
    return SGR_OK;
  };
  // The host-driven loop was launch-gap bound (7+ operations per round, ~40 us): each
  // pass is captured once per all-gather capacity bucket into a CUDA graph (exchange
  // included: NCCL collectives are capturable) and replayed. Capacities are rounded up to
  // a quarter-octave (>= 4096 records, <= cap_max): the padding is at most 25 % of the
  // records, and every rank derives the same bucket from the same counts. All state a
  // pass reads (round number, ping-pong parity, worklist counts) lives on the device, so
  // a replay is the same pass as a fresh launch. Opt-in (SGR_DIST_GRAPHS=1): on one B200
  // (NCCL world 1) replay saved nothing per round and instantiation (one graph per bucket,
  // per coloring) cost 0.3-0.5 ms (cfg1 2.97 -> 3.47 ms, cfg4 46.9 -> 47.2 ms).
  const char* genv = getenv("SGR_DIST_GRAPHS");
  const bool use_graphs = genv && genv[0] == '1';
  std::map<int32_t, cudaGraphExec_t> graphs;
  cudaStream_t gs = nullptr;  // capture stream (the caller's may be the legacy stream)
  if (use_graphs && status == SGR_OK) DCK(cudaStreamCreateWithFlags(&gs, cudaStreamNonBlocking));
  auto cap_bucket = [&](int32_t c) -> int32_t {
    int64_t b = 4096;
    if (c > 4096) {
      int64_t p = 1;
      while (p * 2 <= c) p *= 2;
      const int64_t step = p / 4;
      b = (c + step - 1) / step * step;
    }
    return (int32_t)std::min<int64_t>(b, cap_max);
  };
  auto consume_one = [&]() {
    const int q = (int)(consumed % (kLag + 1));
    cudaEventSynchronize(sev[q]);
    ++consumed;
    if (done) return;  // passes after the end (or an overflow) are no-ops: ignore them
    int64_t t = 0;
    int32_t mx = 0;
    for (int w = 0; w < world; ++w) {
      t += slots[(q * world + w) * 2];
      mx = std::max(mx, slots[(q * world + w) * 2]);
      if (slots[(q * world + w) * 2 + 1]) overflow_seen = true;
    }
    if (overflow_seen) {  // stop; rerun with int32 words
      done = true;
      return;
    }
    known_cap = std::min(known_cap, mx);
    vertices += t;
    if (t > 0) ++rounds;
    else done = true;
  };
  while (status == SGR_OK && !done) {
    if (rounds + (issued - consumed) >= r.max_rounds + 1 && !done) {
      // every pass in flight could still find W non-empty: drain before issuing more
      while (consumed < issued) consume_one();
      if (done) break;
      if (rounds > r.max_rounds) {
        set_error("sgr_color_dist: max_rounds (%d) reached", r.max_rounds);
        status = SGR_ENOCONV;
        break;
      }
    }
    const int32_t cap_k = use_graphs ? cap_bucket(known_cap) : known_cap;
    if (use_graphs) {
      auto it = graphs.find(cap_k);
      if (it == graphs.end()) {
        cudaGraph_t g = nullptr;
        DCK(cudaStreamBeginCapture(gs, cudaStreamCaptureModeThreadLocal));
        const sgr_status cs = enqueue_pass(cap_k, gs);
        const cudaError_t ce = cudaStreamEndCapture(gs, &g);
        if (cs != SGR_OK) {
          if (g) cudaGraphDestroy(g);
          status = cs;
          break;
        }
        DCK(ce);
        cudaGraphExec_t ex = nullptr;
        const cudaError_t ie = cudaGraphInstantiate(&ex, g, 0);
        cudaGraphDestroy(g);
        DCK(ie);
        it = graphs.emplace(cap_k, ex).first;
      }
      DCK(cudaGraphLaunch(it->second, s));
    } else {
      status = enqueue_pass(cap_k, s);
      if (status != SGR_OK) break;
    }
    const int q = (int)(issued % (kLag + 1));
    DCK(cudaMemcpy2DAsync(slots + q * world * 2, sizeof(uint2), recv, (size_t)(cap_k + 1) * sizeof(uint2),
                          sizeof(uint2), world, cudaMemcpyDeviceToHost, s));
    DCK(cudaEventRecord(sev[q], s));
    ++issued;
    if (issued - consumed > kLag) consume_one();
  }
  while (consumed < issued) consume_one();
  if (status == SGR_OK && rounds > r.max_rounds) {
    set_error("sgr_color_dist: max_rounds (%d) reached", r.max_rounds);
    status = SGR_ENOCONV;
  }
  for (int q = 0; q <= kLag; ++q) cudaEventDestroy(sev[q]);
  for (auto& kv : graphs) cudaGraphExecDestroy(kv.second);
  if (gs) cudaStreamDestroy(gs);
  if (slots) cudaFreeHost(slots);
  cudaEventRecord(ev1, s);
  if (status == SGR_OK) {
    RoundArgs<C>& a0 = args[0];
    if constexpr (packed<C>()) {
      k_unpack<<<reduce_grid(n), 256, 0, s>>>(a0.col[0], colors_out, n, &a0.ctrl->max_color);
    } else {
      if (a0.col[0] != (C*)colors_out)
        DCK(cudaMemcpyAsync(colors_out, a0.col[0], (size_t)n * 4, cudaMemcpyDeviceToDevice, s));
      k_max_color<<<reduce_grid(n), 256, 0, s>>>(colors_out, n, &a0.ctrl->max_color);
    }
    DCK(cudaGetLastError());
    std::vector<Ctrl> fin(P);
    for (int i = 0; i < P; ++i)
      DCK(cudaMemcpyAsync(&fin[i], args[i].ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
    DCK(cudaStreamSynchronize(s));
    int overflow = overflow_seen ? 1 : 0;
    for (int i = 0; i < P; ++i) overflow |= fin[i].overflow;
    for (int i = 0; i < P; ++i)
      if (fin[i].violations & 8) {
        set_error("sgr_color_dist: a rank sent more records than its previous worklist "
                  "held (asymmetric CSR?)");
        status = SGR_EINVAL;
      }
    if (overflow && !packed<C>()) {
      set_error("sgr_color_dist: 32-bit color overflow");
      status = SGR_EUNSUPPORTED;
    }
    if (overflow && packed<C>()) *overflow_out = 1;  // every rank saw the same flags
    if (stats) {
      memset(stats, 0, sizeof(*stats));
      for (int i = 0; i < P; ++i) {
        sgr_stats t;
        memset(&t, 0, sizeof(t));
        fill_stats(fin[i], 0, 0, &t, (int)sizeof(C));
        stats->edges_scanned += t.edges_scanned;
        stats->entries_read += t.entries_read;
        stats->entries_written += t.entries_written;
        stats->bytes_algorithmic += t.bytes_algorithmic;
        stats->chunk_items += t.chunk_items;
        for (int q = 0; q < 3; ++q) {
          stats->bin_vertices[q] += t.bin_vertices[q];
          stats->bin_edges[q] += t.bin_edges[q];
          stats->bin_warp_cycles[q] += t.bin_warp_cycles[q];
        }
      }
      int64_t nnz_parts = 0;
      for (auto& pt : parts) nnz_parts += pt.nnz;
      stats->edges_scanned += nnz_parts;  // round 1 (local rows)
      stats->rounds = (int32_t)rounds;
      stats->num_colors = fin[0].max_color;
      // F_1 + advance + fill per part, 5 launches per part per exchange round, final
      stats->launches = (int32_t)(P * 3 + (rounds + 1) * P * 5 + 2);
      stats->vertices_processed = vertices;
      stats->grid_blocks = grid;
      stats->color_bits = packed<C>() ? 16 : 32;
      stats->transport = world > 1 ? SGR_XCHG_ALLGATHER : SGR_XCHG_NONE;
      cudaEventElapsedTime(&stats->elapsed_ms, ev0, ev1);
    }
  }
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  cudaFreeHost(counts_host);
  cudaFreeAsync(recv, s);
  for (auto& pt : parts) {
    cudaFreeAsync(pt.ws, s);
    cudaFreeAsync(pt.send, s);
    if (pt.own_colors) cudaFreeAsync(pt.colors, s);
  }
  cudaStreamSynchronize(s);
  return status;
}

// ---------------------------------------------------------------------------------------
// Device-side exchange (k_persistent_dist): every part writes its color words straight into
// all replicas and the rounds run in one cooperative launch per device, with a barrier
// across parts. Parts on one device share the launch (block groups); on several GPUs
// each rank is one part and the other replicas are NVLink peer memory (CUDA IPC), with
// `xsync` ordering the setup steps across ranks (an NCCL all-reduce; nullptr on one device).
struct DevPart {
  int64_t lo = 0, hi = 0, nnz = 0;
  sgr_csr csr{};          // owned rows: local offsets, global column ids
  void* ws = nullptr;     // workspace of layout(n, nnz)
  int32_t* colors = nullptr;
  bool own_colors = false;
};
struct PeerView {         // multi-GPU: the other ranks' workspaces (IPC-mapped), by rank
  std::vector<void*> ws;  // ws[me] = own
  std::vector<int64_t> ranges;  // nranks + 1 vertex-range boundaries of all ranks
  int me = 0;
};
using XSync = std::function<sgr_status(cudaStream_t, int32_t* dflag, int op_max)>;

template <int TB, class C, bool Hub, bool Multi>
static int dist_grid(int B) {
  const int smax = (int)round_smem<C, Hub>(round_max_block<C, Hub>());
  cudaFuncSetAttribute(k_persistent_dist<TB, C, Hub, Multi>, cudaFuncAttributeMaxDynamicSharedMemorySize, smax);
  int per_sm = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_persistent_dist<TB, C, Hub, Multi>, B,
                                                    round_smem<C, Hub>(B)) != cudaSuccess ||
      per_sm <= 0)
    per_sm = 1;
  return per_sm * num_sms();
}

template <int TB, class C>
static sgr_status run_dev(std::vector<DevPart>& parts, int nranks, int me0, int64_t n,
                          int32_t* colors_out, sgr_stats* stats, const PeerView* peers,
                          const XSync& xsync, const Resolved& r, int* overflow_out) {
  cudaStream_t s = r.stream;
  const int B = r.block;
  if (peers && !packed<C>()) {  // int32 replicas are not in the peer-mapped workspace
    set_error("sgr_color_dist: device exchange needs 16-bit words");
    return SGR_EUNSUPPORTED;
  }
  if (!block_ok(B, 64, round_max_block<C, true>())) {
    set_error("sgr_color_dist: block_size %d not supported by the round kernels", B);
    return SGR_EINVAL;
  }
  keep_pool_memory();
  const int P = (int)parts.size();
  std::vector<Layout> Ls;
  std::vector<RoundArgs<C>> args(P);
  for (int i = 0; i < P; ++i) {
    DevPart& pt = parts[i];
    Ls.push_back(layout(n, pt.nnz, r));
    if (!pt.ws) DCK(cudaMallocAsync(&pt.ws, Ls[i].total, s));
    if (!packed<C>() && (i > 0 || !colors_out)) {
      DCK(cudaMallocAsync((void**)&pt.colors, (size_t)n * 4, s));
      pt.own_colors = true;
    } else {
      pt.colors = colors_out;
    }
    sgr_csr shifted{pt.csr.row_ptr - pt.lo, pt.csr.col_idx};
    build_args<C>(args[i], &shifted, n, pt.nnz, pt.colors, pt.ws, Ls[i], r);
    args[i].v_begin = (int32_t)pt.lo;
    args[i].v_end = (int32_t)pt.hi;
    Ctrl hc;
    memset(&hc, 0, sizeof(hc));
    hc.k = 1;
    hc.max_rounds = r.max_rounds;
    DCK(cudaMemcpyAsync(args[i].ctrl, &hc, sizeof(Ctrl), cudaMemcpyHostToDevice, s));
    DCK(cudaMemsetAsync((char*)pt.ws + Ls[i].zero_begin, 0, Ls[i].zero_end - Ls[i].zero_begin, s));
  }
  // pointer tables: every part's (col[0], col[1]) of the OTHER replicas, all Ctrl, all
  // cross counters. Plain colors: replica i's col[0] is its colors buffer (not in ws), so
  // on several GPUs only packed words (both buffers in the workspace) can be peer-mapped.
  auto col_of = [&](int rank, int b) -> C* {
    if (peers) {
      char* w = (char*)peers->ws[rank];
      const size_t cb = align_up((size_t)n * sizeof(C), 256);
      return (C*)(w + Ls[0].off_col + (b ? cb : 0));
    }
    return args[rank].col[b];
  };
  auto ctrl_of = [&](int rank) -> Ctrl* {
    return peers ? (Ctrl*)peers->ws[rank] : args[rank].ctrl;
  };
  const int per = 2 * (nranks - 1) + 2 * nranks;  // pointers per part
  std::vector<void*> tab((size_t)per * P);
  for (int i = 0; i < P; ++i) {
    const int me = me0 + i;
    void** t = tab.data() + (size_t)per * i;
    int q = 0;
    for (int j = 0; j < nranks; ++j)
      if (j != me) {
        t[2 * q] = col_of(j, 0);
        t[2 * q + 1] = col_of(j, 1);
        ++q;
      }
    for (int j = 0; j < nranks; ++j) {
      t[2 * (nranks - 1) + j] = ctrl_of(j);
      t[2 * (nranks - 1) + nranks + j] = &ctrl_of(j)->xbar;
    }
  }
  void** dtab = nullptr;
  RoundArgs<C>* dargs = nullptr;
  int32_t* dflag = nullptr;
  DCK(cudaMallocAsync((void**)&dtab, tab.size() * sizeof(void*), s));
  DCK(cudaMallocAsync((void**)&dargs, sizeof(RoundArgs<C>) * P, s));
  DCK(cudaMallocAsync((void**)&dflag, 64, s));
  DCK(cudaMemcpyAsync(dtab, tab.data(), tab.size() * sizeof(void*), cudaMemcpyHostToDevice, s));
  for (int i = 0; i < P; ++i) {
    void** t = dtab + (size_t)per * i;
    args[i].rep = (C* const*)t;
    args[i].nrep = nranks - 1;
    args[i].rctrl = (Ctrl* const*)(t + 2 * (nranks - 1));
    args[i].xbar = (uint32_t* const*)(t + 2 * (nranks - 1) + nranks);
    args[i].nranks = nranks;
    args[i].me = me0 + i;
  }
  sgr_status status = SGR_OK;
  // every part's vertex range (host); boundary masks when <= 8 parts (SURVEY §8(e)
  // boundary filtering: a color word goes only to the replicas that read it)
  std::vector<int64_t> rg;
  if (peers) {
    rg = peers->ranges;
  } else {
    rg.push_back(parts[0].lo);
    for (auto& pt : parts) rg.push_back(pt.hi);
  }
  std::vector<uint8_t*> masks(P, nullptr);
  int64_t* dranges = nullptr;
  if (nranks > 1 && nranks <= 8) {
    // masks are used only when at most a quarter of the vertices are boundary vertices
    // (slab partitions of meshes): on skewed graphs nearly every vertex has remote
    // neighbours, and the per-store mask load would cost more than the stores it saves
    DCK(cudaMallocAsync((void**)&dranges, rg.size() * 8 + 8 * (size_t)P, s));
    unsigned long long* dbound = (unsigned long long*)(dranges + rg.size());
    DCK(cudaMemcpyAsync(dranges, rg.data(), rg.size() * 8, cudaMemcpyHostToDevice, s));
    DCK(cudaMemsetAsync(dbound, 0, 8 * (size_t)P, s));
    for (int i = 0; i < P; ++i) {
      const int64_t own = parts[i].hi - parts[i].lo;
      DCK(cudaMallocAsync((void**)&masks[i], (size_t)std::max<int64_t>(own, 1), s));
      const int gm = (int)std::max<int64_t>(1, std::min<int64_t>((own + 7) / 8, (int64_t)num_sms() * 16));
      k_remote_mask<C><<<gm, 256, 0, s>>>(args[i], dranges, masks[i], dbound + i);
    }
    DCK(cudaGetLastError());
    std::vector<unsigned long long> bound(P, 0);
    DCK(cudaMemcpyAsync(bound.data(), dbound, 8 * (size_t)P, cudaMemcpyDeviceToHost, s));
    DCK(cudaStreamSynchronize(s));
    // over this device's parts together: masks pay where boundary vertices are rare (a
    // slab's cut planes); on skewed graphs the store per remote replica is cheaper than a
    // mask load on every write (measured: R-MAT s16 on 8 parts 1.3 -> 2.5 ms with masks in
    // its sparse high-id parts)
    int64_t b_all = 0, own_all = 0;
    for (int i = 0; i < P; ++i) {
      b_all += (int64_t)bound[i];
      own_all += parts[i].hi - parts[i].lo;
    }
    if (4 * b_all <= own_all)
      for (int i = 0; i < P; ++i) args[i].rmask = masks[i];
  }
  // C_1 in both buffers of every replica, before any part broadcasts C_2 into it
  for (int i = 0; i < P; ++i) k_fill_c1<C><<<first_grid(n), 256, 0, s>>>(args[i]);
  DCK(cudaGetLastError());
  if (xsync && (status = xsync(s, dflag, 0)) != SGR_OK) return status;
  // F_1 per part (its C_2 words go into every replica), then the first advance
  for (int i = 0; i < P; ++i) {
    k_first<TB, C><<<first_grid(parts[i].hi - parts[i].lo), 256, 0, s>>>(args[i], r.sorted);
    k_advance<<<1, 32, 0, s>>>(args[i].ctrl, 1, 0);
  }
  DCK(cudaGetLastError());
  // the build every part runs: hub if any part put a vertex into bin 2 (all ranks agree)
  std::vector<int32_t> big(P, 0);
  for (int i = 0; i < P; ++i)
    DCK(cudaMemcpyAsync(&big[i], &args[i].ctrl->big_count, 4, cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  int32_t hub = 0;
  for (int32_t b : big) hub |= b != 0;
  if (xsync) {  // max over ranks; also orders every rank's F_1 broadcast before the rounds
    DCK(cudaMemcpyAsync(dflag, &hub, 4, cudaMemcpyHostToDevice, s));
    if ((status = xsync(s, dflag, 1)) != SGR_OK) return status;
    DCK(cudaMemcpyAsync(&hub, dflag, 4, cudaMemcpyDeviceToHost, s));
    DCK(cudaStreamSynchronize(s));
  }
  const bool multi = P > 1;
  const int gmax = hub ? (multi ? dist_grid<TB, C, true, true>(B) : dist_grid<TB, C, true, false>(B))
                       : (multi ? dist_grid<TB, C, false, true>(B) : dist_grid<TB, C, false, false>(B));
  const int gB = std::max(1, gmax / P);  // blocks per part
  const int grid = gB * P;
  for (int i = 0; i < P; ++i) {
    args[i].gfirst = gB * i;
    args[i].gnum = gB;
  }
  DCK(cudaMemcpyAsync(dargs, args.data(), sizeof(RoundArgs<C>) * P, cudaMemcpyHostToDevice, s));
  cudaEvent_t ev0, ev1;
  cudaEventCreate(&ev0);
  cudaEventCreate(&ev1);
  cudaEventRecord(ev0, s);
  {
    RoundArgs<C> a0 = args[0];
    const RoundArgs<C>* pa = dargs;
    int np = P;
    void* kargs[] = {(void*)&a0, (void*)&pa, (void*)&np};
    const void* fn = hub ? (multi ? (const void*)k_persistent_dist<TB, C, true, true>
                                  : (const void*)k_persistent_dist<TB, C, true, false>)
                         : (multi ? (const void*)k_persistent_dist<TB, C, false, true>
                                  : (const void*)k_persistent_dist<TB, C, false, false>);
    const cudaError_t le = cudaLaunchCooperativeKernel(fn, grid, B, kargs,
                                                       hub ? round_smem<C, true>(B) : round_smem<C, false>(B), s);
    if (le != cudaSuccess) return cuda_fail(le, "cooperative launch of k_persistent_dist", __LINE__);
  }
  cudaEventRecord(ev1, s);
  RoundArgs<C>& a0 = args[0];
  // every vertex's final color is exact in its owner's replica (other replicas only hold
  // the boundary vertices they read): assemble colors_out range by range, from the local
  // parts' replicas and (several GPUs) the peers' mapped ones
  for (int j = 0; j < nranks; ++j) {
    const int64_t lo = rg[j], len = rg[j + 1] - rg[j];
    if (len <= 0) continue;
    const int i = j - me0;  // local part index, if this device owns rank j
    const C* src = (i >= 0 && i < P) ? args[i].col[0] : col_of(j, 0);
    if constexpr (packed<C>()) {
      k_unpack<<<reduce_grid(len), 256, 0, s>>>(src + lo, colors_out + lo, len, &a0.ctrl->max_color);
    } else {
      if (src != (const C*)colors_out)
        DCK(cudaMemcpyAsync(colors_out + lo, src + lo, (size_t)len * 4, cudaMemcpyDeviceToDevice, s));
    }
  }
  if constexpr (!packed<C>()) k_max_color<<<reduce_grid(n), 256, 0, s>>>(colors_out, n, &a0.ctrl->max_color);
  DCK(cudaGetLastError());
  std::vector<Ctrl> fin(P);
  for (int i = 0; i < P; ++i)
    DCK(cudaMemcpyAsync(&fin[i], args[i].ctrl, sizeof(Ctrl), cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  // no rank may release its workspace while another can still read its counters
  if (xsync && (status = xsync(s, dflag, 0)) != SGR_OK) return status;
  int overflow = 0;
  for (int i = 0; i < P; ++i) overflow |= fin[i].overflow;
  if (overflow && !packed<C>()) {
    set_error("sgr_color_dist: 32-bit color overflow");
    status = SGR_EUNSUPPORTED;
  }
  if (overflow && packed<C>()) *overflow_out = 1;
  if (fin[0].status == 1 && !overflow) {
    set_error("sgr_color_dist: max_rounds (%d) reached", r.max_rounds);
    status = SGR_ENOCONV;
  }
  if (stats && status == SGR_OK) {
    memset(stats, 0, sizeof(*stats));
    int64_t nnz_parts = 0, verts = 0;
    for (int i = 0; i < P; ++i) {
      sgr_stats t;
      memset(&t, 0, sizeof(t));
      fill_stats(fin[i], 0, 0, &t, (int)sizeof(C));
      stats->edges_scanned += t.edges_scanned;
      stats->entries_read += t.entries_read;
      stats->entries_written += t.entries_written;
      stats->bytes_algorithmic += t.bytes_algorithmic;
      stats->chunk_items += t.chunk_items;
      verts += t.vertices_processed;
      for (int q = 0; q < 3; ++q) {
        stats->bin_vertices[q] += t.bin_vertices[q];
        stats->bin_edges[q] += t.bin_edges[q];
      }
      nnz_parts += parts[i].nnz;
    }
    stats->edges_scanned += nnz_parts;  // round 1 (this device's parts)
    stats->vertices_processed = verts + n * P / std::max(nranks, 1);
    stats->rounds = fin[0].k - 1;
    stats->num_colors = fin[0].max_color;
    stats->launches = 3 * P + 2;
    stats->grid_blocks = grid;
    stats->color_bits = packed<C>() ? 16 : 32;
    stats->transport = nranks > 1 ? SGR_XCHG_DEVICE : SGR_XCHG_NONE;
    cudaEventElapsedTime(&stats->elapsed_ms, ev0, ev1);
  }
  cudaEventDestroy(ev0);
  cudaEventDestroy(ev1);
  cudaFreeAsync(dtab, s);
  cudaFreeAsync(dargs, s);
  cudaFreeAsync(dflag, s);
  if (dranges) cudaFreeAsync(dranges, s);
  for (auto* m : masks)
    if (m) cudaFreeAsync(m, s);
  for (auto& pt : parts) {
    if (!peers) cudaFreeAsync(pt.ws, s);
    pt.ws = peers ? pt.ws : nullptr;
    if (pt.own_colors) cudaFreeAsync(pt.colors, s);
    pt.own_colors = false;
  }
  cudaStreamSynchronize(s);
  return status;
}

template <class... A>
static sgr_status dispatch_dev(const Resolved& r, A&&... args) {
  int overflow = 0;
  if (r.color_bits == 16) {
    const sgr_status st = r.tiebreak ? run_dev<1, Packed>(args..., r, &overflow)
                                     : run_dev<0, Packed>(args..., r, &overflow);
    if (st != SGR_OK || !overflow) return st;
  }
  Resolved r32 = r;
  r32.color_bits = 32;
  return r.tiebreak ? run_dev<1, int32_t>(args..., r32, &overflow)
                    : run_dev<0, int32_t>(args..., r32, &overflow);
}

// Packed (16-bit) words first; if any partition's first fit exceeded the color cap, every
// rank saw the flag in the same exchange and the whole coloring is redone with int32 words.
template <class... A>
static sgr_status dispatch(const Resolved& r, A&&... args) {
  int overflow = 0;
  if (r.color_bits == 16) {
    const sgr_status st = r.tiebreak ? run_parts<1, Packed>(args..., r, &overflow)
                                     : run_parts<0, Packed>(args..., r, &overflow);
    if (st != SGR_OK || !overflow) return st;
  }
  Resolved r32 = r;
  r32.color_bits = 32;
  return r.tiebreak ? run_parts<1, int32_t>(args..., r32, &overflow)
                    : run_parts<0, int32_t>(args..., r32, &overflow);
}

#if SGR_HAVE_NCCL
// Device-side exchange across GPUs (k_persistent_dist, one part per rank): the workspaces
// (replicas, counters) are cudaMalloc'd, their IPC handles all-gathered over NCCL and
// mapped into every rank (NVLink peer memory), so each rank's pass stores its color words
// straight into all replicas and the ranks meet at a device-side barrier. SGR_EUNSUPPORTED
// (the caller then uses the NCCL all-gather transport) when a peer cannot be mapped.
static sgr_status color_dist_device(DistComm* c, const sgr_csr* local, int64_t n, int64_t v_begin,
                                    int64_t v_end, int64_t nnz_local, int32_t* colors_out,
                                    sgr_stats* stats, const Resolved& r) {
  cudaStream_t s = r.stream;
  Resolved r16 = r;
  r16.color_bits = 16;
  const Layout L = layout(n, nnz_local, r16);
  std::vector<DevPart> dp(1);
  dp[0].lo = v_begin;
  dp[0].hi = v_end;
  dp[0].nnz = nnz_local;
  dp[0].csr = *local;
  if (c->world == 1) {  // no other replica: the rounds of one part, no exchange at all
    return dispatch_dev(r, dp, 1, 0, n, colors_out, stats, (const PeerView*)nullptr, XSync());
  }
  if (r.color_bits == 32) return SGR_EUNSUPPORTED;  // the same on every rank (same opts)
  void* ws = nullptr;
  DCK(cudaMalloc(&ws, L.total));  // IPC needs a cudaMalloc allocation
  cudaIpcMemHandle_t h;
  DCK(cudaIpcGetMemHandle(&h, ws));
  char* dh = nullptr;
  DCK(cudaMalloc((void**)&dh, sizeof(h) * (c->world + 1)));
  DCK(cudaMemcpy(dh + sizeof(h) * c->world, &h, sizeof(h), cudaMemcpyHostToDevice));
  ncclResult_t rc = ncclAllGather(dh + sizeof(h) * c->world, dh, sizeof(h), ncclChar, c->comm, s);
  std::vector<cudaIpcMemHandle_t> hs(c->world);
  if (rc == ncclSuccess) DCK(cudaMemcpyAsync(hs.data(), dh, sizeof(h) * c->world, cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  cudaFree(dh);
  if (rc != ncclSuccess) {
    cudaFree(ws);
    set_error("ncclAllGather (IPC handles): %s", ncclGetErrorString(rc));
    return SGR_ENCCL;
  }
  PeerView pv;
  pv.me = c->rank;
  {  // every rank's [v_begin, v_end): the ranges for the masks and the final assembly
    int64_t* dr = nullptr;
    DCK(cudaMalloc((void**)&dr, 16 * (size_t)(c->world + 1)));
    const int64_t mine[2] = {v_begin, v_end};
    DCK(cudaMemcpy(dr + 2 * c->world, mine, 16, cudaMemcpyHostToDevice));
    const ncclResult_t e = ncclAllGather(dr + 2 * c->world, dr, 2, ncclInt64, c->comm, s);
    std::vector<int64_t> all(2 * (size_t)c->world);
    if (e == ncclSuccess) DCK(cudaMemcpyAsync(all.data(), dr, 16 * (size_t)c->world, cudaMemcpyDeviceToHost, s));
    DCK(cudaStreamSynchronize(s));
    cudaFree(dr);
    if (e != ncclSuccess) {
      cudaFree(ws);
      set_error("ncclAllGather (ranges): %s", ncclGetErrorString(e));
      return SGR_ENCCL;
    }
    // the device path needs rank-ordered contiguous ranges covering V (what sgr_partition
    // gives); anything else takes the all-gather transport (every rank sees the same data)
    bool contiguous = all[0] == 0 && all[2 * (c->world - 1) + 1] == n;
    for (int q = 0; q + 1 < c->world; ++q) contiguous &= all[2 * q + 1] == all[2 * q + 2];
    if (!contiguous) {
      cudaFree(ws);
      return SGR_EUNSUPPORTED;
    }
    pv.ranges.push_back(all[0]);
    for (int q = 0; q < c->world; ++q) pv.ranges.push_back(all[2 * q + 1]);
  }
  pv.ws.assign(c->world, nullptr);
  pv.ws[c->rank] = ws;
  bool mapped = true;
  for (int q = 0; q < c->world && mapped; ++q) {
    if (q == c->rank) continue;
    if (cudaIpcOpenMemHandle(&pv.ws[q], hs[q], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
      cudaGetLastError();
      mapped = false;
    }
  }
  // every rank must take the same path: agree on the mapping outcome
  int32_t* dflag = nullptr;
  DCK(cudaMalloc((void**)&dflag, 4));
  int32_t ok = mapped ? 1 : 0;
  DCK(cudaMemcpy(dflag, &ok, 4, cudaMemcpyHostToDevice));
  rc = ncclAllReduce(dflag, dflag, 1, ncclInt32, ncclMin, c->comm, s);
  DCK(cudaMemcpyAsync(&ok, dflag, 4, cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  cudaFree(dflag);
  sgr_status st = SGR_EUNSUPPORTED;
  if (rc == ncclSuccess && ok) {
    dp[0].ws = ws;
    XSync xs = [c](cudaStream_t st2, int32_t* f, int op_max) -> sgr_status {
      const ncclResult_t e = ncclAllReduce(f, f, 1, ncclInt32, op_max ? ncclMax : ncclSum, c->comm, st2);
      if (e != ncclSuccess) {
        set_error("ncclAllReduce: %s", ncclGetErrorString(e));
        return SGR_ENCCL;
      }
      return SGR_OK;
    };
    int overflow = 0;
    st = r.tiebreak ? run_dev<1, Packed>(dp, c->world, c->rank, n, colors_out, stats, &pv, xs, r16, &overflow)
                    : run_dev<0, Packed>(dp, c->world, c->rank, n, colors_out, stats, &pv, xs, r16, &overflow);
    if (st == SGR_OK && overflow) st = SGR_EUNSUPPORTED;  // every rank saw it: int32 via NCCL
  }
  for (int q = 0; q < c->world; ++q)
    if (q != c->rank && pv.ws[q]) cudaIpcCloseMemHandle(pv.ws[q]);
  cudaFree(ws);
  return st;
}
#endif

}  // namespace sgr

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

sgr_status sgr_color_partitioned(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t P,
                                 const int64_t* ranges, int32_t* colors_out, sgr_stats* stats,
                                 const sgr_opts* opts) {
  if (!csr || n < 0 || nnz < 0 || P < 1 || !ranges || n >= ((int64_t)1 << 31)) return SGR_EINVAL;
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n == 0) return SGR_OK;
  if (!csr->row_ptr || !colors_out || (nnz > 0 && !csr->col_idx)) return SGR_EINVAL;
  if (((uintptr_t)csr->col_idx & 15u) != 0) {
    set_error("sgr_color_partitioned: col_idx must be 16-byte aligned");
    return SGR_EINVAL;
  }
  if (ranges[0] != 0 || ranges[P] != n) return SGR_EINVAL;
  for (int p = 0; p < P; ++p)
    if (ranges[p + 1] < ranges[p]) return SGR_EINVAL;
  const Resolved r = resolve_opts(opts, n);
  // local CSRs: offsets relative to the range's first row (host copy of row_ptr needed)
  std::vector<int64_t> rp(n + 1);
  if (cudaMemcpy(rp.data(), csr->row_ptr, (size_t)(n + 1) * 8, cudaMemcpyDeviceToHost) != cudaSuccess)
    return cuda_fail(cudaGetLastError(), "row_ptr D2H", __LINE__);
  std::vector<Part> parts(P);
  std::vector<int64_t*> local_rp(P, nullptr);
  std::vector<int32_t*> local_ci(P, nullptr);
  cudaStream_t s = r.stream;
  for (int p = 0; p < P; ++p) {
    Part& pt = parts[p];
    pt.lo = ranges[p];
    pt.hi = ranges[p + 1];
    const int64_t b = rp[pt.lo], e = rp[pt.hi];
    pt.nnz = e - b;
    std::vector<int64_t> lrp(pt.hi - pt.lo + 1);
    for (int64_t v = pt.lo; v <= pt.hi; ++v) lrp[v - pt.lo] = rp[v] - b;
    DCK(cudaMallocAsync((void**)&local_rp[p], lrp.size() * 8, s));
    DCK(cudaMallocAsync((void**)&local_ci[p], (size_t)std::max<int64_t>(pt.nnz, 4) * 4, s));
    DCK(cudaMemcpyAsync(local_rp[p], lrp.data(), lrp.size() * 8, cudaMemcpyHostToDevice, s));
    if (pt.nnz > 0)
      DCK(cudaMemcpyAsync(local_ci[p], csr->col_idx + b, (size_t)pt.nnz * 4, cudaMemcpyDeviceToDevice, s));
    DCK(cudaStreamSynchronize(s));  // lrp is a host temporary
    pt.csr = sgr_csr{local_rp[p], local_ci[p]};
  }
  sgr_status st;
  const char* hl = getenv("SGR_DIST_HOSTLOOP");
  if (!(hl && hl[0] == '1')) {
    // device-side exchange: one cooperative launch, a block group per partition, every
    // color word stored into all replicas (k_persistent_dist)
    std::vector<DevPart> dp(P);
    for (int p = 0; p < P; ++p) {
      dp[p].lo = parts[p].lo;
      dp[p].hi = parts[p].hi;
      dp[p].nnz = parts[p].nnz;
      dp[p].csr = parts[p].csr;
    }
    st = dispatch_dev(r, dp, P, 0, n, colors_out, stats, (const PeerView*)nullptr, XSync());
  } else {
    // host-driven rounds with an explicit all-gather (the NCCL transport's protocol) done by
    // device copies between the partitions of this device
    Gather gather = [](std::vector<Part>& ps, uint2* recv, int32_t cap, cudaStream_t st2) -> sgr_status {
      for (size_t q = 0; q < ps.size(); ++q)
        DCK(cudaMemcpyAsync(recv + q * (size_t)(cap + 1), ps[q].send, (size_t)(cap + 1) * sizeof(uint2),
                            cudaMemcpyDeviceToDevice, st2));
      return SGR_OK;
    };
    st = dispatch(r, parts, P, 0, n, colors_out, stats, gather, (int64_t)0);
  }
  for (int p = 0; p < P; ++p) {
    cudaFreeAsync(local_rp[p], s);
    cudaFreeAsync(local_ci[p], s);
  }
  cudaStreamSynchronize(s);
  return st;
}

sgr_status sgr_nccl_unique_id(void* id_out) {
#if SGR_HAVE_NCCL
  if (!id_out) return SGR_EINVAL;
  ncclUniqueId id;
  const ncclResult_t rc = ncclGetUniqueId(&id);
  if (rc != ncclSuccess) {
    set_error("ncclGetUniqueId: %s", ncclGetErrorString(rc));
    return SGR_ENCCL;
  }
  static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId size");
  memcpy(id_out, &id, sizeof(id));
  return SGR_OK;
#else
  (void)id_out;
  set_error("built without NCCL");
  return SGR_EUNSUPPORTED;
#endif
}

sgr_status sgr_comm_init(void** comm, int32_t rank, int32_t world, const void* id, int32_t device) {
  if (!comm || !id || world < 1 || rank < 0 || rank >= world) return SGR_EINVAL;
#if SGR_HAVE_NCCL
  if (cudaSetDevice(device) != cudaSuccess) return cuda_fail(cudaGetLastError(), "cudaSetDevice", __LINE__);
  DistComm* c = new DistComm();
  c->rank = rank;
  c->world = world;
  c->device = device;
  ncclUniqueId uid;
  memcpy(&uid, id, sizeof(uid));
  const ncclResult_t rc = ncclCommInitRank(&c->comm, world, uid, rank);
  if (rc != ncclSuccess) {
    delete c;
    set_error("ncclCommInitRank: %s", ncclGetErrorString(rc));
    return SGR_ENCCL;
  }
  *comm = c;
  return SGR_OK;
#else
  (void)device;
  set_error("built without NCCL");
  return SGR_EUNSUPPORTED;
#endif
}

sgr_status sgr_comm_destroy(void* comm) {
  if (!comm) return SGR_OK;
  DistComm* c = (DistComm*)comm;
#if SGR_HAVE_NCCL
  if (c->comm) ncclCommDestroy(c->comm);
#endif
  delete c;
  return SGR_OK;
}

sgr_status sgr_color_dist(void* comm, const sgr_csr* local, int64_t n_global, int64_t v_begin,
                          int64_t v_end, int64_t nnz_local, int32_t* colors_out, sgr_stats* stats,
                          const sgr_opts* opts) {
  if (!comm || !local || n_global < 0 || v_begin < 0 || v_end < v_begin || v_end > n_global ||
      nnz_local < 0 || n_global >= ((int64_t)1 << 31))
    return SGR_EINVAL;
  if (stats) memset(stats, 0, sizeof(*stats));
  if (n_global == 0) return SGR_OK;
  if (!local->row_ptr || !colors_out || (nnz_local > 0 && !local->col_idx)) return SGR_EINVAL;
  if (((uintptr_t)local->col_idx & 15u) != 0) {
    set_error("sgr_color_dist: col_idx must be 16-byte aligned");
    return SGR_EINVAL;
  }
#if SGR_HAVE_NCCL
  DistComm* c = (DistComm*)comm;
  const Resolved r = resolve_opts(opts, n_global);
  const char* tr = getenv("SGR_DIST_TRANSPORT");  // "nccl": the host-driven all-gather path
  if (!(tr && strcmp(tr, "nccl") == 0)) {
    const sgr_status ds = color_dist_device(c, local, n_global, v_begin, v_end, nnz_local,
                                            colors_out, stats, r);
    if (ds != SGR_EUNSUPPORTED) return ds;
    // no peer access between the ranks' GPUs (or int32 words needed): NCCL transport below
  }
  std::vector<Part> parts(1);
  parts[0].lo = v_begin;
  parts[0].hi = v_end;
  parts[0].nnz = nnz_local;
  parts[0].csr = *local;
  // every rank must size its buffers by the LARGEST range: agree on it first
  int64_t* d_sz = nullptr;
  cudaStream_t s = r.stream;
  DCK(cudaMallocAsync((void**)&d_sz, 8 * (size_t)(c->world + 1), s));
  const int64_t mine = v_end - v_begin;
  DCK(cudaMemcpyAsync(d_sz + c->world, &mine, 8, cudaMemcpyHostToDevice, s));
  ncclResult_t rc = ncclAllGather(d_sz + c->world, d_sz, 1, ncclInt64, c->comm, s);
  if (rc != ncclSuccess) {
    set_error("ncclAllGather: %s", ncclGetErrorString(rc));
    return SGR_ENCCL;
  }
  std::vector<int64_t> sizes(c->world);
  DCK(cudaMemcpyAsync(sizes.data(), d_sz, 8 * (size_t)c->world, cudaMemcpyDeviceToHost, s));
  DCK(cudaStreamSynchronize(s));
  cudaFreeAsync(d_sz, s);
  Gather gather = [c](std::vector<Part>& ps, uint2* recv, int32_t cap, cudaStream_t st) -> sgr_status {
    const ncclResult_t e = ncclAllGather(ps[0].send, recv, (size_t)(cap + 1) * 2, ncclUint32,
                                         c->comm, st);
    if (e != ncclSuccess) {
      set_error("ncclAllGather: %s", ncclGetErrorString(e));
      return SGR_ENCCL;
    }
    return SGR_OK;
  };
  // partitions on other ranks may be larger than ours: every buffer is sized by the
  // largest range, so all ranks use the same padded record counts
  int64_t cap_all = 0;
  for (int64_t z : sizes) cap_all = std::max(cap_all, z);
  return dispatch(r, parts, c->world, c->rank, n_global, colors_out, stats, gather, cap_all);
#else
  (void)comm; (void)local; (void)n_global; (void)v_begin; (void)v_end; (void)nnz_local;
  (void)colors_out; (void)stats; (void)opts;
  set_error("built without NCCL");
  return SGR_EUNSUPPORTED;
#endif
}

}  // extern "C"
