// sgr_round.cuh — sm_100a kernels of the deterministic SGR round.
//
// One fused pass F_k per round k >= 2 computes, for every v in W_k (Alg. 5):
//   conflict(v) = exists w in adj(v): X[w] == X[v] and lose(v, w)     (Alg. 5 l.12-15)
//   tent(v)     = min{c > 0 : c not in {X[w] : w in adj(v)}}            (Alg. 5 l.4-8)
//   Y[v]        = conflict(v) ? tent(v) : X[v];  v joins W_{k+1} iff conflict(v)
// X = C_k is round k's color snapshot and Y the ping-pong buffer: it holds C_{k-1}, which
// differs from C_{k+1} only inside W_k, exactly the set the pass writes (DESIGN.md §3,
// proof (iv)). Detection of round k and assignment of round k+1 read the same snapshot, so
// one adjacency scan serves both. F_1 needs no color gathers (every color is 1).
//
// The pass is bound by the rate of scattered color gathers (~1 distinct 128-byte line per
// SM-cycle, tools/gather_bench.cu) and by load latency. Work binning is static:
//   bin 0  deg <= small_max (<= 32): 4 lanes per vertex (coalesced row reads), <= 8 entries
//          per lane, the next vertex's row loaded while the current one's gathers are in
//          flight, u64 register mask per lane, OR-reduced in-group
//   bin 1  deg <= med_max (<= 256): 8 lanes per vertex, <= 32 entries per lane, 512-byte
//          forbidden table (one byte per color) in shared memory
//   bin 2  larger rows, one warp per chunk of <= kChunk entries of the vertex's (trimmed)
//          list, staged into shared memory by TMA; lane L gathers slots 32 j + L, so one
//          gather instruction reads 32 consecutive (sorted) neighbours. A vertex with several
//          chunks merges the chunks' 1024-bit partial sets with atomicOr and is decided in a
//          finalize phase after a grid barrier (one lane per vertex).
//
// Live-neighbour trimming (bin 2, packed colors; DESIGN.md §3 proof (vii)): a neighbour
// that has left the worklist never changes color again. Colors are stored as 16-bit words
// (last round the vertex was in W, mod 16) << 12 | color, so one gather also says whether
// the neighbour is still live (last == k mod 16; a neighbour that left exactly 16 r rounds
// ago looks live and is kept one more round, which is harmless: only live neighbours must
// never be dropped). Each bin-2 vertex keeps its adjacency list in a
// double-buffered copy adj[2] (same offsets as col_idx) and a 1024-bit set F of the colors
// of the neighbours it has dropped; every pass reads the current list, drops the neighbours
// that are no longer live (their colors go to F), and writes the compacted list for the
// next round. Conflict and first fit are computed from F ∪ {colors of the listed
// neighbours}, exactly the colors of all neighbours. Lists may also keep neighbours that
// have left W (that is the untrimmed semantics), so they are only rewritten when more than
// 1/16 of their entries are dead (single chunk: in place; several chunks: a keep bit per
// item, decided in the finalize phase). The chunk windows of the lists are
// staged into shared memory with TMA bulk copies (cp.async.bulk, mbarrier completion),
// double-buffered per warp so the next chunk streams in while the current chunk's gathers
// are in flight.
// Worklist pushes: warp ballot + popc + one atomicAdd per warp.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "sgr_common.cuh"

#ifndef SGR_QB
#define SGR_QB 2  // bin-2 batch: kJB = 4 * SGR_QB window slots per lane (32 kJB per warp)
#endif
constexpr int kQB = SGR_QB;
constexpr int kJB = 4 * kQB;  // entries per lane per batch
#ifndef SGR_NO_TMA
#define SGR_NO_TMA 0
#endif
#ifndef SGR_LAZY
#define SGR_LAZY 4  // bin 2 single-chunk lists: rewrite only if > cnt >> SGR_LAZY entries dropped
#endif
#ifndef SGR_MCLAZY
#define SGR_MCLAZY 1  // multi-chunk lists: keep uncompacted while <= 1/16 of entries are dead
#endif
#ifndef SGR_MCLAZY_SHIFT
#define SGR_MCLAZY_SHIFT 4  // dead-entry threshold: len >> SGR_MCLAZY_SHIFT
#endif
#ifndef SGR_CLRMAX
#define SGR_CLRMAX 1  // bin 2: clear the chunk's tables only up to the largest color seen
#endif
// Small-color passes: pass k reads C_k, whose colors are <= k (round 1 colors everything 1
// and a first fit is at most one above the largest neighbour color), so for k <= 62 every
// forbidden set fits a 64-bit register mask: bins 1 and 2 OR bits into registers and
// reduce them across lanes instead of storing bytes into shared tables and scanning them.
#ifndef SGR_SMALLMASK
#define SGR_SMALLMASK 1
#endif
// Early exit of bin-2 chunk scans (small passes): once a vertex is known to conflict and
// every color 1..k is forbidden (fixed set | colors seen so far; C_k holds no color above
// k), its first fit is k + 1 whatever the rest of its list holds, so the chunk's remaining
// batches are not gathered. Their entries stay listed (counted live: the lazy-trimming
// semantics of a listed neighbour that has left W). Chunks of a multi-chunk vertex share
// their progress through the slot's accumulators (colors 0..63 as one 64-bit word, the
// conflict flag), read back one batch later.
#ifndef SGR_EARLY
#define SGR_EARLY 0  // measured: cfg4 35.0 -> 35.9 ms (entries read -6 %), off
#endif
#ifndef SGR_B2_STATIC
#define SGR_B2_STATIC 0  // experiments: bin-2 items round-robin (no cursor claims)
#endif
#ifndef SGR_EARLY_MC
#define SGR_EARLY_MC 1  // early exit for multi-chunk vertices too (shared progress)
#endif
#ifndef SGR_TRACE_ENTRIES
#define SGR_TRACE_ENTRIES 0
#endif
#ifndef SGR_BARSLEEP
#define SGR_BARSLEEP 20  // grid-barrier poll back-off (ns); 0 = spin
#endif
#ifndef SGR_B1_BATCH_HUB
#define SGR_B1_BATCH_HUB 8  // bin 1, hub build: row entries per lane per batch (8 or 16)
#endif
#ifndef SGR_SMALL_FIRST
#define SGR_SMALL_FIRST 0  // pass order 0, 1, 2 instead of 2, 1, 0
#endif
#ifndef SGR_HUB_B0T
#define SGR_HUB_B0T 0  // hub build: thread-per-vertex bin 0
#endif
#ifndef SGR_BIN0_THREAD
#define SGR_BIN0_THREAD 0  // bin 0: one thread per vertex (else 4-lane groups)
#endif
#ifndef SGR_DENSE_SPAN
#define SGR_DENSE_SPAN 16  // dense passes only if the mean row width is below n / 16
#endif
#ifndef SGR_SMALL_U8
#define SGR_SMALL_U8 1  // bin 0 (4-lane groups), passes k <= 255: byte gathers + shl masks
#endif
#ifndef SGR_FLAT_B0T
#define SGR_FLAT_B0T 1  // flat build, non-local rows: thread-per-vertex bin 0 (runtime choice)
#endif

namespace sgr {

constexpr int kBins = 3;
constexpr int kBlock = 256;             // default threads per block (8 warps; opts->block_size)
constexpr int kWarps = kBlock / 32;
constexpr int kMaxWarps = 32;           // static per-warp arrays: any block up to 1024 threads
constexpr int kGroup = 8;               // lanes per vertex in bins 0 and 1
constexpr int kG0 = 4;                  // lanes per vertex in bin 0
constexpr int kK0 = 8;                  // entries per lane, bin 0 (4 x 8 = 32 = max small)
constexpr int kMaxSmall = kG0 * kK0;    // 32
// Per-warp push buffer of bins 0/1 (int32 entries), flushed with one atomicAdd once it
// holds >= size - 32 entries. The flat build (stencils, ER: most processed vertices conflict
// again, so the two list counters take an atomic per 32 pushes from every warp) uses a
// larger buffer: stencil -6.6 %, ER +1.8 %; the hub build keeps 64 (larger: +0.3 %).
#ifndef SGR_PUSHBUF
#define SGR_PUSHBUF 64
#endif
#ifndef SGR_PUSHBUF_FLAT
#define SGR_PUSHBUF_FLAT 256
#endif
template <bool Hub>
constexpr int kPushBufOf = Hub ? SGR_PUSHBUF : SGR_PUSHBUF_FLAT;
constexpr int kPushBuf = SGR_PUSHBUF;
constexpr int kK1 = 32;                 // entries per lane, bin 1 (8 x 32 = 256)
constexpr int kMaxMed = kGroup * kK1;   // 256
constexpr int kTile0 = 8;               // bin-0 tiles: <= 8 steps of 8 vertices
constexpr int kTile1 = 4;               // bin-1 tiles: <= 4 steps of 4 vertices
// Forbidden-color sets in shared memory: SGR_BITTBL = 1 one bit per color (shared atomicOr),
// 0 one byte per color (plain byte stores). Bit sets leave more of the SM's unified
// L1/shared storage to the L1 cache that serves the color gathers.
#ifndef SGR_BITTBL
#define SGR_BITTBL 0
#endif
constexpr int kMedTbl = 512;            // bin-1 set: colors < 512 (first fit <= 257)
constexpr int kBigTbl = 1024;           // bin-2 set: colors < 1024
constexpr int kTblDiv = SGR_BITTBL ? 8 : 1;
constexpr int kMedTblB = kMedTbl / kTblDiv;  // bytes
constexpr int kBigTblB = kBigTbl / kTblDiv;
constexpr int kTblBytes = 2 * kBigTblB;      // per-warp tables: 4 x bin-1 | 2 x bin-2
#ifndef SGR_WIN
#define SGR_WIN 1024
#endif
constexpr int kWin = SGR_WIN;           // window entries (32 lanes x kWin / 128 int4)
constexpr int kChunk = kWin - 4;        // bin-2 chunk: entries per warp item; the 16-byte-
                                        // aligned window (<= kWin entries) covers it
static_assert(kWin == 512 || kWin == 768 || kWin == 1024, "window: 512, 768 or 1024 entries");

// Working color word. Packed (default): uint16_t = (last round mod 16) << 12 | color, color
// <= 4095 (a larger first fit sets the overflow flag and the coloring is redone with plain
// int32 words, which have no round field and no trimming).
using Packed = uint16_t;
constexpr uint32_t kColorMask = 0xfffu;
constexpr int kRoundShift = 12;
template <class C>
__host__ __device__ constexpr bool packed() { return sizeof(C) == 2; }

// Two builds of the round kernels: Hub (bins 0-2) and flat (bins 0-1 only), chosen per
// coloring by whether F_1 put any vertex into bin 2 (bins are static, so then bin 2 stays
// empty). The flat build needs no TMA stages, so it leaves most of the SM's unified
// L1/shared storage to the L1 cache that serves the color gathers, and runs 3 blocks/SM.
//
// dynamic shared memory per warp: [2 TMA stages (Hub, packed)] [tables] [push buffer]
// [bin-2 item buffer, 2 mbarriers (Hub)]
constexpr int kStage = kWin * 4;        // bytes per TMA stage: one bin-2 window
// blocks per SM the round kernels are compiled for: the packed Hub build is shared-memory
// bound to 2 (86 KB per block); the others can afford 3 (<= 85 registers)
#ifndef SGR_MINB
#define SGR_MINB 2
#endif
#ifndef SGR_FLATB
#define SGR_FLATB 3
#endif
template <class C, bool Hub = true>
constexpr int kMinBlocks = (packed<C>() && Hub) ? SGR_MINB : (Hub ? 3 : SGR_FLATB);
// Launch bounds of the round kernels: the register budget of kMinBlocks 256-thread blocks
// per SM (packed hub build 2 -> 128 registers, the others 3 -> 85), expressed as ONE block
// of up to kMaxThreads threads, so any block size up to that (opts->block_size, the
// paper's Fig. 8 parameter) launches with the same per-thread register allocation.
#ifndef SGR_HUB_MAXT
#define SGR_HUB_MAXT 0  // experiments: override the packed hub build's threads-per-SM budget
#endif
template <class C, bool Hub = true>
constexpr int kMaxThreads = (SGR_HUB_MAXT && packed<C>() && Hub) ? SGR_HUB_MAXT : kBlock * kMinBlocks<C, Hub>;
// Dense passes of the flat build stage a warp step's 32 rows in the warp's shared memory
// (its tables and push buffer, unused by those passes): at least this many entries, so 32
// rows of the small bin (<= 32 entries each, 16-byte window alignment included) fit.
#ifndef SGR_DENSE_CAP
#define SGR_DENSE_CAP 1056
#endif
template <class C, bool Hub = true> struct WarpSmem {
  static constexpr int kBuf = (packed<C>() && Hub) ? 2 * kStage : 0;
  static constexpr int kPush = kBuf + kTblBytes;         // push buffer (kPushBuf int32)
  static constexpr int kItems = kPush + kPushBufOf<Hub> * 4;  // bin-2 item buffer (32 int64)
  static constexpr int kBars = kItems + (Hub ? 32 * 8 : 0);  // 2 mbarriers
  static constexpr int kUsed = kBars + (Hub ? 16 : 0);
  static constexpr int kBytes = Hub ? kUsed : (kUsed > 4 * SGR_DENSE_CAP ? kUsed : 4 * SGR_DENSE_CAP);
};

// Work counts of one worklist W_k (32 bytes: one pair of vector loads).
struct alignas(32) Counts {
  int32_t t;                 // bin 0 vertices
  int32_t m;                 // bin 1 vertices
  int32_t c;                 // bin 2 chunk items
  int32_t cv;                // bin 2 vertices
  int32_t fin;               // pass k: multi-chunk bin-2 vertices awaiting the finalize phase
  int32_t pad[3];            // pad[0]: pass k's bin-2 work cursor; pad[1]: multi-chunk
                             // vertices in W_k (0: pass k needs no finalize phase)
};
// W_k's counts live in ring slot k % 3: pass k reads slot k % 3 and pushes W_{k+1} into
// slot (k+1) % 3, while slot (k+2) % 3 (W_{k-1}, read by the finished pass k-1) is folded
// into the totals and zeroed. So no single thread has to advance anything between passes:
// after the barrier every block reads the next counts itself.
__host__ __device__ __forceinline__ int rs(int k) { return k % 3; }

// Device-resident loop state (in the workspace).
struct Ctrl {
  int32_t k;                 // index of the next fused pass F_k (k = 2 after F_1)
  int32_t active;            // 1 while W_k is non-empty (host / graph loop modes)
  int32_t status;            // 0 ok, 1 = max_rounds reached with W non-empty
  int32_t max_rounds;
  int32_t overflow;          // a packed color exceeded 12 bits (4095)
  int32_t round_cap;
  uint32_t bar_count;        // grid barrier (persistent kernel)
  uint32_t bar_gen;
  int32_t big_count;         // slots handed to bin-2 vertices by F_1
  int32_t max_color;
  int32_t violations;
  uint32_t xbar;             // cross-part barrier counter (k_persistent_dist; other parts add)
  int32_t cmp_cnt[2];        // bitmap -> worklist compaction (dense -> sparse): bin cursors
  int32_t dcol_bad;          // k_dense: some w - v does not fit 16 bits (dcol unusable)
  int32_t pad;
  unsigned long long span_sum;  // F_1: sum over rows of (last - first entry) — row locality
  Counts ring[3];
  unsigned long long edges_acc[3][kBins];    // per ring slot: sum of deg(v) over the pass's
  unsigned long long entries_acc[3][kBins];  // vertices / list entries actually read
  unsigned long long verts_total[kBins + 1];   // [kBins] = F_1
  unsigned long long edges_total[kBins + 1];
  unsigned long long entries_total[kBins + 1];
  unsigned long long pushes_total[kBins + 1];
  unsigned long long items_total;
  unsigned long long list_writes_total;   // compacted list entries written (bin 2, packed)
  unsigned long long bin_cycles[kBins];   // warp-cycles spent in each bin (SM clock)
  int32_t tile_cur[3][2];                // per ring slot: bin-0 / bin-1 tile cursors
  unsigned long long phase_cycles[8];     // bin 2 (trimmed) phases: issue, wait, gather, post;
                                          // [4] grid barriers, [5] finalize, [6] counters
  int32_t* round_sizes;
  int64_t* round_edges;
  int64_t* round_ns;          // %globaltimer at the end of each pass (profiling)
};

template <class C>
struct RoundArgs {
  const int64_t* row_ptr;
  const int32_t* col_idx;
  C* col[2];                  // color ping-pong: C_k lives in col[(k - 1) & 1]
  int32_t* wl_t[2];           // bin 0 vertex lists, W_k in [k & 1]
  int32_t* wl_m[2];           // bin 1 vertex lists
  int64_t* wl_c[2];           // bin 2 chunk items: (v << 32) | chunk
  int32_t* big_id;            // slot of each bin-2 vertex (F_1)
  uint32_t* acc_bits;         // [slot][32] partial forbidden sets of the running pass
  unsigned long long* acc_cnt;  // [slot] chunks finished | conflicts << 32
  int32_t* adj[2];            // trimmed adjacency lists (packed mode), offsets = row_ptr
  int32_t* len[2];            // [v] list length for the pass of parity p
  uint32_t* fixed;            // [slot][32] colors of dropped (finalized) neighbours
  int64_t* fin;               // finalize list: multi-chunk vertices of the pass
                              // (slot << 32 | buf << 31 | v)
  uint32_t* bm[2];            // worklist membership bitmaps (flat build's dense passes): W_k
  int16_t* dcol;              // dense passes: w - v per CSR entry (aliases adj[0], which only
                              // the hub build uses), nullptr when unavailable
                              // in bm[k & 1], bit v & 31 of word v >> 5
  Ctrl* ctrl;
  int64_t nnz;
  int32_t n;
  int32_t small_max;
  int32_t med_max;
  int32_t v_begin;            // owned vertex range [v_begin, v_end) (multi-GPU: a partition)
  int32_t v_end;
  int32_t color_cap;          // packed mode: largest color a 16-bit word holds (<= 4095)
  // Device-side exchange (k_persistent_dist): every color word this part
  // writes for its own vertices is also stored into the other replicas (other partitions
  // of this device, or NVLink peer memory of other GPUs), so no exchange step exists.
  C* const* rep;              // [2 * nrep]: replica q's (col[0], col[1]); nullptr: none
  int32_t nrep;
  int32_t gfirst, gnum;       // this part's block group in a multi-part launch (gnum 0: grid)
  int32_t nranks, me;         // parts / ranks taking part in the coloring, this one's index
  Ctrl* const* rctrl;         // [nranks] every part's Ctrl (own included): global counts
  uint32_t* const* xbar;      // [nranks] every part's cross-part barrier counter
  // Boundary filtering: bit q of rmask[v - v_begin] is set iff part q owns a
  // neighbour of v, i.e. replica q will ever read v's color; interior vertices (mask 0) are
  // written to the own replica only. nullptr: broadcast to every replica (> 8 parts).
  const uint8_t* rmask;
  int32_t flat_bin0;          // opts->flat_bin0: 0 automatic, 1 4-lane groups, 2 thread per vertex
};

// This part's block group: the whole grid, or (multi-part launch) blocks
// [gfirst, gfirst + gnum).
template <class C>
__device__ __forceinline__ int grp_block(const RoundArgs<C>& a) {
  return a.gnum ? (int)blockIdx.x - a.gfirst : (int)blockIdx.x;
}
template <class C>
__device__ __forceinline__ int grp_size(const RoundArgs<C>& a) { return a.gnum ? a.gnum : (int)gridDim.x; }

// Parameter-struct selects without dynamic indexing (which would spill it to the stack).
template <class T>
__device__ __forceinline__ T sel(int par, T a0, T a1) { return par ? a1 : a0; }

__device__ __forceinline__ int32_t ld_cg(const int32_t* p) { return __ldcg(p); }
__device__ __forceinline__ uint32_t ld_cg(const uint32_t* p) { return __ldcg(p); }

// ---- color words: int32_t = plain color; Packed = (last round mod 16) << 12 | color ------
// Snapshot reads. A per-pass launch may use the read-only path (the buffer is not written
// while it runs). The persistent kernel writes each buffer in alternate passes, so its
// reads must be coherent: SGR_GATHER_CA = 0 reads at L2 (ld.global.cg); 1 uses plain
// L1-cached loads, relying on the PTX memory model: every pass starts after the grid
// barrier's ld.acquire.gpu (thread 0) + bar.sync, which orders these weak loads after the
// previous pass's writes (the acquire invalidates the SM's L1).
#ifndef SGR_GATHER_CA
#define SGR_GATHER_CA 1
#endif
template <bool Persist, class C>
__device__ __forceinline__ uint32_t ldraw(const C* p) {
  if constexpr (Persist) {
#if SGR_GATHER_CA
    return (uint32_t)*p;
#else
    return (uint32_t)__ldcg(p);
#endif
  } else {
    return (uint32_t)__ldg(p);
  }
}
// Bin-2 neighbour gathers (hub lists: scattered over the whole color array) at L2 only:
// they would otherwise allocate L1 lines that are rarely reused, evicting the lines that
// the bin-0/1 gathers and the row reads do reuse (cfg4 -3.6 %, ER -2 % measured with all
// gathers at L2; the stencil's bin-0 gathers need L1: +8 % there). Coherent either way.
#ifndef SGR_B2_CG
#define SGR_B2_CG 1
#endif
template <bool Persist, class C>
__device__ __forceinline__ uint32_t ldraw_b2(const C* p) {
  if constexpr (Persist && SGR_B2_CG) return (uint32_t)__ldcg(p);
  else return ldraw<Persist>(p);
}
template <class C>
__device__ __forceinline__ int32_t cval(uint32_t raw) {
  if constexpr (packed<C>()) return (int32_t)(raw & kColorMask);
  else return (int32_t)raw;
}
template <bool Persist, class C>
__device__ __forceinline__ int32_t ldc(const C* p) { return cval<C>(ldraw<Persist>(p)); }
// Bins 0/1 in the hub build (skewed graphs: rows of scattered small-degree vertices) gather
// at L2 as well (cfg4 a further -1.1 %); the flat build (no bin 2: stencils, ER) keeps them
// L1-cached, where stencil neighbours share lines across vertices (L2-only: +8 %).
#ifndef SGR_HUB01_CG
#define SGR_HUB01_CG 1
#endif
template <bool Persist, bool Hub, class C>
__device__ __forceinline__ int32_t ldc01(const C* p) {
  if constexpr (Persist && Hub && SGR_HUB01_CG) return cval<C>((uint32_t)__ldcg(p));
  else return cval<C>(ldraw<Persist>(p));
}
// The color as a byte: in passes k <= 255 every color of C_k is <= k, so a word's low byte
// (little endian) is its color — no decode. Same cache path as ldc01.
template <bool Persist, bool Hub, class C>
__device__ __forceinline__ uint32_t ldc8(const C* p) {
  const unsigned char* b = reinterpret_cast<const unsigned char*>(p);
  if constexpr (Persist && ((Hub && SGR_HUB01_CG) || !SGR_GATHER_CA)) return (uint32_t)__ldcg(b);
  else if constexpr (Persist) return (uint32_t)*b;
  else return (uint32_t)__ldg(b);
}

template <class C>
__device__ __forceinline__ C cpack(int32_t color, int32_t last, const RoundArgs<C>& a) {
  if constexpr (packed<C>()) {
    if (color > a.color_cap) {  // color_cap = 4095 unless a test lowers it
      a.ctrl->overflow = 1;
      return (C)kColorMask;
    }
    return (C)((((uint32_t)last & 15u) << kRoundShift) | (uint32_t)color);
  } else {
    (void)last;
    (void)a;
    return (C)color;
  }
}

// Y[v] = word, and the same word into every other replica's buffer of that parity (pass
// k writes col[k & 1]; F_1's C_2 is parity 1). Other parts never write v (only its owner
// does) and read that buffer only as the NEXT pass's snapshot, after the pass barrier.
template <class C>
__device__ __forceinline__ void put_y(const RoundArgs<C>& a, C* Y, int k, int32_t v, C word) {
  Y[v] = word;
  if (a.nrep) {
    const uint32_t mk = a.rmask ? (uint32_t)a.rmask[v - a.v_begin] : 0xffffffffu;
    for (int q = 0; q < a.nrep; ++q) {
      const int rank = q < a.me ? q : q + 1;  // rep[] skips this part's own replica
      if ((mk >> rank) & 1u) a.rep[2 * q + (k & 1)][v] = word;
    }
  }
}

// rmask of the owned vertices: OR over each row of the bit of the part owning the neighbour
// (ranges: nranks + 1 boundaries, device memory), the own part excluded; one warp per
// vertex (hub rows are long). *boundary counts the owned vertices with a nonzero mask.
template <class C>
__global__ void k_remote_mask(RoundArgs<C> a, const int64_t* __restrict__ ranges, uint8_t* mask,
                              unsigned long long* boundary) {
  const int lane = threadIdx.x & 31;
  const int64_t wpb = blockDim.x >> 5;
  unsigned long long cnt = 0;
  for (int64_t v = a.v_begin + (int64_t)blockIdx.x * wpb + (threadIdx.x >> 5); v < a.v_end;
       v += (int64_t)gridDim.x * wpb) {
    uint32_t m = 0;
    const int64_t e = ldg_i64(a.row_ptr + v + 1);
    for (int64_t j = ldg_i64(a.row_ptr + v) + lane; j < e; j += 32) {
      const int64_t w = ld_ro(a.col_idx + j);
      int q = 0;
      while (q + 1 < a.nranks && __ldg(ranges + q + 1) <= w) ++q;  // <= 8 parts: linear
      m |= 1u << q;
    }
    m = __reduce_or_sync(0xffffffffu, m) & ~(1u << a.me);
    if (lane == 0) {
      mask[v - a.v_begin] = (uint8_t)m;
      cnt += m ? 1ull : 0ull;
    }
  }
  block_add(cnt, boundary);
}

__device__ __forceinline__ int bin_of(int64_t d, int small_max, int med_max) {
  return d <= small_max ? 0 : (d <= med_max ? 1 : 2);
}

__device__ __forceinline__ int32_t num_chunks(int64_t len) {
  return (int32_t)((len + kChunk - 1) / kChunk);
}

__device__ __forceinline__ void prefetch_l2(const void* p) {
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p));
}

// Release / acquire fence at GPU scope (lighter than the fence.sc.gpu of __threadfence()).
// Phase-cycle accounting (SM clock per bin / bin-2 phase; experiments only, stats
// bin_warp_cycles): compiled out unless SGR_PHASE_CYCLES=1, so the production kernel
// carries no clock reads or counter atomics for it.
#ifndef SGR_PHASE_CYCLES
#define SGR_PHASE_CYCLES 0
#endif
__device__ __forceinline__ long long pclock() {
#if SGR_PHASE_CYCLES
  return clock64();
#else
  return 0;
#endif
}

__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }

__device__ __forceinline__ int64_t make_item(int32_t v, int32_t c) {
  return (int64_t)(((uint64_t)(uint32_t)v << 32) | (uint32_t)c);
}
// Bin-2 items of the trimmed mode carry the adjacency buffer holding the vertex's list in
// bit 31 of the chunk field.
constexpr uint32_t kBufBit = 0x80000000u;
// Multi-chunk items of a list kept uncompacted this pass (SGR_MCLAZY): its chunks leave the
// list where it is (dead entries included) and only count their live entries; the finalize
// phase decides from the dead fraction whether the next pass compacts it.
constexpr uint32_t kKeepBit = 0x40000000u;
constexpr uint32_t kChunkMask = 0x3fffffffu;

// Ticket increment with release+acquire semantics at GPU scope: every write this thread
// (and, through the preceding __syncwarp, its warp) made is visible to whoever observes
// the new count, and this thread observes the others'.
__device__ __forceinline__ unsigned long long atom_add_acq_rel(unsigned long long* p,
                                                               unsigned long long v) {
  unsigned long long r;
  asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;" : "=l"(r) : "l"(p), "l"(v) : "memory");
  return r;
}
// Work-cursor claim by one lane: inline PTX so the compiler does not turn it into a
// warp-aggregated atomic whose result broadcast (a shuffle right after the atomic) waits
// for the round trip at the claim; the caller consumes the result one work item later
// (ncu, cfg4: 4.5 % of the round kernel's stall samples sat on that shuffle).
// (a lane-dependent address, equal to p on lane 0, the one lane that executes it, keeps
// ptxas from proving the address warp-uniform)
__device__ __forceinline__ int lane0_add(int* p, int v) {
  uint32_t lt;
  asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(lt));
  int* q = p + lt;  // lane 0: lanemask_lt = 0, q == p
  int r;
  asm volatile("atom.relaxed.gpu.global.add.s32 %0, [%1], %2;" : "=r"(r) : "l"(q), "r"(v));
  return r;
}
__device__ __forceinline__ int claim_add(int* p) { return lane0_add(p, 1); }
// Generic-proxy global writes before later async-proxy (TMA) reads of the same locations.
__device__ __forceinline__ void fence_proxy_async_global() {
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

// ---- TMA bulk copies + mbarriers (Blackwell async proxy) -------------------------------
__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_init_fence() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
#ifndef SGR_L2HINT
#define SGR_L2HINT 1
#endif
#ifndef SGR_ROWNA
#define SGR_ROWNA 0
#endif
// One elected thread: announce `bytes` of transaction and start the bulk copy global->smem.
// SGR_L2HINT: the lists stream through L2 with evict-first priority (they are read once
// per pass), so the color arrays the gathers hit stay resident.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes,
                                            uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
               : "memory");
#if SGR_L2HINT
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1], %2, [%3], %4;" ::"r"(smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar)), "l"(pol)
      : "memory");
#else
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
#endif
}

// Row entries of bins 0 and 1 (streamed once per pass). SGR_ROWNA: bypass L1 allocation,
// leaving L1 to the color gathers.
// Row entries of bins 0/1. SGR_HUB_ROWNA: in the hub build (whose gathers bypass L1) read
// them without allocating in L1 either.
#ifndef SGR_HUB_ROWNA
#define SGR_HUB_ROWNA 0
#endif
template <bool Hub>
__device__ __forceinline__ int32_t ld_row_h(const int32_t* p) {
  if constexpr (Hub && SGR_HUB_ROWNA) {
    int32_t r;
    asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
  } else {
    return ld_ro(p);
  }
}
__device__ __forceinline__ int32_t ld_row(const int32_t* p) {
#if SGR_ROWNA
  int32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
#else
  return ld_ro(p);
#endif
}
__device__ __forceinline__ int4 ld_row4(const int4* p) { return ld_ro(p); }
__device__ __forceinline__ void prefetch_l1(const void* p) {
  asm volatile("prefetch.global.L1 [%0];" ::"l"(p));
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile(
        "{\n .reg .pred P;\n mbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n"
        " selp.u32 %0, 1, 0, P;\n}"
        : "=r"(done)
        : "r"(smem_addr(b)), "r"(parity)
        : "memory");
  } while (!done);
}

// ---------------------------------------------------------------------------------------
// F_1: round-1 detection + round-2 assignment without color gathers. After round 1 every
// color is 1 (first fit against an all-zero snapshot), so with rows sorted ascending
//   LOWID: conflict(v) <=> first entry < v ;  PAPER: conflict(v) <=> last entry > v
// (a self-loop can never satisfy the strict inequality); tent(v) = mex({1}) = 2.
// Writes col[0] = C_1 (all 1), col[1] = C_2, and W_2 into the bins' lists [0]; bin-2
// vertices of W_2 get a slot and (packed mode) their list length len[0][v] = deg(v).
template <int TB, class C>
__global__ void __launch_bounds__(1024) k_first(RoundArgs<C> a, int sorted) {
  Ctrl* ctrl = a.ctrl;
  C* __restrict__ X = a.col[0];
  C* __restrict__ Y = a.col[1];
  const int lane = threadIdx.x & 31;
  const int64_t n = a.v_end;
  unsigned long long span_acc = 0;  // this thread's rows: sum of widths (dense-pass decision)
  for (int64_t base = (int64_t)a.v_begin + (int64_t)blockIdx.x * blockDim.x; base < n;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t vi = base + threadIdx.x;
    bool conflict = false;
    int64_t s = 0, e = 0;
    const int32_t v = (int32_t)vi;
    uint32_t span = 0;  // last - first entry of the row: its width in id space
    if (vi < n) {
      s = ldg_i64(a.row_ptr + v);
      e = ldg_i64(a.row_ptr + v + 1);
      if (e > s) {
        if (sorted) {
          const int32_t first = ldg_i32(a.col_idx + s), last = ldg_i32(a.col_idx + e - 1);
          if constexpr (TB == 1) conflict = last > v;
          else conflict = first < v;
          span = (uint32_t)max(last - first, 0);
        } else {
          for (int64_t j = s; j < e && !conflict; ++j) conflict = lose<TB>(v, ldg_i32(a.col_idx + j));
        }
      }
      X[v] = cpack<C>(1, 1, a);
      put_y<C>(a, Y, 1, v, cpack<C>(conflict ? 2 : 1, conflict ? 2 : 1, a));
    }
    const int b = bin_of(e - s, a.small_max, a.med_max);
    Counts* w2 = &ctrl->ring[rs(2)];
    if (a.bm[0]) {  // W_2's membership bitmap (single GPU: v_begin = 0, warps word-aligned)
      const unsigned mw = __ballot_sync(0xffffffffu, conflict);
      if (lane == 0 && base + threadIdx.x < n) a.bm[0][(base + threadIdx.x) >> 5] = mw;
      span_acc += span;  // row locality: summed per block at the end (one atomic each)
    }
    {  // bins 0/1: one atomicAdd per BLOCK and bin (~40 % of all vertices enter W_2, so
       // per-warp atomics on the two list counters serialize over the whole grid)
      __shared__ int32_t fcnt[2][kMaxWarps], fbase[2][kMaxWarps];
      const int wid = threadIdx.x >> 5;
      const unsigned m0 = __ballot_sync(0xffffffffu, conflict && b == 0);
      const unsigned m1 = __ballot_sync(0xffffffffu, conflict && b == 1);
      if (lane == 0) {
        fcnt[0][wid] = __popc(m0);
        fcnt[1][wid] = __popc(m1);
      }
      __syncthreads();
      if (threadIdx.x < 2) {
        const int q = threadIdx.x;
        int32_t run = 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
          fbase[q][w] = run;
          run += fcnt[q][w];
        }
        const int32_t b0 = run ? atomicAdd(q == 0 ? &w2->t : &w2->m, run) : 0;
        for (int w = 0; w < (int)(blockDim.x >> 5); ++w) fbase[q][w] += b0;
      }
      __syncthreads();
      const unsigned lt = (1u << lane) - 1u;
      if (conflict && b == 0) a.wl_t[0][fbase[0][wid] + __popc(m0 & lt)] = v;
      if (conflict && b == 1) a.wl_m[0][fbase[1][wid] + __popc(m1 & lt)] = v;
      __syncthreads();  // fcnt / fbase are rewritten by the next iteration
    }
    // bin 2: ceil(deg / kChunk) items per vertex and an accumulator slot
    const bool big = conflict && b == 2;
    const int32_t nch = big ? num_chunks(e - s) : 0;
    const unsigned mb = __ballot_sync(0xffffffffu, big);
    if (mb) {
      int sb = 0;
      if (lane == __ffs(mb) - 1) sb = atomicAdd(&ctrl->big_count, __popc(mb));
      sb = __shfl_sync(0xffffffffu, sb, __ffs(mb) - 1);
      if (big) {
        a.big_id[v] = sb + __popc(mb & ((1u << lane) - 1u));
        if constexpr (packed<C>()) a.len[0][v] = (int32_t)(e - s);
      }
      int incl = nch;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
      }
      const int total = __shfl_sync(0xffffffffu, incl, 31);
      int ib = 0;
      const unsigned mmc = __ballot_sync(0xffffffffu, nch > 1);
      if (lane == 0) {
        ib = atomicAdd(&w2->c, total);
        atomicAdd(&w2->cv, __popc(mb));
        if (mmc) atomicAdd(&w2->pad[1], __popc(mmc));
      }
      ib = __shfl_sync(0xffffffffu, ib, 0) + incl - nch;
      for (int32_t t = 0; t < nch; ++t) a.wl_c[0][ib + t] = make_item(v, t);
    }
  }
  if (a.nrep) __threadfence_system();  // C_2 stores into peer replicas: visible system-wide
  if (a.bm[0]) block_add(span_acc, &ctrl->span_sum);
}

// ---------------------------------------------------------------------------------------
// Forbidden-set helpers (shared memory; bits or bytes per color, see SGR_BITTBL).

__device__ __forceinline__ void set_add(uint8_t* tbl, uint32_t c) {
#if SGR_BITTBL
  atomicOr(reinterpret_cast<uint32_t*>(tbl) + (c >> 5), 1u << (c & 31u));
#else
  tbl[c] = 1;
#endif
}

// Zero `bytes` of a set, the `nl` lanes of a group sharing the work (lane index l < nl).
__device__ __forceinline__ void set_clear(uint8_t* p, int bytes, int l, int nl) {
  if ((bytes / 16) % nl == 0) {
    uint4* t = reinterpret_cast<uint4*>(p);
    for (int q = l; q < bytes / 16; q += nl) t[q] = make_uint4(0u, 0u, 0u, 0u);
  } else {
    uint32_t* t = reinterpret_cast<uint32_t*>(p);
    for (int q = l; q < bytes / 4; q += nl) t[q] = 0u;
  }
}

// First free color >= 1 of a warp-owned table of N bytes (N multiple of 128); -1 if full.
template <int N>
__device__ __forceinline__ int32_t tbl_first_free_warp(const uint8_t* tbl, int lane) {
  const uint32_t* t32 = reinterpret_cast<const uint32_t*>(tbl);
#pragma unroll 1
  for (int it = 0; it < N / 128; ++it) {
    uint32_t word = t32[it * 32 + lane];
    if (it == 0 && lane == 0) word |= 0xffu;  // color 0 is never a candidate
    const uint32_t z = __vcmpeq4(word, 0u);
    const unsigned b = __ballot_sync(0xffffffffu, z != 0u);
    if (b) {
      const int fl = __ffs(b) - 1;
      const uint32_t zz = __shfl_sync(0xffffffffu, z, fl);
      return (it * 32 + fl) * 4 + (__ffs(zz) - 1) / 8;
    }
  }
  return -1;
}

// 32 bits = colors [32 * lane, 32 * lane + 32) of a 1024-color set. Byte sets: multiplying a
// word of four 0/1 bytes by 0x01020408 gathers the bytes into bits 24-27.
__device__ __forceinline__ uint32_t tbl_bits32(const uint8_t* tbl, int lane) {
#if SGR_BITTBL
  return reinterpret_cast<const uint32_t*>(tbl)[lane];
#else
  const uint4* t = reinterpret_cast<const uint4*>(tbl) + lane * 2;
  const uint4 a = t[0], b = t[1];
  const uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
  uint32_t bits = 0;
#pragma unroll
  for (int q = 0; q < 8; ++q) bits |= ((w[q] * 0x01020408u) >> 24) << (4 * q);
  return bits;
#endif
}

// First free color of a 1024-bit set spread over the warp (lane l holds colors
// [32 l, 32 l + 32); bit 0 of lane 0 must already be set); -1 if all are taken.
__device__ __forceinline__ int32_t bits_first_free(uint32_t word) {
  const unsigned fb = __ballot_sync(0xffffffffu, word != 0xffffffffu);
  if (!fb) return -1;
  const int fl = __ffs(fb) - 1;
  const uint32_t w2 = __shfl_sync(0xffffffffu, word, fl);
  return fl * 32 + __ffs(~w2) - 1;
}

// Exact warp first fit over the FULL original row from `base` (all colors in [1, base)
// forbidden): the rare fallback when a first fit exceeds the 1024-color table. Reads the
// snapshot X, which holds the final colors of dropped neighbours, so it is exact in the
// trimmed mode as well.
template <bool Persist, class C>
__device__ __noinline__ int32_t warp_first_fit_rescan(const int32_t* __restrict__ col_idx,
                                                      const C* X, int64_t s, int64_t e,
                                                      int32_t base, int lane) {
  for (;;) {
    uint64_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
    if (base == 0) m0 = 1;
    for (int64_t j = s + lane; j < e; j += 32) {
      const uint32_t idx = (uint32_t)(ldc<Persist>(X + ld_ro(col_idx + j)) - base);
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

// ---------------------------------------------------------------------------------------
// Bin 2, plain 32-bit colors (no trimming): one warp processes one chunk [cs, ce) of the
// full row [s, e), read as int4 from the 16-byte-aligned window; outside [cs, ce) masked.
template <int TB, bool Persist, class C>
__device__ __forceinline__ void process_chunk_plain(const RoundArgs<C>& a, int k, int32_t v,
                                                    int32_t c, int64_t s, int64_t e,
                                                    const C* X, C* Y, int64_t* out,
                                                    int32_t* out_cnt, int32_t* out_vcnt,
                                                    uint8_t* tbl, int lane,
                                                    unsigned long long& edges,
                                                    unsigned long long& entries) {
  const int64_t cs = s + (int64_t)c * kChunk, ce = min(e, cs + kChunk);
  const int64_t wbase = cs & ~(int64_t)3;  // 16-byte aligned window start
  const int32_t nch = num_chunks(e - s);
  const int4* col4 = reinterpret_cast<const int4*>(a.col_idx + wbase);
  int32_t w[kWin / 32];
#pragma unroll
  for (int q = 0; q < kWin / 128; ++q) {
    const int64_t p0 = wbase + 4 * (lane + 32 * q);
    int4 t = make_int4(-1, -1, -1, -1);
    if (p0 + 3 >= cs && p0 < ce) {
      if (p0 + 4 <= a.nnz) {
        t = ld_ro(col4 + lane + 32 * q);
      } else {  // the array's last, partial 16-byte group: never read past nnz
        t.x = ld_ro(a.col_idx + p0);
        if (p0 + 1 < a.nnz) t.y = ld_ro(a.col_idx + p0 + 1);
        if (p0 + 2 < a.nnz) t.z = ld_ro(a.col_idx + p0 + 2);
      }
    }
    w[4 * q + 0] = (p0 + 0 >= cs && p0 + 0 < ce) ? t.x : -1;
    w[4 * q + 1] = (p0 + 1 >= cs && p0 + 1 < ce) ? t.y : -1;
    w[4 * q + 2] = (p0 + 2 >= cs && p0 + 2 < ce) ? t.z : -1;
    w[4 * q + 3] = (p0 + 3 >= cs && p0 + 3 < ce) ? t.w : -1;
  }
  const int32_t xv = ldc<Persist>(X + v);
  uint32_t lb = 0;  // lose(v, w) bits
#pragma unroll
  for (int u = 0; u < kWin / 32; ++u) lb |= (w[u] >= 0 && lose<TB>(v, w[u])) ? (1u << u) : 0u;
#pragma unroll
  for (int u = 0; u < kWin / 32; ++u) w[u] = (w[u] >= 0) ? ldc<Persist>(X + w[u]) : 0;  // now colors
  bool conf = false;
#pragma unroll
  for (int u = 0; u < kWin / 32; ++u) {
    if ((uint32_t)w[u] < (uint32_t)kBigTbl) set_add(tbl, (uint32_t)w[u]);
    conf |= (w[u] == xv) & ((lb >> u) & 1u);
  }
  if (lane == 0) {
    entries += (unsigned long long)(ce - cs);
    if (c == 0) edges += (unsigned long long)(e - s);
  }
  __syncwarp();
  const bool any = __any_sync(0xffffffffu, conf);
  if (nch == 1) {
    int32_t tent = 0;
    if (any) {
#if SGR_BITTBL
      tent = bits_first_free(tbl_bits32(tbl, lane) | (lane == 0 ? 1u : 0u));
#else
      tent = tbl_first_free_warp<kBigTbl>(tbl, lane);
#endif
      if (tent < 0) tent = warp_first_fit_rescan<Persist>(a.col_idx, X, s, e, kBigTbl, lane);
    }
    if (lane == 0) {
      put_y<C>(a, Y, k, v, any ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
      if (any) {
        out[atomicAdd(out_cnt, 1)] = make_item(v, 0);
        atomicAdd(out_vcnt, 1);
      }
    }
  } else {
    const int32_t slot = __ldg(a.big_id + v);
    uint32_t* accb = a.acc_bits + (int64_t)slot * 32;
    const uint32_t bits = tbl_bits32(tbl, lane);
    if (bits) atomicOr(accb + lane, bits);
    __syncwarp();  // orders every lane's atomicOr before lane 0's release below
    unsigned long long old = 0;
    if (lane == 0) {
      fence_acq_rel_gpu();  // release: every lane's partial set before the ticket
      old = atomicAdd(a.acc_cnt + slot, 1ull | ((unsigned long long)any << 32));
    }
    old = __shfl_sync(0xffffffffu, old, 0);
    if ((uint32_t)old == (uint32_t)(nch - 1)) {  // this warp finished the vertex's last chunk
      fence_acq_rel_gpu();  // acquire: the other chunks' partial sets
      uint32_t word = ld_cg(accb + lane);
      accb[lane] = 0u;
      if (lane == 0) a.acc_cnt[slot] = 0ull;
      const bool conf_all = ((old >> 32) + (any ? 1ull : 0ull)) != 0ull;
      int32_t tent = 0;
      if (conf_all) {
        if (lane == 0) word |= 1u;  // color 0
        tent = bits_first_free(word);
        if (tent < 0) tent = warp_first_fit_rescan<Persist>(a.col_idx, X, s, e, kBigTbl, lane);
      }
      int32_t ob = 0;
      if (lane == 0) {
        put_y<C>(a, Y, k, v, conf_all ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
        if (conf_all) {
          ob = atomicAdd(out_cnt, nch);
          atomicAdd(out_vcnt, 1);
        }
      }
      if (conf_all) {
        ob = __shfl_sync(0xffffffffu, ob, 0);
        for (int32_t t = lane; t < nch; t += 32) out[ob + t] = make_item(v, t);
      }
    }
  }
  __syncwarp();  // every lane's table reads (first-fit scan) before any lane clears
  set_clear(tbl, kBigTblB, lane, 32);
  __syncwarp();
}

// ---------------------------------------------------------------------------------------
// Bin 2, packed colors, trimmed lists (see the header comment). Per warp: a 2-stage TMA
// pipeline over the warp's chunk items i, i + NW, i + 2 NW, ...
struct ChunkHdr {
  int32_t v, c, len, slot, buf, keep;
  int64_t s, e;   // original row [s, e): list start in adj[*] and col_idx
  uint32_t fo;    // single-chunk vertex: this lane's word of its fixed set (prefetched)
  uint32_t xraw;  // X[v] word (prefetched; decoded at use, so the load is not waited for)
};

template <int TB, bool Persist>
__device__ __forceinline__ void bin2_trimmed(const RoundArgs<Packed>& a, int k, int p,
                                             const Packed* X, Packed* Y, uint8_t* wsm,
                                             int gw, int NW, int lane, int nC,
                                             unsigned long long& edges,
                                             unsigned long long& entries, uint32_t& ph) {
  using C = Packed;
  Ctrl* ctrl = a.ctrl;
  if (gw >= nC) return;
  const int64_t* items = sel(p, (const int64_t*)a.wl_c[0], (const int64_t*)a.wl_c[1]);
  int64_t* out = sel(p ^ 1, a.wl_c[0], a.wl_c[1]);
  int32_t* out_cnt = &ctrl->ring[rs(k + 1)].c;
  int32_t* out_vcnt = &ctrl->ring[rs(k + 1)].cv;
  int32_t* len_cur = sel(p, a.len[0], a.len[1]);
  int32_t* len_nxt = sel(p ^ 1, a.len[0], a.len[1]);
  int32_t* bufs = reinterpret_cast<int32_t*>(wsm);
  uint8_t* tbl_all = wsm + WarpSmem<C>::kBuf;
  uint8_t* tbl_drop = tbl_all + kBigTblB;
  uint64_t* bars = reinterpret_cast<uint64_t*>(wsm + WarpSmem<C>::kBars);
  // Next-round items are buffered per warp and flushed with one atomicAdd per <= 32 items
  // (the bin's item and vertex counters are single hot addresses).
  int64_t* ibuf = reinterpret_cast<int64_t*>(wsm + WarpSmem<C>::kItems);
  int ipend = 0, vpend = 0;  // warp-uniform
  auto iflush = [&]() {
    if (ipend == 0) return;
    __syncwarp();
    int ob = 0;
    if (lane == 0) ob = atomicAdd(out_cnt, ipend);
    ob = __shfl_sync(0xffffffffu, ob, 0);
    if (lane < ipend) out[ob + lane] = ibuf[lane];
    __syncwarp();
    ipend = 0;
  };

  // Pass 2 reads the rows straight from col_idx (every list is still the full row); later
  // passes read the compacted lists in adj[buf].
  auto list_src = [&](int buf) -> const int32_t* {
    return k == 2 ? a.col_idx : sel(buf, (const int32_t*)a.adj[0], (const int32_t*)a.adj[1]);
  };
  auto issue = [&](const ChunkHdr& h, int st) {  // lane 0 only
    const int64_t cs = h.s + (int64_t)h.c * kChunk;
    const int64_t ce = min(h.s + (int64_t)h.len, cs + kChunk);
    const int64_t w0 = cs & ~(int64_t)3;
    int64_t wend = (ce + 3) & ~(int64_t)3;  // 16-byte-aligned window [w0, wend)
    int32_t* dst = bufs + st * (kStage / 4);
    const int32_t* src = list_src(h.buf);
    fence_proxy_async();  // generic-proxy reads of this stage happen-before the async write
    if (k == 2 && wend > a.nnz) {
      // pass 2 reads col_idx, which holds exactly nnz entries (the adjacency buffers are
      // padded): the array's last partial 16-byte group is copied by plain loads, so the
      // bulk copy never reads past nnz (compute-sanitizer memcheck, round 2)
      const int64_t full = max(a.nnz & ~(int64_t)3, w0);
      for (int64_t q = full; q < ce; ++q) dst[q - w0] = ld_ro(src + q);
      wend = full;
    }
    const uint32_t bytes = (uint32_t)((wend - w0) * 4);
    if (bytes) {
      tma_load_1d(dst, src + w0, bytes, bars + st);
    } else {  // nothing left for the bulk copy: complete the phase with a plain arrival
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bars + st)) : "memory");
    }
  };
  auto finish_hdr = [&](int64_t it, ChunkHdr& h) {  // everything but the item itself
    h.v = (int32_t)((uint64_t)it >> 32);
    h.c = (int32_t)((uint32_t)it & kChunkMask);
    h.buf = ((uint32_t)it & kBufBit) ? 1 : 0;
    h.keep = ((uint32_t)it & kKeepBit) ? 1 : 0;
    h.s = ldg_i64(a.row_ptr + h.v);
    h.e = ldg_i64(a.row_ptr + h.v + 1);
    h.len = ld_cg(len_cur + h.v);
    h.slot = __ldg(a.big_id + h.v);
  };
  auto load_hdr = [&](int i, ChunkHdr& h) { finish_hdr(__ldcg(items + i), h); };
  // second-stage header loads, issued one chunk ahead (they need slot / v)
  auto finish_hdr2 = [&](ChunkHdr& h) {
    // unconditional loads (a select on the result would wait for it); fo is only used when
    // the vertex has a single chunk, and fixed + slot * 32 is always a valid address
    h.fo = ld_cg(a.fixed + (int64_t)h.slot * 32 + lane);
    h.xraw = ldraw<Persist>(X + h.v);
  };
  auto zero_hdr = [](ChunkHdr& h) {
    h.v = h.c = h.len = h.slot = h.buf = h.keep = 0;
    h.s = h.e = 0;
    h.fo = 0u;
    h.xraw = 0u;
  };

  // Work distribution: the warp's first four items are gw + j NW (j < 4); after that it
  // takes the next unclaimed item from a per-pass cursor, so warps that drew short chunks
  // take more of them. Software pipeline over the warp's items: while chunk i is processed,
  // the next chunk's list window streams in (TMA) and its fixed set and own color load, the
  // one after's header loads, the third one's item id and the fourth one's claim are in
  // flight, so nothing the next iteration needs is waited for at the end of this one.
  int* cursor = &ctrl->ring[rs(k)].pad[0];
  unsigned long long lwrites = 0;  // warp-uniform
  unsigned long long pc0 = 0, pc1 = 0, pc2 = 0, pc3 = 0;  // phase cycles (lane 0 adds)
  long long tq = pclock();
  int i = gw, in = gw + NW, inn = gw + 2 * NW, innn = gw + 3 * NW;
  ChunkHdr cur, nxt;
  load_hdr(i, cur);
  finish_hdr2(cur);
#if !SGR_NO_TMA
  if (lane == 0) issue(cur, 0);
#endif
  zero_hdr(nxt);
  if (in < nC) load_hdr(in, nxt);
  int64_t it_nn = inn < nC ? __ldcg(items + inn) : 0;
  int st = 0;
  while (i < nC) {
#if !SGR_NO_TMA
    if (in < nC && lane == 0) issue(nxt, st ^ 1);
#endif
    if (in < nC) finish_hdr2(nxt);
    ChunkHdr nn;
    zero_hdr(nn);
    if (inn < nC) finish_hdr(it_nn, nn);
    const int64_t it_nnn = innn < nC ? __ldcg(items + innn) : 0;
    // the item after innn, less 4 NW (monotone: once past nC, stop claiming). The raw
    // cursor value is kept and 4 NW added at the broadcast: any arithmetic on it here
    // would wait for the atomic's round trip right at the claim.
    int claim = nC;
    if (SGR_B2_STATIC) claim = innn + NW - 4 * NW;
    else if (lane == 0 && innn < nC) claim = claim_add(cursor);

    // ---- chunk `cur` in stage st: slots [off0, off0 + cnt) of the 16-byte-aligned window
    const int32_t v = cur.v;
    const int64_t cs = cur.s + (int64_t)cur.c * kChunk;
    const int32_t cnt = (int32_t)(min(cur.s + (int64_t)cur.len, cs + kChunk) - cs);
    const int32_t off0 = (int32_t)(cs & 3);
    const int32_t nslots = off0 + cnt;
    const int32_t nb = (nslots + 128 * kQB - 1) / (128 * kQB);  // batches of kQB int4 per lane
    const int32_t nch = num_chunks(cur.len);
    const int32_t xv = cval<C>(cur.xraw);
    // a neighbour still in W_k was written by pass k-1 with last = k; one that has left W
    // has last < k and is recognised unless last = k mod 16, in which case it simply stays
    // in the list one more round (never the reverse: live neighbours are never dropped)
    const uint32_t klive = (uint32_t)k & 15u;
#if SGR_NO_TMA
    {  // A/B: the warp stages its own window (16-byte loads + shared stores), no TMA
      const int4* g4 = reinterpret_cast<const int4*>(list_src(cur.buf) + (cs & ~(int64_t)3));
      int4* s4 = reinterpret_cast<int4*>(bufs + st * (kStage / 4));
      for (int q = 0; 4 * 32 * q < nslots; ++q)
        if (4 * (lane + 32 * q) < nslots) s4[lane + 32 * q] = __ldcg(g4 + lane + 32 * q);
      __syncwarp();
    }
#else
    const long long ta = pclock();
    pc0 += (unsigned long long)(ta - tq);
    mbar_wait(bars + st, (ph >> st) & 1u);
    ph ^= 1u << st;
    const long long tb = pclock();
    pc1 += (unsigned long long)(tb - ta);
#endif
    // live entries are compacted into the front of this stage as the batches go (a batch's
    // outputs land below its own slots, whose ids every lane already holds in registers)
    int32_t* sbuf = bufs + st * (kStage / 4);
    bool conf = false;
    uint32_t cmax = 0;  // SGR_CLRMAX: largest table index this lane set
    const unsigned lt_mask = (1u << lane) - 1u;
    const bool small = SGR_SMALLMASK && k <= 62;  // uniform: every color of X is <= k
    uint64_t mall = 0, mdrop = 0;                 // small passes: colors seen / dropped
    // batch bb: window slots 32 (kJB bb + j) + lane, j < kJB: consecutive lanes read
    // consecutive (sorted) list entries, so neighbours close in id share a cache line
    // within one gather instruction
    auto fetch = [&](int bb, int32_t (&id)[kJB], uint32_t (&raw)[kJB], uint32_t& okm) {
      okm = 0;
#pragma unroll
      for (int j = 0; j < kJB; ++j) {
        const int32_t r = 32 * (kJB * bb + j) + lane;
        id[j] = sbuf[r];
        okm |= (r >= off0 && r < nslots) ? (1u << j) : 0u;
      }
#pragma unroll
      for (int j = 0; j < kJB; ++j) raw[j] = ((okm >> j) & 1u) ? ldraw_b2<Persist>(X + id[j]) : 0u;
    };
    uint32_t lvb = 0;  // live bit of window slot 32 (kJB bb + j) + lane, at bit kJB bb + j
    auto consume = [&](int bb, const int32_t (&id)[kJB], const uint32_t (&raw)[kJB], uint32_t okm) {
      (void)bb;
#pragma unroll
      for (int j = 0; j < kJB; ++j) {
        bool live = false;
        if ((okm >> j) & 1u) {
          // colors >= 1023 are clamped onto byte 1023; a first fit of 1023 or more is
          // recomputed exactly from the full row (warp_first_fit_rescan)
          live = (raw[j] >> kRoundShift) == klive;
          if (small) {
            const uint64_t bit = 1ull << (raw[j] & 63u);
            mall |= bit;
            mdrop |= live ? 0ull : bit;
          } else {
            const uint32_t ci = min(raw[j] & kColorMask, (uint32_t)(kBigTbl - 1));
#if SGR_CLRMAX
            cmax = max(cmax, ci);
#endif
            set_add(tbl_all, ci);
            if (!live) set_add(tbl_drop, ci);
          }
          conf |= (int32_t)(raw[j] & kColorMask) == xv && lose<TB>(v, id[j]);
        }
        lvb |= live ? (1u << (kJB * bb + j)) : 0u;
      }
    };
    const int32_t slot = cur.slot;
    uint32_t* accb = a.acc_bits + (int64_t)slot * 32;
    int nbr = nb;  // batches gathered (< nb after an early exit)
#if SGR_EARLY
    // colors 1..k (k <= 62), and the fixed set's colors 0..63 (lanes 0/1 hold them)
    const uint64_t need = ((2ull << k) - 1ull) & ~1ull;
    const uint64_t fx64 = (uint64_t)__shfl_sync(0xffffffffu, cur.fo, 0) |
                          ((uint64_t)__shfl_sync(0xffffffffu, cur.fo, 1) << 32);
    unsigned long long seen_pub = 0ull, conf_pub = 0ull;  // lane 0: the last read-back
#endif
    for (int bb = 0; bb < nb; ++bb) {
      int32_t id[kJB];
      uint32_t raw[kJB];
      uint32_t okm;
      fetch(bb, id, raw, okm);
      consume(bb, id, raw, okm);
#if SGR_EARLY
      if (small && bb + 1 < nb && (SGR_EARLY_MC || nch == 1)) {
        const uint64_t wm = warp_or64(mall);
        const bool wc = __any_sync(0xffffffffu, conf);
        uint64_t seen = wm | fx64;
        bool cf = wc;
        if (nch > 1) {
          // publish this chunk's colors and conflict; the values read back (the other
          // chunks' progress) are used at the next check, so the atomics' latency hides
          // under one batch of gathers
          const uint64_t sp = __shfl_sync(0xffffffffu, seen_pub, 0);
          const uint64_t cp = __shfl_sync(0xffffffffu, conf_pub, 0);
          seen |= sp;
          cf = cf || (cp & 1ull);
          if (lane == 0) {
            seen_pub = atomicOr(reinterpret_cast<unsigned long long*>(accb), (unsigned long long)wm);
            conf_pub = atomicOr(a.acc_cnt + slot, wc ? 1ull : 0ull);
          }
        }
        if (cf && (seen & need) == need) {
          nbr = bb + 1;
          break;
        }
      }
#endif
    }
#if SGR_EARLY
    if (nbr < nb) {  // unread window slots stay listed: counted as live entries
      for (int bb = nbr; bb < nb; ++bb) {
#pragma unroll
        for (int j = 0; j < kJB; ++j) {
          const int32_t r = 32 * (kJB * bb + j) + lane;
          lvb |= (r >= off0 && r < nslots) ? (1u << (kJB * bb + j)) : 0u;
        }
      }
    }
#endif
#if !SGR_NO_TMA
    const long long tc = pclock();
    pc2 += (unsigned long long)(tc - tb);
#endif
    if (lane == 0) {
      entries += (unsigned long long)(min(nslots, 32 * kJB * nbr) - off0);
      if (cur.c == 0) edges += (unsigned long long)(cur.e - cur.s);
    }
    __syncwarp();
    const bool any = __any_sync(0xffffffffu, conf);
    // this lane's 32-bit word of the chunk's color set / dropped set (colors [32 lane, +32))
    auto set_word = [&](const uint8_t* tbl, uint64_t m) -> uint32_t {
      if (!small) return tbl_bits32(tbl, lane);
      const uint64_t w = warp_or64(m);
      return lane == 0 ? (uint32_t)w : (lane == 1 ? (uint32_t)(w >> 32) : 0u);
    };
    // live entries counted from the per-lane bits; the stage is compacted (in place, window
    // order, one ballot per 32 slots) only when the list is actually rewritten
    const uint32_t live_total = __reduce_add_sync(0xffffffffu, (uint32_t)__popc(lvb));
    auto compact = [&]() {
      uint32_t pos = 0;
      for (int bb = 0; bb < nb; ++bb) {
#pragma unroll
        for (int j = 0; j < kJB; ++j) {
          const bool lv = (lvb >> (kJB * bb + j)) & 1u;
          const int32_t id = sbuf[32 * (kJB * bb + j) + lane];
          const unsigned bal = __ballot_sync(0xffffffffu, lv);
          if (lv) sbuf[pos + __popc(bal & lt_mask)] = id;  // <= its own slot: already read
          pos += (uint32_t)__popc(bal);
        }
      }
      __syncwarp();
    };
    // the compacted live list (front of the stage) to global memory, coalesced
    auto write_live = [&](int32_t* base) {
      compact();
      for (uint32_t q = lane; q < live_total; q += 32) base[q] = sbuf[q];
    };

    uint32_t* fx = a.fixed + (int64_t)slot * 32;
    int32_t* lst_same = sel(cur.buf, a.adj[0], a.adj[1]);
    int32_t* lst_other = sel(cur.buf, a.adj[1], a.adj[0]);
    if (nch == 1) {
      if (any) {
        const uint32_t fo = cur.fo;
        const uint32_t word = set_word(tbl_all, mall) | fo | (lane == 0 ? 1u : 0u);
        int32_t tent = bits_first_free(word);
        if (tent < 0 || tent >= kBigTbl - 1) {  // beyond the exact range of the table
          tent = warp_first_fit_rescan<Persist>(a.col_idx, X, cur.s, cur.e, kBigTbl - 1, lane);
        }
        const uint32_t drop = set_word(tbl_drop, mdrop);
        if (drop & ~fo) fx[lane] = fo | drop;
        // single chunk: the warp owns the whole list, so it is compacted in place, and not
        // rewritten at all when nothing was dropped (pass 2 read col_idx: always written)
        // SGR_LAZY > 0: keep the list (dead entries included) unless more than cnt >> SGR_LAZY
        // entries dropped — listed dead neighbours are simply the untrimmed semantics
        const bool rewrite = k == 2 || (SGR_LAZY ? (uint32_t)cnt - live_total > ((uint32_t)cnt >> SGR_LAZY)
                                                 : live_total < (uint32_t)cnt);
        if (rewrite) {
          write_live(lst_same + cur.s);
          lwrites += live_total;
        }
        if (lane == 0) {
          len_nxt[v] = rewrite ? (int32_t)live_total : cnt;
          put_y<C>(a, Y, k, v, cpack<C>(tent, k + 1, a));
          // live <= kChunk: one chunk, the list stays in its buffer
          ibuf[ipend] = make_item(v, (int32_t)(cur.buf ? kBufBit : 0u));
        }
        ++ipend;
        ++vpend;
        if (ipend == 32) iflush();
      } else if (lane == 0) {
        put_y<C>(a, Y, k, v, cpack<C>(xv, k, a));
      }
    } else {
      // several chunks: publish this chunk's partial forbidden set, dropped colors and
      // compacted live entries; the finalize phase after the pass decides conflict and
      // first fit once every chunk is in (no per-chunk fences or tickets)
      // (the atomics whose results are needed are issued first, consumed last)
      int32_t lbase = 0, fpos = 0;
      const bool keep = cur.keep != 0;
      if (lane == 0) {
        if (keep) {  // list stays: count live entries in the slot's accumulator (bits 32-63)
          if (live_total) atomicAdd(a.acc_cnt + slot, (unsigned long long)live_total << 32);
        } else if (live_total) {
          lbase = atomicAdd(len_nxt + v, (int32_t)live_total);
        }
        if (cur.c == 0) fpos = lane0_add(&ctrl->ring[rs(k)].fin, 1);  // used at the end
        if (any) atomicOr(a.acc_cnt + slot, 1ull);  // conflict flag (bit 0)
      }
      const uint32_t drop = set_word(tbl_drop, mdrop);
      if (SGR_EARLY && small) {  // colors 0..63 as one 64-bit word, as the early-exit checks
        const uint64_t wm = warp_or64(mall);
        if (lane == 0 && wm) atomicOr(reinterpret_cast<unsigned long long*>(accb), (unsigned long long)wm);
      } else {
        const uint32_t bits = set_word(tbl_all, mall);
        if (bits) atomicOr(accb + lane, bits);
      }
      if (drop) atomicOr(fx + lane, drop);
      if (!keep) {
        lbase = __shfl_sync(0xffffffffu, lbase, 0);
        write_live(lst_other + cur.s + lbase);
        lwrites += live_total;
      }
      if (lane == 0 && cur.c == 0)
        a.fin[fpos] = (int64_t)(((uint64_t)(uint32_t)slot << 32) | (uint32_t)v |
                                (cur.buf ? kBufBit : 0u) | (keep ? (1ull << 63) : 0ull));
    }
    __syncwarp();  // every lane's table reads before the clear
#if SGR_CLRMAX
    if (!small) {  // both sets, only the 16-byte groups up to the largest color set in this chunk
      const uint32_t nq = (__reduce_max_sync(0xffffffffu, cmax) >> 4) + 1;
      uint4* ta = reinterpret_cast<uint4*>(tbl_all);
      uint4* td = reinterpret_cast<uint4*>(tbl_drop);
      for (uint32_t q = lane; q < nq; q += 32) {
        ta[q] = make_uint4(0u, 0u, 0u, 0u);
        td[q] = make_uint4(0u, 0u, 0u, 0u);
      }
    }
#else
    if (!small) set_clear(tbl_all, kTblBytes, lane, 32);  // both sets
#endif
    __syncwarp();
#if !SGR_NO_TMA
    tq = pclock();
    pc3 += (unsigned long long)(tq - tc);
#endif
    st ^= 1;
    i = in;
    in = inn;
    inn = innn;
    innn = 4 * NW + __shfl_sync(0xffffffffu, claim, 0);
    cur = nxt;
    nxt = nn;
    it_nn = it_nnn;
  }
  iflush();
  if (lane == 0 && vpend) atomicAdd(out_vcnt, vpend);
  if (lane == 0 && lwrites) atomicAdd(&ctrl->list_writes_total, lwrites);
  // once per pass: this thread's list writes before the next pass's TMA (async-proxy) reads
  fence_proxy_async_global();
  if (SGR_PHASE_CYCLES && lane == 0) {
    atomicAdd(&ctrl->phase_cycles[0], pc0);
    atomicAdd(&ctrl->phase_cycles[1], pc1);
    atomicAdd(&ctrl->phase_cycles[2], pc2);
    atomicAdd(&ctrl->phase_cycles[3], pc3);
  }
}

// Finalize phase of a trimmed pass (after every chunk of the pass is done): for each
// multi-chunk bin-2 vertex, the merged forbidden set is the OR of its chunks' partial sets
// and its fixed set; conflict is the OR of the chunks' flags (Alg. 5 l.12-15), the first
// fit the lowest free color (l.8). Writes Y[v], pushes the vertex's next-round chunk items
// (its compacted list now lives in the other buffer), and resets the accumulators.
template <int TB, bool Persist>
__device__ __forceinline__ void finalize_body(const RoundArgs<Packed>& a, int k) {
  using C = Packed;
  Ctrl* ctrl = a.ctrl;
  const int p = k & 1;
  const int lane = threadIdx.x & 31;
  const int gw = (int)((grp_block(a) * blockDim.x + threadIdx.x) >> 5);
  const int NW = (int)((grp_size(a) * blockDim.x) >> 5);
  const int nF = ld_cg(&ctrl->ring[rs(k)].fin);
  const C* X = sel((k - 1) & 1, (const C*)a.col[0], (const C*)a.col[1]);
  C* Y = sel(k & 1, a.col[0], a.col[1]);
  int64_t* out = sel(p ^ 1, a.wl_c[0], a.wl_c[1]);
  int32_t* len_cur = sel(p, a.len[0], a.len[1]);
  int32_t* len_nxt = sel(p ^ 1, a.len[0], a.len[1]);
  // B <= 32 vertices per warp (spread over every warp of the grid), one per lane: its
  // conflict flag, its two 1024-bit sets (partial sets of its chunks, fixed set) as 16
  // vector loads issued together, first fit by a scan of the merged words, item pushes with
  // one aggregated atomicAdd per counter per warp
  const int B = min(32, (nF + NW - 1) / NW);
  // every warp runs the same number of iterations (block-level aggregation below)
  const int iters = nF > 0 ? (nF + NW * B - 1) / (NW * B) : 0;
  __shared__ int32_t fin_tot[3][kMaxWarps];   // per warp: items, vertices, multi-chunk vertices
  __shared__ int32_t fin_base[kMaxWarps];
  const int nwb = (int)(blockDim.x >> 5);
  const int wid = threadIdx.x >> 5;
  for (int it = 0; it < iters; ++it) {
    const int base = gw * B + it * NW * B;
    const int i = base + lane;
    const bool valid = lane < B && i < nF;
    const uint64_t f = valid ? (uint64_t)__ldcg(a.fin + i) : 0ull;
    const int32_t v = (int32_t)((uint32_t)f & ~kBufBit);
    const int32_t slot = (int32_t)((f >> 32) & 0x7fffffffull);
    const bool kept = (f >> 63) != 0ull;  // this pass left the list uncompacted
    bool conf = false, keep_next = false;
    int32_t nch2 = 0, tent = -1, len_list = 0;
    uint32_t xraw = 0u;
    uint4* accb = reinterpret_cast<uint4*>(a.acc_bits + (int64_t)slot * 32);
    if (valid) {
      const uint4* fxb = reinterpret_cast<const uint4*>(a.fixed + (int64_t)slot * 32);
      uint4 m[8];
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const uint4 x = __ldcg(accb + q), y = __ldcg(fxb + q);
        m[q] = make_uint4(x.x | y.x, x.y | y.y, x.z | y.z, x.w | y.w);
      }
      const unsigned long long cc = __ldcg(a.acc_cnt + slot);
      conf = (cc & 1ull) != 0ull;
      xraw = ldraw<Persist>(X + v);
      const int32_t lcur = ld_cg(len_cur + v);  // the list this pass read
      const int32_t lnxt = ld_cg(len_nxt + v);  // compacting pass: live entries written
      // next pass: the same list (kept) or the compacted one; keep it next pass too unless
      // more than 1/16 of its entries are dead (kept) / were dropped this pass (compacted)
      len_list = kept ? lcur : lnxt;
      const int32_t dead = kept ? lcur - (int32_t)(cc >> 32) : lcur - lnxt;
      keep_next = SGR_MCLAZY && dead <= (lcur >> SGR_MCLAZY_SHIFT);
      nch2 = conf ? num_chunks(len_list) : 0;
      m[0].x |= 1u;  // color 0
#pragma unroll
      for (int q = 7; q >= 0; --q) {  // lowest word with a zero bit
        const uint32_t w4[4] = {m[q].x, m[q].y, m[q].z, m[q].w};
#pragma unroll
        for (int t = 3; t >= 0; --t)
          if (w4[t] != 0xffffffffu) tent = 32 * (4 * q + t) + __ffs(~w4[t]) - 1;
      }
#pragma unroll
      for (int q = 0; q < 8; ++q) accb[q] = make_uint4(0u, 0u, 0u, 0u);
    }
    int32_t incl = nch2;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int32_t t = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += t;
    }
    const int32_t total = __shfl_sync(0xffffffffu, incl, 31);
    const unsigned cm = __ballot_sync(0xffffffffu, conf);
    // item slots: one atomicAdd per BLOCK and counter (every warp of the grid finalizes at
    // the same moment, so per-warp atomics on two hot addresses would serialize)
    const unsigned mmc = __ballot_sync(0xffffffffu, nch2 > 1);  // multi-chunk next pass
    if (lane == 0) {
      fin_tot[0][wid] = total;
      fin_tot[1][wid] = (int32_t)__popc(cm);
      fin_tot[2][wid] = (int32_t)__popc(mmc);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
      int32_t run = 0, vs = 0, mc = 0;
      for (int q = 0; q < nwb; ++q) {
        fin_base[q] = run;
        run += fin_tot[0][q];
        vs += fin_tot[1][q];
        mc += fin_tot[2][q];
      }
      const int32_t b0 = run ? atomicAdd(&ctrl->ring[rs(k + 1)].c, run) : 0;
      if (vs) atomicAdd(&ctrl->ring[rs(k + 1)].cv, vs);
      if (mc) atomicAdd(&ctrl->ring[rs(k + 1)].pad[1], mc);
      for (int q = 0; q < nwb; ++q) fin_base[q] += b0;
    }
    __syncthreads();
    int32_t ob = 0;
    if (lane == 0) ob = fin_base[wid];
    // first fits beyond the exact range of the table: warp rescans of the full rows (rare)
    unsigned rm = __ballot_sync(0xffffffffu, conf && (tent < 0 || tent >= kBigTbl - 1));
    while (rm) {
      const int j = __ffs(rm) - 1;
      rm &= rm - 1u;
      const int32_t vj = __shfl_sync(0xffffffffu, v, j);
      const int32_t t = warp_first_fit_rescan<Persist>(a.col_idx, X, ldg_i64(a.row_ptr + vj),
                                                       ldg_i64(a.row_ptr + vj + 1), kBigTbl - 1, lane);
      if (lane == j) tent = t;
    }
    ob = __shfl_sync(0xffffffffu, ob, 0) + incl - nch2;
    if (valid) {
      a.acc_cnt[slot] = 0ull;
      len_cur[v] = 0;  // consumed; the pass after next accumulates into it
      if (conf && kept) len_nxt[v] = len_list;  // the same list again
      put_y<C>(a, Y, k, v, conf ? cpack<C>(tent, k + 1, a) : cpack<C>(cval<C>(xraw), k, a));
      const uint32_t obuf = (uint32_t)f & kBufBit;
      const uint32_t nbuf = (kept ? obuf : (obuf ^ kBufBit)) | (keep_next ? kKeepBit : 0u);
      for (int32_t t = 0; t < nch2; ++t) out[ob + t] = make_item(v, (int32_t)(t | nbuf));
    }
  }
}

// Bin 1: each 8-lane group of the warp processes one vertex (v < 0: idle group) in batches
// of 64 row entries (8 per lane: all eight loads, then all eight gathers); only as many
// batches as the row needs are issued. 32-bit relative indices throughout.
template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void process_group(const RoundArgs<C>& a, int k, int32_t v,
                                              int64_t s, int64_t e, const C* X, C* Y,
                                              uint8_t* gtbl, int gl, unsigned gmask,
                                              bool& push, unsigned long long& edges) {
  const int32_t cnt = v >= 0 ? (int32_t)(e - s) : 0;  // <= 256
  const int32_t* row = a.col_idx + s;
  const int32_t xv = v >= 0 ? ldc<Persist>(X + v) : 0;
  bool conf = false;
  const bool small = SGR_SMALLMASK && k <= 62;  // uniform: colors of X are <= k < 64
  uint64_t msk = 0;
  constexpr int B = Hub ? SGR_B1_BATCH_HUB : 8;  // entries per lane per batch
  const int32_t nb = (cnt + 8 * B - 1) / (8 * B);
  for (int32_t bb = 0; bb < nb; ++bb) {
    int32_t w[B];
#pragma unroll
    for (int u = 0; u < B; ++u) {
      const int32_t r = 8 * B * bb + gl + kGroup * u;
      w[u] = r < cnt ? ld_row_h<Hub>(row + r) : -1;
    }
    uint32_t lb = 0;
#pragma unroll
    for (int u = 0; u < B; ++u) lb |= (w[u] >= 0 && lose<TB>(v, w[u])) ? (1u << u) : 0u;
#pragma unroll
    for (int u = 0; u < B; ++u) w[u] = w[u] >= 0 ? ldc01<Persist, Hub>(X + w[u]) : -1;  // colors
#pragma unroll
    for (int u = 0; u < B; ++u) {
      if (w[u] >= 0) {
        // deg <= 256 => first fit <= 257: colors >= 511 are clamped onto an unused byte
        if (small) msk |= 1ull << (w[u] & 63);
        else set_add(gtbl, (uint32_t)min(w[u], kMedTbl - 1));
        conf |= w[u] == xv && ((lb >> u) & 1u);
      }
    }
  }
  if (v >= 0 && gl == 0) edges += (unsigned long long)cnt;
  __syncwarp();
  const bool any = (__ballot_sync(0xffffffffu, conf) & gmask) != 0u;
  int32_t tent = 0;
  if (small) {  // OR the group's masks (xor butterfly inside the 8-lane group)
#pragma unroll
    for (int o = 4; o > 0; o >>= 1) msk |= __shfl_xor_sync(0xffffffffu, msk, o);
    tent = __ffsll((long long)~(msk | 1ull)) - 1;  // bit c = color c; color 0 never free
  } else if (v >= 0 && any) {  // the group scans its table 32 bytes (8 words) per step
    const uint32_t* t32 = reinterpret_cast<const uint32_t*>(gtbl);
#if SGR_BITTBL
    {  // 512 bits = 16 words, two per lane of the group
      uint32_t w0 = t32[2 * gl], w1 = t32[2 * gl + 1];
      if (gl == 0) w0 |= 1u;  // color 0
      const int f = (~w0) ? (__ffs(~w0) - 1) : ((~w1) ? 32 + __ffs(~w1) - 1 : 64);
      const unsigned b = __ballot_sync(gmask, f < 64) & gmask;
      const int fl = __ffs(b) - 1;  // the group's lane 0 always has a free color (deg <= 256)
      tent = (fl & 7) * 64 + __shfl_sync(gmask, f, fl);
    }
#else
    for (int it = 0; it < kMedTbl / 32; ++it) {
      uint32_t word = t32[it * 8 + gl];
      if (it == 0 && gl == 0) word |= 0xffu;
      const uint32_t z = __vcmpeq4(word, 0u);
      const unsigned b = __ballot_sync(gmask, z != 0u) & gmask;
      if (b) {
        const int fl = __ffs(b) - 1;  // absolute lane
        const uint32_t zz = __shfl_sync(gmask, z, fl);
        tent = (it * 8 + (fl & 7)) * 4 + (__ffs(zz) - 1) / 8;
        break;
      }
    }
#endif
  }
  __syncwarp();  // the group's table reads (first-fit scan) before any lane clears
  if (!small) set_clear(gtbl, kMedTblB, gl, kGroup);
  __syncwarp();
  if (v >= 0 && gl == 0) put_y<C>(a, Y, k, v, any ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
  push = (v >= 0) && any && gl == 0;
}

// Per-warp buffered worklist push (bins 0/1): lanes with `pred` append `v` to a shared-
// memory buffer; when 32 or more are pending the warp flushes them with ONE atomicAdd on the
// global counter and a contiguous store. All 32 lanes must call; `pending` is warp-uniform.
template <int kBufN = kPushBuf>
__device__ __forceinline__ void push_buffered(bool pred, int32_t v, int32_t* pbuf, int& pending,
                                              int32_t* list, int32_t* count, int lane) {
  const unsigned m = __ballot_sync(0xffffffffu, pred);
  if (pred) pbuf[pending + __popc(m & ((1u << lane) - 1u))] = v;
  pending += __popc(m);
  if (pending >= kBufN - 32) {
    __syncwarp();
    int base = 0;
    if (lane == 0) base = atomicAdd(count, pending);
    base = __shfl_sync(0xffffffffu, base, 0);
    for (int t = lane; t < pending; t += 32) list[base + t] = pbuf[t];
    __syncwarp();
    pending = 0;
  }
}
__device__ __forceinline__ void push_flush(int32_t* pbuf, int& pending, int32_t* list,
                                           int32_t* count, int lane) {
  if (pending == 0) return;
  __syncwarp();
  int base = 0;
  if (lane == 0) base = atomicAdd(count, pending);
  base = __shfl_sync(0xffffffffu, base, 0);
  for (int t = lane; t < pending; t += 32) list[base + t] = pbuf[t];
  __syncwarp();
  pending = 0;
}

// Step stream of a warp over a bin-0/1 list (flat build): tiles of kT steps of VPW list
// positions; a warp's first tile is its own (gw), later ones come from a per-pass cursor,
// each claimed one tile ahead (so the atomic's latency is never waited for). Warps that
// spent long on bin 2 take fewer small-vertex tiles: the pass ends together.
template <int VPW>
struct StepStream {
  int tile, j, next;   // warp-uniform except `next` (lane 0's claim, broadcast at use)
  int ntiles, kT;
  int* cursor;
  int NW;
  // tiles of kT <= kTmax steps; short lists get kT = 1 (one step per warp first, as many
  // first tiles as warps) so thin passes spread over the grid
  __device__ __forceinline__ void init(int gw, int nW, int nX, int kTmax, int* cur, int lane) {
    NW = nW;
    cursor = cur;
    kT = max(1, min(kTmax, nX / (NW * VPW)));
    ntiles = (nX + kT * VPW - 1) / (kT * VPW);
    tile = gw;
    j = 0;
    next = ntiles;
    if (lane == 0 && tile < ntiles) next = claim_add(cursor);  // NW added at the broadcast
  }
  // list position of the current step's first vertex (0x7fffffff: done)
  __device__ __forceinline__ int base() const { return tile < ntiles ? (tile * kT + j) * VPW : 0x7fffffff; }
  __device__ __forceinline__ void advance(int lane) {
    if (++j == kT) {
      j = 0;
      tile = NW + __shfl_sync(0xffffffffu, next, 0);
      next = ntiles;
      if (lane == 0 && tile < ntiles) next = claim_add(cursor);
    }
  }
};

// Bin 0 driver: 4-lane groups, 8 vertices per warp per step; list entries and row offsets
// prefetched two steps ahead, the row entries one step ahead (so they are in flight while
// the current vertices' color gathers are), pushes buffered per warp.
template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void bin0(const RoundArgs<C>& a, int k, const int32_t* list, int nX,
                                     int32_t* out, int32_t* out_cnt, const C* X, C* Y,
                                     uint8_t* wsm, int gw, int NW, int lane,
                                     unsigned long long& edges, unsigned long long& entries) {
  constexpr int G = kG0, VPW = 32 / kG0;
  if (gw * VPW >= nX) return;
  const int g = lane / G, gl = lane % G;
  const unsigned gmask = ((1u << G) - 1u) << (g * G);
  int32_t* pbuf = reinterpret_cast<int32_t*>(wsm + WarpSmem<C, Hub>::kPush);
  int pending = 0;
  const int step = NW * VPW;
  auto load_row = [&](int32_t vv, int64_t ss, int64_t ee, int32_t (&w)[kK0]) {
    const int32_t cnt = vv >= 0 ? (int32_t)(ee - ss) : 0;
    const int32_t* row = a.col_idx + ss;
#pragma unroll
    for (int u = 0; u < kK0; ++u) w[u] = (gl + G * u < cnt) ? ld_row_h<Hub>(row + gl + G * u) : -1;
  };
  int i = gw * VPW + g;
  int32_t v = i < nX ? ld_cg(list + i) : -1;
  int64_t s = v >= 0 ? ldg_i64(a.row_ptr + v) : 0, e = v >= 0 ? ldg_i64(a.row_ptr + v + 1) : 0;
  int32_t w[kK0];
  load_row(v, s, e, w);
  int32_t v1 = i + step < nX ? ld_cg(list + i + step) : -1;
  int64_t s1 = v1 >= 0 ? ldg_i64(a.row_ptr + v1) : 0, e1 = v1 >= 0 ? ldg_i64(a.row_ptr + v1 + 1) : 0;
  for (int base = gw * VPW; base < nX; base += step) {
    const int32_t v2 = i + 2 * step < nX ? ld_cg(list + i + 2 * step) : -1;
    const int32_t xv = v >= 0 ? ldc<Persist>(X + v) : 0;
    uint32_t lb = 0;
#pragma unroll
    for (int u = 0; u < kK0; ++u) lb |= (w[u] >= 0 && lose<TB>(v, w[u])) ? (1u << u) : 0u;
    bool conf = false;
    uint32_t mask = 0;  // bit i = color i + 1 present (deg <= 32 => first fit <= 33)
    int32_t wn[kK0];
    if (SGR_SMALL_U8 && k <= 255) {
      // byte gathers (ldc8) and a shl.b32 mask: colors >= 32 drop out, the placeholder 0
      // lands on bit 0. Only a group with every color 1..31 present needs color 32: it
      // redoes its scan exactly (rare).
      uint32_t c8[kK0];
#pragma unroll
      for (int u = 0; u < kK0; ++u) c8[u] = (w[u] >= 0) ? ldc8<Persist, Hub>(X + w[u]) : 0u;
      load_row(v1, s1, e1, wn);  // next vertex's row, in flight with the gathers above
      uint32_t m = 0u;
#pragma unroll
      for (int u = 0; u < kK0; ++u) {
        uint32_t bit;
        asm("shl.b32 %0, 1, %1;" : "=r"(bit) : "r"(c8[u]));
        m |= bit;
        conf |= (c8[u] == (uint32_t)xv) & ((lb >> u) & 1u);
      }
#pragma unroll
      for (int o = G / 2; o > 0; o >>= 1) m |= __shfl_xor_sync(0xffffffffu, m, o);
      mask = m >> 1;
      if (__any_sync(0xffffffffu, (mask & 0x7fffffffu) == 0x7fffffffu)) {
        const bool full = (mask & 0x7fffffffu) == 0x7fffffffu;
        uint32_t mx = 0u;
#pragma unroll
        for (int u = 0; u < kK0; ++u) {
          const int32_t c = (full && w[u] >= 0) ? ldc01<Persist, Hub>(X + w[u]) : 0;
          mx |= ((uint32_t)(c - 1) < 32u) ? (1u << (c - 1)) : 0u;
        }
#pragma unroll
        for (int o = G / 2; o > 0; o >>= 1) mx |= __shfl_xor_sync(0xffffffffu, mx, o);
        if (full) mask = mx;
      }
    } else {
      int32_t c[kK0];
#pragma unroll
      for (int u = 0; u < kK0; ++u) c[u] = (w[u] >= 0) ? ldc01<Persist, Hub>(X + w[u]) : 0;
      load_row(v1, s1, e1, wn);  // next vertex's row, in flight with the gathers above
#pragma unroll
      for (int u = 0; u < kK0; ++u) {
        mask |= ((uint32_t)(c[u] - 1) < 32u) ? (1u << (c[u] - 1)) : 0u;
        conf |= (c[u] == xv) & ((lb >> u) & 1u);
      }
#pragma unroll
      for (int o = G / 2; o > 0; o >>= 1) mask |= __shfl_xor_sync(0xffffffffu, mask, o);
    }
    const bool any = (__ballot_sync(0xffffffffu, conf) & gmask) != 0u;
    if (v >= 0 && gl == 0) {
      const int32_t tent = ~mask ? __ffs(~mask) : 33;
      put_y<C>(a, Y, k, v, any ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
      edges += (unsigned long long)(e - s);
      entries += (unsigned long long)(e - s);
    }
    push_buffered<kPushBufOf<Hub>>(v >= 0 && any && gl == 0, v, pbuf, pending, out, out_cnt, lane);
    const int64_t s2 = v2 >= 0 ? ldg_i64(a.row_ptr + v2) : 0;
    const int64_t e2 = v2 >= 0 ? ldg_i64(a.row_ptr + v2 + 1) : 0;
    i += step;
    v = v1;
    s = s1;
    e = e1;
#pragma unroll
    for (int u = 0; u < kK0; ++u) w[u] = wn[u];
    v1 = v2;
    s1 = s2;
    e1 = e2;
  }
  push_flush(pbuf, pending, out, out_cnt, lane);
}

template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void bin0_tiled(const RoundArgs<C>& a, int k, const int32_t* list, int nX,
                                           int* tile_cursor,
                                     int32_t* out, int32_t* out_cnt, const C* X, C* Y,
                                     uint8_t* wsm, int gw, int NW, int lane,
                                     unsigned long long& edges, unsigned long long& entries) {
  constexpr int G = kG0, VPW = 32 / kG0;
  if (gw * VPW >= nX) return;
  const int g = lane / G, gl = lane % G;
  const unsigned gmask = ((1u << G) - 1u) << (g * G);
  int32_t* pbuf = reinterpret_cast<int32_t*>(wsm + WarpSmem<C, Hub>::kPush);
  int pending = 0;
  const int step = NW * VPW;
  auto load_row = [&](int32_t vv, int64_t ss, int64_t ee, int32_t (&w)[kK0]) {
    const int32_t cnt = vv >= 0 ? (int32_t)(ee - ss) : 0;
    const int32_t* row = a.col_idx + ss;
#pragma unroll
    for (int u = 0; u < kK0; ++u) w[u] = (gl + G * u < cnt) ? ld_row_h<Hub>(row + gl + G * u) : -1;
  };
  (void)step;
  StepStream<VPW> gen;  // runs two steps ahead of the step being processed
  gen.init(gw, NW, nX, kTile0, tile_cursor, lane);
  auto pos = [&](int b) { return b < nX ? b + g : nX; };
  int b0 = gen.base();
  gen.advance(lane);
  int b1 = gen.base();
  int i = pos(b0);
  int32_t v = i < nX ? ld_cg(list + i) : -1;
  int64_t s = v >= 0 ? ldg_i64(a.row_ptr + v) : 0, e = v >= 0 ? ldg_i64(a.row_ptr + v + 1) : 0;
  int32_t w[kK0];
  load_row(v, s, e, w);
  int32_t v1 = pos(b1) < nX ? ld_cg(list + pos(b1)) : -1;
  int64_t s1 = v1 >= 0 ? ldg_i64(a.row_ptr + v1) : 0, e1 = v1 >= 0 ? ldg_i64(a.row_ptr + v1 + 1) : 0;
  while (b0 < nX) {
    gen.advance(lane);
    const int b2 = gen.base();
    const int32_t v2 = pos(b2) < nX ? ld_cg(list + pos(b2)) : -1;
    const int32_t xv = v >= 0 ? ldc<Persist>(X + v) : 0;
    uint32_t lb = 0;
#pragma unroll
    for (int u = 0; u < kK0; ++u) lb |= (w[u] >= 0 && lose<TB>(v, w[u])) ? (1u << u) : 0u;
    bool conf = false;
    uint32_t mask = 0;  // bit i = color i + 1 present (deg <= 32 => first fit <= 33)
    int32_t wn[kK0];
    if (SGR_SMALL_U8 && k <= 255) {
      // byte gathers (ldc8) and a shl.b32 mask: colors >= 32 drop out, the placeholder 0
      // lands on bit 0. Only a group with every color 1..31 present needs color 32: it
      // redoes its scan exactly (rare).
      uint32_t c8[kK0];
#pragma unroll
      for (int u = 0; u < kK0; ++u) c8[u] = (w[u] >= 0) ? ldc8<Persist, Hub>(X + w[u]) : 0u;
      load_row(v1, s1, e1, wn);  // next vertex's row, in flight with the gathers above
      uint32_t m = 0u;
#pragma unroll
      for (int u = 0; u < kK0; ++u) {
        uint32_t bit;
        asm("shl.b32 %0, 1, %1;" : "=r"(bit) : "r"(c8[u]));
        m |= bit;
        conf |= (c8[u] == (uint32_t)xv) & ((lb >> u) & 1u);
      }
#pragma unroll
      for (int o = G / 2; o > 0; o >>= 1) m |= __shfl_xor_sync(0xffffffffu, m, o);
      mask = m >> 1;
      if (__any_sync(0xffffffffu, (mask & 0x7fffffffu) == 0x7fffffffu)) {
        const bool full = (mask & 0x7fffffffu) == 0x7fffffffu;
        uint32_t mx = 0u;
#pragma unroll
        for (int u = 0; u < kK0; ++u) {
          const int32_t c = (full && w[u] >= 0) ? ldc01<Persist, Hub>(X + w[u]) : 0;
          mx |= ((uint32_t)(c - 1) < 32u) ? (1u << (c - 1)) : 0u;
        }
#pragma unroll
        for (int o = G / 2; o > 0; o >>= 1) mx |= __shfl_xor_sync(0xffffffffu, mx, o);
        if (full) mask = mx;
      }
    } else {
      int32_t c[kK0];
#pragma unroll
      for (int u = 0; u < kK0; ++u) c[u] = (w[u] >= 0) ? ldc01<Persist, Hub>(X + w[u]) : 0;
      load_row(v1, s1, e1, wn);  // next vertex's row, in flight with the gathers above
#pragma unroll
      for (int u = 0; u < kK0; ++u) {
        mask |= ((uint32_t)(c[u] - 1) < 32u) ? (1u << (c[u] - 1)) : 0u;
        conf |= (c[u] == xv) & ((lb >> u) & 1u);
      }
#pragma unroll
      for (int o = G / 2; o > 0; o >>= 1) mask |= __shfl_xor_sync(0xffffffffu, mask, o);
    }
    const bool any = (__ballot_sync(0xffffffffu, conf) & gmask) != 0u;
    if (v >= 0 && gl == 0) {
      const int32_t tent = ~mask ? __ffs(~mask) : 33;
      put_y<C>(a, Y, k, v, any ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
      edges += (unsigned long long)(e - s);
      entries += (unsigned long long)(e - s);
    }
    push_buffered<kPushBufOf<Hub>>(v >= 0 && any && gl == 0, v, pbuf, pending, out, out_cnt, lane);
    const int64_t s2 = v2 >= 0 ? ldg_i64(a.row_ptr + v2) : 0;
    const int64_t e2 = v2 >= 0 ? ldg_i64(a.row_ptr + v2 + 1) : 0;
    b0 = b1;
    b1 = b2;
    v = v1;
    s = s1;
    e = e1;
#pragma unroll
    for (int u = 0; u < kK0; ++u) w[u] = wn[u];
    v1 = v2;
    s1 = s2;
    e1 = e2;
  }
  push_flush(pbuf, pending, out, out_cnt, lane);
}

// Bin 0, one thread per vertex (SGR_BIN0_THREAD): lane L of the warp takes list position
// 32 step + L. Its row (<= 32 entries) is read as <= 9 int4 of the 16-byte-aligned window,
// then every entry's color is gathered at once (<= 32 loads in flight per lane, 1024 per
// warp), and mask / first fit / conflict are per-lane register work (no shuffles). When the
// worklist is ordered (stencils), the 32 lanes' j-th neighbours are 32 consecutive ids: one
// cache line per gather instruction. The next step's list entry and row offsets are
// prefetched, its row warmed into L1.
template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void bin0_thread(const RoundArgs<C>& a, int k, const int32_t* list,
                                            int nX, int32_t* out, int32_t* out_cnt, const C* X,
                                            C* Y, uint8_t* wsm, int gw, int NW, int lane,
                                            unsigned long long& edges,
                                            unsigned long long& entries) {
  constexpr int kQ = 9;  // int4 per window: offset <= 3 + 32 entries
  if (gw * 32 >= nX) return;
  int32_t* pbuf = reinterpret_cast<int32_t*>(wsm + WarpSmem<C, Hub>::kPush);
  int pending = 0;
  const int step = NW * 32;
  int i = gw * 32 + lane;
  int32_t v = i < nX ? ld_cg(list + i) : -1;
  int64_t s = v >= 0 ? ldg_i64(a.row_ptr + v) : 0, e = v >= 0 ? ldg_i64(a.row_ptr + v + 1) : 0;
  for (int base = gw * 32; base < nX; base += step) {
    const int in = i + step;
    const int32_t vn = in < nX ? ld_cg(list + in) : -1;
    const int32_t xv = v >= 0 ? ldc<Persist>(X + v) : 0;
    const int64_t w0 = s & ~(int64_t)3;
    const int32_t off = (int32_t)(s - w0), cnt = (int32_t)(e - s);
    const int32_t nq = (off + cnt + 3) >> 2;
    int32_t id[4 * kQ];
    const int4* win = reinterpret_cast<const int4*>(a.col_idx + w0);
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
      int4 t = make_int4(0, 0, 0, 0);
      if (q < nq) {
        if (w0 + 4 * q + 4 <= a.nnz) {
          t = ld_row4(win + q);
        } else {  // the array's last, partial 16-byte group: never read past nnz
          const int64_t p0 = w0 + 4 * q;
          t.x = ld_row(a.col_idx + p0);
          if (p0 + 1 < a.nnz) t.y = ld_row(a.col_idx + p0 + 1);
          if (p0 + 2 < a.nnz) t.z = ld_row(a.col_idx + p0 + 2);
        }
      }
      id[4 * q + 0] = t.x;
      id[4 * q + 1] = t.y;
      id[4 * q + 2] = t.z;
      id[4 * q + 3] = t.w;
    }
    // valid slots [off, off + cnt) of the window
    const uint64_t vm = cnt > 0 ? (((cnt >= 64 ? ~0ull : ((1ull << cnt) - 1ull))) << off) : 0ull;
    uint64_t lb = 0;
#pragma unroll
    for (int r = 0; r < 4 * kQ; ++r)
      lb |= (((vm >> r) & 1ull) && lose<TB>(v, id[r])) ? (1ull << r) : 0ull;
    int32_t c[4 * kQ];
#pragma unroll
    for (int r = 0; r < 4 * kQ; ++r) c[r] = ((vm >> r) & 1ull) ? ldc01<Persist, Hub>(X + id[r]) : 0;
    const int64_t sn = vn >= 0 ? ldg_i64(a.row_ptr + vn) : 0;
    const int64_t en = vn >= 0 ? ldg_i64(a.row_ptr + vn + 1) : 0;
    bool conf = false;
    uint32_t mask = 0;  // bit i = color i + 1 present (deg <= 32 => first fit <= 33)
#pragma unroll
    for (int r = 0; r < 4 * kQ; ++r) {
      mask |= ((uint32_t)(c[r] - 1) < 32u) ? (1u << (c[r] - 1)) : 0u;
      conf |= (c[r] == xv) & (((lb >> r) & 1ull) != 0ull);
    }
    if (v >= 0) {
      const int32_t tent = ~mask ? __ffs(~mask) : 33;
      put_y<C>(a, Y, k, v, conf ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
      edges += (unsigned long long)cnt;
      entries += (unsigned long long)cnt;
    }
    push_buffered<kPushBufOf<Hub>>(v >= 0 && conf, v, pbuf, pending, out, out_cnt, lane);
    if (en > sn) prefetch_l1(a.col_idx + sn);
    i = in;
    v = vn;
    s = sn;
    e = en;
  }
  push_flush(pbuf, pending, out, out_cnt, lane);
}

// Bins 0/1 driver: warp w takes list positions 4w + g, 4(w + NW) + g, ... (g = group); the
// next position's list entry and row offsets are prefetched, its row warmed into L2.
template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void bin1(const RoundArgs<C>& a, int k, const int32_t* list, int nX,
                                      int32_t* out, int32_t* out_cnt, const C* X, C* Y,
                                      uint8_t* wsm, int gw, int NW, int lane,
                                      unsigned long long& edges, unsigned long long& entries) {
  const int g = lane >> 3, gl = lane & 7;
  const unsigned gmask = 0xffu << (g * 8);
  uint8_t* gtbl = wsm + WarpSmem<C, Hub>::kBuf + g * kMedTblB;
  int32_t* pbuf = reinterpret_cast<int32_t*>(wsm + WarpSmem<C, Hub>::kPush);
  int pending = 0;
  const int step = NW * 4;
  int i = gw * 4 + g;
  int32_t v = i < nX ? ld_cg(list + i) : -1;
  int64_t s = v >= 0 ? ldg_i64(a.row_ptr + v) : 0, e = v >= 0 ? ldg_i64(a.row_ptr + v + 1) : 0;
  for (int base = gw * 4; base < nX; base += step) {
    const int in = i + step;
    const int32_t vn = in < nX ? ld_cg(list + in) : -1;
    const int64_t sn = vn >= 0 ? ldg_i64(a.row_ptr + vn) : 0;
    const int64_t en = vn >= 0 ? ldg_i64(a.row_ptr + vn + 1) : 0;
    if (sn + 32 * gl < en) prefetch_l2(a.col_idx + sn + 32 * gl);  // 1 line / lane
    bool push = false;
    if (v >= 0 && gl == 0) entries += (unsigned long long)(e - s);
    process_group<TB, Persist, C, Hub>(a, k, v, s, e, X, Y, gtbl, gl, gmask, push, edges);
    push_buffered<kPushBufOf<Hub>>(push, v, pbuf, pending, out, out_cnt, lane);
    i = in;
    v = vn;
    s = sn;
    e = en;
  }
  push_flush(pbuf, pending, out, out_cnt, lane);
}

template <int TB, bool Persist, class C, bool Hub>
__device__ __forceinline__ void bin1_tiled(const RoundArgs<C>& a, int k, const int32_t* list, int nX,
                                            int* tile_cursor,
                                      int32_t* out, int32_t* out_cnt, const C* X, C* Y,
                                      uint8_t* wsm, int gw, int NW, int lane,
                                      unsigned long long& edges, unsigned long long& entries) {
  const int g = lane >> 3, gl = lane & 7;
  const unsigned gmask = 0xffu << (g * 8);
  uint8_t* gtbl = wsm + WarpSmem<C, Hub>::kBuf + g * kMedTblB;
  int32_t* pbuf = reinterpret_cast<int32_t*>(wsm + WarpSmem<C, Hub>::kPush);
  int pending = 0;
  if (gw * 4 >= nX) return;
  StepStream<4> gen;  // one step ahead of the step being processed
  gen.init(gw, NW, nX, kTile1, tile_cursor, lane);
  int b0 = gen.base();
  int i = b0 < nX ? b0 + g : nX;
  int32_t v = i < nX ? ld_cg(list + i) : -1;
  int64_t s = v >= 0 ? ldg_i64(a.row_ptr + v) : 0, e = v >= 0 ? ldg_i64(a.row_ptr + v + 1) : 0;
  while (b0 < nX) {
    gen.advance(lane);
    const int b1 = gen.base();
    const int in = b1 < nX ? b1 + g : nX;
    const int32_t vn = in < nX ? ld_cg(list + in) : -1;
    const int64_t sn = vn >= 0 ? ldg_i64(a.row_ptr + vn) : 0;
    const int64_t en = vn >= 0 ? ldg_i64(a.row_ptr + vn + 1) : 0;
    if (sn + 32 * gl < en) prefetch_l2(a.col_idx + sn + 32 * gl);  // 1 line / lane
    bool push = false;
    if (v >= 0 && gl == 0) entries += (unsigned long long)(e - s);
    process_group<TB, Persist, C, Hub>(a, k, v, s, e, X, Y, gtbl, gl, gmask, push, edges);
    push_buffered<kPushBufOf<Hub>>(push, v, pbuf, pending, out, out_cnt, lane);
    b0 = b1;
    i = in;
    v = vn;
    s = sn;
    e = en;
  }
  push_flush(pbuf, pending, out, out_cnt, lane);
}

// One fused pass F_k over all three bins; every warp of the grid calls it. Static
// round-robin assignment (warp w takes items w, w + NW, ...), with the next item's list
// entry and row offsets prefetched while the current one is processed.
template <int TB, bool Persist, class C, bool Hub, bool T0 = false>
__device__ __forceinline__ void round_body(const RoundArgs<C>& a, int k, const Counts& w,
                                           uint8_t* wsm,
                                           unsigned long long (&edges)[kBins],
                                           unsigned long long (&entries)[kBins],
                                           uint32_t& ph, unsigned long long (&cyc)[kBins]) {
  Ctrl* ctrl = a.ctrl;
  const int p = k & 1;
  const int lane = threadIdx.x & 31;
  const int gw = (int)((grp_block(a) * blockDim.x + threadIdx.x) >> 5);
  const int NW = (int)((grp_size(a) * blockDim.x) >> 5);
  const C* X = sel((k - 1) & 1, (const C*)a.col[0], (const C*)a.col[1]);
  C* Y = sel(k & 1, a.col[0], a.col[1]);
  uint8_t* wtbl = wsm + WarpSmem<C, Hub>::kBuf;
  (void)wtbl;
  auto run_bin2 = [&]() {
    // ---- bin 2 (Hub build only; the flat build runs when bin 2 is empty)
    if constexpr (!Hub) {
    } else if constexpr (packed<C>()) {
      bin2_trimmed<TB, Persist>(a, k, p, X, Y, wsm, gw, NW, lane, w.c, edges[2], entries[2], ph);
    } else {
      const int nC = w.c;
      const int64_t* items = sel(p, (const int64_t*)a.wl_c[0], (const int64_t*)a.wl_c[1]);
      int64_t* out = sel(p ^ 1, a.wl_c[0], a.wl_c[1]);
      int i = gw;
      int64_t it = i < nC ? __ldcg(items + i) : 0;
      int32_t v = (int32_t)((uint64_t)it >> 32);
      int64_t s = i < nC ? ldg_i64(a.row_ptr + v) : 0, e = i < nC ? ldg_i64(a.row_ptr + v + 1) : 0;
      while (i < nC) {
        const int in = i + NW;
        const int64_t itn = in < nC ? __ldcg(items + in) : 0;
        const int32_t vn = (int32_t)((uint64_t)itn >> 32);
        const int64_t sn = in < nC ? ldg_i64(a.row_ptr + vn) : 0;
        const int64_t en = in < nC ? ldg_i64(a.row_ptr + vn + 1) : 0;
        if (in < nC) {  // warm L2 with the next item's 4 KB window (one 128-byte line per lane)
          const int64_t csn = sn + (int64_t)(int32_t)(uint32_t)itn * kChunk;
          const int64_t ln = (csn & ~(int64_t)3) + 32 * lane;
          if (ln < en) prefetch_l2(a.col_idx + ln);
        }
        process_chunk_plain<TB, Persist, C>(a, k, v, (int32_t)(uint32_t)it, s, e, X, Y, out,
                                            &ctrl->ring[rs(k + 1)].c, &ctrl->ring[rs(k + 1)].cv, wtbl,
                                            lane, edges[2], entries[2]);
        i = in;
        it = itn;
        v = vn;
        s = sn;
        e = en;
      }
    }
  };
  auto run_bin1 = [&]() {
    // ---- bin 1: four vertices per warp (one per 8-lane group), 512-byte tables
    // flat build: tiles claimed from a per-pass cursor (ER -4.7 %); hub build: round-robin
    // (tiles there: +0.4 % R-MAT s24, +4 % s16)
    if constexpr (!Hub)
      bin1_tiled<TB, Persist, C, Hub>(
          a, k, sel(p, (const int32_t*)a.wl_m[0], (const int32_t*)a.wl_m[1]), w.m,
          &ctrl->tile_cur[rs(k)][1], sel(p ^ 1, a.wl_m[0], a.wl_m[1]),
          &ctrl->ring[rs(k + 1)].m, X, Y, wsm, gw, NW, lane, edges[1], entries[1]);
    else
      bin1<TB, Persist, C, Hub>(
          a, k, sel(p, (const int32_t*)a.wl_m[0], (const int32_t*)a.wl_m[1]),
          w.m, sel(p ^ 1, a.wl_m[0], a.wl_m[1]), &ctrl->ring[rs(k + 1)].m, X, Y,
          wsm, gw, NW, lane, edges[1], entries[1]);
  };
  auto run_bin0 = [&]() {
    // ---- bin 0: eight vertices per warp, register masks
    // thread per vertex (SGR_BIN0_THREAD; SGR_HUB_B0T: in the hub build only, where the
    // small rows are scattered and short) or 4-lane groups
    if constexpr (SGR_BIN0_THREAD || (Hub && SGR_HUB_B0T))
      bin0_thread<TB, Persist, C, Hub>(
          a, k, sel(p, (const int32_t*)a.wl_t[0], (const int32_t*)a.wl_t[1]),
          w.t, sel(p ^ 1, a.wl_t[0], a.wl_t[1]), &ctrl->ring[rs(k + 1)].t, X, Y,
          wsm, gw, NW, lane, edges[0], entries[0]);
    else if constexpr (!Hub) {
      // T0 (a separate instantiation of the flat build, so the two bin-0 mappings do not
      // share one register allocation): thread per vertex, a lane's whole row in flight
      if constexpr (T0)
        bin0_thread<TB, Persist, C, Hub>(
            a, k, sel(p, (const int32_t*)a.wl_t[0], (const int32_t*)a.wl_t[1]),
            w.t, sel(p ^ 1, a.wl_t[0], a.wl_t[1]), &ctrl->ring[rs(k + 1)].t, X, Y,
            wsm, gw, NW, lane, edges[0], entries[0]);
      else
        bin0_tiled<TB, Persist, C, Hub>(
            a, k, sel(p, (const int32_t*)a.wl_t[0], (const int32_t*)a.wl_t[1]), w.t,
            &ctrl->tile_cur[rs(k)][0], sel(p ^ 1, a.wl_t[0], a.wl_t[1]),
            &ctrl->ring[rs(k + 1)].t, X, Y, wsm, gw, NW, lane, edges[0], entries[0]);
    }
    else
      bin0<TB, Persist, C, Hub>(
          a, k, sel(p, (const int32_t*)a.wl_t[0], (const int32_t*)a.wl_t[1]),
          w.t, sel(p ^ 1, a.wl_t[0], a.wl_t[1]), &ctrl->ring[rs(k + 1)].t, X, Y,
          wsm, gw, NW, lane, edges[0], entries[0]);
  };
  // Order within the pass. Default 2, 1, 0: the large chunk items first (claimed from a
  // cursor), the static small-vertex bins fill the tail. SGR_SMALL_FIRST: 0, 1, 2 (the
  // dynamic bin-2 claims absorb the static bins' imbalance before the barrier).
  long long t0 = pclock();
#if SGR_SMALL_FIRST
  run_bin0();
  long long t1 = pclock();
  cyc[0] += (unsigned long long)(t1 - t0);
  run_bin1();
  long long t2 = pclock();
  cyc[1] += (unsigned long long)(t2 - t1);
  run_bin2();
  cyc[2] += (unsigned long long)(pclock() - t2);
#else
  run_bin2();
  long long t1 = pclock();
  cyc[2] += (unsigned long long)(t1 - t0);
  run_bin1();
  long long t2 = pclock();
  cyc[1] += (unsigned long long)(t2 - t1);
  run_bin0();
  cyc[0] += (unsigned long long)(pclock() - t2);
#endif
}

// ---------------------------------------------------------------------------------------
// Dense passes (flat build, single GPU). While |W_k| > n / SGR_DENSE_DIV (stencils: W = V
// for ~100 of 314 rounds; ER's first rounds) the grid walks V in id order instead of the
// worklists: a warp takes one 32-vertex word of the membership bitmap bm[k & 1] per step,
// one thread per vertex. The 32 rows are one contiguous col_idx segment: the warp copies its
// 16-byte-aligned window into shared memory with asynchronous 16-byte copies (all in flight
// at once), then every lane issues ALL gathers of its row together (a row of <= 32 entries:
// up to 32 loads in flight per lane, 1024 per warp), and the j-th gathers of the 32 lanes
// are the 32 consecutive vertices' j-th neighbours (one or two lines on a stencil). The pass
// writes Y for members, the next bitmap word (ballot of the members that conflict; no
// worklist reads or pushes) and W_{k+1}'s per-bin counts: the sparse pass's exact results.
// When the next pass is sparse, a compaction phase first turns its bitmap into worklists.
#ifndef SGR_DENSE
#define SGR_DENSE 1
#endif
#ifndef SGR_DENSE_DIV
#define SGR_DENSE_DIV 8  // n/2 before the byte-gather dense rows; n/3, n/4, n/8: 8.74, 8.70, 8.64 ms (cfg2)
#endif
#ifndef SGR_DENSE_AHEAD
#define SGR_DENSE_AHEAD 1  // next word staged ahead: cfg2 8.49 -> 8.17 ms
#endif
#ifndef SGR_DENSE_PF2
#define SGR_DENSE_PF2 0  // offsets two words ahead: cfg2 8.18 -> 8.16 ms (noise), off
#endif
#ifndef SGR_DENSE_MAXT
#define SGR_DENSE_MAXT 768  // k_dense launch bounds (768: 80 registers, 3 blocks of 256 / SM)
#endif
#ifndef SGR_DENSE_PF
#define SGR_DENSE_PF 1
#endif
#ifndef SGR_DENSE_U8
#define SGR_DENSE_U8 1  // dense rows of <= 32 entries in passes k <= 255: byte gathers, bit masks
#endif

template <int TB, bool Persist, class C, bool D16>
__device__ __forceinline__ void dense_body(const RoundArgs<C>& a, int k, const C* X, C* Y,
                                           uint8_t* wsm, unsigned long long (&edges)[kBins],
                                           unsigned long long (&entries)[kBins],
                                           int32_t (&nxt)[2]) {
  const int lane = threadIdx.x & 31;
  const int gw = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const int NW = (int)((gridDim.x * blockDim.x) >> 5);
  const uint32_t* bcur = a.bm[k & 1];
  uint32_t* bnxt = a.bm[(k + 1) & 1];
  int32_t* stage0 = reinterpret_cast<int32_t*>(wsm);  // the warp's tables + push buffer
  // D16 && SGR_DENSE_AHEAD: two half-size stages; the next word's rows are copied into the
  // other half before this word is processed, so they land while its gathers run
  constexpr bool kAh = D16 && SGR_DENSE_AHEAD;
  constexpr int kCap = WarpSmem<C, false>::kBytes / 4 / (kAh ? 2 : 1);
  constexpr int kE = D16 ? 8 : 4;  // entries per 16-byte copy
  const int nwords = (a.n + 31) >> 5;
  // the 32 rows of a word are one contiguous segment: its 16-byte-aligned window (capped at
  // the stage) by asynchronous 16-byte copies, all in flight at once, zero-filled past nnz.
  // D16: the segment of dcol (2-byte w - v), half the bytes of col_idx's.
  auto stage_rows = [&](int64_t s0, int64_t e0, int32_t* dst, int64_t& seg0, int32_t& len) {
    seg0 = __shfl_sync(0xffffffffu, s0, 0) & ~(int64_t)(kE - 1);
    const int64_t seg1 = __shfl_sync(0xffffffffu, e0, 31);
    const int32_t nq = (int32_t)min((seg1 - seg0 + kE - 1) / kE, (int64_t)(kCap / 4));
    len = kE * nq;  // staged entries [seg0, seg0 + len)
    for (int32_t q = lane; q < nq; q += 32) {
      const int64_t p0 = seg0 + kE * q;
      const uint32_t bytes = (uint32_t)min((int64_t)16, (a.nnz - p0) * (16 / kE));
      const void* src = D16 ? (const void*)(a.dcol + p0) : (const void*)(a.col_idx + p0);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_addr(dst + 4 * q)),
                   "l"(src), "r"(bytes)
                   : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int half = 0;          // kAh: half holding the current word's rows
  bool ahead = false;    // kAh: they were staged while the previous word was processed
  int64_t seg0_a = 0;
  int32_t len_a = 0;
  // the next word's bitmap word and row offsets are loaded one word ahead (SGR_DENSE_PF):
  // they head the word's dependency chain (offsets -> staged rows -> gathers)
  auto ld_word = [&](int g, uint32_t& wd, int64_t& s, int64_t& e) {
    wd = g < nwords ? __ldcg(bcur + g) : 0u;
    const int32_t v = (g << 5) + lane;
    const bool inr = g < nwords && v < a.n;
    s = inr ? ldg_i64(a.row_ptr + v) : a.nnz;
    e = inr ? ldg_i64(a.row_ptr + v + 1) : a.nnz;
  };
  uint32_t word_n = 0u, word_nn = 0u;
  int64_t s_n = 0, e_n = 0, s_nn = 0, e_nn = 0;
  if (SGR_DENSE_PF) ld_word(gw, word_n, s_n, e_n);
  if (SGR_DENSE_PF2) ld_word(gw + NW, word_nn, s_nn, e_nn);
  for (int g = gw; g < nwords; g += NW) {
    uint32_t word;
    int64_t s, e;
    if (SGR_DENSE_PF2) {  // offsets two words ahead: the next word's stage needs them now
      word = word_n;
      s = s_n;
      e = e_n;
      word_n = word_nn;
      s_n = s_nn;
      e_n = e_nn;
      ld_word(g + 2 * NW, word_nn, s_nn, e_nn);
    } else if (SGR_DENSE_PF) {
      word = word_n;
      s = s_n;
      e = e_n;
      ld_word(g + NW, word_n, s_n, e_n);
    } else {
      ld_word(g, word, s, e);
    }
    uint32_t out = 0u;
    if (word) {
      const int32_t v = (g << 5) + lane;
      int32_t* stage = stage0 + (kAh ? half * kCap : 0);
      int64_t seg0;
      int32_t len;
      if (kAh && ahead) {
        seg0 = seg0_a;
        len = len_a;
      } else {
        __syncwarp();
        stage_rows(s, e, stage, seg0, len);
      }
      ahead = false;
      if (kAh && SGR_DENSE_PF && word_n) {  // the next word's rows into the other half
        stage_rows(s_n, e_n, stage0 + (half ^ 1) * kCap, seg0_a, len_a);
        ahead = true;
        asm volatile("cp.async.wait_group 1;" ::: "memory");
      } else {
        asm volatile("cp.async.wait_group 0;" ::: "memory");
      }
      __syncwarp();
      half ^= kAh ? 1 : 0;
      const bool mem = (word >> lane) & 1u;
      bool conf = false;
      const int16_t* st16 = reinterpret_cast<const int16_t*>(stage);
      // staged entry i -> neighbour id
      auto nb = [&](int32_t i) -> int32_t { return D16 ? v + (int32_t)st16[i] : stage[i]; };
      if (mem) {
        const int32_t xv = ldc<Persist>(X + v);
        const int32_t d = (int32_t)(e - s);
        const int32_t off = (int32_t)(s - seg0);
        int32_t tent = 0;
        bool done = false;
#if SGR_DENSE_U8
        if (d <= 32 && off + d <= len && k <= 255 && xv < 32) {
          // pass k reads C_k, whose colors are <= k <= 255: a word's low byte is its color
          // (byte gathers, nothing to decode). Colors as bits of one 32-bit mask (shl.b32
          // yields 0 for shifts >= 32; the color-0 placeholder of unused slots lands on bit 0,
          // never a color) and the colors of the neighbours v loses to as a second mask, so
          // the conflict test is one bit of it. A first fit beyond 31 takes the exact loop.
          uint32_t c[32];
          uint32_t lb = 0u;  // bit j: v loses to the j-th neighbour
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            c[j] = 0u;
            if (j < d) {
              const int32_t w = nb(off + j);
              lb |= lose<TB>(v, w) ? (1u << j) : 0u;
              c[j] = *reinterpret_cast<const uint8_t*>(X + w);  // little endian: low byte
            }
          }
          uint32_t m = 1u, ml = 0u;
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            uint32_t bit;
            asm("shl.b32 %0, 1, %1;" : "=r"(bit) : "r"(c[j]));
            m |= bit;
            if ((lb >> j) & 1u) ml |= bit;
          }
          if (~m) {
            tent = __ffs(~m) - 1;
            conf = (ml >> xv) & 1u;
            done = true;
          }
        }
        if (done) {
        } else
#endif
        if (d <= 32 && off + d <= len) {  // the whole row is staged: every gather at once
          int32_t c[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) c[j] = j < d ? ldc<Persist>(X + nb(off + j)) : 0;
          uint32_t m = 0;  // bit c - 1 = color c present (first fit <= 33)
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const uint32_t ci = (uint32_t)(c[j] - 1);
            m |= ci < 32u ? (1u << ci) : 0u;
            if (c[j] == xv && j < d) conf |= lose<TB>(v, nb(off + j));
          }
          tent = ~m ? __ffs(~m) : 33;
        } else {  // long or unstaged row: batches of 8, 4 x 64-bit masks (deg <= 256)
          uint64_t m0 = 0, m1 = 0, m2 = 0, m3 = 0;
          for (int32_t j = 0; j < d; j += 8) {
            int32_t w[8], c[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              const int32_t q = off + j + u;
              w[u] = j + u < d ? (q < len ? nb(q) : ld_row(a.col_idx + s + j + u)) : -1;
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) c[u] = w[u] >= 0 ? ldc<Persist>(X + w[u]) : 0;
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              const uint32_t ci = (uint32_t)(c[u] - 1);
              const uint64_t bit = 1ull << (ci & 63u);
              m0 |= ci < 64u ? bit : 0ull;
              m1 |= ci - 64u < 64u ? bit : 0ull;
              m2 |= ci - 128u < 64u ? bit : 0ull;
              m3 |= ci - 192u < 64u ? bit : 0ull;
              conf |= w[u] >= 0 && c[u] == xv && lose<TB>(v, w[u]);
            }
          }
          tent = 257;
          if (~m3) tent = 192 + __ffsll((long long)~m3);
          if (~m2) tent = 128 + __ffsll((long long)~m2);
          if (~m1) tent = 64 + __ffsll((long long)~m1);
          if (~m0) tent = __ffsll((long long)~m0);
        }
        put_y<C>(a, Y, k, v, conf ? cpack<C>(tent, k + 1, a) : cpack<C>(xv, k, a));
        // constant indices only: a runtime bin index would put the counters on the stack
        const bool b0 = d <= a.small_max;
        const unsigned long long d0 = b0 ? (unsigned long long)d : 0ull;
        const unsigned long long d1 = b0 ? 0ull : (unsigned long long)d;
        edges[0] += d0;
        edges[1] += d1;
        entries[0] += d0;
        entries[1] += d1;
        nxt[0] += (conf && b0) ? 1 : 0;
        nxt[1] += (conf && !b0) ? 1 : 0;
      }
      out = __ballot_sync(0xffffffffu, mem && conf);
    }
    if (lane == 0) bnxt[g] = out;
  }
  __syncwarp();
}

// W_k's bin worklists from its bitmap (the first sparse pass after dense ones, once per
// coloring): members in id order, pushed with one atomicAdd per warp and bin; the counts
// were produced by the dense pass. The warp's shared tables are re-zeroed (the dense passes
// used them as row stages).
template <class C>
__device__ __forceinline__ void dense_to_lists(const RoundArgs<C>& a, int k, uint8_t* wsm) {
  const int lane = threadIdx.x & 31;
  const int gw = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const int NW = (int)((gridDim.x * blockDim.x) >> 5);
  set_clear(wsm + WarpSmem<C, false>::kBuf, kTblBytes, lane, 32);
  const uint32_t* bm = a.bm[k & 1];
  int32_t* lt = sel(k & 1, a.wl_t[0], a.wl_t[1]);
  int32_t* lm = sel(k & 1, a.wl_m[0], a.wl_m[1]);
  const int nwords = (a.n + 31) >> 5;
  for (int g = gw; g < nwords; g += NW) {
    const uint32_t word = __ldcg(bm + g);
    if (!word) continue;  // warp-uniform
    const int32_t v = (g << 5) + lane;
    const bool mem = (word >> lane) & 1u;
    const int64_t d = mem ? ldg_i64(a.row_ptr + v + 1) - ldg_i64(a.row_ptr + v) : 0;
    const bool b0 = mem && d <= a.small_max, b1 = mem && d > a.small_max;
    const unsigned m0 = __ballot_sync(0xffffffffu, b0), m1 = __ballot_sync(0xffffffffu, b1);
    int o0 = 0, o1 = 0;
    if (lane == 0) {
      if (m0) o0 = atomicAdd(&a.ctrl->cmp_cnt[0], __popc(m0));
      if (m1) o1 = atomicAdd(&a.ctrl->cmp_cnt[1], __popc(m1));
    }
    o0 = __shfl_sync(0xffffffffu, o0, 0);
    o1 = __shfl_sync(0xffffffffu, o1, 0);
    const unsigned lt_mask = (1u << lane) - 1u;
    if (b0) lt[o0 + __popc(m0 & lt_mask)] = v;
    if (b1) lm[o1 + __popc(m1 & lt_mask)] = v;
  }
  __syncwarp();
}

// Block sum of two per-thread counts, added to *d0 / *d1 with one atomic each.
__device__ __forceinline__ void block_add2(int32_t (&x)[2], int32_t* d0, int32_t* d1) {
  __shared__ int32_t red2[2][kMaxWarps];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int32_t a0 = __reduce_add_sync(0xffffffffu, x[0]);
  const int32_t a1 = __reduce_add_sync(0xffffffffu, x[1]);
  if (lane == 0) {
    red2[0][wid] = a0;
    red2[1][wid] = a1;
  }
  __syncthreads();
  if (threadIdx.x < 2) {
    int32_t t = 0;
    for (int q = 0; q < (int)(blockDim.x >> 5); ++q) t += red2[threadIdx.x][q];
    if (t) atomicAdd(threadIdx.x == 0 ? d0 : d1, t);
  }
}

// Block reduction of the per-thread counters, one atomicAdd each per block.
__device__ __forceinline__ void block_add6(unsigned long long (&x)[kBins],
                                           unsigned long long (&y)[kBins], Ctrl* ctrl, int k) {
  __shared__ unsigned long long red[2 * kBins][kMaxWarps];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
  for (int q = 0; q < 2 * kBins; ++q) {
    unsigned long long z = q < kBins ? x[q] : y[q - kBins];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) z += __shfl_xor_sync(0xffffffffu, z, o);
    if (lane == 0) red[q][wid] = z;
  }
  __syncthreads();
  if (wid == 0) {
#pragma unroll
    for (int q = 0; q < 2 * kBins; ++q) {
      unsigned long long z = lane < (int)(blockDim.x >> 5) ? red[q][lane] : 0ull;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) z += __shfl_xor_sync(0xffffffffu, z, o);
      if (lane == 0 && z) {
        if (q < kBins) atomicAdd(&ctrl->edges_acc[rs(k)][q], z);
        else atomicAdd(&ctrl->entries_acc[rs(k)][q - kBins], z);
      }
    }
  }
}

// Counts written by other blocks' atomics: read at L2 (ld.global.cg), never a stale L1 line.
__device__ __forceinline__ Counts ld_counts(const Counts* p) {
  const int4* q = reinterpret_cast<const int4*>(p);
  const int4 x = __ldcg(q), y = __ldcg(q + 1);
  Counts w;
  w.t = x.x; w.m = x.y; w.c = x.z; w.cv = x.w;
  w.fin = y.x; w.pad[0] = y.y; w.pad[1] = y.z; w.pad[2] = y.w;
  return w;
}

__device__ __forceinline__ void stamp_round(Ctrl* c, int idx) {
  if (c->round_ns && idx < c->round_cap) {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    c->round_ns[idx] = (int64_t)t;
  }
}

// After F_1 (one thread): W_2's counts are in ring slot 2.
__device__ __forceinline__ void first_body(Ctrl* c) {
  const Counts w = ld_counts(&c->ring[rs(2)]);
  c->pushes_total[kBins] = (unsigned long long)(w.t + w.m + w.cv);
  c->k = 2;
  c->active = (w.t + w.m + w.c) > 0 && !__ldcg(&c->overflow);
  if (c->active && c->max_rounds < 2) {
    c->status = 1;
    c->active = 0;
  }
  stamp_round(c, 0);
}

// Fold finished pass F_k into the totals and the trace (one thread, any time after every
// block of pass k is done and before pass k+2 pushes into slot k % 3), then zero slot k % 3.
// A pass over an empty W_k changes nothing, so surplus passes are no-ops.
__device__ __forceinline__ void fold_pass(Ctrl* c, int k) {
  const Counts win = ld_counts(&c->ring[rs(k)]), wout = ld_counts(&c->ring[rs(k + 1)]);
  const int vin[kBins] = {win.t, win.m, win.cv};
  const int vout[kBins] = {wout.t, wout.m, wout.cv};
  unsigned long long e_all = 0, x_all = 0;
  int tot_in = 0;
  for (int q = 0; q < kBins; ++q) {
    const unsigned long long e = __ldcg(&c->edges_acc[rs(k)][q]);
    const unsigned long long x = __ldcg(&c->entries_acc[rs(k)][q]);
    // fire-and-forget reductions: the folding thread never waits on the totals
    atomicAdd(&c->verts_total[q], (unsigned long long)vin[q]);
    atomicAdd(&c->edges_total[q], e);
    atomicAdd(&c->entries_total[q], x);
    atomicAdd(&c->pushes_total[q], (unsigned long long)vout[q]);
    c->edges_acc[rs(k)][q] = 0ull;
    c->entries_acc[rs(k)][q] = 0ull;
    e_all += e;
    x_all += x;
    tot_in += vin[q];
  }
  atomicAdd(&c->items_total, (unsigned long long)win.c);
  c->ring[rs(k)] = Counts{};
  c->tile_cur[rs(k)][0] = 0;
  c->tile_cur[rs(k)][1] = 0;
  if (k - 1 < c->round_cap) {
    if (c->round_sizes) c->round_sizes[k - 1] = tot_in;
    // SGR_TRACE_ENTRIES (experiment builds only): trace the list entries actually read
    if (c->round_edges) c->round_edges[k - 1] = (int64_t)(SGR_TRACE_ENTRIES ? x_all : e_all);
  }
  stamp_round(c, k - 1);
}

__device__ __forceinline__ int items_of(const Counts& w) { return w.t + w.m + w.c; }

// Host / graph loop modes, after pass F_k (and its finalize): fold it, advance k and decide
// whether W_{k+1} is non-empty. Multi-GPU ranks advance in lockstep (force).
__device__ __forceinline__ void advance_body(Ctrl* ctrl, bool first, bool force = false) {
  Ctrl* c = ctrl;
  if (first) {
    first_body(c);
    return;
  }
  const int k = c->k;
  if (items_of(ld_counts(&c->ring[rs(k)])) == 0 && !force) {
    c->active = 0;
    return;
  }
  fold_pass(c, k);
  c->k = k + 1;
  c->active = items_of(ld_counts(&c->ring[rs(k + 1)])) > 0 && !__ldcg(&c->overflow);
  if (c->active && k + 1 > c->max_rounds) {  // W_{k+1} non-empty beyond the cap
    c->status = 1;
    c->active = 0;
  }
}

static __global__ void k_advance(Ctrl* ctrl, int first, int force = 0) {
  if (threadIdx.x == 0 && blockIdx.x == 0) advance_body(ctrl, first != 0, force != 0);
}

// ---------------------------------------------------------------------------------------
// Multi-GPU exchange. After pass F_k the rank's next worklists hold its
// owned part of W_{k+1}; every other replica needs those vertices' new color words.
// Record = (v, word); slot 0 of a send buffer carries (count, 0).
template <class C>
__global__ void k_pack(RoundArgs<C> a, uint2* send, int32_t cap, int pre = 0) {
  Ctrl* ctrl = a.ctrl;
  // W_k's lists are the new ones: k = ctrl->k once advanced, ctrl->k + 1 when the pack runs
  // before the advance (pre = 1; the round loop advances in k_apply)
  const int k = ctrl->k + pre;
  const int p = k & 1;
  const C* Y = sel((k - 1) & 1, (const C*)a.col[0], (const C*)a.col[1]);
  const Counts w = ctrl->ring[rs(k)];
  const int nT = w.t, nM = w.m, nC = w.c;
  const int32_t* lt = sel(p, (const int32_t*)a.wl_t[0], (const int32_t*)a.wl_t[1]);
  const int32_t* lm = sel(p, (const int32_t*)a.wl_m[0], (const int32_t*)a.wl_m[1]);
  const int64_t* lc = sel(p, (const int64_t*)a.wl_c[0], (const int64_t*)a.wl_c[1]);
  int32_t* count = reinterpret_cast<int32_t*>(&send[0].x);
  if (blockIdx.x == 0 && threadIdx.x == 0) send[0].y = (uint32_t)ctrl->overflow;
  const int64_t total = (int64_t)nT + nM + nC;
  for (int64_t base = (int64_t)blockIdx.x * blockDim.x; base < total;
       base += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = base + threadIdx.x;
    int32_t v = -1;
    if (i < nT) v = lt[i];
    else if (i < nT + nM) v = lm[i - nT];
    else if (i < total) {
      const int64_t it = lc[i - nT - nM];
      if (((uint32_t)it & kChunkMask) == 0u) v = (int32_t)((uint64_t)it >> 32);  // chunk 0
    }
    const unsigned m = __ballot_sync(0xffffffffu, v >= 0);
    if (m) {
      const int lane = threadIdx.x & 31;
      int b = 0;
      if (lane == __ffs(m) - 1) b = atomicAdd(count, __popc(m));
      b = __shfl_sync(0xffffffffu, b, __ffs(m) - 1);
      if (v >= 0) {
        const int slot = b + __popc(m & ((1u << lane) - 1u));
        if (slot < cap) send[1 + slot] = make_uint2((uint32_t)v, (uint32_t)Y[v]);
      }
    }
  }
}

// Apply every other part's records to this replica: both ping-pong buffers, because a
// remote vertex is only ever written by these updates.
template <class C>
__global__ void k_apply(RoundArgs<C> a, const uint2* recv, int32_t parts, int32_t stride,
                        int32_t me, uint2* send_reset = nullptr, int adv = 0) {
  // Round loop: this launch also carries the lockstep advance of pass k (the pack already
  // read W_{k+1}) and re-arms the send count for the next pack (the all-gather has consumed
  // it) — two fewer stream operations per round.
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    if (adv) advance_body(a.ctrl, false, true);
    if (send_reset) send_reset[0].x = 0u;
  }
  for (int q = 0; q < parts; ++q) {
    if (q == me) continue;
    const uint2* r = recv + (int64_t)q * stride;
    int32_t cnt = (int32_t)r[0].x;
    // A count above the slot capacity means W_{k+1} is not inside W_k on that rank, which
    // the method guarantees for a symmetric CSR (DESIGN.md §3 proof ii): never read past
    // the sender's block; flag it (bit 8 of violations, reported as SGR_EINVAL).
    if (cnt > stride - 1 || cnt < 0) {
      if (threadIdx.x == 0 && blockIdx.x == 0) atomicOr(&a.ctrl->violations, 8);
      cnt = cnt < 0 ? 0 : stride - 1;
    }
    for (int32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < cnt; i += gridDim.x * blockDim.x) {
      const uint2 rec = r[1 + i];
      a.col[0][rec.x] = (C)rec.y;
      a.col[1][rec.x] = (C)rec.y;
    }
  }
}

// Initialise both color buffers of a replica to C_1 (every vertex colored 1 in round 1).
template <class C>
__global__ void k_fill_c1(RoundArgs<C> a) {
  const C one = packed<C>() ? (C)((1u << kRoundShift) | 1u) : (C)1;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n;
       i += (int64_t)gridDim.x * blockDim.x) {
    a.col[0][i] = one;
    a.col[1][i] = one;
  }
}

// Kernel prologue: zero the warp tables, initialise the warp's two TMA mbarriers.
template <class C, bool Hub = true>
__device__ __forceinline__ uint8_t* warp_smem_init(uint8_t* smem) {
  const int wid = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint8_t* wsm = smem + wid * WarpSmem<C, Hub>::kBytes;
  set_clear(wsm + WarpSmem<C, Hub>::kBuf, kTblBytes, lane, 32);
  if constexpr (packed<C>() && Hub) {
    if (lane == 0) {
      uint64_t* bars = reinterpret_cast<uint64_t*>(wsm + WarpSmem<C, Hub>::kBars);
      mbar_init(bars + 0, 1);  // bin-2 stages: one elected arrival per phase
      mbar_init(bars + 1, 1);
      mbar_init_fence();
    }
  }
  __syncthreads();
  return wsm;
}

// One pass per launch (host / graph loop modes, distributed rounds); k_advance (or the
// distributed k_apply) follows it on the stream. Hub = false is the flat build (bins 0/1
// only), for colorings whose F_1 put no vertex into bin 2 (the caller reads big_count).
template <int TB, class C, bool Hub = true>
__global__ void __launch_bounds__(kMaxThreads<C, Hub>, 1) k_round(RoundArgs<C> a) {
  extern __shared__ __align__(16) uint8_t dsmem[];
  Ctrl* ctrl = a.ctrl;
  if (!ctrl->active) return;  // uniform across the grid
  uint8_t* wsm = warp_smem_init<C, Hub>(dsmem);
  unsigned long long edges[kBins] = {0, 0, 0}, entries[kBins] = {0, 0, 0};
  unsigned long long cyc[kBins] = {0, 0, 0};
  uint32_t ph = 0;
  const int k = ctrl->k;
  const Counts w = ctrl->ring[rs(k)];
  round_body<TB, false, C, Hub>(a, k, w, wsm, edges, entries, ph, cyc);
  block_add6(edges, entries, ctrl, k);
  // bin cycle stats: one atomic per block and bin (per-warp atomics were ~7K same-address
  // reductions per launch, on every pass of the host-driven loops)
  __shared__ unsigned long long cred[kBins][kMaxWarps];
  if (!SGR_PHASE_CYCLES) return;
  if ((threadIdx.x & 31) == 0)
    for (int q = 0; q < kBins; ++q) cred[q][threadIdx.x >> 5] = cyc[q];
  __syncthreads();
  if (threadIdx.x < kBins) {
    unsigned long long z = 0;
    for (int i = 0; i < (int)(blockDim.x >> 5); ++i) z += cred[threadIdx.x][i];
    atomicAdd(&ctrl->bin_cycles[threadIdx.x], z);
  }
}

// Finalize phase as its own launch (host / graph loop modes), between k_round and k_advance.
template <int TB, class C>
__global__ void __launch_bounds__(kBlock) k_finalize(RoundArgs<C> a) {
  if constexpr (packed<C>()) {
    if (!a.ctrl->active) return;
    finalize_body<TB, false>(a, a.ctrl->k);
  }
}

__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_gpu(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t atom_add_acq_rel_u32(uint32_t* p, uint32_t v) {
  uint32_t r;
  asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "r"(v) : "memory");
  return r;
}

// Grid-wide barrier of the persistent kernel (every block resident).
// Monotonic arrival counter (zeroed per coloring): thread 0 of each block adds 1 with
// release semantics (publishing, via the preceding bar.sync, every write of its block) and
// waits with acquire loads until barrier number `epoch` has all gridDim.x arrivals. No
// last-arriver reset/release step: one L2 round trip less per barrier.
__device__ __forceinline__ void red_release_gpu_u32(uint32_t* p, uint32_t v) {
  asm volatile("red.release.gpu.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void grid_sync(Ctrl* ctrl, uint32_t& epoch) {
  __syncthreads();
  ++epoch;
  if (threadIdx.x == 0) {
    red_release_gpu_u32(&ctrl->bar_count, 1u);
    const uint32_t target = epoch * gridDim.x;
    // poll with relaxed loads (served by L2; an acquire load would invalidate this SM's L1
    // on every poll, evicting the lines the SM's other blocks are still gathering from),
    // then one acquire load once the count is reached
    while ((int32_t)(ld_relaxed_gpu(&ctrl->bar_count) - target) < 0) {
      if (SGR_BARSLEEP) __nanosleep(SGR_BARSLEEP);
    }
    (void)ld_acquire_gpu(&ctrl->bar_count);
  }
  __syncthreads();
}

// All rounds in one cooperative launch (every block resident). Each block tracks k itself
// and reads W_k's counts after the barrier that ends pass k-1; block 0 folds pass k-1 into
// the totals while pass k runs. The host enqueues both builds; each returns at once unless
// it is the right one for this coloring (Hub iff F_1 put a vertex into bin 2), so the
// choice needs no host round trip.
// Flat build, bin-0 mapping: graphs with non-local rows (F_1's mean row width >= n / 16:
// ER-like, the graphs that get no dense passes) and a color array beyond ~8 MB take the
// thread-per-vertex instantiation (T0; cfg3 ER 2^24 -6 %): a lane's whole row in flight at
// once covers the L2 latency of scattered gathers. Local rows keep the 4-lane groups, whose
// gathers share lines (stencil +4 % with threads), as do small graphs whose colors stay
// near (rmat-er s20 +5 %). Uniform over the grid; read after F_1 (same stream).
template <class C>
__device__ __forceinline__ bool flat_thread_bin0(const RoundArgs<C>& a) {
  if (a.bm[0] == nullptr || a.flat_bin0 == 1) return false;
  if (a.flat_bin0 == 2) return true;
  return SGR_FLAT_B0T && a.n >= (1 << 22) &&
         __ldcg(&a.ctrl->span_sum) > (unsigned long long)a.n * (unsigned long long)a.n / SGR_DENSE_SPAN;
}

template <int TB, class C, bool Hub, bool T0 = false>
__global__ void __launch_bounds__(kMaxThreads<C, Hub>, 1) k_persistent(RoundArgs<C> a) {
  extern __shared__ __align__(16) uint8_t dsmem[];
  Ctrl* ctrl = a.ctrl;
  if ((ld_cg(&ctrl->big_count) != 0) != Hub) return;  // uniform across the grid
  if constexpr (!Hub) {
    if (flat_thread_bin0(a) != T0) return;  // the other flat instantiation runs
  }
  if (!ld_cg(&ctrl->active)) return;                   // F_1 left W_2 empty
  uint8_t* wsm = warp_smem_init<C, Hub>(dsmem);
  uint32_t ph = 0;  // mbarrier phase bits of the warp's two TMA stages
  unsigned long long cyc[kBins] = {0, 0, 0};
  unsigned long long pcx[3] = {0, 0, 0};  // barrier waits, finalize, counter reduction
  uint32_t epoch = 0;                     // grid barriers passed
  const int max_rounds = ld_cg(&ctrl->max_rounds);
  // the last block folds the finished pass: it is the one that draws work last (items go to
  // the lowest warp ids first), so the fold is off the critical path of thin rounds
  const bool leader = blockIdx.x == gridDim.x - 1 && threadIdx.x == 0;
  // pass 2, or the first sparse pass after k_dense's dense passes (it sets ctrl->k)
  int k = ld_cg(&ctrl->k);
  for (;; ++k) {
    const Counts w = ld_counts(&ctrl->ring[rs(k)]);
    const int overflow = ld_cg(&ctrl->overflow);
    if (leader && k > 2) fold_pass(ctrl, k - 1);
    const bool active = items_of(w) > 0 && !overflow;
    if (!active || k > max_rounds) {  // uniform: every block read the same values
      if (leader) {
        ctrl->k = k;
        ctrl->active = 0;
        if (active) ctrl->status = 1;  // W_k non-empty beyond the cap
      }
      break;
    }
    unsigned long long edges[kBins] = {0, 0, 0}, entries[kBins] = {0, 0, 0};
    round_body<TB, true, C, Hub, T0>(a, k, w, wsm, edges, entries, ph, cyc);
    const long long t0 = pclock();
    block_add6(edges, entries, ctrl, k);
    const long long t1 = pclock();
    pcx[2] += (unsigned long long)(t1 - t0);
    // multi-chunk vertices: decided once all chunks are in (no finalize phase, and no
    // barrier for it, when W_k has none — most thin rounds of a skewed graph's tail)
    bool fin_phase = false;
    if constexpr (packed<C>() && Hub) fin_phase = w.pad[1] != 0;  // uniform over the grid
    if (fin_phase) {
      grid_sync(ctrl, epoch);
      const long long t2 = pclock();
      if constexpr (packed<C>() && Hub) finalize_body<TB, true>(a, k);
      const long long t3 = pclock();
      pcx[0] += (unsigned long long)(t2 - t1);
      pcx[1] += (unsigned long long)(t3 - t2);
      grid_sync(ctrl, epoch);
      pcx[0] += (unsigned long long)(pclock() - t3);
    } else {
      grid_sync(ctrl, epoch);
      pcx[0] += (unsigned long long)(pclock() - t1);
    }
  }
  if (SGR_PHASE_CYCLES && (threadIdx.x & 31) == 0) {
    for (int q = 0; q < kBins; ++q) atomicAdd(&ctrl->bin_cycles[q], cyc[q]);
    for (int q = 0; q < 3; ++q) atomicAdd(&ctrl->phase_cycles[4 + q], pcx[q]);
  }
}

// ---------------------------------------------------------------------------------------
// Multi-part persistent kernel: the distributed rounds with the exchange done
// on the device. Each part (a vertex range with its own rows, worklists and a full color
// replica) runs the same fused pass as k_persistent in its own block group; put_y stores
// every color word the part writes into all replicas as well (other parts of this device,
// or NVLink peer memory when each GPU holds one part), so after the pass barrier every
// replica holds C_{k+1} and no exchange step, host round trip or collective launch remains.
// The pass barrier spans all parts: a group barrier on the part's own counter, then the
// group's first block signals every other part's cross counter (red.release.sys) and waits
// for all of theirs (ld.acquire.sys), then a second group barrier. Loop decisions use the
// counts of ALL parts (termination, color overflow, the finalize phase), read after it.
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int32_t ld_relaxed_sys_i32(const int32_t* p) {
  int32_t v;
  asm volatile("ld.relaxed.sys.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_release_sys_u32(uint32_t* p, uint32_t v) {
  asm volatile("red.release.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Barrier of one block group (nblk blocks) on `ctrl->bar_count` (as grid_sync).
__device__ __forceinline__ void group_sync(Ctrl* ctrl, uint32_t& epoch, int nblk) {
  __syncthreads();
  ++epoch;
  if (threadIdx.x == 0) {
    red_release_gpu_u32(&ctrl->bar_count, 1u);
    const uint32_t target = epoch * (uint32_t)nblk;
    while ((int32_t)(ld_relaxed_gpu(&ctrl->bar_count) - target) < 0) {
      if (SGR_BARSLEEP) __nanosleep(SGR_BARSLEEP);
    }
    (void)ld_acquire_gpu(&ctrl->bar_count);
  }
  __syncthreads();
}

template <class C>
__device__ __forceinline__ void part_sync(const RoundArgs<C>& a, uint32_t& epoch, uint32_t& xepoch) {
  const int nblk = grp_size(a);
  group_sync(a.ctrl, epoch, nblk);
  if (a.nranks > 1) {
    if (grp_block(a) == 0 && threadIdx.x == 0) {
      ++xepoch;
      for (int q = 0; q < a.nranks; ++q)
        if (q != a.me) red_release_sys_u32(a.xbar[q], 1u);
      const uint32_t target = xepoch * (uint32_t)(a.nranks - 1);
      uint32_t* mine = a.xbar[a.me];
      while ((int32_t)(ld_relaxed_sys(mine) - target) < 0) {
        if (SGR_BARSLEEP) __nanosleep(SGR_BARSLEEP);
      }
      (void)ld_acquire_sys(mine);
    } else {
      ++xepoch;
    }
    group_sync(a.ctrl, epoch, nblk);
  }
}

// Counts of pass k over all parts (thread 0 reads them, the block shares them).
struct GlobalCounts {
  int64_t items;
  int32_t overflow;
  int32_t multi;  // multi-chunk bin-2 vertices anywhere (the finalize phase is global)
};
template <class C>
__device__ __forceinline__ GlobalCounts global_counts(const RoundArgs<C>& a, int k) {
  __shared__ GlobalCounts gc;
  if (threadIdx.x == 0) {
    GlobalCounts g{0, 0, 0};
    for (int q = 0; q < a.nranks; ++q) {
      const Counts* r = &a.rctrl[q]->ring[rs(k)];
      g.items += (int64_t)ld_relaxed_sys_i32(&r->t) + ld_relaxed_sys_i32(&r->m) + ld_relaxed_sys_i32(&r->c);
      g.multi |= ld_relaxed_sys_i32(&r->pad[1]) != 0;
      g.overflow |= ld_relaxed_sys_i32(&a.rctrl[q]->overflow);
    }
    gc = g;
  }
  __syncthreads();
  const GlobalCounts g = gc;
  __syncthreads();  // gc is rewritten by the next call
  return g;
}

template <int TB, class C, bool Hub>
__device__ __forceinline__ void dist_body(const RoundArgs<C>& a, uint8_t* dsmem) {
  Ctrl* ctrl = a.ctrl;
  uint8_t* wsm = warp_smem_init<C, Hub>(dsmem);
  uint32_t ph = 0;
  unsigned long long cyc[kBins] = {0, 0, 0};
  uint32_t epoch = 0, xepoch = 0;
  const int max_rounds = ld_cg(&ctrl->max_rounds);
  const bool leader = grp_block(a) == grp_size(a) - 1 && threadIdx.x == 0;
  // every part's F_1 (and its broadcast of C_2) finished before this launch (stream order /
  // the host's cross-rank sync), so pass 2 can start at once
  int k = 2;
  for (;; ++k) {
    const Counts w = ld_counts(&ctrl->ring[rs(k)]);
    const GlobalCounts g = global_counts(a, k);
    if (leader && k > 2) fold_pass(ctrl, k - 1);
    const bool active = g.items > 0 && !g.overflow;
    if (!active || k > max_rounds) {  // uniform over all parts
      if (leader) {
        ctrl->k = k;
        ctrl->active = 0;
        if (active) ctrl->status = 1;
        if (g.overflow) ctrl->overflow = 1;  // every part reruns with int32 words
      }
      break;
    }
    unsigned long long edges[kBins] = {0, 0, 0}, entries[kBins] = {0, 0, 0};
    round_body<TB, true, C, Hub>(a, k, w, wsm, edges, entries, ph, cyc);
    block_add6(edges, entries, ctrl, k);
    bool fin_phase = false;
    if constexpr (packed<C>() && Hub) fin_phase = g.multi != 0;  // uniform over all parts
    if (fin_phase) {  // a part's multi-chunk vertices are all its own: a group barrier
      group_sync(ctrl, epoch, grp_size(a));
      if constexpr (packed<C>() && Hub) finalize_body<TB, true>(a, k);
    }
    part_sync(a, epoch, xepoch);
  }
}

// Multi = false: one part per launch (each GPU of a multi-GPU coloring, or one partition):
// its arguments stay kernel parameters. Multi = true: `nparts` block groups on this device,
// each block copying its part's arguments from `parts`.
template <int TB, class C, bool Hub, bool Multi>
__global__ void __launch_bounds__(kMaxThreads<C, Hub>, 1) k_persistent_dist(RoundArgs<C> a0,
                                                                        const RoundArgs<C>* __restrict__ parts,
                                                                        int nparts) {
  extern __shared__ __align__(16) uint8_t dsmem[];
  if constexpr (Multi) {
    const int gB = (int)gridDim.x / nparts;
    const int p = min((int)blockIdx.x / gB, nparts - 1);
    const RoundArgs<C> a = parts[p];
    dist_body<TB, C, Hub>(a, dsmem);
  } else {
    (void)parts;
    (void)nparts;
    dist_body<TB, C, Hub>(a0, dsmem);
  }
}

// The dense passes as their own cooperative launch (between the two builds of
// k_persistent), so the sparse kernel's register allocation is not shaped by the dense
// code: it runs passes 2, 3, ... while they qualify (flat graph, bitmaps present, mean row
// width below n / SGR_DENSE_SPAN, |W_k| > n / SGR_DENSE_DIV), builds the first sparse
// pass's worklists from its bitmap and leaves ctrl->k there; the host zeroes the barrier
// counter before k_persistent starts.
// Dense passes pay only where consecutive vertices have neighbours close in id (meshes):
// their thread-per-vertex gathers then share lines. 27-point stencil: mean row width ~2 N^2
// = n / 52 at N = 104; on ER (mean width ~0.9 n) dense passes measured 6.3 -> 7.2 ms.
#ifndef SGR_DENSE16
#define SGR_DENSE16 1
#endif
// dcol[q] = col_idx[q] - v for every entry q of row v (16 bits; ctrl->dcol_bad if any does
// not fit). A warp takes 32 consecutive rows (one contiguous segment: the flat build's rows
// have <= 256 entries, so segment offsets fit 32 bits) and strides over its entries, 8 loads
// per lane in flight, finding each entry's row by a 5-step binary search over the lanes' row
// starts: reads and writes coalesced.
template <class C>
__device__ __forceinline__ void build_dcol(const RoundArgs<C>& a) {
  const int lane = threadIdx.x & 31;
  const int gw = (int)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const int NW = (int)((gridDim.x * blockDim.x) >> 5);
  const int nwords = (a.n + 31) >> 5;
  bool bad = false;
  for (int g = gw; g < nwords; g += NW) {
    const int32_t v = (g << 5) + lane;
    const int64_t S = ldg_i64(a.row_ptr + (g << 5));
    const int64_t E = ldg_i64(a.row_ptr + min((g << 5) + 32, a.n));
    const int32_t s = v < a.n ? (int32_t)(ldg_i64(a.row_ptr + v) - S) : INT32_MAX;
    const int32_t len = (int32_t)(E - S);
    for (int32_t i0 = 0; i0 < len; i0 += 256) {
      int32_t w[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int32_t i = i0 + 32 * u + lane;
        w[u] = i < len ? ld_ro(a.col_idx + S + i) : 0;
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const int32_t i = i0 + 32 * u + lane;
        int L = 0;
#pragma unroll
        for (int step = 16; step; step >>= 1)
          if (__shfl_sync(0xffffffffu, s, L + step) <= i) L += step;
        if (i < len) {
          const int32_t d = w[u] - ((g << 5) + L);
          bad |= d < -32768 || d > 32767;
          a.dcol[S + i] = (int16_t)d;
        }
      }
    }
  }
  if (__any_sync(0xffffffffu, bad) && lane == 0) atomicOr(&a.ctrl->dcol_bad, 1);
}

template <int TB, class C>
__global__ void __launch_bounds__(SGR_DENSE_MAXT, 1) k_dense(RoundArgs<C> a) {
  extern __shared__ __align__(16) uint8_t dsmem[];
  Ctrl* ctrl = a.ctrl;
  if (!SGR_DENSE || a.bm[0] == nullptr) return;
  if (ld_cg(&ctrl->big_count) != 0 || !ld_cg(&ctrl->active)) return;  // uniform
  if (__ldcg(&ctrl->span_sum) > (unsigned long long)a.n * (unsigned long long)a.n / SGR_DENSE_SPAN)
    return;
  uint8_t* wsm = warp_smem_init<C, false>(dsmem);
  uint32_t epoch = 0;
  const int max_rounds = ld_cg(&ctrl->max_rounds);
  const bool leader = blockIdx.x == gridDim.x - 1 && threadIdx.x == 0;
  int k = 2;
  bool d16 = false;
  if (SGR_DENSE16 && a.dcol != nullptr) {
    build_dcol(a);  // once per coloring: ~1.5 col_idx worth of traffic, then half per pass
    grid_sync(ctrl, epoch);
    d16 = ld_cg(&ctrl->dcol_bad) == 0;
  }
  for (;; ++k) {
    const Counts w = ld_counts(&ctrl->ring[rs(k)]);
    const bool dense = items_of(w) > 0 && !ld_cg(&ctrl->overflow) && k <= max_rounds &&
                       (int64_t)(w.t + w.m) * SGR_DENSE_DIV > (int64_t)a.n;
    if (!dense) break;  // uniform; k_persistent folds pass k - 1 and goes on from k
    if (leader && k > 2) fold_pass(ctrl, k - 1);
    const C* X = sel((k - 1) & 1, (const C*)a.col[0], (const C*)a.col[1]);
    C* Y = sel(k & 1, a.col[0], a.col[1]);
    unsigned long long edges[kBins] = {0, 0, 0}, entries[kBins] = {0, 0, 0};
    int32_t nx[2] = {0, 0};
    if (d16) dense_body<TB, true, C, true>(a, k, X, Y, wsm, edges, entries, nx);
    else dense_body<TB, true, C, false>(a, k, X, Y, wsm, edges, entries, nx);
    block_add2(nx, &ctrl->ring[rs(k + 1)].t, &ctrl->ring[rs(k + 1)].m);
    block_add6(edges, entries, ctrl, k);
    grid_sync(ctrl, epoch);
  }
  if (k > 2) dense_to_lists(a, k, wsm);  // W_k's lists (in bm[k & 1]) for the sparse passes
  if (leader) ctrl->k = k;
}

// Final colors (packed words) into the caller's int32 output, and their maximum.
static __global__ void k_unpack(const Packed* __restrict__ src, int32_t* __restrict__ dst, int64_t n,
                                int32_t* max_out) {
  int32_t m = 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t c = (int32_t)(src[i] & kColorMask);
    dst[i] = c;
    m = max(m, c);
  }
  m = (int32_t)__reduce_max_sync(0xffffffffu, (unsigned)m);
  if ((threadIdx.x & 31) == 0 && m) atomicMax(max_out, m);
}

}  // namespace sgr
