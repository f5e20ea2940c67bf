/*
 * sgr.h — C ABI of the B200 (sm_100a) deterministic speculative-greedy (SGR) coloring
 * library, libsgr.so. Every function is extern "C", never throws, and returns an
 * sgr_status (0 = OK, < 0 = error; sgr_last_error() gives a thread-local message).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, "P:N" = line N):
 *   Vertex coloring: "assign colors to all the vertices of a graph such that no neighboring
 *   vertices have the same color", by the data-driven speculative greedy
 *   method, Algorithm 5: rounds of first-fit assignment over a worklist
 *   (Alg. 5 l.4-10) followed by conflict detection that returns the losing endpoint of
 *   every monochromatic edge to the next worklist (Alg. 5 l.12-18, pushed with a
 *   prefix-sum / aggregated atomic), until the worklist is empty (l.3, l.19).
 *   Rounds are Jacobi-style (reading C1): assignment in round r reads the
 *   colors as they were when round r started, so the result is a deterministic function
 *   of (graph, tie-break) only — independent of GPU count, launch shape, bins or timing —
 *   and is bit-identical to the CPU oracle (oracle/, test infrastructure).
 *
 * Graph input: CSR "R" (row offsets, n+1) and "C" (column indices, nnz), stored
 * "in the order they are defined" with no relabeling (reading C19). Contract:
 *   - row_ptr is int64, row_ptr[0] = 0, nondecreasing, row_ptr[n] = nnz;
 *   - col_idx is int32, 0 <= col_idx[e] < n, each row sorted ascending (or any order with
 *     opts->unsorted_rows; sorted input without the flag is what F_1 relies on: unsorted
 *     rows without it can give an improper coloring), and the col_idx pointer is 16-byte
 *     aligned (rows are read with 16-byte vector loads);
 *   - the pattern is symmetric (w in adj(v) <=> v in adj(w)); asymmetric input is
 *     undefined (conflicts may go unseen);
 *   - self-loops and duplicate entries are allowed and provably never change the result;
 *   - n < 2^31; n = 0 is OK (no kernels); nnz = 0 gives all colors 1 in one round.
 * Output: colors_out[v] in [1, deg(v)+1] (colors are positive integers), a
 *   proper coloring.
 *
 * Ownership: the caller owns every buffer passed in; the library never frees or retains
 * caller memory after a call returns. Device scratch is either the caller's `workspace`
 * (>= sgr_workspace_bytes()) or taken from the stream-ordered allocator and released
 * before return.
 * Synchronization: sgr_color / sgr_color_ex / sgr_color_host return when colors_out and
 * *stats are valid (they synchronize opts->stream once at the end). The step entry points
 * (sgr_assign, sgr_commit, sgr_detect, sgr_compact) are asynchronous on opts->stream.
 * Errors: SGR_EINVAL for a null required pointer, n < 0, nnz < 0, n >= 2^31, aliasing
 * that the operation forbids, or (with opts->validate) a CSR that breaks the contract;
 * SGR_ECUDA for a CUDA error (message in sgr_last_error()); SGR_ENOCONV if opts->max_rounds
 * was reached (cannot happen with the default cap n+1: |W| strictly shrinks every round).
 */
#ifndef SGR_H
#define SGR_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SGR_OK = 0,
  SGR_EINVAL = -1,
  SGR_ENOMEM = -2,
  SGR_ECUDA = -3,
  SGR_ENCCL = -4,
  SGR_ENOCONV = -5,
  SGR_EUNSUPPORTED = -6
} sgr_status;

/* Which endpoint of a conflicting edge (v, w), color[v] = color[w], goes back to the
 * worklist (DESIGN.md §3 reading C4). */
typedef enum {
  SGR_TIEBREAK_LOWID_KEEPS = 0, /* the higher id recolors: lose(v,w) = v > w (default) */
  SGR_TIEBREAK_PAPER = 1        /* Alg. 2 l.14 / Alg. 4 l.17 / Alg. 5 l.14: v < w -> v */
} sgr_tiebreak;

typedef enum {
  SGR_LOOP_AUTO = 0,       /* = SGR_LOOP_PERSISTENT */
  SGR_LOOP_GRAPH = 1,      /* one kernel per round, batches of rounds replayed as a CUDA graph */
  SGR_LOOP_PERSISTENT = 2, /* all rounds in one cooperative kernel, grid barrier per round */
  SGR_LOOP_HOST = 3        /* one kernel per round, launched from the host in batches */
} sgr_loop_mode;

/* Device CSR (both pointers in device memory). */
typedef struct {
  const int64_t* row_ptr; /* n+1 */
  const int32_t* col_idx; /* nnz */
} sgr_csr;

typedef struct {
  int32_t tiebreak;      /* sgr_tiebreak; default LOWID_KEEPS */
  int32_t max_rounds;    /* 0 = n+1 (never reached) */
  int32_t loop_mode;     /* sgr_loop_mode */
  int32_t color_bits;    /* 16 (default): 16-bit words (12-bit color + round mod 16), with
                            live-neighbour trimming of high-degree rows; a color above 4095
                            triggers an automatic 32-bit rerun. 32: plain int32 colors,
                            full rows every round */
  int32_t bin_small_max; /* degree bins: d <= small -> 8 lanes/vertex, register mask (<= 62);
                            0 = 32 */
  int32_t bin_med_max;   /* small < d <= med -> 8 lanes/vertex, smem table (<= 256); 0 = 256
                            (128 when n <= 2^20);
                            d > med -> one warp per 1024-entry aligned chunk of the row */
  void* stream;          /* cudaStream_t; NULL = legacy default stream */
  int32_t* round_sizes;  /* optional DEVICE buffer: |W_r| for r = 1..R (R capped by cap) */
  int64_t* round_edges;  /* optional DEVICE buffer: sum of deg(v), v in W_r, r = 1..R   */
  int32_t round_cap;     /* capacity of round_sizes / round_edges */
  int32_t validate;      /* != 0: check the CSR contract on the device first (slow) */
  int32_t rounds_per_batch; /* rounds issued between termination checks; 0 = 8 */
  int32_t profile;       /* != 0: time every kernel launch with CUDA events */
  float* round_ms;       /* optional HOST buffer (round_cap): with profile != 0 and the host
                            loop, device time of each round pass k = 2, 3, ... */
  int64_t* round_ns;     /* optional DEVICE buffer (round_cap): %globaltimer (ns) when pass
                            k = 2, 3, ... ended, written by the loop control (profiling) */
  int32_t color_cap;     /* test hook: 0 = 4095, the largest color a 16-bit word holds; a
                            smaller cap sends colorings whose colors exceed it down the
                            automatic 32-bit rerun path (results are unchanged) */
  int32_t block_size;    /* threads per block (the paper's Fig. 8 parameter, P:267-273;
                            performance only, never the result). 0 = 256. A multiple of 32:
                            per-vertex kernels (F_1, steps, topology-driven, final) take
                            32..1024; the fused round kernels 64..512 when the graph has
                            rows of degree > bin_med_max (hub build), else 64..768.
                            Anything else: SGR_EINVAL. */
  int32_t unsorted_rows; /* != 0: rows may be in any order. F_1 then scans whole rows
                            instead of reading the first / last entry (sorted rows are the
                            default contract: with unsorted rows and this flag 0 the
                            coloring can be improper). opts->validate reports unsorted rows
                            (bit 4) only when this flag is 0. */
  int32_t flat_bin0;     /* test hook, graphs without rows of degree > bin_med_max (flat
                            build, persistent loop): bin-0 mapping. 0 = automatic (one
                            thread per vertex for non-local rows — mean row width >= n/16 —
                            and n >= 2^22, else 4-lane groups), 1 = 4-lane groups, 2 = one
                            thread per vertex. Never changes a result. */
} sgr_opts;

/* Kernel classes (stats->kernel_*): F_1, the fused round pass(es), loop control, final. */
enum { SGR_K_FIRST = 0, SGR_K_ROUND = 1, SGR_K_CTRL = 2, SGR_K_FINAL = 3, SGR_K_COUNT = 4 };

typedef struct {
  int32_t rounds;             /* R = number of assignment rounds (P4 path: 4)           */
  int32_t num_colors;         /* max color                                               */
  int64_t vertices_processed; /* sum over rounds of |W_r|                                */
  int64_t edges_scanned;      /* sum over rounds of sum_{v in W_r} deg(v) (A * nnz)      */
  int64_t entries_read;       /* adjacency entries the passes actually read (rounds >= 2;
                                 < edges_scanned - nnz when neighbour lists are trimmed) */
  int64_t bytes_algorithmic;  /* DESIGN.md §6 byte model, summed over all launches       */
  float elapsed_ms;           /* device time from the first kernel to the final count   */
  int32_t launches;           /* kernels launched by this call                           */
  float kernel_ms[SGR_K_COUNT];      /* opts->profile: device time per kernel class      */
  int64_t kernel_launches[SGR_K_COUNT];
  int64_t kernel_bytes[SGR_K_COUNT]; /* algorithmic bytes per kernel class             */
  int64_t bin_vertices[3];           /* rounds >= 2, per degree bin (thread/group/chunk) */
  int64_t bin_edges[3];
  int64_t chunk_items;               /* warp work items processed in the chunk bin       */
  int64_t bin_warp_cycles[3];        /* SM cycles warps spent in each bin (all rounds)   */
  int32_t grid_blocks;               /* blocks of the round kernel                        */
  int32_t color_bits;                /* width the coloring finished with (16 or 32)       */
  int64_t entries_written;           /* compacted neighbour-list entries written (bin 2)  */
  int32_t transport;                 /* partitioned / multi-GPU colorings: how replicas were
                                        kept equal — SGR_XCHG_* below; 0 otherwise         */
} sgr_stats;

/* stats->transport of sgr_color_partitioned / sgr_color_dist. */
enum {
  SGR_XCHG_NONE = 0,        /* single part: nothing to exchange                          */
  SGR_XCHG_DEVICE = 1,      /* one cooperative launch, every color word stored into all
                               replicas (parts of one device, or NVLink peer memory), device
                               barrier across parts (k_persistent_dist)                     */
  SGR_XCHG_ALLGATHER = 2    /* host-driven rounds, padded all-gather of (v, color) records
                               per round (NCCL between GPUs, device copies on one GPU)      */
};

void sgr_opts_default(sgr_opts* opts);

/* Scratch the library needs for a graph of this size (device bytes). */
size_t sgr_workspace_bytes(int64_t n, int64_t nnz, const sgr_opts* opts);

/* Color the graph. csr and colors_out (n int32) are device pointers. stats: host, nullable. */
sgr_status sgr_color(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                     sgr_stats* stats);

/* Same, with options and optional caller workspace (device, >= sgr_workspace_bytes). */
sgr_status sgr_color_ex(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                        sgr_stats* stats, const sgr_opts* opts, void* workspace,
                        size_t workspace_bytes);

/* End to end from HOST buffers: copies row_ptr/col_idx host->device, colors, copies the
 * colors device->host. Host buffers should be pinned for full PCIe/C2C speed. */
sgr_status sgr_color_host(const int64_t* row_ptr, const int32_t* col_idx, int64_t n,
                          int64_t nnz, int32_t* colors_out, sgr_stats* stats,
                          const sgr_opts* opts);

/* Pipelined end to end over `count` HOST graphs (the batch a user colors one after the
 * other): graph i+1's row_ptr/col_idx upload and graph i-1's colors download run on two
 * internal copy streams while graph i is colored (sgr_color_ex) on opts->stream, with two
 * device buffer sets sized by the largest graph (stream-ordered allocator, released before
 * return). Arguments are arrays of `count` entries: row_ptr[i] (n[i]+1 int64 offsets),
 * col_idx[i] (nnz[i] int32 ids, may be NULL when nnz[i] == 0), colors_out[i] (n[i] int32);
 * the same host buffers may appear more than once (read-only inputs; outputs should be
 * distinct). Host buffers must be pinned for the copies to overlap the coloring (pageable
 * memory makes them synchronous). stats: NULL or an array of `count` records, one per
 * graph. Each colors_out[i] equals sgr_color_host's result for graph i. Returns at the
 * first failing graph (its status; later graphs untouched); synchronizes all streams. */
sgr_status sgr_color_host_batch(const int64_t* const* row_ptr, const int32_t* const* col_idx,
                                const int64_t* n, const int64_t* nnz, int32_t* const* colors_out,
                                int32_t count, sgr_stats* stats, const sgr_opts* opts);

/* Topology-driven mapping of the same method: the paper's Algorithm 4 (T-base,
 * P:194-196) under the Jacobi reading. Every iteration visits all n vertices, one thread
 * per vertex: the uncolored ones take a first fit against the iteration's snapshot, then
 * every vertex is checked for a conflict (Alg. 4 l.15-21) and the host reads the `changed`
 * count (l.22). Same contract, same result (colors, rounds, |W_r|) as sgr_color; slower by
 * design (it rescans V every iteration) — the comparison the paper makes against Alg. 5.
 * Uses opts->tiebreak, max_rounds, stream and round_sizes/round_cap (|W_r| per iteration);
 * device scratch from the stream-ordered allocator; synchronizes the stream. */
sgr_status sgr_color_topo(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* colors_out,
                          sgr_stats* stats, const sgr_opts* opts);

/* Reduced-round variants (DESIGN.md §3 reading C20). Different
 * semantics from sgr_color: a round's assignment loop (Alg. 5 l.4-10) runs as `substeps`
 * ordered sub-steps over a fixed id partition — partition 0: v mod substeps ("strided"),
 * 1: floor(v * substeps / n) ("blocked") — and sub-step j sees the colors written by the
 * sub-steps before it (the paper's in-place writes, P:169/174/190, made deterministic);
 * then detection and compaction as Alg. 5 l.12-15. Deterministic, equal to the oracle's
 * O3 (colors, rounds, |W_r|); substeps = 1 is sgr_color's result. Partition 2 is the
 * paper-faithful NONDETERMINISTIC mode: one in-place assignment per round whose first fits
 * read colors other warps are writing (substeps ignored); the result is a proper coloring
 * whose colors and rounds may vary from run to run. Plain int32 colors, host-driven
 * rounds (one count readback per round). Uses opts tiebreak, max_rounds, stream,
 * block_size and round_sizes / round_edges / round_cap; synchronizes the stream. */
sgr_status sgr_color_gs(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t substeps,
                        int32_t partition, int32_t* colors_out, sgr_stats* stats,
                        const sgr_opts* opts);

/* ---- one-round step entry points: Algorithm 5 split line by line (all device pointers,
 * asynchronous on opts->stream; opts may be NULL) ---------------------------------------- */

/* Alg. 5 l.4-10 against a snapshot: tent_out[i] = min{c > 0 : c != colors_in[w] for all
 * w in adj(wl[i])}. colors_in must not alias tent_out. The step is Alg. 5 l.5-6 literally:
 * w ranges over every entry of the row, so a listed self-loop forbids v's own snapshot
 * color (DESIGN.md §3 reading C7; inside sgr_color this never changes a result, proof v). */
sgr_status sgr_assign(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors_in, int32_t* tent_out, const sgr_opts* opts);

/* Alg. 5 l.9 applied after the whole assignment step: colors[wl[i]] = tent[i]. */
sgr_status sgr_commit(const int32_t* wl, const int32_t* tent, int64_t wl_len, int32_t* colors,
                      const sgr_opts* opts);

/* Alg. 5 l.13-14 for the listed vertices: conflict_out[i] = 1 iff some w in adj(v),
 * v = wl[i], has colors[w] == colors[v] and v loses by opts->tiebreak; else 0. */
sgr_status sgr_detect(const sgr_csr* csr, int64_t n, const int32_t* wl, int64_t wl_len,
                      const int32_t* colors, uint8_t* conflict_out, const sgr_opts* opts);

/* Alg. 5 l.15 / P:228-230: wl_out = [wl[i] : flags[i] != 0] in input order (block scan +
 * one aggregated offset per block); *count_out (device int64) = its length. */
sgr_status sgr_compact(const int32_t* wl, const uint8_t* flags, int64_t len, int32_t* wl_out,
                       int64_t* count_out, const sgr_opts* opts);

/* Device-side CSR contract check; *violations (host) gets the sgr_gen_validate-style
 * bitmask (1 offsets, 2 range, 4 unsorted). Symmetry is not checked on the device. */
sgr_status sgr_validate_csr(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t* violations,
                            void* stream);

/* ---- multi-GPU: contiguous vertex ranges, one NCCL exchange per round -- */

/* nnz-balanced contiguous ranges: ranges[p] = min{v : row_ptr[v] >= ceil(p*nnz/P)},
 * ranges[0] = 0, ranges[P] = n. row_ptr is a HOST array here. */
sgr_status sgr_partition(const int64_t* row_ptr, int64_t n, int32_t P, int64_t* ranges);

/* NCCL communicator wrapper: nccl_unique_id is the 128-byte ncclUniqueId that rank 0
 * created (sgr_nccl_unique_id) and every rank received out of band. */
sgr_status sgr_nccl_unique_id(void* id_out_128B);
sgr_status sgr_comm_init(void** comm, int32_t rank, int32_t world, const void* nccl_unique_id,
                         int32_t device);
sgr_status sgr_comm_destroy(void* comm);

/* One call per rank, collective over comm. `local` holds the rank's OWNED rows
 * [v_begin, v_end) with local row offsets (local.row_ptr[0] = 0, length v_end-v_begin+1)
 * and GLOBAL column ids. colors_out: device, n_global int32, filled on every rank. */
sgr_status sgr_color_dist(void* comm, const sgr_csr* local, int64_t n_global, int64_t v_begin,
                          int64_t v_end, int64_t nnz_local, int32_t* colors_out,
                          sgr_stats* stats, const sgr_opts* opts);

/* P logical partitions on ONE device: same per-rank kernels, exchange and commit as
 * sgr_color_dist, with the all-gather done by device copies (for testing the distributed
 * path bit-exactly on a single GPU). csr is the full device CSR; ranges: host, P+1. */
sgr_status sgr_color_partitioned(const sgr_csr* csr, int64_t n, int64_t nnz, int32_t P,
                                 const int64_t* ranges, int32_t* colors_out, sgr_stats* stats,
                                 const sgr_opts* opts);

const char* sgr_strerror(sgr_status s);
const char* sgr_last_error(void);
const char* sgr_version(void);

#ifdef __cplusplus
}
#endif
#endif
