/*
 * sgr_oracle.h — CPU ORACLE for deterministic speculative-greedy (SGR) coloring.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library. The product path
 * (libsgr.so, include/sgr.h) never links, includes or calls anything here, and this
 * file shares no code, header, table or helper with it.
 *
 * Plain, slow, obviously correct: every function restates an algorithm of
 * /root/reference/PAPER.md ("P:N" = line N) step by step, in the paper's order and
 * notation (color, colorMask, adj(v), W_in/W_out), with the readings of SURVEY.md §8(c)
 * listed in DESIGN.md §3.
 *
 * Graph input: CSR R = row_ptr (n+1, int64) and C = col_idx (int32); the pattern
 * must be symmetric. Colors are positive integers, 0 = uncolored.
 * All pointers are host pointers owned by the caller. Functions return 0 on success,
 * -1 on invalid arguments, -2 on allocation failure, 1 if max_rounds was reached first.
 */
#ifndef SGR_ORACLE_H
#define SGR_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Conflict rule of Alg. 2 l.14 / Alg. 4 l.17 / Alg. 5 l.14 and its mirror (reading C4). */
#define ORACLE_TIEBREAK_LOWID_KEEPS 0 /* conflicting edge: the HIGHER id recolors (v > w)  */
#define ORACLE_TIEBREAK_PAPER 1       /* the paper's literal rule: v < w -> v recolors     */

/* Per-round record of Algorithm 5's loop (r = 1..R). */
typedef struct {
  int64_t w_size;    /* |W_in| entering round r                               */
  int64_t w_edges;   /* sum of |adj(v)| over v in W_in (scanned CSR entries)   */
  int64_t next_size; /* |W_out| produced by round r's conflict detection        */
  int32_t max_color; /* max(color) after round r's assignment                   */
  int32_t pad;
} oracle_round;

/* O1 — Algorithm 1 (colorMask labelled by v), natural id order. */
int oracle_alg1(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int32_t* color);

/* O2 — Algorithm 5 with Jacobi rounds (reading C1): every assignment of a round
 * reads the color snapshot taken when the round starts. Recolored vertices keep their stale
 * color (C2). detect_over_v != 0 runs conflict detection over all of V exactly as Alg. 5
 * l.12 says; 0 runs it over W_in only (reading C3, provably identical).
 * nthreads > 1 runs the per-vertex loops (independent given the snapshot) with OpenMP;
 * W_out is always assembled in ascending id order, so the result does not depend on it.
 * trace (nullable) receives min(R, trace_cap) records; *rounds_out (nullable) = R.
 * max_rounds > 0 stops after that many rounds (returns 1 if W_in was still non-empty). */
int oracle_jacobi(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int tiebreak,
                  int detect_over_v, int nthreads, int64_t max_rounds, int32_t* color,
                  oracle_round* trace, int64_t trace_cap, int64_t* rounds_out);

/* One assignment step (Alg. 5 l.4-10) of the Jacobi round: for i < wl_len, v = wl[i],
 * tent[i] = min{ c > 0 : colorMask[c] != v } after colorMask[snapshot[w]] <- v, w in adj(v). */
int oracle_assign(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, const int32_t* wl,
                  int64_t wl_len, const int32_t* snapshot, int32_t* tent);

/* One detection step (Alg. 5 l.12-18) restricted to the listed vertices:
 * conflict[i] = 1 iff some w in adj(wl[i]) has color[w] == color[v] and the tiebreak says
 * v loses (PAPER: v < w; LOWID_KEEPS: v > w). */
int oracle_detect(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, const int32_t* wl,
                  int64_t wl_len, const int32_t* color, int tiebreak, uint8_t* conflict);

/* O2 simulated on P logical ranks that each own a contiguous vertex range and a private
 * full color replica; after each assignment step every rank publishes the (v, color)
 * pairs it assigned into an explicit outbox, and every rank applies every outbox to its
 * replica before detection. Must equal oracle_jacobi for any P and any valid ranges.
 * ranges (nullable) = P+1 boundaries (0 = ranges[0] <= ... <= ranges[P] = n); NULL splits V
 * into P equal-count ranges. */
int oracle_jacobi_partitioned(const int64_t* row_ptr, const int32_t* col_idx, int64_t n,
                              int tiebreak, int P, const int64_t* ranges, int32_t* color,
                              int64_t* rounds_out);

/* O3 — reduced-round variant (DESIGN.md §3 reading C20): Algorithm 5
 * with each round's assignment loop (l.4-10) split into K sub-steps taken in order
 * j = 0..K-1. Vertex v belongs to sub-step part(v) = v mod K (partition 0, "strided") or
 * floor(v * K / n) (partition 1, "blocked", ids in order). Sub-step j assigns its members of
 * W_in against the colors as the previous sub-step left them — the in-place writes of
 * Alg. 5 l.9 become visible between sub-steps — and, within the sub-step,
 * against that sub-step's snapshot (Jacobi). Detection (l.12-18) follows the K sub-steps
 * as in O2. K = 1 is O2; K = n, blocked, is Algorithm 1 in one round. Same trace, return
 * values and max_rounds meaning as oracle_jacobi; single-threaded. */
int oracle_gauss_seidel(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int tiebreak,
                        int64_t K, int partition, int64_t max_rounds, int32_t* color,
                        oracle_round* trace, int64_t trace_cap, int64_t* rounds_out);

/* Number of worker threads oracle_jacobi would use for nthreads <= 0 (OpenMP max). */
int oracle_max_threads(void);

#ifdef __cplusplus
}
#endif
#endif
