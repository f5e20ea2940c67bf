/*
 * sgr_oracle.c — CPU oracle for deterministic SGR coloring. TEST INFRASTRUCTURE ONLY
 * (see sgr_oracle.h): only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline
 * and --impl reference legs load it; the CUDA product path never does.
 *
 * Each function follows the paper's pseudo-code line by line; "P:N" cites
 * /root/reference/PAPER.md line N, "Alg. k l.j" the pseudo-code line. Readings of the
 * paper where it is silent or garbled are SURVEY.md §8(c) C1-C19, listed in DESIGN.md §3.
 *
 * Pins (tests/test_oracle.py, -m "not gpu"): networkx greedy_color in natural order for
 * O1; hand-derived traces (tests/golden/hand_traces.json) for O2; closed-form round counts
 * on paths and grids; brute-force chromatic numbers on tiny graphs; the id-reversal
 * relation between the two tie-break rules; invariants (proper coloring, color <= deg+1,
 * W_out strictly inside W_in, R <= n).
 */
#include "sgr_oracle.h"

#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static int64_t max_degree(const int64_t* row_ptr, int64_t n) {
  int64_t d = 0;
  for (int64_t v = 0; v < n; ++v)
    if (row_ptr[v + 1] - row_ptr[v] > d) d = row_ptr[v + 1] - row_ptr[v];
  return d;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* ---------------------------------------------------------------------------------------
 * O1 — Algorithm 1, Sequential Greedy, natural vertex order (graphs are
 * processed "in the order they are defined").
 * color[] starts at 0 = "not yet colored"; colorMask[] starts at a value a not in V (-1)
 * and is labelled with the current vertex v, so it is never re-initialised.
 * A color never exceeds deg(v)+1 (at most deg(v) colors are forbidden), so colorMask needs
 * maxdeg+2 entries (index 0 absorbs uncolored neighbours).
 * ------------------------------------------------------------------------------------- */
int oracle_alg1(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int32_t* color) {
  if (n < 0 || !row_ptr || (n > 0 && !color)) return -1;
  const int64_t maxdeg = max_degree(row_ptr, n);
  int64_t* colorMask = (int64_t*)malloc((size_t)(maxdeg + 2) * sizeof(int64_t));
  if (!colorMask) return -2;
  for (int64_t i = 0; i < maxdeg + 2; ++i) colorMask[i] = -1; /* a not in V */
  for (int64_t v = 0; v < n; ++v) color[v] = 0;

  for (int64_t v = 0; v < n; ++v) {                              /* l.2 for v in V   */
    for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {      /* l.3 w in adj(v)  */
      int32_t w = col_idx[e];
      colorMask[color[w]] = v;                                   /* l.4              */
    }
    int64_t c = 1;                                               /* l.6 min{i>0 : colorMask[i] != v} */
    while (colorMask[c] == v) ++c;
    color[v] = (int32_t)c;                                       /* l.7              */
  }
  free(colorMask);
  return 0;
}

/* lose(v, w): does v go back to the worklist on a conflicting edge (v, w)?
 * PAPER: Alg. 2 l.14, Alg. 4 l.17, Alg. 5 l.14: "v < w".
 * LOWID_KEEPS: the mirror image "v > w" (reading C4). Both are false for w == v, so a
 * self-loop never makes a conflict (reading C7). */
static int lose(int tiebreak, int64_t v, int64_t w) {
  return tiebreak == ORACLE_TIEBREAK_PAPER ? (v < w) : (v > w);
}

/* First-fit of one vertex against a color array (Alg. 5 l.5-8). colorMask entries are
 * labelled with `label`, a value never used before on this mask (the paper labels with v,
 * which is unique per pass over V; a Jacobi run visits v once per round, so the label is
 * the (round, v) pair). */
static int32_t first_fit(const int64_t* row_ptr, const int32_t* col_idx, int64_t v,
                         const int32_t* colors, int64_t* colorMask, int64_t label) {
  for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {       /* l.5 w in adj(v)  */
    int32_t w = col_idx[e];
    colorMask[colors[w]] = label;                                /* l.6              */
  }
  int64_t c = 1;                                                 /* l.8              */
  while (colorMask[c] == label) ++c;
  return (int32_t)c;
}

/* Conflict test of one vertex (Alg. 5 l.13-16). */
static int has_conflict(const int64_t* row_ptr, const int32_t* col_idx, int64_t v,
                        const int32_t* color, int tiebreak) {
  for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {       /* l.13 w in adj(v) */
    int32_t w = col_idx[e];
    if (color[v] == color[w] && lose(tiebreak, v, w)) return 1;  /* l.14            */
  }
  return 0;
}

/* ---------------------------------------------------------------------------------------
 * O2 — Algorithm 5, Data-driven Parallel Graph Coloring, Jacobi rounds.
 * ------------------------------------------------------------------------------------- */
int oracle_jacobi(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int tiebreak,
                  int detect_over_v, int nthreads, int64_t max_rounds, int32_t* color,
                  oracle_round* trace, int64_t trace_cap, int64_t* rounds_out) {
  if (n < 0 || !row_ptr || (n > 0 && (!color || (!col_idx && row_ptr[n] > 0)))) return -1;
  if (tiebreak != ORACLE_TIEBREAK_PAPER && tiebreak != ORACLE_TIEBREAK_LOWID_KEEPS) return -1;
#ifdef _OPENMP
  const int T = nthreads > 0 ? nthreads : omp_get_max_threads();
#else
  const int T = 1;
  (void)nthreads;
#endif
  const int64_t maxdeg = max_degree(row_ptr, n);
  const int64_t masklen = maxdeg + 2;
  int32_t* W_in = (int32_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
  int32_t* W_out = (int32_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
  int32_t* snapshot = (int32_t*)malloc((size_t)(n > 0 ? n : 1) * sizeof(int32_t));
  uint8_t* flag = (uint8_t*)calloc((size_t)(n > 0 ? n : 1), 1);
  int64_t* masks = (int64_t*)malloc((size_t)T * (size_t)masklen * sizeof(int64_t));
  if (!W_in || !W_out || !snapshot || !flag || !masks) {
    free(W_in); free(W_out); free(snapshot); free(flag); free(masks);
    return -2;
  }
  for (int64_t i = 0; i < (int64_t)T * masklen; ++i) masks[i] = -1; /* a not in V */

  for (int64_t v = 0; v < n; ++v) color[v] = 0;
  int64_t w_len = n;                                             /* l.2 W_in <- V    */
  for (int64_t v = 0; v < n; ++v) W_in[v] = (int32_t)v;
  int64_t r = 0;
  int status = 0;

  while (w_len > 0) {                                            /* l.3              */
    if (max_rounds > 0 && r == max_rounds) {
      status = 1;
      break;
    }
    ++r;
    /* Jacobi (C1): the whole round reads the colors as they were when it started. */
    memcpy(snapshot, color, (size_t)n * sizeof(int32_t));
    int64_t w_edges = 0;

    /* l.4-10: first-fit for every v in W_in, against the snapshot. */
#pragma omp parallel for num_threads(T) schedule(dynamic, 256) reduction(+ : w_edges)
    for (int64_t i = 0; i < w_len; ++i) {
#ifdef _OPENMP
      int64_t* colorMask = masks + (int64_t)omp_get_thread_num() * masklen;
#else
      int64_t* colorMask = masks;
#endif
      const int64_t v = W_in[i];
      color[v] = first_fit(row_ptr, col_idx, v, snapshot, colorMask, (r - 1) * n + v); /* l.9 */
      w_edges += row_ptr[v + 1] - row_ptr[v];
    }

    /* l.11-18: W_out <- { v : exists w in adj(v), color[v] = color[w] and lose(v, w) }. */
    int64_t out_len = 0;
    if (detect_over_v) {                                         /* l.12 over V      */
#pragma omp parallel for num_threads(T) schedule(dynamic, 1024)
      for (int64_t v = 0; v < n; ++v) flag[v] = (uint8_t)has_conflict(row_ptr, col_idx, v, color, tiebreak);
      for (int64_t v = 0; v < n; ++v)
        if (flag[v]) W_out[out_len++] = (int32_t)v;              /* l.15             */
    } else {                                                     /* C3: over W_in    */
#pragma omp parallel for num_threads(T) schedule(dynamic, 256)
      for (int64_t i = 0; i < w_len; ++i)
        flag[W_in[i]] = (uint8_t)has_conflict(row_ptr, col_idx, W_in[i], color, tiebreak);
      for (int64_t i = 0; i < w_len; ++i)
        if (flag[W_in[i]]) W_out[out_len++] = W_in[i];          /* l.15 (ascending) */
    }

    if (trace && r - 1 < trace_cap) {
      int32_t mc = 0;
#pragma omp parallel for num_threads(T) reduction(max : mc)
      for (int64_t v = 0; v < n; ++v) mc = color[v] > mc ? color[v] : mc;
      trace[r - 1].w_size = w_len;
      trace[r - 1].w_edges = w_edges;
      trace[r - 1].next_size = out_len;
      trace[r - 1].max_color = mc;
      trace[r - 1].pad = 0;
    }
    /* l.19: swap(W_in, W_out) */
    int32_t* t = W_in;
    W_in = W_out;
    W_out = t;
    w_len = out_len;
  }
  if (rounds_out) *rounds_out = r;
  free(W_in); free(W_out); free(snapshot); free(flag); free(masks);
  return status;
}

/* ---------------------------------------------------------------------------------------
 * O3 — K-sub-step Gauss-Seidel rounds (reading C20).
 * The paper's kernels write color[v] in place inside the parallel loop of Alg. 5 l.4-10
 * (P:169), so later threads may read earlier threads' new colors. O3 makes
 * that deterministic: the loop runs as K sub-steps in a fixed order, each one Jacobi
 * against the colors left by the sub-steps before it.
 * ------------------------------------------------------------------------------------- */
static int64_t gs_part(int64_t v, int64_t n, int64_t K, int partition) {
  return partition == 1 ? (int64_t)(((__int128)v * K) / n) : v % K;
}

int oracle_gauss_seidel(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int tiebreak,
                        int64_t K, int partition, int64_t max_rounds, int32_t* color,
                        oracle_round* trace, int64_t trace_cap, int64_t* rounds_out) {
  if (n < 0 || !row_ptr || (n > 0 && (!color || (!col_idx && row_ptr[n] > 0)))) return -1;
  if (tiebreak != ORACLE_TIEBREAK_PAPER && tiebreak != ORACLE_TIEBREAK_LOWID_KEEPS) return -1;
  if (K < 1 || (partition != 0 && partition != 1)) return -1;
  const int64_t masklen = max_degree(row_ptr, n) + 2;
  const size_t nn = (size_t)(n > 0 ? n : 1);
  int32_t* W_in = (int32_t*)malloc(nn * sizeof(int32_t));
  int32_t* W_out = (int32_t*)malloc(nn * sizeof(int32_t));
  int32_t* snapshot = (int32_t*)malloc(nn * sizeof(int32_t));
  int64_t* colorMask = (int64_t*)malloc((size_t)masklen * sizeof(int64_t));
  if (!W_in || !W_out || !snapshot || !colorMask) {
    free(W_in); free(W_out); free(snapshot); free(colorMask);
    return -2;
  }
  for (int64_t i = 0; i < masklen; ++i) colorMask[i] = -1;      /* a not in V       */
  for (int64_t v = 0; v < n; ++v) color[v] = 0;
  int64_t w_len = n;                                             /* l.2 W_in <- V    */
  for (int64_t v = 0; v < n; ++v) W_in[v] = (int32_t)v;
  int64_t r = 0, label = 0;
  int status = 0;
  while (w_len > 0) {                                            /* l.3              */
    if (max_rounds > 0 && r == max_rounds) {
      status = 1;
      break;
    }
    ++r;
    int64_t w_edges = 0;
    for (int64_t j = 0; j < K; ++j) {                            /* sub-steps in order */
      /* sub-step j reads the colors as the previous sub-steps left them (Jacobi inside) */
      memcpy(snapshot, color, (size_t)n * sizeof(int32_t));
      for (int64_t i = 0; i < w_len; ++i) {                      /* l.4 v in W_in    */
        const int64_t v = W_in[i];
        if (gs_part(v, n, K, partition) != j) continue;
        color[v] = first_fit(row_ptr, col_idx, v, snapshot, colorMask, label++); /* l.5-9 */
        w_edges += row_ptr[v + 1] - row_ptr[v];
      }
    }
    int64_t out_len = 0;                                         /* l.11-18 over W_in */
    for (int64_t i = 0; i < w_len; ++i)
      if (has_conflict(row_ptr, col_idx, W_in[i], color, tiebreak)) W_out[out_len++] = W_in[i];
    if (trace && r - 1 < trace_cap) {
      int32_t mc = 0;
      for (int64_t v = 0; v < n; ++v) mc = color[v] > mc ? color[v] : mc;
      trace[r - 1].w_size = w_len;
      trace[r - 1].w_edges = w_edges;
      trace[r - 1].next_size = out_len;
      trace[r - 1].max_color = mc;
      trace[r - 1].pad = 0;
    }
    int32_t* t = W_in;                                           /* l.19             */
    W_in = W_out;
    W_out = t;
    w_len = out_len;
  }
  if (rounds_out) *rounds_out = r;
  free(W_in); free(W_out); free(snapshot); free(colorMask);
  return status;
}

int oracle_assign(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, const int32_t* wl,
                  int64_t wl_len, const int32_t* snapshot, int32_t* tent) {
  if (n < 0 || wl_len < 0 || !row_ptr || (wl_len > 0 && (!wl || !snapshot || !tent))) return -1;
  /* An arbitrary snapshot may hold colors above maxdeg+1: size colorMask for both. */
  int64_t masklen = max_degree(row_ptr, n) + 2;
  for (int64_t v = 0; wl_len > 0 && v < n; ++v) {
    if (snapshot[v] < 0) return -1;
    if ((int64_t)snapshot[v] + 2 > masklen) masklen = (int64_t)snapshot[v] + 2;
  }
  int64_t* colorMask = (int64_t*)malloc((size_t)masklen * sizeof(int64_t));
  if (!colorMask) return -2;
  for (int64_t i = 0; i < masklen; ++i) colorMask[i] = -1;
  for (int64_t i = 0; i < wl_len; ++i) {                         /* l.4              */
    if (wl[i] < 0 || wl[i] >= n) { free(colorMask); return -1; }
    tent[i] = first_fit(row_ptr, col_idx, wl[i], snapshot, colorMask, i);
  }
  free(colorMask);
  return 0;
}

int oracle_detect(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, const int32_t* wl,
                  int64_t wl_len, const int32_t* color, int tiebreak, uint8_t* conflict) {
  if (n < 0 || wl_len < 0 || !row_ptr || (wl_len > 0 && (!wl || !color || !conflict))) return -1;
  if (tiebreak != ORACLE_TIEBREAK_PAPER && tiebreak != ORACLE_TIEBREAK_LOWID_KEEPS) return -1;
  for (int64_t i = 0; i < wl_len; ++i) {                         /* l.12             */
    if (wl[i] < 0 || wl[i] >= n) return -1;
    conflict[i] = (uint8_t)has_conflict(row_ptr, col_idx, wl[i], color, tiebreak);
  }
  return 0;
}

/* ---------------------------------------------------------------------------------------
 * O2 on P logical ranks with an explicit exchange (the CPU test of the multi-GPU idea,
 * SURVEY §8(e)): rank p owns [ranges[p], ranges[p+1]) and a full private replica.
 * ------------------------------------------------------------------------------------- */
int oracle_jacobi_partitioned(const int64_t* row_ptr, const int32_t* col_idx, int64_t n,
                              int tiebreak, int P, const int64_t* ranges, int32_t* color,
                              int64_t* rounds_out) {
  if (n < 0 || P < 1 || !row_ptr || (n > 0 && !color)) return -1;
  if (tiebreak != ORACLE_TIEBREAK_PAPER && tiebreak != ORACLE_TIEBREAK_LOWID_KEEPS) return -1;
  int64_t* lo = (int64_t*)malloc((size_t)(P + 1) * sizeof(int64_t));
  if (!lo) return -2;
  for (int p = 0; p <= P; ++p) lo[p] = ranges ? ranges[p] : (n * p) / P;
  if (lo[0] != 0 || lo[P] != n) { free(lo); return -1; }
  for (int p = 0; p < P; ++p)
    if (lo[p + 1] < lo[p]) { free(lo); return -1; }

  const size_t nn = (size_t)(n > 0 ? n : 1);
  const int64_t masklen = max_degree(row_ptr, n) + 2;
  int32_t* replica = (int32_t*)calloc((size_t)P * nn, sizeof(int32_t)); /* all uncolored */
  int32_t* snapshot = (int32_t*)malloc(nn * sizeof(int32_t));
  int32_t* W = (int32_t*)malloc(nn * sizeof(int32_t));      /* rank p's part at W + lo[p] */
  int64_t* wlen = (int64_t*)malloc((size_t)P * sizeof(int64_t));
  int32_t* out_v = (int32_t*)malloc(nn * sizeof(int32_t));  /* outbox of rank p at + lo[p] */
  int32_t* out_c = (int32_t*)malloc(nn * sizeof(int32_t));
  int64_t* colorMask = (int64_t*)malloc((size_t)masklen * sizeof(int64_t));
  if (!replica || !snapshot || !W || !wlen || !out_v || !out_c || !colorMask) {
    free(lo); free(replica); free(snapshot); free(W); free(wlen); free(out_v); free(out_c);
    free(colorMask);
    return -2;
  }
  for (int64_t i = 0; i < masklen; ++i) colorMask[i] = -1;
  for (int p = 0; p < P; ++p) {
    wlen[p] = lo[p + 1] - lo[p];
    for (int64_t v = lo[p]; v < lo[p + 1]; ++v) W[v] = (int32_t)v;
  }
  int64_t r = 0;
  for (;;) {
    int64_t total = 0;
    for (int p = 0; p < P; ++p) total += wlen[p];
    if (total == 0) break;
    ++r;
    /* assignment on every rank against its own replica's snapshot -> outbox */
    for (int p = 0; p < P; ++p) {
      int32_t* rep = replica + (size_t)p * nn;
      memcpy(snapshot, rep, (size_t)n * sizeof(int32_t));
      for (int64_t i = 0; i < wlen[p]; ++i) {
        int64_t v = W[lo[p] + i];
        out_v[lo[p] + i] = (int32_t)v;
        out_c[lo[p] + i] = first_fit(row_ptr, col_idx, v, snapshot, colorMask, (r - 1) * n + v);
      }
    }
    /* exchange: every rank applies every rank's outbox (an allgather of (v, color) pairs) */
    for (int p = 0; p < P; ++p) {
      int32_t* rep = replica + (size_t)p * nn;
      for (int q = 0; q < P; ++q)
        for (int64_t i = 0; i < wlen[q]; ++i) rep[out_v[lo[q] + i]] = out_c[lo[q] + i];
    }
    /* detection on every rank over its own worklist, against its replica */
    for (int p = 0; p < P; ++p) {
      const int32_t* rep = replica + (size_t)p * nn;
      int64_t k = 0;
      for (int64_t i = 0; i < wlen[p]; ++i) {
        int32_t v = W[lo[p] + i];
        if (has_conflict(row_ptr, col_idx, v, rep, tiebreak)) W[lo[p] + k++] = v;
      }
      wlen[p] = k;
    }
  }
  /* all replicas must agree; rank 0's is the result */
  int status = 0;
  for (int p = 1; p < P && status == 0; ++p)
    if (memcmp(replica, replica + (size_t)p * nn, (size_t)n * sizeof(int32_t)) != 0) status = -3;
  memcpy(color, replica, (size_t)n * sizeof(int32_t));
  if (rounds_out) *rounds_out = r;
  free(lo); free(replica); free(snapshot); free(W); free(wlen); free(out_v); free(out_c);
  free(colorMask);
  return status;
}
