/* sim_locality.c — experiment (not product, not oracle): per-round color-gather locality of
 * the Jacobi-SGR passes on an R-MAT graph, to size the "dense renumbering" idea of
 * VERDICT r1 item 4 before building it.
 *
 * For every pass k >= 2 it counts, per degree bin, the color gathers of an exactly trimmed
 * pass (bin 2 lists = live neighbours, i.e. neighbours in W_k; bins 0/1 full rows) and the
 * distinct 128-byte lines each 32-lane gather instruction touches with 16-bit color words:
 *   orig : lists hold vertex ids (64 ids per line)
 *   dense: lists hold ranks in S_e, the worklist at the start of the current epoch; a new
 *          epoch starts when |W_k| <= |S_e| / 2 (ranks preserve id order, so lists stay
 *          sorted and the tie-break can compare ranks).
 * bin 2: 32 consecutive list entries per instruction; bin 1: 4 vertices x 8 consecutive
 * entries; bin 0: 8 vertices x 4 entries (worklists in ascending id order).
 *
 *   gcc -O2 -fopenmp -o /tmp/sim_locality tools/sim_locality.c \
 *       -Lpaper_conf_ipps_licqfsty16_b200/lib -l:libsgr_gen.so -Iinclude
 *   LD_LIBRARY_PATH=paper_conf_ipps_licqfsty16_b200/lib /tmp/sim_locality 22
 */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "sgr_gen.h"

static int cmp_u32(const void* a, const void* b) {
  uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
  return x < y ? -1 : x > y;
}
static int distinct(uint32_t* v, int m) {
  qsort(v, m, sizeof(uint32_t), cmp_u32);
  int d = 0;
  for (int i = 0; i < m; ++i)
    if (i == 0 || v[i] != v[i - 1]) ++d;
  return d;
}

int main(int argc, char** argv) {
  int scale = argc > 1 ? atoi(argv[1]) : 20;
  int shift = argc > 2 ? atoi(argv[2]) : 6; /* log2 ids per line: 6 = u16 words, 128 B */
  sgr_gen_graph g;
  if (sgr_gen_rmat(scale, 8, 0.57, 0.19, 0.19, 4, 0, &g)) return 1;
  const int64_t n = g.n;
  const int64_t* R = g.row_ptr;
  const int32_t* C = g.col_idx;
  int32_t* X = calloc(n, 4);  /* snapshot */
  int32_t* Y = calloc(n, 4);
  uint8_t* inW = calloc(n, 1);
  int32_t* W = malloc(n * 4);
  int32_t* W2 = malloc(n * 4);
  int32_t* rank = malloc(n * 4);
  int64_t wl = 0;
  /* round 1: all colors 1; W_2 = vertices with a lower neighbour */
  for (int64_t v = 0; v < n; ++v) X[v] = 1;
  for (int64_t v = 0; v < n; ++v)
    if (R[v + 1] > R[v] && C[R[v]] < v) W[wl++] = (int32_t)v;
  memcpy(Y, X, n * 4);
  for (int64_t i = 0; i < wl; ++i) { Y[W[i]] = 2; inW[W[i]] = 1; }
  int64_t S = 0; /* epoch size */
  double tot_g[3] = {0}, tot_lo[3] = {0}, tot_ld[3] = {0}, tot_skip[3] = {0};
  double hot[4] = {0};  /* bin-2 gathers with id < 2^12, 2^14, 2^16, 2^18 */
  printf("k |W| | g0 l0 | g1 l1 live1 | g2 l2orig l2dense | epoch\n");
  for (int k = 2; wl > 0; ++k) {
    /* snapshot X = C_k */
    int32_t* t = X; X = Y; Y = t;
    memcpy(Y, X, n * 4);
    if (S == 0 || wl * 2 <= S) { /* new epoch: ranks of W_k in id order */
      int64_t r = 0;
      for (int64_t v = 0; v < n; ++v) rank[v] = inW[v] ? (int32_t)r++ : -1;
      S = wl;
    }
    double g[3] = {0}, lo[3] = {0}, ld[3] = {0}, skip[3] = {0};
    /* bins 0/1: instruction groups over the ascending worklist */
    int64_t nw2 = 0;
    double hotl[4] = {0};
#pragma omp parallel for schedule(dynamic, 4096) reduction(+ : g[:3], lo[:3], ld[:3], skip[:3], hotl[:4])
    for (int64_t i = 0; i < wl; ++i) {
      const int32_t v = W[i];
      const int64_t d = R[v + 1] - R[v];
      { /* conflict-first: a vertex that does not conflict needs no entry w > v (lowid) */
        int conf = 0;
        for (int64_t j = R[v]; j < R[v + 1] && C[j] < v; ++j)
          if (X[C[j]] == X[v]) { conf = 1; break; }
        if (!conf) {
          const int b = d <= 32 ? 0 : (d <= 256 ? 1 : 2);
          for (int64_t j = R[v]; j < R[v + 1]; ++j)
            if (C[j] > v && (b < 2 || inW[C[j]])) skip[b] += 1;
        }
      }
      if (d > 32 && d <= 256) { /* bin 1 if it were trimmed: live entries */
        for (int64_t j = R[v]; j < R[v + 1]; ++j) ld[1] += inW[C[j]] ? 1 : 0;
      }
      if (d > 256) { /* bin 2: exact live list, 32 consecutive entries per instruction */
        uint32_t a[32], b[32];
        int m = 0;
        for (int64_t j = R[v]; j < R[v + 1]; ++j) {
          const int32_t w = C[j];
          if (!inW[w]) continue;
          for (int h = 0; h < 4; ++h) hotl[h] += w < (1 << (12 + 2 * h)) ? 1 : 0;
          a[m] = (uint32_t)w >> shift;
          b[m] = (uint32_t)rank[w] >> shift;
          if (++m == 32) {
            g[2] += 32; lo[2] += distinct(a, 32); ld[2] += distinct(b, 32); m = 0;
          }
        }
        if (m) { g[2] += m; lo[2] += distinct(a, m); ld[2] += distinct(b, m); }
      }
    }
    /* bins 0/1 in instruction groups (serial over groups, parallel inside is not needed) */
    for (int bin = 0; bin < 2; ++bin) {
      const int vpw = bin == 0 ? 8 : 4, lpv = bin == 0 ? 4 : 8;
      int32_t grp[8];
      int ng = 0;
      for (int64_t i = 0; i <= wl; ++i) {
        int flush = i == wl;
        if (!flush) {
          const int32_t v = W[i];
          const int64_t d = R[v + 1] - R[v];
          if ((bin == 0 && d <= 32) || (bin == 1 && d > 32 && d <= 256)) grp[ng++] = v;
          flush = ng == vpw;
        }
        if (flush && ng) {
          int64_t maxd = 0;
          for (int q = 0; q < ng; ++q) {
            const int64_t d = R[grp[q] + 1] - R[grp[q]];
            if (d > maxd) maxd = d;
          }
          for (int64_t base = 0; base < maxd; base += lpv) {
            uint32_t a[32];
            int m = 0;
            for (int q = 0; q < ng; ++q)
              for (int l = 0; l < lpv; ++l) {
                const int64_t j = R[grp[q]] + base + l;
                if (j < R[grp[q] + 1]) a[m++] = (uint32_t)C[j] >> shift;
              }
            g[bin] += m;
            lo[bin] += distinct(a, m);
          }
          ng = 0;
        }
      }
    }
    /* the Jacobi pass itself: detect (round k-1 colors = X) + assign against X */
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < wl; ++i) {
      const int32_t v = W[i];
      int conf = 0;
      for (int64_t j = R[v]; j < R[v + 1]; ++j)
        if (X[C[j]] == X[v] && C[j] < v) { conf = 1; break; }
      if (!conf) { inW[v] = 2; continue; } /* leaves */
      /* first fit against X */
      uint64_t m[8] = {0};
      int big = 0;
      for (int64_t j = R[v]; j < R[v + 1]; ++j) {
        const int32_t c = X[C[j]];
        if (c < 512) m[c >> 6] |= 1ull << (c & 63); else big = 1;
      }
      (void)big;
      m[0] |= 1;
      int tent = -1;
      for (int q = 0; q < 8 && tent < 0; ++q)
        if (~m[q]) tent = q * 64 + __builtin_ctzll(~m[q]);
      Y[v] = tent;
    }
    for (int64_t i = 0; i < wl; ++i) {
      const int32_t v = W[i];
      if (inW[v] == 2) inW[v] = 0; else W2[nw2++] = v;
    }
    printf("%d %lld | %.0f %.0f | %.0f %.0f %.0f | %.0f %.0f %.0f | %lld\n", k, (long long)wl, g[0],
           lo[0], g[1], lo[1], ld[1], g[2], lo[2], ld[2], (long long)S);
    for (int q = 0; q < 3; ++q) { tot_g[q] += g[q]; tot_lo[q] += lo[q]; tot_ld[q] += ld[q]; tot_skip[q] += skip[q]; }
    for (int h = 0; h < 4; ++h) hot[h] += hotl[h];
    if (k < 40) printf("   hot %.3f %.3f %.3f %.3f of bin2\n", hotl[0] / (g[2] + 1e-9), hotl[1] / (g[2] + 1e-9), hotl[2] / (g[2] + 1e-9), hotl[3] / (g[2] + 1e-9));
    if (k < 40) printf("   skip %.0f %.0f %.0f\n", skip[0], skip[1], skip[2]);
    int32_t* tw = W; W = W2; W2 = tw;
    wl = nw2;
  }
  printf("TOTAL gathers bin0 %.3g bin1 %.3g (live %.3g) bin2 %.3g | lines bin0 %.3g bin1 %.3g bin2 orig %.3g dense %.3g\n",
         tot_g[0], tot_g[1], tot_ld[1], tot_g[2], tot_lo[0], tot_lo[1], tot_lo[2], tot_ld[2]);
  printf("HOT bin-2 gathers with id < 2^12/14/16/18: %.3f %.3f %.3f %.3f\n", hot[0] / tot_g[2], hot[1] / tot_g[2], hot[2] / tot_g[2], hot[3] / tot_g[2]);
  printf("SKIPPABLE (conflict-first) bin0 %.3g bin1 %.3g bin2 %.3g\n", tot_skip[0], tot_skip[1], tot_skip[2]);
  return 0;
}
