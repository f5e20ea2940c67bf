/*
 * sgr_gen.h — seeded synthetic CSR graph generators (host C ABI).
 *
 * This module produces the INPUTS of the coloring path and nothing else: it holds none
 * of the method's arithmetic (no masks, no first-fit, no conflict rule), so the CPU
 * oracle (oracle/) and the CUDA path (libsgr.so) may both consume its graphs.
 *
 * Workloads (Table I; BASELINE.json configs):
 *   - R-MAT [36]: per pair, `scale` independent quadrant draws, MSB first,
 *     a=(0,0) b=(0,1) c=(1,0) d=(1,1) (SURVEY §8(c) reading C13). Draw (i, l) is a
 *     32-bit uniform taken from splitmix64(seed, i, l/2) (low half for even l, high half
 *     for odd l): a counter-based generator, so the graph depends only on the seed and
 *     never on the thread count.
 *   - Erdos-Renyi G(n, m-pairs): pair i = (U(2i) mod n, U(2i+1) mod n) via multiply-high.
 *   - 2D 5/9-point and 3D 7/27-point stencils, natural order v = x + nx*(y + ny*z),
 *     no diagonal (reading C14).
 * Every generator symmetrizes, drops self-loops, sorts every row ascending and removes
 * duplicates, so the output satisfies the input contract of include/sgr.h.
 *
 * Ownership: the generator allocates row_ptr/col_idx with malloc(); the caller releases
 * them with sgr_gen_free(). All functions return 0 on success, -1 on bad arguments,
 * -2 on allocation failure. Thread-safe; uses OpenMP internally when available.
 */
#ifndef SGR_GEN_H
#define SGR_GEN_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int64_t n;        /* vertices */
  int64_t nnz;      /* directed CSR entries (each undirected edge appears twice) */
  int64_t* row_ptr; /* n+1 entries, row_ptr[0]=0, row_ptr[n]=nnz (malloc'd) */
  int32_t* col_idx; /* nnz entries, rows sorted ascending, no loops, no dups (malloc'd) */
} sgr_gen_graph;

/* R-MAT: n = 2^scale, pairs = edge_factor * n, probabilities (a,b,c,1-a-b-c).
 * permute != 0 relabels vertices with a seeded Fisher-Yates permutation (Graph500 style). */
int sgr_gen_rmat(int scale, int64_t edge_factor, double a, double b, double c, uint64_t seed,
                 int permute, sgr_gen_graph* out);

/* Erdos-Renyi: `pairs` uniform (u, v) draws, symmetrized (average degree ~ 2*pairs/n). */
int sgr_gen_er(int64_t n, int64_t pairs, uint64_t seed, sgr_gen_graph* out);

/* 2D stencil on nx*ny: points = 5 (von Neumann) or 9 (Moore). */
int sgr_gen_stencil2d(int64_t nx, int64_t ny, int points, sgr_gen_graph* out);

/* 3D stencil on nx*ny*nz: points = 7 or 27 (HPCG-style, P:11 [6]). */
int sgr_gen_stencil3d(int64_t nx, int64_t ny, int64_t nz, int points, sgr_gen_graph* out);

/* Build a symmetric, sorted, loop-free, duplicate-free CSR from an arbitrary edge list
 * (src[i], dst[i]), i < m, ids in [0, n). */
int sgr_gen_from_edges(int64_t n, int64_t m, const int64_t* src, const int64_t* dst,
                       sgr_gen_graph* out);

/* Seeded relabeling: out = P(in) with the same Fisher-Yates permutation sgr_gen_rmat uses. */
int sgr_gen_permute(const sgr_gen_graph* in, uint64_t seed, sgr_gen_graph* out);

/* Validate a CSR. Returns a bitmask of violations (0 = valid):
 *   1 row_ptr not monotone / row_ptr[0]!=0 / row_ptr[n]!=nnz   2 column out of range
 *   4 row not sorted ascending   8 duplicate entry   16 self-loop   32 not symmetric */
int sgr_gen_validate(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int64_t nnz);

void sgr_gen_free(sgr_gen_graph* g);

/* The counter-based generator itself, exported so tests can pin it. */
uint64_t sgr_gen_splitmix64(uint64_t x);

#ifdef __cplusplus
}
#endif
#endif
