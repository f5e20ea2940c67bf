// sgr_gen.cpp — seeded synthetic CSR generators. See include/sgr_gen.h for the contract.
//
// Input-side only: nothing here knows about colors, masks or conflicts. Shared by the CPU
// oracle tests and the CUDA path tests/bench as "the seeded input generator" module.
//
// Workload recipes follow PAPER.md P:234 (R-MAT [36] with (a,b,c,d)), Table I
// (rmat-er / rmat-g: 2^20 vertices, ~20 directed edges per vertex) and BASELINE.json's five
// configs; the R-MAT bit convention is SURVEY §8(c) reading C13, the stencil one C14.
#include "../../include/sgr_gen.h"

#include <algorithm>
#include <atomic>
#include <cstdlib>
#include <cstring>
#include <vector>

#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// Counter-based stream: value number `ctr` of stream `stream` under `seed`.
inline uint64_t rng_at(uint64_t seed, uint64_t stream, uint64_t ctr) {
  return splitmix64(splitmix64(seed ^ (stream * 0xD1B54A32D192ED03ull)) + ctr);
}

inline uint64_t mulhi64(uint64_t a, uint64_t b) {
  return (uint64_t)(((__uint128_t)a * (__uint128_t)b) >> 64);
}

void prefix_sum_inplace(int64_t* a, int64_t len) {  // exclusive, a[len] = total
  int64_t run = 0;
  for (int64_t i = 0; i < len; ++i) {
    int64_t d = a[i];
    a[i] = run;
    run += d;
  }
  a[len] = run;
}

// Build a symmetric, sorted, loop-free, dedup'd CSR from m undirected pairs produced by
// `pair(i, &u, &v)`. Deterministic regardless of thread count: rows are sorted at the end.
template <class PairFn>
int build_csr(int64_t n, int64_t m, PairFn pair, sgr_gen_graph* out) {
  if (!out || n < 0 || m < 0 || n > INT32_MAX) return -1;
  out->n = n;
  out->nnz = 0;
  out->row_ptr = nullptr;
  out->col_idx = nullptr;
  int64_t* deg = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
  if (!deg) return -2;
  // pass 1: degrees (each undirected pair contributes to both endpoints)
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    int64_t u, v;
    pair(i, &u, &v);
    if (u == v) continue;
    __atomic_fetch_add(&deg[u], 1, __ATOMIC_RELAXED);
    __atomic_fetch_add(&deg[v], 1, __ATOMIC_RELAXED);
  }
  prefix_sum_inplace(deg, n);  // deg now = provisional offsets
  const int64_t total = deg[n];
  int32_t* tmp = (int32_t*)malloc((size_t)std::max<int64_t>(total, 1) * sizeof(int32_t));
  int64_t* cur = (int64_t*)malloc(((size_t)n + 1) * sizeof(int64_t));
  if (!tmp || !cur) {
    free(deg);
    free(tmp);
    free(cur);
    return -2;
  }
  memcpy(cur, deg, ((size_t)n + 1) * sizeof(int64_t));
  // pass 2: scatter (pairs are regenerated: the generator is counter-based)
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; ++i) {
    int64_t u, v;
    pair(i, &u, &v);
    if (u == v) continue;
    int64_t pu = __atomic_fetch_add(&cur[u], 1, __ATOMIC_RELAXED);
    int64_t pv = __atomic_fetch_add(&cur[v], 1, __ATOMIC_RELAXED);
    tmp[pu] = (int32_t)v;
    tmp[pv] = (int32_t)u;
  }
  free(cur);
  // pass 3: sort + unique each row; record unique degree
  int64_t* ndeg = (int64_t*)malloc(((size_t)n + 1) * sizeof(int64_t));
  if (!ndeg) {
    free(deg);
    free(tmp);
    return -2;
  }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < n; ++v) {
    int32_t* b = tmp + deg[v];
    int32_t* e = tmp + deg[v + 1];
    std::sort(b, e);
    ndeg[v] = std::unique(b, e) - b;
  }
  prefix_sum_inplace(ndeg, n);
  const int64_t nnz = ndeg[n];
  int32_t* col = (int32_t*)malloc((size_t)std::max<int64_t>(nnz, 1) * sizeof(int32_t));
  if (!col) {
    free(deg);
    free(tmp);
    free(ndeg);
    return -2;
  }
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < n; ++v) {
    memcpy(col + ndeg[v], tmp + deg[v], (size_t)(ndeg[v + 1] - ndeg[v]) * sizeof(int32_t));
  }
  free(tmp);
  free(deg);
  out->nnz = nnz;
  out->row_ptr = ndeg;
  out->col_idx = col;
  return 0;
}

// Seeded Fisher-Yates permutation of [0, n).
std::vector<int32_t> make_perm(int64_t n, uint64_t seed) {
  std::vector<int32_t> p((size_t)n);
  for (int64_t i = 0; i < n; ++i) p[(size_t)i] = (int32_t)i;
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)mulhi64(rng_at(seed, 7, (uint64_t)i), (uint64_t)(i + 1));
    std::swap(p[(size_t)i], p[(size_t)j]);
  }
  return p;
}

}  // namespace

extern "C" {

uint64_t sgr_gen_splitmix64(uint64_t x) { return splitmix64(x); }

int sgr_gen_rmat(int scale, int64_t edge_factor, double a, double b, double c, uint64_t seed,
                 int permute, sgr_gen_graph* out) {
  if (scale < 0 || scale > 30 || edge_factor < 0 || a < 0 || b < 0 || c < 0 ||
      a + b + c > 1.0 + 1e-12)
    return -1;
  const int64_t n = (int64_t)1 << scale;
  const int64_t m = edge_factor * n;
  // Quadrant thresholds on a 32-bit uniform: u < ta -> a, < tb -> b, < tc -> c, else d.
  const double two32 = 4294967296.0;
  const uint64_t ta = (uint64_t)(a * two32);
  const uint64_t tb = (uint64_t)((a + b) * two32);
  const uint64_t tc = (uint64_t)((a + b + c) * two32);
  std::vector<int32_t> perm;
  if (permute) perm = make_perm(n, seed ^ 0x5bd1e995ull);
  const int32_t* pp = permute ? perm.data() : nullptr;
  auto pair = [=](int64_t i, int64_t* u, int64_t* v) {
    int64_t r = 0, q = 0;
    uint64_t word = 0;
    for (int l = 0; l < scale; ++l) {
      if ((l & 1) == 0) word = rng_at(seed, 1, (uint64_t)i * 16 + (uint64_t)(l >> 1));
      uint64_t x = (l & 1) ? (word >> 32) : (word & 0xffffffffull);
      int rb, cb;
      if (x < ta) {
        rb = 0; cb = 0;
      } else if (x < tb) {
        rb = 0; cb = 1;
      } else if (x < tc) {
        rb = 1; cb = 0;
      } else {
        rb = 1; cb = 1;
      }
      r = (r << 1) | rb;
      q = (q << 1) | cb;
    }
    if (pp) {
      r = pp[r];
      q = pp[q];
    }
    *u = r;
    *v = q;
  };
  return build_csr(n, m, pair, out);
}

int sgr_gen_er(int64_t n, int64_t pairs, uint64_t seed, sgr_gen_graph* out) {
  if (n < 0 || pairs < 0 || (n == 0 && pairs > 0)) return -1;
  auto pair = [=](int64_t i, int64_t* u, int64_t* v) {
    *u = (int64_t)mulhi64(rng_at(seed, 2, 2 * (uint64_t)i), (uint64_t)n);
    *v = (int64_t)mulhi64(rng_at(seed, 2, 2 * (uint64_t)i + 1), (uint64_t)n);
  };
  return build_csr(n, pairs, pair, out);
}

static int stencil_impl(int64_t nx, int64_t ny, int64_t nz, int rx, int ry, int rz, bool box,
                        sgr_gen_graph* out) {
  if (!out || nx < 0 || ny < 0 || nz < 0) return -1;
  const int64_t n = nx * ny * nz;
  if (n > INT32_MAX) return -1;
  out->n = n;
  out->nnz = 0;
  int64_t* rp = (int64_t*)malloc(((size_t)n + 1) * sizeof(int64_t));
  if (!rp) return -2;
  // neighbour offsets in (dz, dy, dx) lexicographic order => ascending ids in natural order
  auto is_nbr = [&](int dx, int dy, int dz) {
    if (dx == 0 && dy == 0 && dz == 0) return false;
    if (box) return true;
    return (dx != 0) + (dy != 0) + (dz != 0) == 1;  // axis neighbours only
  };
  auto row = [&](int64_t v, int32_t* dst) -> int64_t {
    int64_t x = v % nx, y = (v / nx) % ny, z = v / (nx * ny);
    int64_t k = 0;
    for (int dz = -rz; dz <= rz; ++dz)
      for (int dy = -ry; dy <= ry; ++dy)
        for (int dx = -rx; dx <= rx; ++dx) {
          if (!is_nbr(dx, dy, dz)) continue;
          int64_t X = x + dx, Y = y + dy, Z = z + dz;
          if (X < 0 || X >= nx || Y < 0 || Y >= ny || Z < 0 || Z >= nz) continue;
          if (dst) dst[k] = (int32_t)(X + nx * (Y + ny * Z));
          ++k;
        }
    return k;
  };
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < n; ++v) rp[v] = row(v, nullptr);
  prefix_sum_inplace(rp, n);
  const int64_t nnz = rp[n];
  int32_t* col = (int32_t*)malloc((size_t)std::max<int64_t>(nnz, 1) * sizeof(int32_t));
  if (!col) {
    free(rp);
    return -2;
  }
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < n; ++v) row(v, col + rp[v]);
  out->nnz = nnz;
  out->row_ptr = rp;
  out->col_idx = col;
  return 0;
}

int sgr_gen_stencil2d(int64_t nx, int64_t ny, int points, sgr_gen_graph* out) {
  if (points != 5 && points != 9) return -1;
  return stencil_impl(nx, ny, 1, 1, 1, 0, points == 9, out);
}

int sgr_gen_stencil3d(int64_t nx, int64_t ny, int64_t nz, int points, sgr_gen_graph* out) {
  if (points != 7 && points != 27) return -1;
  return stencil_impl(nx, ny, nz, 1, 1, 1, points == 27, out);
}

int sgr_gen_from_edges(int64_t n, int64_t m, const int64_t* src, const int64_t* dst,
                       sgr_gen_graph* out) {
  if (m > 0 && (!src || !dst)) return -1;
  for (int64_t i = 0; i < m; ++i)
    if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return -1;
  auto pair = [=](int64_t i, int64_t* u, int64_t* v) {
    *u = src[i];
    *v = dst[i];
  };
  return build_csr(n, m, pair, out);
}

int sgr_gen_permute(const sgr_gen_graph* in, uint64_t seed, sgr_gen_graph* out) {
  if (!in || !out) return -1;
  const int64_t n = in->n;
  std::vector<int32_t> perm = make_perm(n, seed ^ 0x5bd1e995ull);
  // Enumerate directed entries (v -> col) as pairs; each undirected edge appears twice,
  // which build_csr dedupes.
  std::vector<int64_t> rowof((size_t)in->nnz);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < n; ++v)
    for (int64_t e = in->row_ptr[v]; e < in->row_ptr[v + 1]; ++e) rowof[(size_t)e] = v;
  const int64_t* rf = rowof.data();
  const int32_t* ci = in->col_idx;
  const int32_t* pp = perm.data();
  auto pair = [=](int64_t i, int64_t* u, int64_t* v) {
    *u = pp[rf[i]];
    *v = pp[ci[i]];
  };
  return build_csr(n, in->nnz, pair, out);
}

int sgr_gen_validate(const int64_t* row_ptr, const int32_t* col_idx, int64_t n, int64_t nnz) {
  if (n < 0 || nnz < 0 || !row_ptr || (nnz > 0 && !col_idx)) return 1;
  if (row_ptr[0] != 0 || row_ptr[n] != nnz) return 1;
  for (int64_t v = 0; v < n; ++v)
    if (row_ptr[v + 1] < row_ptr[v]) return 1;
  std::atomic<int> bad{0};
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < n; ++v) {
    int flags = 0;
    for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
      int64_t w = col_idx[e];
      if (w < 0 || w >= n) {
        flags |= 2;
        continue;
      }
      if (e > row_ptr[v]) {
        if (col_idx[e - 1] > w) flags |= 4;
        if (col_idx[e - 1] == w) flags |= 8;
      }
      if (w == v) flags |= 16;
    }
    if (flags) bad.fetch_or(flags);
  }
  int flags = bad.load();
  if (flags & (2 | 4)) return flags;  // symmetry check below needs sorted, in-range rows
  // symmetry: for each entry v->w, w's row contains v (binary search in the sorted row)
  std::atomic<int> asym{0};
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < n; ++v) {
    for (int64_t e = row_ptr[v]; e < row_ptr[v + 1]; ++e) {
      int64_t w = col_idx[e];
      const int32_t* b = col_idx + row_ptr[w];
      const int32_t* en = col_idx + row_ptr[w + 1];
      if (!std::binary_search(b, en, (int32_t)v)) {
        asym.store(32);
        break;
      }
    }
  }
  return flags | asym.load();
}

void sgr_gen_free(sgr_gen_graph* g) {
  if (!g) return;
  free(g->row_ptr);
  free(g->col_idx);
  g->row_ptr = nullptr;
  g->col_idx = nullptr;
  g->n = g->nnz = 0;
}

}  // extern "C"
