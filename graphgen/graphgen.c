/* graphgen.c — seeded synthetic input graphs for the HEC hot path.
 *
 * This module holds NO arithmetic of the coarsening method: it only builds the
 * input G0 (undirected, unit weights, CSR with int64 row_ptr and ascending int32
 * columns, no self-loops, no duplicates) that both the oracle and the CUDA path
 * consume.  Shapes follow BASELINE.json configs:
 *   grid2d   nx*ny 4-neighbour mesh        id = i*ny + j          (config 1)
 *   mesh27   nx*ny*nz 27-point stencil     id = (i*ny + j)*nz + k (config 2)
 *   rmat     Graph500-like R-MAT, the counter-based "G-spec" of SURVEY §8(d):
 *            per-bit splitmix64 draws with (A,B,C,D)=(0.57,0.19,0.19,0.05),
 *            a seeded vertex permutation, symmetrise + dedup, largest connected
 *            component, relabel ascending (configs 3-5; the paper's preprocessing
 *            "LCC + relabel").
 * The output is a pure function of (shape, seed): independent of thread count.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdio.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t gg_splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t gg_hash(uint64_t x) { return gg_splitmix64(x); }

/* ---------------------------------------------------------------- meshes */
int64_t gg_grid2d_nnz(int64_t nx, int64_t ny) {
  return 2 * (nx * (ny - 1) + ny * (nx - 1));
}

void gg_grid2d(int64_t nx, int64_t ny, int64_t *row_ptr, int32_t *col) {
  int64_t n = nx * ny;
  /* degrees first, then an exclusive prefix (neighbours in ascending id order) */
  row_ptr[0] = 0;
  for (int64_t i = 0; i < nx; ++i)
    for (int64_t j = 0; j < ny; ++j) {
      int64_t d = (i > 0) + (j > 0) + (j + 1 < ny) + (i + 1 < nx);
      row_ptr[i * ny + j + 1] = d;
    }
  for (int64_t u = 0; u < n; ++u) row_ptr[u + 1] += row_ptr[u];
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < nx; ++i)
    for (int64_t j = 0; j < ny; ++j) {
      int64_t u = i * ny + j, p = row_ptr[u];
      if (i > 0) col[p++] = (int32_t)(u - ny);
      if (j > 0) col[p++] = (int32_t)(u - 1);
      if (j + 1 < ny) col[p++] = (int32_t)(u + 1);
      if (i + 1 < nx) col[p++] = (int32_t)(u + ny);
    }
}

static inline int64_t span3(int64_t i, int64_t n) { return 1 + (i > 0) + (i + 1 < n); }

int64_t gg_mesh27_nnz(int64_t nx, int64_t ny, int64_t nz) {
  int64_t s = 0;
  for (int64_t i = 0; i < nx; ++i) {
    int64_t si = span3(i, nx);
    for (int64_t j = 0; j < ny; ++j) {
      int64_t sj = span3(j, ny);
      for (int64_t k = 0; k < nz; ++k) s += si * sj * span3(k, nz) - 1;
    }
  }
  return s;
}

void gg_mesh27(int64_t nx, int64_t ny, int64_t nz, int64_t *row_ptr, int32_t *col) {
  int64_t n = nx * ny * nz;
  row_ptr[0] = 0;
  for (int64_t i = 0; i < nx; ++i)
    for (int64_t j = 0; j < ny; ++j)
      for (int64_t k = 0; k < nz; ++k)
        row_ptr[(i * ny + j) * nz + k + 1] = span3(i, nx) * span3(j, ny) * span3(k, nz) - 1;
  for (int64_t u = 0; u < n; ++u) row_ptr[u + 1] += row_ptr[u];
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < nx; ++i)
    for (int64_t j = 0; j < ny; ++j)
      for (int64_t k = 0; k < nz; ++k) {
        int64_t u = (i * ny + j) * nz + k, p = row_ptr[u];
        /* lexicographic (di, dj, dk) == ascending neighbour id */
        for (int di = -1; di <= 1; ++di) {
          int64_t a = i + di; if (a < 0 || a >= nx) continue;
          for (int dj = -1; dj <= 1; ++dj) {
            int64_t b = j + dj; if (b < 0 || b >= ny) continue;
            for (int dk = -1; dk <= 1; ++dk) {
              int64_t c = k + dk; if (c < 0 || c >= nz) continue;
              if (!di && !dj && !dk) continue;
              col[p++] = (int32_t)((a * ny + b) * nz + c);
            }
          }
        }
      }
}

/* ------------------------------------------------------------------ R-MAT */
typedef struct {
  int64_t n, nnz;
  int64_t *row_ptr;
  int32_t *col;
} gg_graph;

static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

/* in-place LSD radix sort of (key, idx) by key (stable, so ties stay in idx order) */
static void radix_sort_kv(uint64_t *key, uint32_t *idx, int64_t N) {
  uint64_t *k2 = (uint64_t *)malloc(sizeof(uint64_t) * N);
  uint32_t *i2 = (uint32_t *)malloc(sizeof(uint32_t) * N);
  for (int pass = 0; pass < 8; ++pass) {
    int sh = pass * 8;
    int64_t cnt[257];
    memset(cnt, 0, sizeof cnt);
    for (int64_t t = 0; t < N; ++t) cnt[((key[t] >> sh) & 255) + 1]++;
    for (int b = 0; b < 256; ++b) cnt[b + 1] += cnt[b];
    for (int64_t t = 0; t < N; ++t) {
      int64_t p = cnt[(key[t] >> sh) & 255]++;
      k2[p] = key[t]; i2[p] = idx[t];
    }
    memcpy(key, k2, sizeof(uint64_t) * N);
    memcpy(idx, i2, sizeof(uint32_t) * N);
  }
  free(k2); free(i2);
}

/* union-find with path halving */
static int32_t uf_find(int32_t *p, int32_t x) {
  while (p[x] != x) { p[x] = p[p[x]]; x = p[x]; }
  return x;
}

#define T1 2448131358ULL /* floor(0.57 * 2^32) */
#define T2 3264175144ULL /* floor(0.76 * 2^32) */
#define T3 4080218931ULL /* floor(0.95 * 2^32) */

static inline void rmat_sample(uint64_t seed_g, int scale, uint64_t k, uint32_t *pu, uint32_t *pv) {
  uint32_t u = 0, v = 0;
  for (int j = 0; j < scale; ++j) {
    uint64_t r = gg_splitmix64((seed_g << 40) | (k << 6) | (uint64_t)j) >> 32;
    if (r >= T3) { u |= 1u << j; v |= 1u << j; }
    else if (r >= T2) { u |= 1u << j; }
    else if (r >= T1) { v |= 1u << j; }
  }
  *pu = u; *pv = v;
}

/* Returns an opaque graph (free with gg_free). NULL on allocation failure. */
void *gg_rmat(int scale, int64_t edgefactor, uint64_t seed_g, int nthreads) {
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  int64_t N = (int64_t)1 << scale;
  int64_t S = edgefactor * N;
  /* 1. vertex permutation pi(i) = rank of i by ascending (key_i, i) */
  uint64_t k0 = gg_splitmix64(seed_g ^ 0xD1B54A32D192ED03ULL);
  uint64_t *key = (uint64_t *)malloc(sizeof(uint64_t) * N);
  uint32_t *idx = (uint32_t *)malloc(sizeof(uint32_t) * N);
  uint32_t *pi = (uint32_t *)malloc(sizeof(uint32_t) * N);
  if (!key || !idx || !pi) return NULL;
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < N; ++i) { key[i] = gg_splitmix64(k0 ^ (uint64_t)i); idx[i] = (uint32_t)i; }
  radix_sort_kv(key, idx, N);
  for (int64_t r = 0; r < N; ++r) pi[idx[r]] = (uint32_t)r;
  free(key); free(idx);

  /* 2. samples -> permuted endpoints; drop self-loops; count both directions */
  uint32_t *eu = (uint32_t *)malloc(sizeof(uint32_t) * S);
  uint32_t *ev = (uint32_t *)malloc(sizeof(uint32_t) * S);
  int64_t *deg = (int64_t *)calloc(N + 1, sizeof(int64_t));
  if (!eu || !ev || !deg) return NULL;
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < S; ++k) {
    uint32_t u, v;
    rmat_sample(seed_g, scale, (uint64_t)k, &u, &v);
    u = pi[u]; v = pi[v];
    eu[k] = u; ev[k] = v;
    if (u != v) {
      __atomic_fetch_add(&deg[u + 1], 1, __ATOMIC_RELAXED);
      __atomic_fetch_add(&deg[v + 1], 1, __ATOMIC_RELAXED);
    }
  }
  free(pi);
  for (int64_t u = 0; u < N; ++u) deg[u + 1] += deg[u];
  int64_t tot = deg[N];
  int32_t *adj = (int32_t *)malloc(sizeof(int32_t) * (tot > 0 ? tot : 1));
  int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * N);
  if (!adj || !cur) return NULL;
  memcpy(cur, deg, sizeof(int64_t) * N);
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < S; ++k) {
    uint32_t u = eu[k], v = ev[k];
    if (u == v) continue;
    int64_t p = __atomic_fetch_add(&cur[u], 1, __ATOMIC_RELAXED);
    adj[p] = (int32_t)v;
    p = __atomic_fetch_add(&cur[v], 1, __ATOMIC_RELAXED);
    adj[p] = (int32_t)u;
  }
  free(eu); free(ev); free(cur);
  /* 3. per-row sort + dedup (in place); new degree in ndeg */
  int64_t *ndeg = (int64_t *)calloc(N + 1, sizeof(int64_t));
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t u = 0; u < N; ++u) {
    int32_t *r = adj + deg[u];
    int64_t d = deg[u + 1] - deg[u];
    if (d == 0) continue;
    qsort(r, (size_t)d, sizeof(int32_t), cmp_i32);
    int64_t w = 1;
    for (int64_t t = 1; t < d; ++t) if (r[t] != r[w - 1]) r[w++] = r[t];
    ndeg[u + 1] = w;
  }
  /* 4. connected components (union-find over u<v), pick the largest; ties -> the
   *    component holding the smallest vertex id. Only vertices with degree>0 can
   *    be in a component of size >= 2; isolated vertices are components of 1. */
  int32_t *par = (int32_t *)malloc(sizeof(int32_t) * N);
  for (int64_t u = 0; u < N; ++u) par[u] = (int32_t)u;
  for (int64_t u = 0; u < N; ++u) {
    const int32_t *r = adj + deg[u];
    for (int64_t t = 0; t < ndeg[u + 1]; ++t) {
      int32_t v = r[t];
      if (v <= u) continue;
      int32_t a = uf_find(par, (int32_t)u), b = uf_find(par, v);
      if (a != b) { if (a < b) par[b] = a; else par[a] = b; }
    }
  }
  int32_t *csize = (int32_t *)calloc(N, sizeof(int32_t));
  for (int64_t u = 0; u < N; ++u) csize[uf_find(par, (int32_t)u)]++;
  int32_t best = 0;
  for (int64_t u = 0; u < N; ++u) /* roots are the smallest id of their set */
    if (par[u] == u && csize[u] > csize[best]) best = (int32_t)u;
  /* 5. relabel kept vertices in ascending old id; build the final CSR */
  int32_t *nid = (int32_t *)malloc(sizeof(int32_t) * N);
  int64_t nk = 0;
  for (int64_t u = 0; u < N; ++u) nid[u] = (par[u] == best) ? (int32_t)(nk++) : -1;
  free(csize);
  gg_graph *g = (gg_graph *)calloc(1, sizeof(gg_graph));
  g->n = nk;
  g->row_ptr = (int64_t *)malloc(sizeof(int64_t) * (nk + 1));
  g->row_ptr[0] = 0;
  {
    int64_t q = 0;
    for (int64_t u = 0; u < N; ++u)
      if (nid[u] >= 0) { g->row_ptr[q + 1] = g->row_ptr[q] + ndeg[u + 1]; ++q; }
  }
  g->nnz = g->row_ptr[nk];
  g->col = (int32_t *)malloc(sizeof(int32_t) * (g->nnz > 0 ? g->nnz : 1));
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t u = 0; u < N; ++u) {
    if (nid[u] < 0) continue;
    int64_t o = g->row_ptr[nid[u]];
    const int32_t *r = adj + deg[u];
    for (int64_t t = 0; t < ndeg[u + 1]; ++t) g->col[o + t] = nid[r[t]];
  }
  free(nid); free(par); free(adj); free(deg); free(ndeg);
  return g;
}

int64_t gg_n(void *h) { return ((gg_graph *)h)->n; }
int64_t gg_nnz(void *h) { return ((gg_graph *)h)->nnz; }
void gg_copy(void *h, int64_t *row_ptr, int32_t *col) {
  gg_graph *g = (gg_graph *)h;
  memcpy(row_ptr, g->row_ptr, sizeof(int64_t) * (g->n + 1));
  memcpy(col, g->col, sizeof(int32_t) * g->nnz);
}
void gg_free(void *h) {
  gg_graph *g = (gg_graph *)h;
  if (!g) return;
  free(g->row_ptr); free(g->col); free(g);
}
