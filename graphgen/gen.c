/*
 * graphgen/gen.c -- seeded synthetic graph generators shared by BOTH sides
 * (the oracle under oracle/ and the CUDA product path).  This file holds no
 * part of the Graffix method: it only produces raw directed edge lists and a
 * raw CSR (rows grouped by source, each row ordered by (destination, edge
 * index)); duplicates and self-loops are left in place so that each side
 * canonicalises independently.
 *
 * Every random draw is counter based: splitmix64(seed ^ f(index)), so any
 * edge can be regenerated from (seed, edge index) alone, on any host.
 *
 * Shapes follow the paper's Table 1 (PAPER.md P@35781-36235):
 *   - R-MAT (GTgraph, P@35965): scale s, edge factor 16, (a,b,c,d) =
 *     (0.45, 0.15, 0.15, 0.25), vertex ids permuted with a seed.
 *   - uniform random (Erdos-Renyi-like "random26"): (src, dst) uniform.
 *   - road-like grid ("USA-road"): side x side lattice; a spanning tree
 *     from the binary-tree maze rule (each cell links north or west), every
 *     other lattice edge kept with p = 0.15, one diagonal per cell with
 *     p = 0.10; symmetric; natural (row-major) ids.
 *   - weights: uniform integers 1..100 (BASELINE.json configs).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t sm64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
static inline uint64_t draw(uint64_t seed, uint64_t stream, uint64_t idx) {
  return sm64(sm64(seed ^ (stream * 0xD6E8FEB86659FD93ull)) ^ idx);
}

uint32_t gg_weight(uint64_t wseed, uint64_t eidx) {
  return 1u + (uint32_t)(draw(wseed, 7, eidx) % 100u);
}

/* R-MAT edge e: `scale` quadrant choices with 32-bit integer thresholds. */
void gg_rmat_edges(int scale, int64_t m, uint64_t seed, uint64_t wseed,
                   uint32_t ta, uint32_t tab, uint32_t tabc, int permute,
                   int32_t *src, int32_t *dst, uint32_t *w) {
  int64_t n = (int64_t)1 << scale;
  int32_t *perm = NULL;
  if (permute) {
    perm = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
    for (int64_t i = 0; i < n; i++) perm[i] = (int32_t)i;
    for (int64_t i = n - 1; i > 0; i--) { /* Fisher-Yates, counter based */
      int64_t j = (int64_t)(draw(seed, 3, (uint64_t)i) % (uint64_t)(i + 1));
      int32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
    }
  }
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < m; e++) {
    uint64_t u = 0, v = 0;
    for (int l = 0; l < scale; l++) {
      uint32_t r = (uint32_t)(draw(seed, 1, (uint64_t)e * 64u + (uint64_t)l) >> 32);
      int sb, db;
      if (r < ta) { sb = 0; db = 0; }
      else if (r < tab) { sb = 0; db = 1; }
      else if (r < tabc) { sb = 1; db = 0; }
      else { sb = 1; db = 1; }
      u = (u << 1) | (uint64_t)sb;
      v = (v << 1) | (uint64_t)db;
    }
    src[e] = perm ? perm[u] : (int32_t)u;
    dst[e] = perm ? perm[v] : (int32_t)v;
    w[e] = gg_weight(wseed, (uint64_t)e);
  }
  free(perm);
}

void gg_uniform_edges(int64_t n, int64_t m, uint64_t seed, uint64_t wseed,
                      int32_t *src, int32_t *dst, uint32_t *w) {
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < m; e++) {
    src[e] = (int32_t)(draw(seed, 1, (uint64_t)e) % (uint64_t)n);
    dst[e] = (int32_t)(draw(seed, 2, (uint64_t)e) % (uint64_t)n);
    w[e] = gg_weight(wseed, (uint64_t)e);
  }
}

/* Road-like grid.  Undirected edge ids: cell*4 + {0: east, 1: south,
 * 2: diagonal SE, 3: anti-diagonal SW}.  Tree edge of cell (r,c) != (0,0):
 * west if r == 0, north if c == 0, else north or west by one random bit.
 * Emits both arcs of every kept undirected edge.  Two-call: with src == NULL
 * only the arc count is returned. */
static inline int road_keep(uint64_t seed, int64_t side, int64_t cell, int kind) {
  int64_t r = cell / side, c = cell % side;
  if (kind == 0) {              /* east: (r,c)-(r,c+1) */
    if (c + 1 >= side) return 0;
    /* tree edge if cell (r,c+1) chose west */
    int64_t nb = cell + 1;
    int64_t nr = r, nc = c + 1;
    int tree = (nr == 0) ? 1 : (draw(seed, 11, (uint64_t)nb) & 1u) ? 1 : 0;
    (void)nc;
    if (tree) return 1;
  } else if (kind == 1) {       /* south: (r,c)-(r+1,c) */
    if (r + 1 >= side) return 0;
    int64_t nb = cell + side;
    int64_t nc = c;
    int tree = (nc == 0) ? 1 : (draw(seed, 11, (uint64_t)nb) & 1u) ? 0 : 1;
    if (tree) return 1;
  } else {                      /* diagonals */
    if (r + 1 >= side) return 0;
    if (kind == 2 && c + 1 >= side) return 0;
    if (kind == 3 && c == 0) return 0;
    uint64_t d = draw(seed, 13, (uint64_t)cell);
    int pick = (d >> 63) ? 3 : 2;          /* at most one diagonal per cell */
    if (pick != kind) return 0;
    return (uint32_t)(d & 0xffffffffu) < (uint32_t)(0.10 * 4294967296.0);
  }
  /* non-tree lattice edge kept with p = 0.15 */
  uint32_t x = (uint32_t)(draw(seed, 12, (uint64_t)cell * 4u + (uint64_t)kind) >> 32);
  return x < (uint32_t)(0.15 * 4294967296.0);
}

int64_t gg_road_edges(int64_t side, uint64_t seed, uint64_t wseed,
                      int32_t *src, int32_t *dst, uint32_t *w) {
  int64_t n = side * side;
  /* pass 1: per-cell counts (parallel), prefix, pass 2: emit */
  int64_t *cnt = (int64_t *)malloc(sizeof(int64_t) * (size_t)(n + 1));
#pragma omp parallel for schedule(static)
  for (int64_t cell = 0; cell < n; cell++) {
    int k = 0;
    for (int kind = 0; kind < 4; kind++) k += road_keep(seed, side, cell, kind);
    cnt[cell] = 2 * k;
  }
  int64_t tot = 0;
  for (int64_t cell = 0; cell < n; cell++) { int64_t t = cnt[cell]; cnt[cell] = tot; tot += t; }
  cnt[n] = tot;
  if (src) {
#pragma omp parallel for schedule(static)
    for (int64_t cell = 0; cell < n; cell++) {
      int64_t o = cnt[cell];
      int64_t r = cell / side, c = cell % side;
      for (int kind = 0; kind < 4; kind++) {
        if (!road_keep(seed, side, cell, kind)) continue;
        int64_t other;
        if (kind == 0) other = cell + 1;
        else if (kind == 1) other = cell + side;
        else if (kind == 2) other = (r + 1) * side + (c + 1);
        else other = (r + 1) * side + (c - 1);
        uint32_t ww = gg_weight(wseed, (uint64_t)cell * 4u + (uint64_t)kind);
        src[o] = (int32_t)cell; dst[o] = (int32_t)other; w[o] = ww; o++;
        src[o] = (int32_t)other; dst[o] = (int32_t)cell; w[o] = ww; o++;
      }
    }
  }
  free(cnt);
  return tot;
}

/* Raw CSR: rows grouped by src; inside a row, ordered by (dst, edge index).
 * Duplicates and self-loops are kept (each side canonicalises). */
static int cmp_u64(const void *a, const void *b) {
  uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b;
  return (x > y) - (x < y);
}

void gg_build_csr(int64_t n, int64_t m, const int32_t *src, const int32_t *dst,
                  const uint32_t *w, int64_t *row_ptr, int32_t *col, uint32_t *ow) {
  memset(row_ptr, 0, sizeof(int64_t) * (size_t)(n + 1));
  for (int64_t e = 0; e < m; e++) row_ptr[src[e] + 1]++;
  for (int64_t v = 0; v < n; v++) row_ptr[v + 1] += row_ptr[v];
  int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  memcpy(cur, row_ptr, sizeof(int64_t) * (size_t)n);
  /* keys: (dst << 31 | e) needs e < 2^31 and dst < 2^33 */
  uint64_t *key = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(m > 0 ? m : 1));
  for (int64_t e = 0; e < m; e++)
    key[cur[src[e]]++] = ((uint64_t)(uint32_t)dst[e] << 31) | (uint64_t)e;
  free(cur);
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t v = 0; v < n; v++) {
    int64_t b = row_ptr[v], d = row_ptr[v + 1] - b;
    if (d > 1) qsort(key + b, (size_t)d, sizeof(uint64_t), cmp_u64);
  }
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < m; i++) {
    uint64_t k = key[i];
    int64_t e = (int64_t)(k & 0x7fffffffull);
    col[i] = (int32_t)(k >> 31);
    ow[i] = w[e];
  }
  free(key);
}
