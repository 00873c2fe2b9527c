/* oracle.c — the serial CPU oracle for SAGE's hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product (libsage.so) never links, loads or
 * calls it, and this file includes no header of the product (it shares no code with it).
 *
 * Every function is the plain definition (or, for the heuristic, the paper's algorithm step by
 * step in its own order) with no blocking, fusion or reordering.  "P:NNN" = line NNN of the
 * paper text (Sha, Li, Tan, "Self-adaptive Graph Traversal on GPUs", SIGMOD'21) as extracted in
 * /root/reference/PAPER.md; readings R1..R31 are the ones listed in DESIGN.md / SURVEY.md §8(c).
 *
 * Pins (tests/test_oracle_*.py, run with -m "not gpu"):
 *   ora_bfs        brute force on n<=12, scipy csgraph, certificate, symmetric |dl|<=1 invariant
 *   ora_sssp       brute-force Bellman-Ford n<=12, scipy dijkstra, w==1 reduces to BFS, certificate
 *   ora_pagerank   dense Google-matrix power iteration, networkx.pagerank, closed forms, sum=1
 *   ora_tiles      Figure 3 worked example, partition invariants
 *   reorder        Figure 5 worked example: stage-1 vector, stage-2 counts 8/4 then 6/2,
 *                  stage-3 locality 1->6, swap 8<->3 and the sorted 2nd-round tiles; objective
 *                   vs brute force; σ bijection; relabelled graph isomorphic.
 *                  The heuristic's QUALITY beyond Figure 5 is parity-unpinned (NP-hard objective,
 *                  Thm 6.1): the oracle is pinned on the worked example and invariants only.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ===================================================================================== */
/* c1. BFS — P:112-120 (Alg. 1 l.1-6: dist = -1 sentinel, dist[nb] := dist[fr] + 1) and the
 * expansion-filtering-contraction pipeline over frontier queues.  The result has a
 * plain definition (hop distance), so the oracle is a FIFO-queue BFS.                        */
int ora_bfs(int64_t n, const int64_t *off, const int32_t *col, int32_t src, int32_t *level) {
  if (src < 0 || src >= n) return 1;
  int32_t *queue = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  if (!queue) return 2;
  for (int64_t v = 0; v < n; ++v) level[v] = -1;
  int64_t head = 0, tail = 0;
  level[src] = 0;
  queue[tail++] = src;
  while (head < tail) {
    int32_t u = queue[head++];
    for (int64_t k = off[u]; k < off[u + 1]; ++k) {
      int32_t v = col[k];
      if (level[v] == -1) {          /* Alg. 1 l.3 */
        level[v] = level[u] + 1;     /* Alg. 1 l.4 */
        queue[tail++] = v;           /* Alg. 1 l.5 filter_in */
      }
    }
  }
  free(queue);
  return 0;
}

/* BFS certificate: accepts `level` iff it equals the hop distance.
 *  level(s)=0; every arc u->v with u reached has v reached and level(v) <= level(u)+1;
 *  every reached v != s has level(v) > 0 and an in-arc from u with level(u) = level(v)-1.
 * Returns 0 if accepted, else a nonzero code naming the violated rule.                       */
int ora_check_bfs(int64_t n, const int64_t *off, const int32_t *col, int32_t src, const int32_t *level) {
  if (src < 0 || src >= n) return 1;
  if (level[src] != 0) return 2;
  uint8_t *has_parent = (uint8_t *)calloc((size_t)(n > 0 ? n : 1), 1);
  for (int64_t u = 0; u < n; ++u) {
    if (level[u] < -1) { free(has_parent); return 3; }
    if (level[u] < 0) continue;
    for (int64_t k = off[u]; k < off[u + 1]; ++k) {
      int32_t v = col[k];
      if (level[v] < 0) { free(has_parent); return 4; }
      if ((int64_t)level[v] > (int64_t)level[u] + 1) { free(has_parent); return 5; }
      if ((int64_t)level[v] == (int64_t)level[u] + 1) has_parent[v] = 1;
    }
  }
  for (int64_t v = 0; v < n; ++v) {
    if (level[v] < 0 || v == src) continue;
    if (level[v] == 0 || !has_parent[v]) { free(has_parent); return 6; }
  }
  free(has_parent);
  return 0;
}

/* ===================================================================================== */
/* c2. SSSP — the paper names it only ("Shortest Path (iteratively update neighbors'
 * distances)").  Reading R4: uint32 weights >= 1, distances accumulated in uint64,
 * UINT32_MAX = unreachable, a finite distance >= UINT32_MAX is an overflow (return 5).
 * Plain definition -> Dijkstra with a binary heap (lazy deletion).                           */
typedef struct { uint64_t d; int32_t v; } ora_hitem;

static void ora_heap_push(ora_hitem *h, int64_t *sz, ora_hitem it) {
  int64_t i = (*sz)++;
  h[i] = it;
  while (i > 0) {
    int64_t p = (i - 1) / 2;
    if (h[p].d <= h[i].d) break;
    ora_hitem t = h[p]; h[p] = h[i]; h[i] = t;
    i = p;
  }
}
static ora_hitem ora_heap_pop(ora_hitem *h, int64_t *sz) {
  ora_hitem top = h[0];
  h[0] = h[--(*sz)];
  int64_t i = 0;
  for (;;) {
    int64_t l = 2 * i + 1, r = l + 1, s = i;
    if (l < *sz && h[l].d < h[s].d) s = l;
    if (r < *sz && h[r].d < h[s].d) s = r;
    if (s == i) break;
    ora_hitem t = h[s]; h[s] = h[i]; h[i] = t;
    i = s;
  }
  return top;
}

int ora_sssp(int64_t n, const int64_t *off, const int32_t *col, const uint32_t *w, int32_t src,
             uint32_t *dist_out) {
  if (src < 0 || src >= n) return 1;
  const uint64_t INF = UINT64_MAX;
  uint64_t *d = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)(n > 0 ? n : 1));
  int64_t cap = off[n] + 1;
  ora_hitem *heap = (ora_hitem *)malloc(sizeof(ora_hitem) * (size_t)cap);
  if (!d || !heap) { free(d); free(heap); return 2; }
  for (int64_t v = 0; v < n; ++v) d[v] = INF;
  int64_t sz = 0;
  d[src] = 0;
  ora_heap_push(heap, &sz, (ora_hitem){0, src});
  while (sz > 0) {
    ora_hitem it = ora_heap_pop(heap, &sz);
    if (it.d != d[it.v]) continue;            /* stale entry */
    int32_t u = it.v;
    for (int64_t k = off[u]; k < off[u + 1]; ++k) {
      int32_t v = col[k];
      uint64_t nd = d[u] + (uint64_t)w[k];
      if (nd < d[v]) {
        d[v] = nd;
        ora_heap_push(heap, &sz, (ora_hitem){nd, v});
      }
    }
  }
  int rc = 0;
  for (int64_t v = 0; v < n; ++v) {
    if (d[v] == INF) dist_out[v] = UINT32_MAX;
    else if (d[v] >= (uint64_t)UINT32_MAX) { dist_out[v] = UINT32_MAX; rc = 5; }
    else dist_out[v] = (uint32_t)d[v];
  }
  free(d);
  free(heap);
  return rc;
}

/* SSSP certificate: dist(s)=0; for every arc from a reached u,
 * dist(v) <= dist(u)+w; every reached v != s has dist(v) > 0 and a tight in-arc.            */
int ora_check_sssp(int64_t n, const int64_t *off, const int32_t *col, const uint32_t *w, int32_t src,
                   const uint32_t *dist) {
  if (src < 0 || src >= n) return 1;
  if (dist[src] != 0) return 2;
  uint8_t *tight = (uint8_t *)calloc((size_t)(n > 0 ? n : 1), 1);
  for (int64_t u = 0; u < n; ++u) {
    if (dist[u] == UINT32_MAX) continue;
    for (int64_t k = off[u]; k < off[u + 1]; ++k) {
      int32_t v = col[k];
      uint64_t nd = (uint64_t)dist[u] + w[k];
      if ((uint64_t)dist[v] > nd) { free(tight); return 4; }   /* also catches unreached v */
      if ((uint64_t)dist[v] == nd) tight[v] = 1;
    }
  }
  for (int64_t v = 0; v < n; ++v) {
    if (dist[v] == UINT32_MAX || v == src) continue;
    if (dist[v] == 0 || !tight[v]) { free(tight); return 6; }
  }
  free(tight);
  return 0;
}

/* ===================================================================================== */
/* c3. PageRank — push form of Alg. 1 l.26-29: increment := pr_in[fr]*0.85/outdeg,
 * atomicAdd(pr_out[nb], increment); "global traversal": the frontier is all of V every
 * iteration.  Readings R5-R7 (teleport (1-d)/N, dangling mass spread uniformly,
 * x0 = 1/N, fixed K iterations, fp64):
 *   D   = sum_{out(u)=0} x_u
 *   y_v = sum_{u->v} x_u / out(u)          (source-major push in CSR order)
 *   x_v = (1-d)/N + d*(y_v + D/N)                                                         */
int ora_pagerank(int64_t n, const int64_t *off, const int32_t *col, double d, int32_t iters, double *x) {
  if (n <= 0) return 1;
  double *y = (double *)malloc(sizeof(double) * (size_t)n);
  if (!y) return 2;
  const double N = (double)n;
  for (int64_t v = 0; v < n; ++v) x[v] = 1.0 / N;
  for (int32_t it = 0; it < iters; ++it) {
    double D = 0.0;
    for (int64_t v = 0; v < n; ++v) y[v] = 0.0;
    for (int64_t u = 0; u < n; ++u) {
      int64_t deg = off[u + 1] - off[u];
      if (deg == 0) { D += x[u]; continue; }
      double inc = x[u] / (double)deg;       /* pr_in[fr] / outdegree_cnt[fr] */
      for (int64_t k = off[u]; k < off[u + 1]; ++k) y[col[k]] += inc;
    }
    for (int64_t v = 0; v < n; ++v) x[v] = (1.0 - d) / N + d * (y[v] + D / N);
  }
  free(y);
  return 0;
}

/* One iteration of c3 from a given iterate x (n doubles) -> x_next: the same three lines of the
 * power iteration above (D, y, x update), so that a GPU result at full size can be checked vertex
 * by vertex against x_K = step(x_{K-1}) without re-running the whole serial iteration.          */
int ora_pagerank_step(int64_t n, const int64_t *off, const int32_t *col, double d, const double *x,
                      double *x_next) {
  if (n <= 0) return 1;
  double *y = (double *)calloc((size_t)n, sizeof(double));
  if (!y) return 2;
  const double N = (double)n;
  double D = 0.0;
  for (int64_t u = 0; u < n; ++u) {
    int64_t deg = off[u + 1] - off[u];
    if (deg == 0) { D += x[u]; continue; }
    double inc = x[u] / (double)deg;
    for (int64_t k = off[u]; k < off[u + 1]; ++k) y[col[k]] += inc;
  }
  for (int64_t v = 0; v < n; ++v) x_next[v] = (1.0 - d) / N + d * (y[v] + D / N);
  free(y);
  return 0;
}

/* ===================================================================================== */
/* BC — Alg. 1 l.8-24: forward BFS that counts shortest paths
 * (l.8-17: dist[nb] := dist[fr]+1 on first visit; sigma[nb] += sigma[fr] when dist[nb] =
 * dist[fr]+1) and backward dependency accumulation by decreasing level (l.19-24: delta[fr] +=
 * sigma[fr]/sigma[nb] * (delta[nb] + 1) for every arc fr->nb with dist[nb] = dist[fr]+1).
 * This is Brandes' algorithm; the oracle writes it out plainly (FIFO BFS, then the BFS order
 * reversed).  sigma and delta are fp64.  For every source s in `sources`, bc[v] += delta_s(v)
 * for v != s (delta_s(s) is not added).  Unreachable vertices get 0.                          */
int ora_bc(int64_t n, const int64_t *off, const int32_t *col, const int32_t *sources, int64_t ns,
           double *bc) {
  int32_t *dist = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  int32_t *order = (int32_t *)malloc(sizeof(int32_t) * (size_t)(n > 0 ? n : 1));
  double *sigma = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  double *delta = (double *)malloc(sizeof(double) * (size_t)(n > 0 ? n : 1));
  if (!dist || !order || !sigma || !delta) { free(dist); free(order); free(sigma); free(delta); return 2; }
  for (int64_t v = 0; v < n; ++v) bc[v] = 0.0;
  for (int64_t k = 0; k < ns; ++k) {
    const int32_t s = sources[k];
    if (s < 0 || s >= n) { free(dist); free(order); free(sigma); free(delta); return 1; }
    for (int64_t v = 0; v < n; ++v) { dist[v] = -1; sigma[v] = 0.0; delta[v] = 0.0; }
    int64_t head = 0, tail = 0;
    dist[s] = 0;
    sigma[s] = 1.0;
    order[tail++] = s;
    while (head < tail) {                         /* forward: Alg. 1 l.8-17 */
      const int32_t u = order[head++];
      for (int64_t e = off[u]; e < off[u + 1]; ++e) {
        const int32_t v = col[e];
        if (dist[v] == -1) { dist[v] = dist[u] + 1; order[tail++] = v; }
        if (dist[v] == dist[u] + 1) sigma[v] += sigma[u];
      }
    }
    for (int64_t i = tail - 1; i >= 0; --i) {     /* backward: Alg. 1 l.19-24 */
      const int32_t u = order[i];
      for (int64_t e = off[u]; e < off[u + 1]; ++e) {
        const int32_t v = col[e];
        if (dist[v] == dist[u] + 1) delta[u] += sigma[u] / sigma[v] * (delta[v] + 1.0);
      }
      if (u != s) bc[u] += delta[u];
    }
  }
  free(dist); free(order); free(sigma); free(delta);
  return 0;
}

/* ===================================================================================== */
/* c4. Tiled Partitioning of one row [b, e) — Alg. 2 as the resident tile log of
 * Alg. 3 l.2-7.  The block-sized tile consumes full tile-size chunks of the row
 * (Alg. 2 l.9-25; the leader keeps neighbor_size mod tile.size() at the row END, l.14-16),
 * then the tile is halved ("binary partition") down to MIN_TILE_SIZE (l.8, l.28); what
 * is left (< MIN) is the fragment (l.32).  Reading R14: with alignment A > 0 a head fragment
 * [b, b+h) first brings the row start to a multiple of A (tile alignment).
 * Writes triples (offset, size, kind) with kind 0 = tile, 1 = fragment; returns the count.   */
int64_t ora_tiles_row(int64_t b, int64_t e, int32_t B, int32_t M, int32_t A, int64_t *triples) {
  int64_t k = 0;
  if (A > 0) {
    int64_t h = (A - (b % A)) % A;
    if (h > e - b) h = e - b;
    if (h > 0) { triples[3*k] = b; triples[3*k+1] = h; triples[3*k+2] = 1; ++k; }
    b += h;
  }
  int64_t q = (e - b) / B;
  for (int64_t j = 0; j < q; ++j) { triples[3*k] = b + j * B; triples[3*k+1] = B; triples[3*k+2] = 0; ++k; }
  int64_t r = e - b - q * B;
  for (int64_t t = B / 2; t >= M; t /= 2) {
    if (r >= t) { triples[3*k] = e - r; triples[3*k+1] = t; triples[3*k+2] = 0; ++k; r -= t; }
  }
  if (r > 0) { triples[3*k] = e - r; triples[3*k+1] = r; triples[3*k+2] = 1; ++k; }
  return k;
}

/* Tile log of a vertex list: (vertex, offset, size, kind) quadruples; returns the count.   */
int64_t ora_tile_log(const int64_t *off, const int32_t *vertices, int64_t count, int32_t B, int32_t M,
                     int32_t A, int64_t *quads) {
  int64_t maxdeg = 0;
  for (int64_t i = 0; i < count; ++i)
    if (off[vertices[i] + 1] - off[vertices[i]] > maxdeg) maxdeg = off[vertices[i] + 1] - off[vertices[i]];
  int64_t *tmp = (int64_t *)malloc(sizeof(int64_t) * 3 * (size_t)(maxdeg / B + 72));
  int64_t k = 0;
  for (int64_t i = 0; i < count; ++i) {
    int32_t u = vertices[i];
    int64_t c = ora_tiles_row(off[u], off[u + 1], B, M, A, tmp);
    for (int64_t j = 0; j < c; ++j) {
      quads[4*k] = u; quads[4*k+1] = tmp[3*j]; quads[4*k+2] = tmp[3*j+1]; quads[4*k+3] = tmp[3*j+2];
      ++k;
    }
  }
  free(tmp);
  return k;
}

/* ===================================================================================== */
/* Objective of §6: sum over sampled tiles of count(distinct(floor(sigma(nbrs)/S))).
 * Tiles = every tile (not fragment) of every vertex under c4 with the current labels (R19/R20). */
static int cmp_i64(const void *a, const void *b) {
  int64_t x = *(const int64_t *)a, y = *(const int64_t *)b;
  return (x > y) - (x < y);
}

int64_t ora_objective_tiles(int64_t ntiles, const int64_t *tile_ptr, const int32_t *members, int32_t S) {
  int64_t total = 0;
  int64_t maxlen = 0;
  for (int64_t t = 0; t < ntiles; ++t)
    if (tile_ptr[t + 1] - tile_ptr[t] > maxlen) maxlen = tile_ptr[t + 1] - tile_ptr[t];
  int64_t *sec = (int64_t *)malloc(sizeof(int64_t) * (size_t)(maxlen > 0 ? maxlen : 1));
  for (int64_t t = 0; t < ntiles; ++t) {
    int64_t len = tile_ptr[t + 1] - tile_ptr[t];
    for (int64_t i = 0; i < len; ++i) sec[i] = members[tile_ptr[t] + i] / S;
    qsort(sec, (size_t)len, sizeof(int64_t), cmp_i64);
    for (int64_t i = 0; i < len; ++i)
      if (i == 0 || sec[i] != sec[i - 1]) ++total;
  }
  free(sec);
  return total;
}

/* The tile sample of a CSR (R19/R20): tile_ptr[ntiles+1] and members[] = the col entries of every
 * tile (kind 0) of every vertex.  Two-call protocol: with tile_ptr == NULL returns ntiles and
 * stores the member count in *nmembers.                                                     */
int64_t ora_sample_tiles(int64_t n, const int64_t *off, const int32_t *col, int32_t B, int32_t M, int32_t A,
                         int64_t *tile_ptr, int32_t *members, int64_t *nmembers) {
  int64_t maxdeg = 0;
  for (int64_t u = 0; u < n; ++u) if (off[u + 1] - off[u] > maxdeg) maxdeg = off[u + 1] - off[u];
  int64_t *tmp = (int64_t *)malloc(sizeof(int64_t) * 3 * (size_t)(maxdeg / B + 72));
  int64_t nt = 0, nm = 0;
  if (tile_ptr) tile_ptr[0] = 0;
  for (int64_t u = 0; u < n; ++u) {
    int64_t c = ora_tiles_row(off[u], off[u + 1], B, M, A, tmp);
    for (int64_t j = 0; j < c; ++j) {
      if (tmp[3*j+2] != 0) continue;
      if (tile_ptr) {
        for (int64_t i = 0; i < tmp[3*j+1]; ++i) members[nm + i] = col[tmp[3*j] + i];
        tile_ptr[nt + 1] = nm + tmp[3*j+1];
      }
      nm += tmp[3*j+1];
      ++nt;
    }
  }
  if (nmembers) *nmembers = nm;
  free(tmp);
  return nt;
}

/* ===================================================================================== */
/* c5. Sampling-based Reordering, one round's three stages (§6; Alg. 4 P:325-354;
 * Figure 5), following the readings:
 *   sec(x) = floor(x / S); for an occurrence of v in tile T its mates are T \ {v}.
 *   Stage 1 (R18): loc1[v] = sum_T |{w in mates : sec(w) = sec(v)}|.
 *   Stage 2 (R21): [lo,hi) = [0, ceil(n/S)) in sectors; while hi-lo > 1:
 *            mid = lo + (hi-lo)/2; L = sum_T |{w : lo <= sec(w) < mid}|,
 *            R = sum_T |{w : mid <= sec(w) < hi}|; L >= R -> hi = mid else lo = mid.
 *            target[v] = lo.
 *   Stage 3 (R22): loc3[v] = sum_T |{w in mates : sec(w) = target[v]}|;
 *            v is a mover iff loc3 > loc1 (and v is a candidate, if a candidate list is given).
 * Each count is taken the plain way: a loop over the occurrence's tile mates.
 * Outputs per vertex: loc1, target, loc3, mover (0/1).                                       */
void ora_reorder_stages(int64_t n, int64_t ntiles, const int64_t *tile_ptr, const int32_t *members,
                        int32_t S, const uint8_t *candidate /* NULL = all */, int64_t *loc1,
                        int64_t *target, int64_t *loc3, uint8_t *mover,
                        int32_t trace_v /* -1 = none */, int64_t *trace_lr /* 4 per step: lo,hi,L,R */,
                        int32_t *trace_steps) {
  const int64_t nsec = (n + S - 1) / S;
  if (trace_steps) *trace_steps = 0;
  int64_t *lo = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  int64_t *hi = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  int64_t *cl = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  int64_t *cr = (int64_t *)malloc(sizeof(int64_t) * (size_t)n);
  /* Stage 1 */
  for (int64_t v = 0; v < n; ++v) loc1[v] = 0;
  for (int64_t t = 0; t < ntiles; ++t)
    for (int64_t i = tile_ptr[t]; i < tile_ptr[t + 1]; ++i) {
      int32_t v = members[i];
      for (int64_t j = tile_ptr[t]; j < tile_ptr[t + 1]; ++j)
        if (j != i && members[j] / S == v / S) loc1[v]++;
    }
  /* Stage 2: binary search, one halving step per sampling sweep */
  for (int64_t v = 0; v < n; ++v) { lo[v] = 0; hi[v] = nsec; }
  for (;;) {
    int any = 0;
    for (int64_t v = 0; v < n; ++v) { cl[v] = 0; cr[v] = 0; if (hi[v] - lo[v] > 1) any = 1; }
    if (!any) break;
    for (int64_t t = 0; t < ntiles; ++t)
      for (int64_t i = tile_ptr[t]; i < tile_ptr[t + 1]; ++i) {
        int32_t v = members[i];
        if (hi[v] - lo[v] <= 1) continue;
        int64_t mid = lo[v] + (hi[v] - lo[v]) / 2;
        for (int64_t j = tile_ptr[t]; j < tile_ptr[t + 1]; ++j) {
          if (j == i) continue;
          int64_t s = members[j] / S;
          if (s >= lo[v] && s < mid) cl[v]++;
          else if (s >= mid && s < hi[v]) cr[v]++;
        }
      }
    if (trace_v >= 0 && trace_v < n && hi[trace_v] - lo[trace_v] > 1 && trace_lr && trace_steps) {
      int32_t k = (*trace_steps)++;
      trace_lr[4*k] = lo[trace_v]; trace_lr[4*k+1] = hi[trace_v];
      trace_lr[4*k+2] = cl[trace_v]; trace_lr[4*k+3] = cr[trace_v];
    }
    for (int64_t v = 0; v < n; ++v) {
      if (hi[v] - lo[v] <= 1) continue;
      int64_t mid = lo[v] + (hi[v] - lo[v]) / 2;
      if (cl[v] >= cr[v]) hi[v] = mid; else lo[v] = mid;
    }
  }
  for (int64_t v = 0; v < n; ++v) target[v] = lo[v];
  /* Stage 3 */
  for (int64_t v = 0; v < n; ++v) loc3[v] = 0;
  for (int64_t t = 0; t < ntiles; ++t)
    for (int64_t i = tile_ptr[t]; i < tile_ptr[t + 1]; ++i) {
      int32_t v = members[i];
      for (int64_t j = tile_ptr[t]; j < tile_ptr[t + 1]; ++j)
        if (j != i && members[j] / S == target[v]) loc3[v]++;
    }
  for (int64_t v = 0; v < n; ++v)
    mover[v] = (uint8_t)((candidate == NULL || candidate[v]) && loc3[v] > loc1[v]);
  free(lo); free(hi); free(cl); free(cr);
}

/* Swap matching (reading R23, pinned by Figure 5's 8<->3): for every sector s,
 *   I = movers with target s, sorted by (gain = loc3-loc1 descending, id ascending);
 *   V = non-movers whose current sector is s, sorted by (loc1 ascending, id ascending);
 *   pair I[k] with V[k] while gain(I[k]) > loc1(V[k]) and swap their labels.
 * Writes sigma_round (new label of each current label, a bijection); returns #swaps.
 * Implemented as plain per-sector selection (O(n * sector size)), no sort library.          */
int64_t ora_reorder_match(int64_t n, int32_t S, const int64_t *loc1, const int64_t *target,
                          const int64_t *loc3, const uint8_t *mover, int32_t *sigma_round) {
  const int64_t nsec = (n + S - 1) / S;
  for (int64_t v = 0; v < n; ++v) sigma_round[v] = (int32_t)v;
  /* bucket movers by target sector (counting sort by sector, ids ascending inside) */
  int64_t *cnt = (int64_t *)calloc((size_t)nsec + 1, sizeof(int64_t));
  int64_t nmov = 0;
  for (int64_t v = 0; v < n; ++v) if (mover[v]) { cnt[target[v] + 1]++; ++nmov; }
  for (int64_t s = 0; s < nsec; ++s) cnt[s + 1] += cnt[s];
  int64_t *bucket = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nmov > 0 ? nmov : 1));
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * (size_t)nsec);
  for (int64_t s = 0; s < nsec; ++s) fill[s] = cnt[s];
  for (int64_t v = 0; v < n; ++v) if (mover[v]) bucket[fill[target[v]]++] = v;
  int64_t swaps = 0;
  int64_t *vic = (int64_t *)malloc(sizeof(int64_t) * (size_t)S);
  for (int64_t s = 0; s < nsec; ++s) {
    int64_t nb = cnt[s + 1] - cnt[s];
    if (nb == 0) continue;
    int64_t *I = bucket + cnt[s];
    /* insertion sort of I by (gain desc, id asc) */
    for (int64_t a = 1; a < nb; ++a) {
      int64_t x = I[a], gx = loc3[x] - loc1[x];
      int64_t b = a - 1;
      while (b >= 0) {
        int64_t y = I[b], gy = loc3[y] - loc1[y];
        if (gy > gx || (gy == gx && y < x)) break;
        I[b + 1] = I[b];
        --b;
      }
      I[b + 1] = x;
    }
    /* victims: non-movers in sector s, by (loc1 asc, id asc) */
    int64_t nv = 0;
    for (int64_t v = s * S; v < (s + 1) * S && v < n; ++v) if (!mover[v]) vic[nv++] = v;
    for (int64_t a = 1; a < nv; ++a) {
      int64_t x = vic[a];
      int64_t b = a - 1;
      while (b >= 0 && (loc1[vic[b]] > loc1[x] || (loc1[vic[b]] == loc1[x] && vic[b] > x))) {
        vic[b + 1] = vic[b];
        --b;
      }
      vic[b + 1] = x;
    }
    for (int64_t k = 0; k < nb && k < nv; ++k) {
      int64_t a = I[k], b = vic[k];
      if (!(loc3[a] - loc1[a] > loc1[b])) break;
      sigma_round[a] = (int32_t)b;
      sigma_round[b] = (int32_t)a;
      ++swaps;
    }
  }
  free(cnt); free(bucket); free(fill); free(vic);
  return swaps;
}

/* Relabel (R24): the row of sigma(v) is sort(sigma(adj v)); weights move with their arcs.
 * off_out[n+1], col_out[m], w_out[m] (w/w_out may be NULL).                                  */
typedef struct { int32_t c; uint32_t w; } ora_arc;
static int cmp_arc(const void *a, const void *b) {
  int32_t x = ((const ora_arc *)a)->c, y = ((const ora_arc *)b)->c;
  return (x > y) - (x < y);
}
void ora_relabel(int64_t n, const int64_t *off, const int32_t *col, const uint32_t *w,
                 const int32_t *sigma, int64_t *off_out, int32_t *col_out, uint32_t *w_out) {
  int32_t *inv = (int32_t *)malloc(sizeof(int32_t) * (size_t)n);
  for (int64_t v = 0; v < n; ++v) inv[sigma[v]] = (int32_t)v;
  off_out[0] = 0;
  for (int64_t nv = 0; nv < n; ++nv) {
    int32_t v = inv[nv];
    off_out[nv + 1] = off_out[nv] + (off[v + 1] - off[v]);
  }
  int64_t maxdeg = 0;
  for (int64_t v = 0; v < n; ++v) if (off[v + 1] - off[v] > maxdeg) maxdeg = off[v + 1] - off[v];
  ora_arc *tmp = (ora_arc *)malloc(sizeof(ora_arc) * (size_t)(maxdeg > 0 ? maxdeg : 1));
  for (int64_t nv = 0; nv < n; ++nv) {
    int32_t v = inv[nv];
    int64_t d = off[v + 1] - off[v];
    for (int64_t k = 0; k < d; ++k) {
      tmp[k].c = sigma[col[off[v] + k]];
      tmp[k].w = w ? w[off[v] + k] : 0u;
    }
    qsort(tmp, (size_t)d, sizeof(ora_arc), cmp_arc);
    for (int64_t k = 0; k < d; ++k) {
      col_out[off_out[nv] + k] = tmp[k].c;
      if (w_out) w_out[off_out[nv] + k] = tmp[k].w;
    }
  }
  free(tmp);
  free(inv);
}
