// sagegen.cpp — seeded synthetic graph generators (TEST / BENCH INFRASTRUCTURE).
//
// This module only produces INPUTS: CSR graphs, weights and source vertices.
// It holds none of SAGE's arithmetic (no traversal, no tiling, no reordering),
// so both the oracle (oracle/) and the CUDA path (paper_conf_sigmod_00020t21_b200/)
// may consume its output.  Everything is a pure function of (parameters, seed):
// a counter-based splitmix64 hash keyed by (seed, tuple index, level group) is the
// only randomness, so the output is identical for any OpenMP thread count.
//
// Graph shapes follow SURVEY.md §8(d):
//   * Graph500 Kronecker/RMAT (A,B,C,D = .57,.19,.19,.05), edgefactor tuples per vertex,
//     IDs scrambled by a seeded bijection, self-loops and duplicate arcs removed, rows
//     sorted; optionally symmetrised (both directions stored).
//   * "twitter-like": Chung-Lu Zipf sources + planted communities (directed).
//   * "uk-like": host blocks in crawl order + tendril chains (directed, high diameter).
//
// Build: g++ -O3 -fopenmp -shared -fPIC sagegen.cpp -o libsagegen.so
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <omp.h>

extern "C" {

static inline uint64_t sg_mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
// Counter-based hash of (seed, a, b).
static inline uint64_t sg_hash3(uint64_t seed, uint64_t a, uint64_t b) {
  return sg_mix64(sg_mix64(seed ^ sg_mix64(a + 0x632BE59BD9B4E019ull)) + b);
}
uint64_t sg_hash(uint64_t seed, uint64_t a, uint64_t b) { return sg_hash3(seed, a, b); }

// ---------------------------------------------------------------------------
// Seeded bijection on [0, 2^bits): odd multiplies and xor-shifts mod 2^bits.
static inline uint64_t sg_perm_pow2(uint64_t x, int bits, uint64_t seed) {
  if (bits <= 0) return 0;
  const uint64_t mask = (bits >= 64) ? ~0ull : ((1ull << bits) - 1);
  const uint64_t k1 = sg_mix64(seed ^ 0x1111) | 1ull, k2 = sg_mix64(seed ^ 0x2222) | 1ull;
  const uint64_t c1 = sg_mix64(seed ^ 0x3333);
  const int s1 = bits / 2 + 1, s2 = bits / 3 + 1;
  x = (x * k1) & mask;
  x ^= (x >> s1);
  x = (x * k2 + c1) & mask;
  x ^= (x >> s2);
  x = (x * k1) & mask;
  return x & mask;
}
// Bijection on [0, n) by cycle-walking the power-of-two permutation.
static inline uint64_t sg_perm(uint64_t x, uint64_t n, uint64_t seed) {
  int bits = 0;
  while ((1ull << bits) < n) ++bits;
  do { x = sg_perm_pow2(x, bits, seed); } while (x >= n);
  return x;
}
uint64_t sg_permute(uint64_t x, uint64_t n, uint64_t seed) { return sg_perm(x, n, seed); }

// ---------------------------------------------------------------------------
// CSR construction from a tuple list: counting sort by source, per-row sort,
// removal of self loops and duplicates.  Output arrays are malloc'ed and handed
// to the caller (free with sg_free).
struct sg_csr_out {
  int64_t n, m;
  int64_t *off;
  int32_t *col;
};

static void sg_build_csr(int64_t n, int64_t t, const int32_t *src, const int32_t *dst, int symmetric,
                         sg_csr_out *out) {
  std::vector<std::atomic<int64_t>> cnt(n + 1);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i <= n; ++i) cnt[i].store(0, std::memory_order_relaxed);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < t; ++i) {
    int32_t u = src[i], v = dst[i];
    if (u == v) continue;
    cnt[u].fetch_add(1, std::memory_order_relaxed);
    if (symmetric) cnt[v].fetch_add(1, std::memory_order_relaxed);
  }
  int64_t *off0 = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
  off0[0] = 0;
  for (int64_t i = 0; i < n; ++i) off0[i + 1] = off0[i] + cnt[i].load(std::memory_order_relaxed);
  const int64_t m0 = off0[n];
  int32_t *col0 = (int32_t *)malloc(sizeof(int32_t) * (m0 > 0 ? m0 : 1));
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < n; ++i) cnt[i].store(off0[i], std::memory_order_relaxed);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < t; ++i) {
    int32_t u = src[i], v = dst[i];
    if (u == v) continue;
    col0[cnt[u].fetch_add(1, std::memory_order_relaxed)] = v;
    if (symmetric) col0[cnt[v].fetch_add(1, std::memory_order_relaxed)] = u;
  }
  // sort + dedupe each row in place; record new degrees
  std::vector<int64_t> deg(n);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; ++u) {
    int32_t *b = col0 + off0[u], *e = col0 + off0[u + 1];
    std::sort(b, e);
    deg[u] = std::unique(b, e) - b;
  }
  int64_t *off = (int64_t *)malloc(sizeof(int64_t) * (n + 1));
  off[0] = 0;
  for (int64_t i = 0; i < n; ++i) off[i + 1] = off[i] + deg[i];
  const int64_t m = off[n];
  int32_t *col = (int32_t *)malloc(sizeof(int32_t) * (m > 0 ? m : 1));
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; ++u) memcpy(col + off[u], col0 + off0[u], sizeof(int32_t) * deg[u]);
  free(col0);
  free(off0);
  out->n = n;
  out->m = m;
  out->off = off;
  out->col = col;
}

void sg_free(void *p) { free(p); }

int sg_csr_from_tuples(int64_t n, int64_t t, const int32_t *src, const int32_t *dst, int symmetric,
                       sg_csr_out *out) {
  for (int64_t i = 0; i < t; ++i)
    if (src[i] < 0 || src[i] >= n || dst[i] < 0 || dst[i] >= n) return 1;
  sg_build_csr(n, t, src, dst, symmetric, out);
  return 0;
}

// ---------------------------------------------------------------------------
// Graph500 Kronecker / RMAT.  Tuple i draws, for each of `scale` levels, a
// quadrant with probabilities (A, B, C, 1-A-B-C) from 16 bits of sg_hash3(seed, i, group).
int sg_rmat(int scale, int edgefactor, uint64_t seed, double A, double B, double C, int symmetric,
            int scramble, sg_csr_out *out) {
  if (scale < 1 || scale > 30) return 1;
  const int64_t n = 1ll << scale;
  const int64_t t = (int64_t)edgefactor * n;
  int32_t *src = (int32_t *)malloc(sizeof(int32_t) * t);
  int32_t *dst = (int32_t *)malloc(sizeof(int32_t) * t);
  const uint32_t tA = (uint32_t)llround(A * 65536.0), tAB = (uint32_t)llround((A + B) * 65536.0),
                 tABC = (uint32_t)llround((A + B + C) * 65536.0);
  const uint64_t pseed = sg_mix64(seed ^ 0xABCDEF12345ull);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < t; ++i) {
    uint64_t u = 0, v = 0;
    for (int g = 0; g * 4 < scale; ++g) {
      uint64_t r = sg_hash3(seed, (uint64_t)i, (uint64_t)g);
      for (int j = 0; j < 4 && g * 4 + j < scale; ++j) {
        uint32_t q = (uint32_t)((r >> (16 * j)) & 0xFFFF);
        int l = g * 4 + j;
        uint64_t ub = (q >= tAB) ? 1 : 0;             // C or D quadrant: row bit
        uint64_t vb = ((q >= tA && q < tAB) || q >= tABC) ? 1 : 0;  // B or D: column bit
        u |= ub << l;
        v |= vb << l;
      }
    }
    if (scramble) {
      u = sg_perm_pow2(u, scale, pseed);
      v = sg_perm_pow2(v, scale, pseed);
    }
    src[i] = (int32_t)u;
    dst[i] = (int32_t)v;
  }
  sg_build_csr(n, t, src, dst, symmetric, out);
  free(src);
  free(dst);
  return 0;
}

// ---------------------------------------------------------------------------
// Zipf-like sampler: inverse-CDF of a continuous power law on [1, n] mapped to a rank,
// then a seeded bijection turns the rank into a vertex ID (so hubs are scattered).
static inline double sg_unit(uint64_t h) { return ((h >> 11) + 0.5) * (1.0 / 9007199254740992.0); }
static inline int64_t sg_zipf_rank(double u, double s, int64_t n) {
  // density ∝ x^-s on [1, n+1); s != 1
  double a = 1.0 - s;
  double lo = 1.0, hi = std::pow((double)n + 1.0, a);
  double x = std::pow(lo + u * (hi - lo), 1.0 / a);
  int64_t r = (int64_t)x - 1;
  if (r < 0) r = 0;
  if (r >= n) r = n - 1;
  return r;
}

// Twitter-like directed graph (proposed parameters).
//   sources: Chung-Lu with out-weight ∝ rank^-s_out   (hubs of "several million" out-degree)
//   targets: with prob mu inside the source's planted community, else Zipf(s_in) over all
//   communities: contiguous rank blocks with sizes ∝ s^-2 on [cmin, cmax]
//   final seeded ID scramble, so the input order carries no locality.
int sg_twitter_like(int64_t n, int64_t tuples, uint64_t seed, double s_out, double s_in, double mu,
                    int64_t cmin, int64_t cmax, sg_csr_out *out) {
  if (n < 2 || n >= (1ll << 31)) return 1;
  // community boundaries over rank space
  std::vector<int64_t> cstart;
  {
    int64_t pos = 0, k = 0;
    while (pos < n) {
      double u = sg_unit(sg_hash3(seed ^ 0xC0FFEE, (uint64_t)k++, 7));
      // size ∝ s^-2 on [cmin, cmax]  (inverse CDF)
      double a = 1.0 / cmin, b = 1.0 / cmax;
      int64_t sz = (int64_t)(1.0 / (a - u * (a - b)));
      if (sz < cmin) sz = cmin;
      cstart.push_back(pos);
      pos += sz;
    }
    cstart.push_back(n);
  }
  const int64_t ncomm = (int64_t)cstart.size() - 1;
  // community of every rank
  std::vector<int32_t> comm_of(n);
#pragma omp parallel for schedule(static)
  for (int64_t c = 0; c < ncomm; ++c)
    for (int64_t r = cstart[c]; r < cstart[c + 1]; ++r) comm_of[r] = (int32_t)c;
  const uint64_t pseed_src = sg_mix64(seed ^ 0x51), pseed_dst = sg_mix64(seed ^ 0x52),
                 pseed_fin = sg_mix64(seed ^ 0x53);
  int32_t *src = (int32_t *)malloc(sizeof(int32_t) * tuples);
  int32_t *dst = (int32_t *)malloc(sizeof(int32_t) * tuples);
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < tuples; ++i) {
    uint64_t h0 = sg_hash3(seed, (uint64_t)i, 0), h1 = sg_hash3(seed, (uint64_t)i, 1),
             h2 = sg_hash3(seed, (uint64_t)i, 2);
    int64_t su = (int64_t)sg_perm((uint64_t)sg_zipf_rank(sg_unit(h0), s_out, n), n, pseed_src);
    int64_t c = comm_of[su];
    int64_t v;
    if (sg_unit(h1) < mu) {
      int64_t lo = cstart[c], sz = cstart[c + 1] - cstart[c];
      v = lo + (int64_t)(h2 % (uint64_t)sz);
    } else {
      v = (int64_t)sg_perm((uint64_t)sg_zipf_rank(sg_unit(h2), s_in, n), n, pseed_dst);
    }
    src[i] = (int32_t)sg_perm((uint64_t)su, n, pseed_fin);
    dst[i] = (int32_t)sg_perm((uint64_t)v, n, pseed_fin);
  }
  sg_build_csr(n, tuples, src, dst, 0, out);
  free(src);
  free(dst);
  return 0;
}

// UK-2007-like directed web graph (proposed parameters), natural crawl order.
//   hosts: contiguous ID blocks, sizes ∝ s^-1.8 on [1, hmax]
//   out-degree: lognormal(mu_ln, sigma_ln) capped at dmax
//   targets: with prob p_local inside the host at a geometric offset (mean `goff`), else a
//            Zipf(s_glob) rank over a scrambled global order
//   tendrils: n_tendrils chains of length U[tmin, tmax] hung off random vertices, giving
//             hundreds of BFS levels ("high diameter").  Tendril vertices are the last IDs.
int sg_uk_like(int64_t n, uint64_t seed, double mu_ln, double sigma_ln, int64_t dmax, int64_t hmax,
               double p_local, double goff, double s_glob, int64_t n_tendrils, int64_t tmin,
               int64_t tmax, sg_csr_out *out) {
  if (n < 16 || n >= (1ll << 31)) return 1;
  // tendril lengths
  std::vector<int64_t> tlen(n_tendrils);
  int64_t tend_total = 0;
  for (int64_t k = 0; k < n_tendrils; ++k) {
    tlen[k] = tmin + (int64_t)(sg_hash3(seed ^ 0x7E4D, (uint64_t)k, 0) % (uint64_t)(tmax - tmin + 1));
    tend_total += tlen[k];
  }
  if (tend_total >= n / 2) return 1;
  const int64_t nc = n - tend_total;  // core vertices [0, nc)
  // hosts
  std::vector<int64_t> hstart;
  {
    int64_t pos = 0, k = 0;
    const double s = 1.8, a = 1.0 - s;
    while (pos < nc) {
      double u = sg_unit(sg_hash3(seed ^ 0x4057, (uint64_t)k++, 3));
      double x = std::pow(1.0 + u * (std::pow((double)hmax + 1.0, a) - 1.0), 1.0 / a);
      int64_t sz = (int64_t)x;
      if (sz < 1) sz = 1;
      hstart.push_back(pos);
      pos += sz;
    }
    hstart.push_back(nc);
  }
  const int64_t nh = (int64_t)hstart.size() - 1;
  std::vector<int32_t> host_of(nc);
#pragma omp parallel for schedule(static)
  for (int64_t h = 0; h < nh; ++h)
    for (int64_t r = hstart[h]; r < hstart[h + 1] && r < nc; ++r) host_of[r] = (int32_t)h;
  // out-degrees of core vertices
  std::vector<int64_t> odeg(nc + 1);
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < nc; ++v) {
    double u1 = sg_unit(sg_hash3(seed, (uint64_t)v, 11)), u2 = sg_unit(sg_hash3(seed, (uint64_t)v, 12));
    double z = std::sqrt(-2.0 * std::log(u1)) * std::cos(6.283185307179586 * u2);
    double d = std::exp(mu_ln + sigma_ln * z);
    int64_t di = (int64_t)d;
    if (di > dmax) di = dmax;
    odeg[v] = di;
  }
  std::vector<int64_t> tpos(nc + 1);
  tpos[0] = 0;
  for (int64_t v = 0; v < nc; ++v) tpos[v + 1] = tpos[v] + odeg[v];
  const int64_t tcore = tpos[nc];
  const int64_t t = tcore + tend_total;  // each tendril vertex has one in-arc (chain)
  int32_t *src = (int32_t *)malloc(sizeof(int32_t) * t);
  int32_t *dst = (int32_t *)malloc(sizeof(int32_t) * t);
  const uint64_t gseed = sg_mix64(seed ^ 0x6106);
  const double pgeo = 1.0 / goff;
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t v = 0; v < nc; ++v) {
    int64_t h = host_of[v], hb = hstart[h], he = hstart[h + 1], hs = he - hb;
    for (int64_t j = 0; j < odeg[v]; ++j) {
      int64_t idx = tpos[v] + j;
      uint64_t r1 = sg_hash3(seed, (uint64_t)idx, 21), r2 = sg_hash3(seed, (uint64_t)idx, 22);
      int64_t w;
      if (hs > 1 && sg_unit(r1) < p_local) {
        // geometric offset with mean goff, random sign, wrapped inside the host
        int64_t off = 1 + (int64_t)(std::log(sg_unit(r2)) / std::log(1.0 - pgeo));
        if ((r1 >> 60) & 1) off = -off;
        int64_t rel = ((v - hb + off) % hs + hs) % hs;
        w = hb + rel;
      } else {
        w = (int64_t)sg_perm((uint64_t)sg_zipf_rank(sg_unit(r2), s_glob, nc), (uint64_t)nc, gseed);
      }
      src[idx] = (int32_t)v;
      dst[idx] = (int32_t)w;
    }
  }
  // tendril chains: anchor (random core vertex) -> t0 -> t1 -> ...
  int64_t base = nc, idx = tcore;
  for (int64_t k = 0; k < n_tendrils; ++k) {
    int64_t anchor = (int64_t)(sg_hash3(seed ^ 0x7E4D, (uint64_t)k, 1) % (uint64_t)nc);
    int64_t prev = anchor;
    for (int64_t j = 0; j < tlen[k]; ++j) {
      src[idx] = (int32_t)prev;
      dst[idx] = (int32_t)(base + j);
      prev = base + j;
      ++idx;
    }
    base += tlen[k];
  }
  sg_build_csr(n, t, src, dst, 0, out);
  free(src);
  free(dst);
  return 0;
}

// Symmetric integer weights w(u,v) = 1 + hash(seed, min(u,v), max(u,v)) mod wmax  (in [1, wmax]).
void sg_weights(int64_t n, const int64_t *off, const int32_t *col, uint64_t seed, uint32_t wmax,
                uint32_t *w) {
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t u = 0; u < n; ++u)
    for (int64_t k = off[u]; k < off[u + 1]; ++k) {
      uint64_t a = (uint64_t)u, b = (uint64_t)col[k];
      if (a > b) std::swap(a, b);
      w[k] = 1u + (uint32_t)(sg_hash3(seed, a, b) % wmax);
    }
}

// `k` sources drawn uniformly (with replacement) among vertices with out-degree > 0.
int sg_sources(int64_t n, const int64_t *off, uint64_t seed, int32_t k, int32_t *out) {
  int64_t tries = 0;
  for (int32_t i = 0; i < k; ++i) {
    for (uint64_t j = 0;; ++j) {
      uint64_t v = sg_hash3(seed, (uint64_t)i, j) % (uint64_t)n;
      if (off[v + 1] > off[v]) {
        out[i] = (int32_t)v;
        break;
      }
      if (++tries > 100000000) return 1;
    }
  }
  return 0;
}

int sg_num_threads(void) { return omp_get_max_threads(); }

}  // extern "C"
