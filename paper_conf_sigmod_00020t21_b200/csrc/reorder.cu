// reorder.cu — Sampling-based Reordering (§6; Alg. 4; Figure 5) on
// the GPU, one round = the paper's three stages over a tile sample, then the relabel.
//
// Readings (the same ones the oracle follows):
//   sample (R19/R20): every TILE (not fragment) of every vertex under the graph's ladder — the
//     all-V resident tile log (the same log PageRank reuses) — with the current labels.
//   sec(x) = x / S.  For an occurrence of v in tile T its mates are T \ {v}.
//   stage 1 (R18): loc1[v] = sum_T |{w in mates : sec(w) = sec(v)}|.
//   stage 2 (R21): [lo, hi) = [0, ceil(n/S)); ceil(log2) halving steps, each a full
//     sweep of the sample: L / R = mates in [lo, mid) / [mid, hi); L >= R -> hi = mid, else lo.
//   stage 3 (R22): loc3[v] = mates in sector target[v]; mover iff loc3 > loc1.
//   match (R23): per sector s, movers targeting s by (gain desc, id asc) are paired with the
//     non-movers of s by (loc1 asc, id asc) while gain > loc1(victim); pairs swap labels.
//   relabel (R24): row of sigma(v) = sort(sigma(adj v)), weights moved with their arcs.
// Tile-access sampling (Alg. 4) is done per tile in shared memory: the tile is staged in smem,
// sorted (bitonic) unless the rows are already sorted, and every count is two binary searches —
// O(t log t) per tile instead of Alg. 4's O(t^2) pairwise compares.
// Every count is an exact integer, so the result is independent of atomic order and equals the
// oracle's permutation exactly.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>
#include <cub/device/device_select.cuh>
#include <vector>

#include "common.cuh"
#include "graph.h"
#include "internal.h"

namespace sage {

struct SampleArgs {
  const long long *off;
  const int *col;
  Ladder L;
  Queues q;                    // resident all-V log
  unsigned long long cnt[kQueues];
  int lgS;
  int sort_tiles;              // rows not known to be sorted -> sort every tile in smem
  unsigned long long *loc1, *loc3;
  void *cd;                    // stage 2: L - R per vertex (int32 when it cannot overflow, else int64)
  int cd32;
  const uint32_t *lohi;        // stage 2: (lo << 1) | e per vertex, interval length f + e (see k_s2_update)
  long long f;                 // this step's floor length (nsec >> step)
  const int *target;
  unsigned long long *objective;
  const uint32_t *vw;          // online sampling: occurrences of each vertex's tiles (null = 1)
  int xlo, xhi;                // this sweep updates the counters of members x in [xlo, xhi) only
};

// first index i in seg[0, len) with seg[i] >= key (seg sorted ascending)
__device__ __forceinline__ int lower_bound_s(const int *seg, int len, long long key) {
  int lo = 0, hi = len;
  while (lo < hi) {
    const int mid = (lo + hi) >> 1;
    if ((long long)seg[mid] < key) lo = mid + 1; else hi = mid;
  }
  return lo;
}

// Bitonic sort of every aligned segment of t elements of buf[0, total) (t power of two).
__device__ __forceinline__ void warp_sort_segments(int *buf, int total, int t) {
  const int lane = (int)lane_id();
  for (int k = 2; k <= t; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      __syncwarp();
      for (int i = lane; i < total; i += 32) {
        const int l = i ^ j;
        if (l > i) {
          const bool asc = (k == t) || ((i & k) == 0);
          const int a = buf[i], b = buf[l];
          if ((a > b) == asc) {
            buf[i] = b;
            buf[l] = a;
          }
        }
      }
    }
  }
  __syncwarp();
}

// One sweep over the sample.  MODE 0: stage 1; 1: one stage-2 step; 2: stage 3; 3: objective.
template <int MODE>
__global__ void __launch_bounds__(256) k_sample(const __grid_constant__ SampleArgs a) {
  extern __shared__ int smem[];
  const int warp = threadIdx.x >> 5, lane = (int)lane_id();
  const int bufn = a.L.B > 32 ? a.L.B : 32;
  int *buf = smem + warp * bufn;
  const long long gwarp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  unsigned long long obj = 0;
  for (int c = 0; c < a.L.ncls; ++c) {
    const int t = a.L.B >> c;
    const long long count = (long long)a.cnt[c];
    const int G = t < 32 ? t : 32;       // lanes per tile
    const int R = 32 / G;                // tiles per warp round
    const int total = t < 32 ? 32 : t;   // staged elements per round
    const long long rounds = (count + R - 1) / R;
    for (long long r = gwarp; r < rounds; r += nwarps) {
      // locate the tile(s)
      const long long ti = r * R + lane / G;
      const bool tv = ti < count;
      long long start = 0;
      unsigned long long wt = 1;   // occurrences of this tile in the sample
      if (tv) {
        int u;
        if (c == 0) {
          start = a.q.cta[ti].start;
          u = a.q.cta[ti].u;
        } else {
          u = a.q.cls[c][ti];
          const long long b = a.off[u], e = a.off[u + 1];
          const RowSplit s = split_row(b, e, a.L);
          start = class_tile_start(e, s.r, t);
        }
        if (a.vw) wt = a.vw[u];
      }
      // stage the members in shared memory
      if (t < 32) {
        buf[lane] = tv ? a.col[start + lane % G] : 0x7fffffff;
      } else {
        for (int i = lane; i < t; i += 32) buf[i] = a.col[start + i];
      }
      __syncwarp();
      if (a.sort_tiles) warp_sort_segments(buf, total, t);
      // per-member counts
      const int per = t < 32 ? 1 : t / 32;
      for (int k = 0; k < per; ++k) {
        const int i = t < 32 ? lane : lane + 32 * k;
        const int *seg = t < 32 ? buf + (lane / G) * G : buf;
        const int pos = t < 32 ? lane % G : i;
        if (!tv || (MODE != 3 && wt == 0)) continue;
        const int x = seg[pos];
        if (MODE != 3 && (x < a.xlo || x >= a.xhi)) continue;
        const long long sx = (long long)x >> a.lgS;
        if (MODE == 0) {
          const int cnt = lower_bound_s(seg, t, (sx + 1) << a.lgS) - lower_bound_s(seg, t, sx << a.lgS) - 1;
          if (cnt > 0) atomicAdd(a.loc1 + x, (unsigned long long)cnt * wt);
        } else if (MODE == 1) {
          const uint32_t lh = a.lohi[x];
          const long long len = a.f + (lh & 1u);
          if (len > 1) {
            const long long lo = lh >> 1, hi = lo + len, mid = lo + len / 2;
            const int ilo = lower_bound_s(seg, t, lo << a.lgS);
            const int imid = lower_bound_s(seg, t, mid << a.lgS);
            const int ihi = lower_bound_s(seg, t, hi << a.lgS);
            const int Lc = imid - ilo - ((sx >= lo && sx < mid) ? 1 : 0);
            const int Rc = ihi - imid - ((sx >= mid && sx < hi) ? 1 : 0);
            // only the sign of L - R decides the step (L >= R -> left): one signed counter
            const long long d = (long long)(Lc - Rc) * (long long)wt;
            if (d != 0) {
              if (a.cd32) atomicAdd(static_cast<int *>(a.cd) + x, (int)d);
              else atomicAdd(static_cast<unsigned long long *>(a.cd) + x, (unsigned long long)d);
            }
          }
        } else if (MODE == 2) {
          const long long tg = a.target[x];
          const int cnt = lower_bound_s(seg, t, (tg + 1) << a.lgS) - lower_bound_s(seg, t, tg << a.lgS) -
                          (sx == tg ? 1 : 0);
          if (cnt > 0) atomicAdd(a.loc3 + x, (unsigned long long)cnt * wt);
        } else {
          if (pos == 0 || ((long long)seg[pos - 1] >> a.lgS) != sx) obj++;
        }
      }
      __syncwarp();
    }
  }
  if (MODE == 3) {
    obj = warp_sum64(obj);
    if (lane == 0 && obj) atomicAdd(a.objective, obj);
  }
}

// Stage-2 intervals: every step halves every open interval, so after k steps of [0, nsec) a
// length is floor(nsec / 2^k) or one more; one bit e per vertex holds which (4 B per vertex
// instead of an explicit (lo, hi) pair: half the random-read footprint of a sweep).
__global__ void k_s2_init(uint32_t *lohi, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) lohi[v] = 0u;
}
// stage-2 decision: L >= R -> hi = mid, else lo = mid (R21), then reset the counts
__global__ void k_s2_update(uint32_t *lohi, void *cd, int cd32, long long n, long long f) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long f2 = f >> 1;   // the next step's floor length
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    const uint32_t lh = lohi[v];
    const long long d = cd32 ? (long long)static_cast<int *>(cd)[v] : static_cast<long long *>(cd)[v];
    long long lo = lh >> 1, len = f + (lh & 1u);
    if (len > 1) {
      const long long half = len / 2;
      if (d >= 0) len = half;                   // L >= R -> left half [lo, mid) (R21)
      else { lo += half; len -= half; }         // right half [mid, hi)
    }
    lohi[v] = ((uint32_t)lo << 1) | (uint32_t)(len - f2);
    if (cd32) static_cast<int *>(cd)[v] = 0;
    else static_cast<long long *>(cd)[v] = 0;
  }
}
// in-degree (label-invariant; bounds the stage-2 counters: |L - R| <= in-degree * (B - 1))
__global__ void k_indeg(const int *__restrict__ col, long long m, unsigned *deg) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += stride) atomicAdd(deg + col[k], 1u);
}
__global__ void k_max_u32(const unsigned *x, long long n, unsigned *out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned mx = 0;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) mx = x[i] > mx ? x[i] : mx;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned y = __shfl_xor_sync(FULL, mx, o);
    mx = y > mx ? y : mx;
  }
  if ((threadIdx.x & 31) == 0 && mx) atomicMax(out, mx);
}
__global__ void k_s2_final(const uint32_t *lohi, int *target, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    target[v] = (int)(lohi[v] >> 1);
}
// movers (R22): loc3 > loc1 (and a candidate); keys for the (gain desc) sort
__global__ void k_movers(const unsigned long long *loc1, const unsigned long long *loc3,
                         const uint8_t *cand, uint8_t *mover, int *ids, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    mover[v] = (uint8_t)((cand == nullptr || cand[v]) && loc3[v] > loc1[v]);
    ids[v] = (int)v;
  }
}
__global__ void k_gain_keys(const int *mids, long long nm, const unsigned long long *loc1,
                            const unsigned long long *loc3, unsigned long long *keys) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nm; i += stride) {
    const int v = mids[i];
    keys[i] = ~(loc3[v] - loc1[v]);        // ascending order of ~gain = descending gain
  }
}
__global__ void k_target_keys(const int *mids, long long nm, const int *target, unsigned *keys) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nm; i += stride)
    keys[i] = (unsigned)target[mids[i]];
}
__global__ void k_iota_sigma(int *s, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) s[v] = (int)v;
}

// Swap matching: one thread per sector (R23).
__global__ void k_match(const unsigned *tkeys, const int *mids, long long nm,
                        const unsigned long long *loc1, const unsigned long long *loc3,
                        const uint8_t *mover, int *sigma_round, long long n, int S, long long nsec,
                        unsigned long long *nswaps) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long sw = 0;
  for (long long s = (long long)blockIdx.x * blockDim.x + threadIdx.x; s < nsec; s += stride) {
    // movers targeting s: [b, e) of the (target, gain desc, id asc) order
    long long lo = 0, hi = nm;
    while (lo < hi) {
      long long mid = (lo + hi) >> 1;
      if ((long long)tkeys[mid] < s) lo = mid + 1; else hi = mid;
    }
    const long long b = lo;
    if (b >= nm || (long long)tkeys[b] != s) continue;
    // victims: non-movers of sector s by (loc1 asc, id asc) — at most S of them
    int vic[64];
    int nv = 0;
    for (long long v = s * S; v < (s + 1) * S && v < n; ++v)
      if (!mover[v]) {
        int k = nv++;
        while (k > 0) {
          const int y = vic[k - 1];
          if (loc1[y] > loc1[v] || (loc1[y] == loc1[v] && y > v)) {
            vic[k] = y;
            --k;
          } else {
            break;
          }
        }
        vic[k] = (int)v;
      }
    for (int k = 0; k < nv && b + k < nm && (long long)tkeys[b + k] == s; ++k) {
      const int x = mids[b + k], y = vic[k];
      if (!(loc3[x] - loc1[x] > loc1[y])) break;
      sigma_round[x] = y;
      sigma_round[y] = x;
      ++sw;
    }
  }
  if (sw) atomicAdd(nswaps, sw);
}

// relabel: per old row v, key = (sigma(v) << cb) | sigma(col)
__global__ void k_relabel_keys(const long long *off, const int *col, const int *sig, long long n,
                               int cb, unsigned long long *keys, long long *deg_new) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const int lane = (int)lane_id();
  for (long long v = gw; v < n; v += nw) {
    const long long b = off[v], e = off[v + 1];
    const unsigned long long hi = (unsigned long long)(unsigned)sig[v] << cb;
    for (long long k = b + lane; k < e; k += 32) keys[k] = hi | (unsigned)sig[col[k]];
    if (lane == 0) deg_new[sig[v]] = e - b;
  }
}
__global__ void k_split_keys(const unsigned long long *keys, long long m, unsigned long long mask, int *col) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += stride)
    col[k] = (int)(keys[k] & mask);
}
__global__ void k_compose_sigma(int *sigma, int *sigma_inv, const int *sr, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    const int nl = sr[sigma[v]];
    sigma[v] = nl;
    sigma_inv[nl] = (int)v;
  }
}

static int ceil_log2(long long x) {
  int r = 0;
  while ((1ll << r) < x) ++r;
  return r;
}

static sage_status sample_args(sage_graph *g, SampleArgs *a, int lgS) {
  sage_status s = ensure_pagerank_log(g);
  if (s != SAGE_OK) return s;
  memset(a, 0, sizeof(*a));
  a->off = (const long long *)g->off;
  a->col = g->col;
  a->L = g->ladder;
  a->q = g->pr.q;
  for (int i = 0; i < kQueues; ++i) a->cnt[i] = g->pr.cnt[i];
  a->lgS = lgS;
  a->sort_tiles = g->rows_sorted ? 0 : 1;
  return SAGE_OK;
}

// A sweep's counter updates are random over the n members; above kPassBytes of counters the sweep
// runs in passes over member ranges (every pass reads the whole sample again).  Measured at C3
// (166 MB of counters): 48 MB passes 2.13 s per round, one pass 1.28 s — the extra sample reads and
// binary searches cost more than the DRAM-resident counter updates they avoid; so one pass up to
// 1 GB of counters.
#ifndef SAGE_PASS_MB
#define SAGE_PASS_MB 1024
#endif
constexpr size_t kPassBytes = (size_t)SAGE_PASS_MB << 20;
template <int MODE>
static sage_status launch_sample(sage_graph *g, const SampleArgs &a0, size_t counter_bytes = 8) {
  const int bufn = g->ladder.B > 32 ? g->ladder.B : 32;
  const size_t smem = sizeof(int) * (size_t)bufn * 8;
  if (smem > 48 * 1024)
    cudaFuncSetAttribute(k_sample<MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  const long long n = g->n;
  const int passes = MODE == 3 ? 1 : (int)std::max<long long>(1, ((long long)counter_bytes * n + kPassBytes - 1) / (long long)kPassBytes);
  for (int p = 0; p < passes; ++p) {
    SampleArgs a = a0;
    a.xlo = (int)(n * p / passes);
    a.xhi = (int)(n * (p + 1) / passes);
    k_sample<MODE><<<g->num_sms * 8, 256, smem, g->stream>>>(a);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(g, e, "reorder sample sweep");
  return SAGE_OK;
}

// Objective of §6 on the current labels: sum over sampled tiles of distinct sectors.
static sage_status objective(sage_graph *g, int lgS, unsigned long long *out) {
  SampleArgs a;
  sage_status s = sample_args(g, &a, lgS);
  if (s != SAGE_OK) return s;
  unsigned long long *d = nullptr;
  if ((s = dalloc(g, (void **)&d, sizeof(unsigned long long))) != SAGE_OK) return s;
  cudaMemsetAsync(d, 0, sizeof(unsigned long long), g->stream);
  a.objective = d;
  if ((s = launch_sample<3>(g, a)) != SAGE_OK) return s;
  cudaMemcpyAsync(out, d, sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  dfree(g, d);
  if (e != cudaSuccess) return cuda_fail(g, e, "objective");
  return SAGE_OK;
}

struct RoundBufs {
  unsigned long long *loc1 = nullptr, *loc3 = nullptr, *cl = nullptr;   // cl: stage-2 L - R
  uint32_t *lohi = nullptr;
  int *target = nullptr, *ids = nullptr, *mids = nullptr, *mids2 = nullptr, *sr = nullptr;
  uint8_t *mover = nullptr, *cand = nullptr;
  unsigned long long *gkeys = nullptr, *gkeys2 = nullptr;
  unsigned *tkeys = nullptr, *tkeys2 = nullptr;
  unsigned long long *scal = nullptr;   // [0] #movers (selected), [1] #swaps
  void *tmp = nullptr;
  size_t tmp_bytes = 0;
};

static void free_round(sage_graph *g, RoundBufs &b) {
  void *ps[] = {b.loc1, b.loc3, b.cl, b.lohi, b.target, b.ids, b.mids, b.mids2, b.sr,
                b.mover, b.cand, b.gkeys, b.gkeys2, b.tkeys, b.tkeys2, b.scal, b.tmp};
  for (void *p : ps) dfree(g, p);
  b = RoundBufs();
}

// One reorder round; *movers / *swaps report what happened (swaps == 0 -> nothing relabelled).
static sage_status one_round(sage_graph *g, RoundBufs &b, int lgS, const uint8_t *cand,
                             long long *movers, long long *swaps, bool stages_only = false,
                             const uint32_t *vw = nullptr) {
  const long long n = g->n;
  const int S = 1 << lgS;
  const long long nsec = (n + S - 1) / S;
  const int grid = g->num_sms * 8;
  SampleArgs a;
  sage_status s = sample_args(g, &a, lgS);
  if (s != SAGE_OK) return s;
  a.vw = vw;
  a.loc1 = b.loc1;
  a.loc3 = b.loc3;
  a.cd = b.cl;
  a.cd32 = (vw == nullptr && g->max_indeg >= 0 &&
            (unsigned long long)g->max_indeg * (unsigned long long)(g->ladder.B > 1 ? g->ladder.B - 1 : 1) <
                0x7fffffffull) ? 1 : 0;
  a.lohi = b.lohi;
  a.target = b.target;
  cudaMemsetAsync(b.loc1, 0, sizeof(unsigned long long) * n, g->stream);
  cudaMemsetAsync(b.loc3, 0, sizeof(unsigned long long) * n, g->stream);
  cudaMemsetAsync(b.cl, 0, sizeof(unsigned long long) * n, g->stream);
  // stage 1
  if ((s = launch_sample<0>(g, a)) != SAGE_OK) return s;
  // stage 2: ceil(log2(nsec)) halving sweeps
  k_s2_init<<<grid, 256, 0, g->stream>>>(b.lohi, n);
  const int steps = ceil_log2(nsec);
  for (int it = 0; it < steps; ++it) {
    a.f = nsec >> it;
    if ((s = launch_sample<1>(g, a, a.cd32 ? 4 : 8)) != SAGE_OK) return s;
    k_s2_update<<<grid, 256, 0, g->stream>>>(b.lohi, a.cd, a.cd32, n, a.f);
  }
  k_s2_final<<<grid, 256, 0, g->stream>>>(b.lohi, b.target, n);
  // stage 3
  if ((s = launch_sample<2>(g, a)) != SAGE_OK) return s;
  // movers, sorted by (target asc, gain desc, id asc) with two stable radix sorts
  k_movers<<<grid, 256, 0, g->stream>>>(b.loc1, b.loc3, cand, b.mover, b.ids, n);
  if (stages_only) return SAGE_OK;
  cub::DeviceSelect::Flagged(b.tmp, b.tmp_bytes, b.ids, b.mover, b.mids, b.scal, (int)n, g->stream);
  unsigned long long hm = 0;
  cudaMemcpyAsync(&hm, b.scal, sizeof(hm), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "reorder stages");
  // DeviceSelect writes an int count into scal[0]
  const long long nm = (long long)(hm & 0xffffffffull);
  *movers = nm;
  *swaps = 0;
  if (nm == 0) return SAGE_OK;
  k_gain_keys<<<grid, 256, 0, g->stream>>>(b.mids, nm, b.loc1, b.loc3, b.gkeys);
  cub::DeviceRadixSort::SortPairs(b.tmp, b.tmp_bytes, b.gkeys, b.gkeys2, b.mids, b.mids2, nm, 0, 64,
                                  g->stream);
  k_target_keys<<<grid, 256, 0, g->stream>>>(b.mids2, nm, b.target, b.tkeys);
  cub::DeviceRadixSort::SortPairs(b.tmp, b.tmp_bytes, b.tkeys, b.tkeys2, b.mids2, b.mids, nm, 0,
                                  std::max(1, ceil_log2(nsec + 1)), g->stream);
  k_iota_sigma<<<grid, 256, 0, g->stream>>>(b.sr, n);
  cudaMemsetAsync(b.scal + 1, 0, sizeof(unsigned long long), g->stream);
  k_match<<<grid, 256, 0, g->stream>>>(b.tkeys2, b.mids, nm, b.loc1, b.loc3, b.mover, b.sr, n, S, nsec,
                                       b.scal + 1);
  unsigned long long hs = 0;
  cudaMemcpyAsync(&hs, b.scal + 1, sizeof(hs), cudaMemcpyDeviceToHost, g->stream);
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "reorder match");
  *swaps = (long long)hs;
  if (hs == 0) return SAGE_OK;
  // ---- relabel: rows permuted, columns mapped, rows sorted, weights carried along
  const long long m = g->m;
  const int cb = std::max(1, ceil_log2(n));
  unsigned long long *keys = nullptr, *keys2 = nullptr;
  long long *deg = nullptr, *off2 = nullptr;
  int *col2 = nullptr;
  uint32_t *w2 = nullptr;
  void *tmp = nullptr;
  size_t tmpb = 0;
  if ((s = dalloc(g, (void **)&keys, sizeof(unsigned long long) * (size_t)std::max(m, 1ll))) != SAGE_OK ||
      (s = dalloc(g, (void **)&keys2, sizeof(unsigned long long) * (size_t)std::max(m, 1ll))) != SAGE_OK ||
      (s = dalloc(g, (void **)&deg, sizeof(long long) * (size_t)(n + 1))) != SAGE_OK ||
      (s = dalloc(g, (void **)&off2, sizeof(long long) * (size_t)(n + 1))) != SAGE_OK ||
      (s = dalloc(g, (void **)&col2, sizeof(int) * (size_t)m + 16)) != SAGE_OK)
    return s;
  if (g->w && (s = dalloc(g, (void **)&w2, sizeof(uint32_t) * (size_t)m + 16)) != SAGE_OK) return s;
  cudaMemsetAsync(deg + n, 0, sizeof(long long), g->stream);
  k_relabel_keys<<<grid, 256, 0, g->stream>>>((const long long *)g->off, g->col, b.sr, n, cb, keys, deg);
  cub::DeviceScan::ExclusiveSum(nullptr, tmpb, deg, off2, (int)(n + 1), g->stream);
  size_t tb2 = 0;
  if (g->w)
    cub::DeviceRadixSort::SortPairs(nullptr, tb2, keys, keys2, g->w, w2, m, 0, 2 * cb, g->stream);
  else
    cub::DeviceRadixSort::SortKeys(nullptr, tb2, keys, keys2, m, 0, 2 * cb, g->stream);
  tmpb = std::max(tmpb, tb2);
  if ((s = dalloc(g, &tmp, tmpb)) != SAGE_OK) return s;
  cub::DeviceScan::ExclusiveSum(tmp, tmpb, deg, off2, (int)(n + 1), g->stream);
  if (g->w)
    cub::DeviceRadixSort::SortPairs(tmp, tmpb, keys, keys2, g->w, w2, m, 0, 2 * cb, g->stream);
  else
    cub::DeviceRadixSort::SortKeys(tmp, tmpb, keys, keys2, m, 0, 2 * cb, g->stream);
  k_split_keys<<<grid, 256, 0, g->stream>>>(keys2, m, (1ull << cb) - 1, col2);
  // sigma <- sigma_round o sigma
  if (!g->sigma) {
    if ((s = dalloc(g, (void **)&g->sigma, sizeof(int) * (size_t)n)) != SAGE_OK ||
        (s = dalloc(g, (void **)&g->sigma_inv, sizeof(int) * (size_t)n)) != SAGE_OK)
      return s;
    k_iota_sigma<<<grid, 256, 0, g->stream>>>(g->sigma, n);
  }
  k_compose_sigma<<<grid, 256, 0, g->stream>>>(g->sigma, g->sigma_inv, b.sr, n);
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "relabel");
  // swap in the new CSR (library-owned from now on)
  if (g->own_off) dfree(g, g->off);
  if (g->own_col) dfree(g, g->col);
  if (g->own_w) dfree(g, g->w);
  g->off = (int64_t *)off2;
  g->col = col2;
  g->w = w2;
  g->own_off = g->own_col = true;
  g->own_w = w2 != nullptr;
  g->rows_sorted = true;
  g->reordered = true;
  g->vec_ok = g->vec == 4 && g->ladder.A >= 4;
  dfree(g, keys);
  dfree(g, keys2);
  dfree(g, deg);
  dfree(g, tmp);
  // the resident log describes the old labels: rebuild lazily
  free_queues(g, &g->pr.q);
  dfree(g, g->pr.dangling);
  g->pr.dangling = nullptr;
  g->pr.valid = false;
  g->pr.win = -1;   // arc locality changes with the labels: measured again
  return SAGE_OK;
}

static sage_status alloc_round(sage_graph *g, RoundBufs &b, bool with_cand) {
  const long long n = g->n;
  sage_status s;
  if (g->max_indeg < 0) {   // once per graph (label-invariant)
    unsigned *deg = nullptr;
    if ((s = dalloc(g, (void **)&deg, sizeof(unsigned) * (size_t)(n + 1))) != SAGE_OK) return s;
    cudaMemsetAsync(deg, 0, sizeof(unsigned) * (size_t)(n + 1), g->stream);
    k_indeg<<<g->num_sms * 8, 256, 0, g->stream>>>(g->col, g->m, deg);
    k_max_u32<<<g->num_sms * 8, 256, 0, g->stream>>>(deg, n, deg + n);
    unsigned hmax = 0;
    cudaMemcpyAsync(&hmax, deg + n, sizeof(hmax), cudaMemcpyDeviceToHost, g->stream);
    cudaError_t e = cudaStreamSynchronize(g->stream);
    dfree(g, deg);
    if (e != cudaSuccess) return cuda_fail(g, e, "in-degree");
    g->max_indeg = (long long)hmax;
  }
  void **ps[] = {(void **)&b.loc1, (void **)&b.loc3, (void **)&b.cl};
  for (auto p : ps)
    if ((s = dalloc(g, p, sizeof(unsigned long long) * (size_t)n)) != SAGE_OK) return s;
  if ((s = dalloc(g, (void **)&b.lohi, sizeof(uint32_t) * (size_t)n)) != SAGE_OK) return s;
  int **pi[] = {&b.target, &b.ids, &b.mids, &b.mids2, &b.sr};
  for (auto p : pi)
    if ((s = dalloc(g, (void **)p, sizeof(int) * (size_t)n)) != SAGE_OK) return s;
  if ((s = dalloc(g, (void **)&b.mover, (size_t)n)) != SAGE_OK) return s;
  if ((s = dalloc(g, (void **)&b.gkeys, sizeof(unsigned long long) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&b.gkeys2, sizeof(unsigned long long) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&b.tkeys, sizeof(unsigned) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&b.tkeys2, sizeof(unsigned) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&b.scal, sizeof(unsigned long long) * 4)) != SAGE_OK)
    return s;
  size_t t1 = 0, t2 = 0, t3 = 0;
  cub::DeviceSelect::Flagged(nullptr, t1, b.ids, b.mover, b.mids, b.scal, (int)n, g->stream);
  cub::DeviceRadixSort::SortPairs(nullptr, t2, b.gkeys, b.gkeys2, b.mids, b.mids2, (long long)n, 0, 64,
                                  g->stream);
  cub::DeviceRadixSort::SortPairs(nullptr, t3, b.tkeys, b.tkeys2, b.mids2, b.mids, (long long)n, 0, 32,
                                  g->stream);
  b.tmp_bytes = std::max(t1, std::max(t2, t3));
  if ((s = dalloc(g, &b.tmp, b.tmp_bytes)) != SAGE_OK) return s;
  if (with_cand && (s = dalloc(g, (void **)&b.cand, (size_t)n)) != SAGE_OK) return s;
  return SAGE_OK;
}

static sage_status load_candidates(sage_graph *g, RoundBufs &b, const std::vector<int32_t> &cand_orig) {
  if (cand_orig.empty()) return SAGE_OK;
  // candidates are ORIGINAL ids: map them to the current labels
  std::vector<uint8_t> hc((size_t)g->n, 0);
  for (int32_t v : cand_orig) hc[(size_t)to_internal_id(g, v)] = 1;
  cudaMemcpyAsync(b.cand, hc.data(), (size_t)g->n, cudaMemcpyHostToDevice, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "candidates");
  return SAGE_OK;
}

}  // namespace sage

using namespace sage;

// ---- online sampling (NEXT #3; §6 P:444 "the sampling is performed along with the tile access",
// threshold |E| P:514; reading R19b): queries record the rows they expanded as per-vertex
// occurrence counts (current labels); once the recorded row lengths since the last round reach
// the threshold, one round runs on that weighted sample after the query has returned its answer.
__global__ void k_samp_levels(const int32_t *__restrict__ level, const long long *__restrict__ off,
                              long long n, uint32_t *w, unsigned long long *acc) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long s = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    if (level[v] >= 0) {
      w[v] += 1u;
      s += (unsigned long long)(off[v + 1] - off[v]);
    }
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(acc, s);
}
__global__ void k_samp_all(const long long *__restrict__ off, long long n, uint32_t k, uint32_t *w,
                           unsigned long long *acc) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long s = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    const long long d = off[v + 1] - off[v];
    if (d > 0) {
      w[v] += k;
      s += (unsigned long long)d * k;
    }
  }
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(acc, s);
}

sage_status sage::online_after_query(sage_graph *g, const int32_t *level_internal, int32_t pr_iters) {
  if (!g->online) return SAGE_OK;
  const long long n = g->n;
  const int grid = g->num_sms * 8;
  if (level_internal)
    k_samp_levels<<<grid, 256, 0, g->stream>>>(level_internal, (const long long *)g->off, n, g->samp_w,
                                              g->samp_acc);
  else if (pr_iters > 0)
    k_samp_all<<<grid, 256, 0, g->stream>>>((const long long *)g->off, n, (uint32_t)pr_iters, g->samp_w,
                                           g->samp_acc);
  unsigned long long acc = 0;
  cudaMemcpyAsync(&acc, g->samp_acc, sizeof(acc), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "online sampling");
  g->online_pending = (long long)acc;
  if ((long long)acc < g->online_thr) return SAGE_OK;
  RoundBufs b;
  sage_status s = alloc_round(g, b, false);
  long long mv = 0, sw = 0;
  if (s == SAGE_OK) s = one_round(g, b, g->online_lgS, nullptr, &mv, &sw, false, g->samp_w);
  free_round(g, b);
  if (s != SAGE_OK) return s;
  if (sw > 0) {
    g->h_sigma.resize((size_t)n);
    cudaMemcpy(g->h_sigma.data(), g->sigma, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToHost);
  }
  cudaMemsetAsync(g->samp_w, 0, sizeof(uint32_t) * (size_t)n, g->stream);
  cudaMemsetAsync(g->samp_acc, 0, sizeof(unsigned long long), g->stream);
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "online reorder");
  g->online_rounds += 1;
  g->online_movers += mv;
  g->online_swaps += sw;
  g->online_pending = 0;
  return SAGE_OK;
}

extern "C" sage_status sage_online_reorder(sage_graph *g, int32_t enable, int32_t sector_width,
                                           int64_t threshold) {
  clear_error();
  if (!g) {
    set_error("null graph");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (!enable) {
    g->online = false;
    return SAGE_OK;
  }
  if (g->comm || g->host_columns) {
    set_error("online reordering is single-GPU with device-resident columns only");
    return SAGE_E_UNSUPPORTED;
  }
  const int S = sector_width ? sector_width : 8;
  if (S < 1 || S > 64 || (S & (S - 1))) {
    set_error("sector_width must be a power of two in [1, 64]");
    return SAGE_E_INVALID;
  }
  int lgS = 0;
  while ((1 << lgS) < S) ++lgS;
  sage_status s;
  if (!g->samp_w) {
    if ((s = dalloc(g, (void **)&g->samp_w, sizeof(uint32_t) * (size_t)std::max<long long>(g->n, 1))) != SAGE_OK ||
        (s = dalloc(g, (void **)&g->samp_acc, sizeof(unsigned long long))) != SAGE_OK)
      return s;
  }
  cudaMemsetAsync(g->samp_w, 0, sizeof(uint32_t) * (size_t)std::max<long long>(g->n, 1), g->stream);
  cudaMemsetAsync(g->samp_acc, 0, sizeof(unsigned long long), g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "online reorder");
  g->online = true;
  g->online_lgS = lgS;
  g->online_thr = threshold > 0 ? threshold : std::max<long long>(g->m, 1);
  g->online_pending = 0;
  return SAGE_OK;
}

extern "C" sage_status sage_online_reorder_info(const sage_graph *g, int64_t *rounds, int64_t *swaps,
                                                int64_t *pending) {
  clear_error();
  if (!g) {
    set_error("null graph");
    return SAGE_E_INVALID;
  }
  if (rounds) *rounds = g->online_rounds;
  if (swaps) *swaps = g->online_swaps;
  if (pending) *pending = g->online_pending;
  return SAGE_OK;
}

extern "C" sage_status sage_reorder(sage_graph *g, int32_t rounds, const sage_reorder_opts *opt,
                                    sage_stats *st) {
  NvtxRange nvtx_("sage_reorder");
  clear_error();
  if (!g || rounds < 0) {
    set_error("null graph or negative rounds");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (g->comm) {
    set_error("sage_reorder is single-GPU only");
    return SAGE_E_UNSUPPORTED;
  }
  if (g->host_columns) {
    set_error("sage_reorder needs device-resident columns (not SAGE_F_HOST_COLUMNS)");
    return SAGE_E_UNSUPPORTED;
  }
  int S = 8;
  if (opt && opt->sector_width) S = opt->sector_width;
  if (S < 1 || S > 64 || (S & (S - 1))) {
    set_error("sector_width must be a power of two in [1, 64]");
    return SAGE_E_INVALID;
  }
  if (opt && opt->n_candidates > 0 && !opt->candidates) {
    set_error("candidates is NULL");
    return SAGE_E_INVALID;
  }
  std::vector<int32_t> cand_orig;
  if (opt && opt->candidates) {
    for (int64_t i = 0; i < opt->n_candidates; ++i) {
      if (opt->candidates[i] < 0 || opt->candidates[i] >= g->n) {
        set_error("candidate %d out of range", opt->candidates[i]);
        return SAGE_E_INVALID;
      }
      cand_orig.push_back(opt->candidates[i]);
    }
  }
  int lgS = 0;
  while ((1 << lgS) < S) ++lgS;
  const long long n = g->n;
  sage_status s;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, g->stream);
  RoundBufs b;
  if ((s = alloc_round(g, b, !cand_orig.empty())) != SAGE_OK) goto fail;
  {
    long long tot_movers = 0, tot_swaps = 0;
    int done = 0;
    for (int r = 0; r < rounds; ++r) {
      if ((s = load_candidates(g, b, cand_orig)) != SAGE_OK) goto fail;
      long long mv = 0, sw = 0;
      if ((s = one_round(g, b, lgS, b.cand, &mv, &sw)) != SAGE_OK) goto fail;
      ++done;
      tot_movers += mv;
      tot_swaps += sw;
      if (sw > 0) {
        g->h_sigma.resize((size_t)n);
        cudaMemcpy(g->h_sigma.data(), g->sigma, sizeof(int32_t) * (size_t)n, cudaMemcpyDeviceToHost);
      }
      if (mv == 0 || sw == 0) break;   // R25: no movers (or an identity round) -> converged
    }
    cudaEventRecord(e1, g->stream);
    cudaError_t e = cudaStreamSynchronize(g->stream);
    if (e != cudaSuccess) {
      s = cuda_fail(g, e, "reorder");
      goto fail;
    }
    float ms = 0;
    cudaEventElapsedTime(&ms, e0, e1);
    if (st) {
      memset(st, 0, sizeof(*st));
      st->levels = done;
      st->vertices_expanded = tot_movers;
      st->vertices_discovered = tot_swaps;
      st->edges_traversed = (int64_t)done * g->m;
      st->arcs_inspected = (int64_t)done * g->m;
      st->ms = ms;
      st->kernel_ms = ms;
      // per round: (3 + steps) sample sweeps reading 4 B/arc + 8 B/arc of per-vertex state and
      // updates, plus the relabel (keys 8 B written+read twice per radix pass is not counted)
      const int steps = ceil_log2((n + S - 1) / S);
      st->model_bytes = (double)done * ((3.0 + steps) * 12.0 * (double)g->m + 24.0 * (double)g->m);
    }
  }
  free_round(g, b);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return SAGE_OK;
fail:
  free_round(g, b);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  return s;
}

extern "C" sage_status sage_reorder_objective(sage_graph *g, int32_t sector_width, int64_t *out) {
  clear_error();
  if (!g || !out || sector_width < 1 || sector_width > (1 << 30) || (sector_width & (sector_width - 1))) {
    set_error("invalid argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (g->comm) {
    set_error("single-GPU only");
    return SAGE_E_UNSUPPORTED;
  }
  int lgS = 0;
  while ((1 << lgS) < sector_width) ++lgS;
  unsigned long long v = 0;
  sage_status s = objective(g, lgS, &v);
  if (s != SAGE_OK) return s;
  *out = (int64_t)v;
  return SAGE_OK;
}

extern "C" sage_status sage_debug_reorder_stages(sage_graph *g, int32_t sector_width,
                                                 const int32_t *candidates, int64_t n_candidates,
                                                 int64_t *loc1_out, int64_t *target_out,
                                                 int64_t *loc3_out, uint8_t *mover_out) {
  clear_error();
  if (!g || !loc1_out || !target_out || !loc3_out || !mover_out || sector_width < 1 ||
      sector_width > 64 || (sector_width & (sector_width - 1)) || (n_candidates > 0 && !candidates)) {
    set_error("invalid argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (g->comm) return SAGE_E_UNSUPPORTED;
  std::vector<int32_t> cand;
  for (int64_t i = 0; i < n_candidates; ++i) {
    if (candidates[i] < 0 || candidates[i] >= g->n) {
      set_error("candidate out of range");
      return SAGE_E_INVALID;
    }
    cand.push_back(candidates[i]);
  }
  int lgS = 0;
  while ((1 << lgS) < sector_width) ++lgS;
  RoundBufs b;
  long long mv = 0, sw = 0;
  sage_status s = alloc_round(g, b, !cand.empty());
  if (s == SAGE_OK) s = load_candidates(g, b, cand);
  if (s == SAGE_OK) s = one_round(g, b, lgS, b.cand, &mv, &sw, true);
  if (s == SAGE_OK) {
    const size_t n = (size_t)g->n;
    cudaStreamSynchronize(g->stream);   // the stages ran on the graph's (non-blocking) stream
    std::vector<unsigned long long> l1(n), l3(n);
    std::vector<int> tg(n);
    cudaMemcpy(l1.data(), b.loc1, 8 * n, cudaMemcpyDeviceToHost);
    cudaMemcpy(l3.data(), b.loc3, 8 * n, cudaMemcpyDeviceToHost);
    cudaMemcpy(tg.data(), b.target, 4 * n, cudaMemcpyDeviceToHost);
    cudaError_t e = cudaMemcpy(mover_out, b.mover, n, cudaMemcpyDeviceToHost);
    if (e != cudaSuccess) s = cuda_fail(g, e, "reorder stages export");
    for (size_t i = 0; i < n; ++i) {
      loc1_out[i] = (int64_t)l1[i];
      loc3_out[i] = (int64_t)l3[i];
      target_out[i] = tg[i];
    }
  }
  free_round(g, b);
  cudaStreamSynchronize(g->stream);
  return s;
}
