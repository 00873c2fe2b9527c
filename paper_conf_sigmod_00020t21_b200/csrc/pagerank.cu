// pagerank.cu — PageRank as SAGE's "global traversal": the frontier is all of V every
// iteration, so the all-V tile log is built ONCE by Tiled Partitioning and kept resident in
// device memory (the scheduling log reused on revisits; reading R15), then consumed
// by the stealing persistent kernel every iteration.
//
// Filter = push form of Alg. 1 l.26-29: every arc u->v adds x_u / out(u) into y_v
// with an fp64 atomic (red.global.add.f64; reading R7: fp32 atomics miss the 1e-6 bar).
// Readings R5/R6: x0 = 1/N; per iteration D = sum of x over dangling vertices,
// x_v <- (1-d)/N + d*(y_v + D/N); fixed number of iterations.
#include <cuda_runtime.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "common.cuh"
#include "graph.h"
#include "internal.h"

namespace sage {

struct PrPush {
  struct Src {
    double c;
  };
#ifndef SAGE_PR_PREFETCH
#define SAGE_PR_PREFETCH 4
#endif
  static constexpr int kPrefetch = SAGE_PR_PREFETCH;
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = true;
  static constexpr bool kEnqueue = false;
  const Queues *next_q = nullptr;
  CounterSet *next_cs = nullptr;
  const double *x;
  double *y;

  __device__ __forceinline__ Src src(bool valid, int u, long long b, long long e) const {
    // x is rewritten by the finalize phase of the previous iteration: read through L2
    return Src{(valid && e > b) ? ldcg(x + u) / (double)(e - b) : 0.0};
  }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N],
                                        const uint32_t (&)[N], bool (&in)[N], int) const {
#pragma unroll
    for (int j = 0; j < N; ++j) in[j] = false;
    if (!valid) return;
#pragma unroll
    for (int j = 0; j < N; ++j) red_add_f64(y + v[j], s.c);
  }
};

// Pull (gather) form for SYMMETRIC graphs (in-neighbours = out-neighbours): the tile of row v
// sums the contributions c_u = x_u / out(u) of its members (fp32 storage, kept L2-resident;
// fp64 accumulation, reading R7) and adds the group's partial sum to y_v with one fp64 atomic per
// lane group and step — the same resident log and stealing consumer, no per-arc atomics.
template <class CT>   // contribution storage: float (d <= 0.9) or double (d > 0.9)
struct PrPull {
  static constexpr int kPrefetch = SAGE_PR_PREFETCH;
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = false;
  const Queues *next_q = nullptr;
  CounterSet *next_cs = nullptr;
  const CT *c;
  double *y;
  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int lpt) const {
    CT cv[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      cv[j] = valid ? __ldcg(c + v[j]) : (CT)0;
    }
    double acc = 0.0;
#pragma unroll
    for (int j = 0; j < N; ++j) acc += (double)cv[j];
    for (int o = lpt >> 1; o > 0; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
    if (valid && (lane_id() & (lpt - 1)) == 0 && acc != 0.0) red_add_f64(y + s.u, acc);
  }
};

struct PrArgs {
  const long long *off;
  const int *col;
  long long n;        // rows here
  double N;           // global vertex count
  double d;
  int iters;
  Ladder L;
  Queues q;
  CounterSet *sets;   // 3 rotating copies of the log's counters (tickets reset each iteration)
  const int *dangling;
  long long n_dangling;
  double *x, *y;
  void *c;            // pull form: x_u / out(u), fp32 or fp64 (see PrPull)
  Ctl *ctl;
  int vec_ok;
  int steal;          // 0 = ablation (sage_pagerank_ex with SAGE_F_NO_STEALING): static tile dealing
};

// Build the all-V resident log: one thread per vertex, warp-aggregated classification.
__global__ void k_build_log(const long long *__restrict__ off, long long v0, long long n, Ladder L, Queues Q,
                            CounterSet *cs, int *dangling, unsigned long long *n_dangling) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long nthr = v0 + ((n - v0 + 31) / 32) * 32;
  for (long long i = v0 + (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nthr; i += stride) {
    const bool in = i < n;
    long long b = 0, e = 0;
    if (in) {
      b = off[i];
      e = off[i + 1];
    }
    const bool act = in && e > b;
    enqueue_warp(act, (int)i, b, e, L, Q, cs);
    const bool dg = in && e == b;
    const unsigned dm = __ballot_sync(FULL, dg);
    if (dm) {
      const int leader = __ffs(dm) - 1;
      unsigned long long base = 0;
      if ((int)lane_id() == leader) base = atomicAdd(n_dangling, (unsigned long long)__popc(dm));
      base = shfl64(base, leader);
      if (dg) dangling[base + __popc(dm & lanemask_lt())] = (int)i;
    }
  }
}

__global__ void k_pr_init(double *x, double *y, long long n, double v0) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    x[i] = v0;
    y[i] = 0.0;
  }
}

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_pagerank(const __grid_constant__ PrArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ PrPush::Src fsrc[kWarps][32];
  __shared__ double red[kWarps];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const double base = (1.0 - a.d) / a.N;
  for (int it = 0; it < a.iters; ++it) {
    CounterSet *cs = &a.sets[it % 3];
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x < kQueues) a.sets[(it + 2) % 3].tk[threadIdx.x].v = 0ull;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.ctl->D[(it + 2) % 3] = 0.0;
    // push phase over the resident log
    PrPush f;
    f.x = a.x;
    f.y = a.y;
    consume_log<VEC>(f, a.L, a.q, cs, a.off, a.col, nullptr, &wsm[warp], fsrc[warp], a.vec_ok, a.steal != 0);
    // dangling mass of this iteration's x
    double dsum = 0.0;
    for (long long i = tid; i < a.n_dangling; i += stride) dsum += ldcg(a.x + a.dangling[i]);
    dsum = warp_sumd(dsum);
    if (lane == 0) red[warp] = dsum;
    __syncthreads();
    if (threadIdx.x == 0) {
      double s = 0.0;
      for (int k = 0; k < kWarps; ++k) s += red[k];
      if (s != 0.0) atomicAdd(&a.ctl->D[it % 3], s);
    }
    grid_barrier(&a.ctl->bar);
    // finalize: x = (1-d)/N + d*(y + D/N); y = 0
    const double D = ldcg(&a.ctl->D[it % 3]);
    const double add = base + a.d * D / a.N;
    for (long long v = tid; v < a.n; v += stride) {
      const double yv = ldcg(a.y + v);
      a.x[v] = add + a.d * yv;
      a.y[v] = 0.0;
    }
    grid_barrier(&a.ctl->bar);
  }
}

template <int VEC, class CT>
__global__ void __launch_bounds__(kBlock, 4) k_pagerank_pull(const __grid_constant__ PrArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ typename PrPull<CT>::Src fsrc[kWarps][32];
  __shared__ double red[kWarps];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const double base = (1.0 - a.d) / a.N;
  for (int it = 0; it < a.iters; ++it) {
    CounterSet *cs = &a.sets[it % 3];
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x < kQueues) a.sets[(it + 2) % 3].tk[threadIdx.x].v = 0ull;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.ctl->D[(it + 2) % 3] = 0.0;
    PrPull<CT> f;
    f.c = static_cast<const CT *>(a.c);
    f.y = a.y;
    consume_log<VEC>(f, a.L, a.q, cs, a.off, a.col, nullptr, &wsm[warp], fsrc[warp], a.vec_ok);
    double dsum = 0.0;
    for (long long i = tid; i < a.n_dangling; i += stride) dsum += ldcg(a.x + a.dangling[i]);
    dsum = warp_sumd(dsum);
    if (lane == 0) red[warp] = dsum;
    __syncthreads();
    if (threadIdx.x == 0) {
      double s = 0.0;
      for (int k = 0; k < kWarps; ++k) s += red[k];
      if (s != 0.0) atomicAdd(&a.ctl->D[it % 3], s);
    }
    grid_barrier(&a.ctl->bar);
    const double D = ldcg(&a.ctl->D[it % 3]);
    const double add = base + a.d * D / a.N;
    for (long long v = tid; v < a.n; v += stride) {
      const double xv = add + a.d * ldcg(a.y + v);
      a.x[v] = xv;
      a.y[v] = 0.0;
      const long long dg = a.off[v + 1] - a.off[v];
      static_cast<CT *>(a.c)[v] = dg ? (CT)(xv / (double)dg) : (CT)0;
    }
    grid_barrier(&a.ctl->bar);
  }
}

// ============================================================================ windowed push
// Push PageRank on graphs whose arcs mostly stay near their source (web graphs in crawl order,
// C4): a CTA takes a chunk of kWinR consecutive rows (the all-V frontier in vertex order; tickets
// over chunks give the stealing) and accumulates every contribution x_u / out(u) whose target lies
// in [chunk - kWinH, chunk + kWinR + kWinH) into a shared-memory window of fp64 (R7) instead of an
// fp64 reduction in L2 / DRAM; the window is flushed with one coalesced red.global.add.f64 per
// nonzero entry after the chunk.  Far targets first try the chunk's hot table (4096 direct-mapped
// slots in shared memory, a slot kept by the first target that claims it, flushed with the window):
// the in-degree-heavy targets then cost one reduction per chunk instead of one per arc — same-
// address reductions serialise in L2 (C4: 54.5 -> 41 ms per iteration).  The rest are reduced in
// global memory directly.  (Binning the far arcs by 32 MB target block and reducing each block
// L2-resident — propagation blocking with a static layout — measured 50 ms: the bin writes cost
// more than the DRAM-resident reductions they replace.)  Inside a chunk, warps take 32-row groups (shared-memory counter): the group's arcs are ONE
// contiguous segment of col, streamed 32 elements per round with the owner row of each element
// found by a 5-step shuffle search over the group's row starts (empty rows share the next row's
// start, and the search takes the last of equal starts, i.e. the non-empty row).
#ifndef SAGE_WIN_HALO
#define SAGE_WIN_HALO 4096
#endif
#ifndef SAGE_WIN_HOTLG
#define SAGE_WIN_HOTLG 12
#endif
constexpr int kWinR = 8192;                 // rows per chunk
constexpr int kWinH = SAGE_WIN_HALO;        // halo on each side
constexpr int kWinS = kWinR + 2 * kWinH;    // window entries (fp64): 128 KB of shared memory
constexpr int kWinBlock = 1024;
constexpr int kWinUnroll = 4;               // rounds of 32 elements in flight per warp
constexpr long long kWinMaxDegree = 1 << 16;  // one warp streams a 32-row group: no huge rows
constexpr double kWinMinLocality = 0.25;     // sampled share of arcs inside the halo
constexpr int kWinHotLg = SAGE_WIN_HOTLG;    // hot far-target table: 4096 slots (48 KB)
constexpr int kWinHot = 1 << kWinHotLg;
constexpr size_t kWinDyn = sizeof(double) * (kWinS + kWinHot) + sizeof(int) * kWinHot;
#ifndef SAGE_WIN_HOT
#define SAGE_WIN_HOT 1
#endif

// A/B builds only: SAGE_WIN_MODE 1 = drop the global reductions, 2 = drop the window additions
// (timing attribution; wrong answers); SAGE_WIN_HOT 0 = no hot-target table
#ifndef SAGE_WIN_MODE
#define SAGE_WIN_MODE 0
#endif
__device__ __forceinline__ void atomic_add_shared_f64(double *p, double v) {
  atomicAdd(p, v);   // CAS loop on shared memory (no native fp64 shared add on sm_100a)
}

struct PrWinArgs {
  const long long *off;
  const int *col;
  long long n;
  double N, d;
  int iters;
  long long nchunks;
  CounterSet *sets;
  const int *dangling;
  long long n_dangling;
  double *x, *y;
  Ctl *ctl;
};

__global__ void __launch_bounds__(kWinBlock, 1) k_pagerank_win(const __grid_constant__ PrWinArgs a) {
  extern __shared__ double win[];   // kWinS window entries, then the hot table (kWinDyn bytes)
  __shared__ long long s_chunk;
  __shared__ int s_grp;
  double *s_hv = win + kWinS;                                  // hot far targets of the chunk:
  int *s_hk = reinterpret_cast<int *>(win + kWinS + kWinHot);  // values, keys (-1 = empty slot)
  __shared__ double red[kWinBlock / 32];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const double base = (1.0 - a.d) / a.N;
  const unsigned long long pol = policy_evict_first();
  for (int i = threadIdx.x; i < kWinS; i += blockDim.x) win[i] = 0.0;
  for (int i = threadIdx.x; i < kWinHot; i += blockDim.x) {
    s_hk[i] = -1;
    s_hv[i] = 0.0;
  }
  for (int it = 0; it < a.iters; ++it) {
    CounterSet *cs = &a.sets[it % 3];
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x < kQueues) a.sets[(it + 2) % 3].tk[threadIdx.x].v = 0ull;
    if (blockIdx.x == 0 && threadIdx.x == 0) a.ctl->D[(it + 2) % 3] = 0.0;
    for (;;) {
      if (threadIdx.x == 0) {
        s_chunk = (long long)atomicAdd(&cs->tk[0].v, 1ull);
        s_grp = 0;
      }
      __syncthreads();
      const long long chunk = s_chunk;
      if (chunk >= a.nchunks) break;
      const long long c0 = chunk * kWinR;
      const long long c1 = c0 + kWinR < a.n ? c0 + kWinR : a.n;
      const long long wlo = c0 - kWinH;
      const int ngroups = (int)((c1 - c0 + 31) >> 5);
      for (;;) {
        int g = 0;
        if (lane == 0) g = atomicAdd(&s_grp, 1);
        g = __shfl_sync(FULL, g, 0);
        if (g >= ngroups) break;
        const long long u = c0 + 32ll * g + lane;
        const bool vu = u < c1;
        const long long rb = vu ? __ldg(a.off + u) : 0;
        const long long re = vu ? __ldg(a.off + u + 1) : 0;
        const double cu = (vu && re > rb) ? ldcg(a.x + u) / (double)(re - rb) : 0.0;
        const long long b0 = shfl64((unsigned long long)rb, 0);
        const int last = __popc(__ballot_sync(FULL, vu)) - 1;
        const long long total = (long long)shfl64((unsigned long long)re, last) - b0;
        const int sj = vu ? (int)(rb - b0) : 0x7fffffff;   // row start within the segment
        for (long long k0 = 0; k0 < total; k0 += 32 * kWinUnroll) {
          int v[kWinUnroll];
#pragma unroll
          for (int r = 0; r < kWinUnroll; ++r) {
            const long long k = k0 + 32 * r + lane;
            v[r] = k < total ? ld_col(a.col + b0 + k, pol) : -1;
          }
#pragma unroll
          for (int r = 0; r < kWinUnroll; ++r) {
            const int k = (int)(k0 + 32 * r) + (int)lane;
            // owner = largest j with s_j <= k (the s_j are non-decreasing)
            int lo = 0;
#pragma unroll
            for (int st = 16; st > 0; st >>= 1) {
              const int s_mid = __shfl_sync(FULL, sj, lo + st);
              if (s_mid <= k) lo += st;
            }
            const double c = __shfl_sync(FULL, cu, lo);
            const unsigned long long rel = (unsigned long long)((long long)v[r] - wlo);
            const bool near = v[r] >= 0 && rel < (unsigned long long)kWinS;
            bool far = v[r] >= 0 && !near;
            if (SAGE_WIN_HOT && far) {
              // a far target keeps a slot of the chunk's hot table once it claims it: the heavy
              // in-degree targets (a few vertices take a large share of the far arcs) are summed
              // in shared memory instead of serialising same-address reductions in L2
              const int slot = (int)((uint32_t)v[r] * 2654435761u >> (32 - kWinHotLg));
              int k = s_hk[slot];
              if (k < 0) {
                k = atomicCAS(&s_hk[slot], -1, v[r]);
                if (k < 0) k = v[r];
              }
              if (k == v[r]) {
                atomic_add_shared_f64(&s_hv[slot], c);
                far = false;
              }
            }
            if (near) {
              if (SAGE_WIN_MODE != 2) atomic_add_shared_f64(&win[rel], c);
            } else if (far && SAGE_WIN_MODE != 1) {
              red_add_f64(a.y + v[r], c);
            }
          }
        }
      }
      __syncthreads();
      // flush the window (coalesced reductions) and leave it zeroed for the next chunk
      for (int i = threadIdx.x; i < kWinS; i += blockDim.x) {
        const double val = win[i];
        if (val != 0.0) {
          red_add_f64(a.y + (wlo + i), val);
          win[i] = 0.0;
        }
      }
      if (SAGE_WIN_HOT)
        for (int i = threadIdx.x; i < kWinHot; i += blockDim.x) {
          const int k = s_hk[i];
          if (k >= 0) {
            red_add_f64(a.y + k, s_hv[i]);
            s_hk[i] = -1;
            s_hv[i] = 0.0;
          }
        }
      __syncthreads();
    }
    // dangling mass of this iteration's x
    double dsum = 0.0;
    for (long long i = tid; i < a.n_dangling; i += stride) dsum += ldcg(a.x + a.dangling[i]);
    dsum = warp_sumd(dsum);
    if (lane == 0) red[warp] = dsum;
    __syncthreads();
    if (threadIdx.x == 0) {
      double s = 0.0;
      for (int k = 0; k < kWinBlock / 32; ++k) s += red[k];
      if (s != 0.0) atomicAdd(&a.ctl->D[it % 3], s);
    }
    grid_barrier(&a.ctl->bar);
    const double D = ldcg(&a.ctl->D[it % 3]);
    const double add = base + a.d * D / a.N;
    for (long long v = tid; v < a.n; v += stride) {
      const double yv = ldcg(a.y + v);
      a.x[v] = add + a.d * yv;
      a.y[v] = 0.0;
    }
    grid_barrier(&a.ctl->bar);
  }
}

// Locality of the arcs (sampled rows): arcs whose target lies within the window's halo of the
// source, and the sampled arcs; decides whether the windowed push pays.
__global__ void k_pr_locality(const long long *__restrict__ off, const int *__restrict__ col, long long n,
                              int sample, unsigned long long *out) {
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const unsigned lane = lane_id();
  unsigned long long near = 0, all = 0;
  for (long long v = gw * sample; v < n; v += nw * sample) {
    const long long b = off[v], e = off[v + 1];
    for (long long k = b + lane; k < e; k += 32) {
      const long long dv = (long long)col[k] - v;
      near += (dv > -kWinH && dv < kWinH) ? 1 : 0;
      all++;
    }
  }
  near = warp_sum64(near);
  all = warp_sum64(all);
  if (lane == 0 && all) {
    atomicAdd(out, near);
    atomicAdd(out + 1, all);
  }
}

template <class CT>
__global__ void k_pr_init_c(const long long *__restrict__ off, CT *c, long long n, double v0) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    const long long dg = off[i + 1] - off[i];
    c[i] = dg ? (CT)(v0 / (double)dg) : (CT)0;
  }
}

void free_pagerank_state(sage_graph *g) {
  PageRankState &p = g->pr;
  free_queues(g, &p.q);
  dfree(g, p.dangling);
  dfree(g, p.x);
  dfree(g, p.y);
  dfree(g, p.c);
  dfree(g, p.cs);
  p = PageRankState();
}

sage_status ensure_pagerank_log(sage_graph *g) {
  PageRankState &p = g->pr;
  if (p.valid) return SAGE_OK;
  sage_status s;
  const long long n = g->n_local;
  if (!p.x) {
    if ((s = dalloc(g, (void **)&p.x, sizeof(double) * (size_t)n)) != SAGE_OK ||
        (s = dalloc(g, (void **)&p.y, sizeof(double) * (size_t)n)) != SAGE_OK ||
        (s = dalloc(g, (void **)&p.cs, sizeof(CounterSet) * 3 + 64)) != SAGE_OK) {
      free_pagerank_state(g);
      return s;
    }
  }
  if ((s = alloc_queues(g, &p.q, n, g->m)) != SAGE_OK ||
      (s = dalloc(g, (void **)&p.dangling, sizeof(int) * (size_t)(n + 1))) != SAGE_OK) {
    free_pagerank_state(g);
    return s;
  }
  unsigned long long *nd = reinterpret_cast<unsigned long long *>(p.cs + 3);
  cudaMemsetAsync(p.cs, 0, sizeof(CounterSet) * 3 + 64, g->stream);
  k_build_log<<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, 0, n, g->ladder,
                                                     p.q, p.cs, p.dangling, nd);
  // replicate the counts into the two other rotating sets
  cudaMemcpyAsync(p.cs + 1, p.cs, sizeof(CounterSet), cudaMemcpyDeviceToDevice, g->stream);
  cudaMemcpyAsync(p.cs + 2, p.cs, sizeof(CounterSet), cudaMemcpyDeviceToDevice, g->stream);
  static CounterSet h;
  unsigned long long hnd = 0;
  cudaMemcpyAsync(&h, p.cs, sizeof(h), cudaMemcpyDeviceToHost, g->stream);
  cudaMemcpyAsync(&hnd, nd, sizeof(hnd), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "PageRank log build");
  for (int i = 0; i < kQueues; ++i) p.cnt[i] = h.cnt[i].v;
  p.n_dangling = (long long)hnd;
  p.valid = true;
  return SAGE_OK;
}

sage_status run_pagerank_multi(sage_graph *g, double damping, int32_t iterations, double *rank_out,
                               sage_stats *st);

}  // namespace sage

using namespace sage;

extern "C" sage_status sage_pagerank_ex(sage_graph *g, double damping, int32_t iterations,
                                        double *rank_out, uint32_t call_flags, sage_stats *st) {
  NvtxRange nvtx_("sage_pagerank");
  clear_error();
  if (!g || !rank_out) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (!(damping >= 0.0 && damping < 1.0) || iterations < 0) {
    set_error("damping must be in [0, 1) and iterations >= 0");
    return SAGE_E_INVALID;
  }
  if (g->comm) return run_pagerank_multi(g, damping, iterations, rank_out, st);
  sage_status s;
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  cudaEvent_t e0, e1, e2;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventCreate(&e2);
  cudaEventRecord(e0, g->stream);
  if ((s = ensure_pagerank_log(g)) != SAGE_OK) return s;
  PageRankState &p = g->pr;
  k_pr_init<<<g->num_sms * 8, 256, 0, g->stream>>>(p.x, p.y, g->n_local, 1.0 / (double)g->n);
  cudaMemsetAsync(g->ts.ctl, 0, offsetof(Ctl, rec), g->stream);
  for (int i = 0; i < 3; ++i)   // fresh stealing tickets for every call
    cudaMemsetAsync(&p.cs[i].tk, 0, sizeof(p.cs[i].tk), g->stream);
  cudaEventRecord(e1, g->stream);
  PrArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.n = g->n_local;
  a.N = (double)g->n;
  a.d = damping;
  a.iters = iterations;
  a.L = g->ladder;
  a.q = p.q;
  a.sets = p.cs;
  a.dangling = p.dangling;
  a.n_dangling = p.n_dangling;
  a.x = p.x;
  a.y = p.y;
  a.ctl = g->ts.ctl;
  a.vec_ok = g->vec_ok ? 1 : 0;
  a.steal = (call_flags & SAGE_F_NO_STEALING) ? 0 : 1;
  // pull (gather) on symmetric graphs unless the paper's push form is requested
  const bool pull = (g->flags & SAGE_F_SYMMETRIC) && !((g->flags | call_flags) & SAGE_F_PUSH_ONLY);
  // pull contributions in fp32 (half the bytes, L2-resident at C2) while the worst-case relative
  // error 6e-8 * d / (1 - d) stays <= 5.4e-7 (d <= 0.9); fp64 above that
  const bool c64 = damping > 0.9;
  if (pull && iterations > 0) {
    const size_t cb = (c64 ? sizeof(double) : sizeof(float)) * (size_t)g->n_local;
    if (p.c && p.c_bytes < cb) {
      dfree(g, p.c);
      p.c = nullptr;
    }
    if (!p.c) {
      if ((s = dalloc(g, &p.c, cb)) != SAGE_OK) return s;
      p.c_bytes = cb;
    }
    if (c64)
      k_pr_init_c<double><<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, (double *)p.c,
                                                                g->n_local, 1.0 / (double)g->n);
    else
      k_pr_init_c<float><<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, (float *)p.c,
                                                               g->n_local, 1.0 / (double)g->n);
    a.c = p.c;
  }
  // windowed push (directed / push form): chosen once per graph when most arcs stay within the
  // window's halo of their source and no row is long enough to stall a warp
  const bool steal = !(call_flags & SAGE_F_NO_STEALING);
  if (!pull && steal && iterations > 0 && p.win < 0) {
    p.win = 0;
    if (g->max_degree <= kWinMaxDegree && g->n_local >= kWinR) {
      unsigned long long *cnt = reinterpret_cast<unsigned long long *>(p.cs + 3) + 2;
      cudaMemsetAsync(cnt, 0, 2 * sizeof(unsigned long long), g->stream);
      k_pr_locality<<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, g->col, g->n_local, 16, cnt);
      unsigned long long h[2] = {0, 0};
      cudaMemcpyAsync(h, cnt, sizeof(h), cudaMemcpyDeviceToHost, g->stream);
      cudaError_t e = cudaStreamSynchronize(g->stream);
      if (e != cudaSuccess) return cuda_fail(g, e, "PageRank locality");
      p.locality = h[1] ? (double)h[0] / (double)h[1] : 0.0;
      // locality, not a window that spans much of a small graph: >= 4x what uniform targets give
      const double uniform = std::min(1.0, 2.0 * kWinH / (double)g->n_local);
      p.win = (p.locality >= kWinMinLocality && p.locality >= 4.0 * uniform) ? 1 : 0;
    }
  }
  if (iterations > 0 && !pull && steal && p.win == 1) {
    PrWinArgs wa;
    wa.off = a.off;
    wa.col = a.col;
    wa.n = a.n;
    wa.N = a.N;
    wa.d = a.d;
    wa.iters = a.iters;
    wa.nchunks = (a.n + kWinR - 1) / kWinR;
    wa.sets = a.sets;
    wa.dangling = a.dangling;
    wa.n_dangling = a.n_dangling;
    wa.x = a.x;
    wa.y = a.y;
    wa.ctl = a.ctl;
    const void *fn = (const void *)k_pagerank_win;
    const size_t dyn = kWinDyn;
    const int grid = coop_grid(g, fn, &g->grid_pr_win, kWinBlock, dyn);
    void *args[] = {&wa};
    if ((s = launch_coop(g, fn, grid, args, "PageRank kernel", kWinBlock, dyn)) != SAGE_OK) return s;
  } else if (iterations > 0) {
    const void *fn = pull ? (c64 ? (g->vec == 4 ? (const void *)k_pagerank_pull<4, double> : (const void *)k_pagerank_pull<1, double>)
                                 : (g->vec == 4 ? (const void *)k_pagerank_pull<4, float> : (const void *)k_pagerank_pull<1, float>))
                          : (g->vec == 4 ? (const void *)k_pagerank<4> : (const void *)k_pagerank<1>);
    int *cache = pull ? (c64 ? &g->grid_pr_pull64 : &g->grid_pr_pull) : &g->grid_pr;
    const int grid = coop_grid(g, fn, cache);
    void *args[] = {&a};
    if ((s = launch_coop(g, fn, grid, args, "PageRank kernel")) != SAGE_OK) return s;
  }
  cudaEventRecord(e2, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "PageRank");
  float ms = 0, kms = 0;
  cudaEventElapsedTime(&ms, e0, e2);
  cudaEventElapsedTime(&kms, e1, e2);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaEventDestroy(e2);
  if (st) {
    memset(st, 0, sizeof(*st));
    st->levels = iterations;
    st->push_levels = iterations;
    st->edges_traversed = (int64_t)iterations * g->m;
    st->arcs_inspected = (int64_t)iterations * g->m;
    st->vertices_expanded = (int64_t)iterations * (g->n_local - p.n_dangling);
    st->ms = ms;
    st->kernel_ms = kms;
    // 40 B per vertex + 12 B per arc, per iteration
    st->model_bytes = (double)iterations * (40.0 * (double)g->n_local + 12.0 * (double)g->m);
  }
  if ((s = translate_out_f64(g, p.x, rank_out)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "PageRank output");
  return online_after_query(g, nullptr, iterations);
}

extern "C" sage_status sage_pagerank(sage_graph *g, double damping, int32_t iterations,
                                     double *rank_out, sage_stats *st) {
  return sage_pagerank_ex(g, damping, iterations, rank_out, 0u, st);
}
