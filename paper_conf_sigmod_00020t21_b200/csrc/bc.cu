// bc.cu — Betweenness Centrality (the paper's third evaluated workload,
// Alg. 1 l.8-24, Table 3) on the same Tiled Partitioning log and stealing consumer.
//
// Forward (Alg. 1 l.8-17): push BFS whose filter claims a neighbour with atomicCAS on its level
// (-1 -> L+1) and, for every arc into the next level (claimed here or by another arc of the same
// level), adds sigma[fr] to sigma[nb] with an fp64 atomic.  Every claimed vertex is appended to a
// BFS-order list (Queues::order), so level L's vertices are a contiguous segment.
// Backward (Alg. 1 l.19-24): levels in decreasing order; the segment of level L is classified
// into tiles again (Tiled Partitioning of the revisited rows) and consumed by the stealing
// consumer with a gather filter: a tile of row u sums (1 + delta[v]) / sigma[v] over members v on
// level L+1 (precomputed once per vertex into sigma[v] when its level is done), and the lane group
// adds sigma[u] * sum to delta[u] with one fp64 atomic — the same value as the paper's per-arc
// atomicAdd(delta[fr], sigma[fr]/sigma[nb] * (delta[nb] + 1)).
// bc[v] += delta[v] for v != source.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "common.cuh"
#include "graph.h"
#include "internal.h"

namespace sage {

struct BcArgs {
  const long long *off;
  const int *col;
  long long n;
  Ladder L;
  Queues q[2];
  Ctl *ctl;
  int *level;
  double *sigma;
  double *delta;
  double *bc;
  int *order;
  unsigned long long *order_cnt;
  long long *seg;       // backward: segment boundaries of the levels (host-computed)
  int nlev;             // backward: number of levels (deepest level = nlev - 1)
  int src;
  int vec_ok;
  int max_levels;
  int *flist;           // deferred contraction: frontier list
};

struct BcFwd {
  struct Src {
    double su;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
  static constexpr bool kDefer = true;   // contraction deferred to a K2' phase (see traversal.cu)
  int *flist = nullptr;
  unsigned long long *flc = nullptr;
  int *level;
  double *sigma;
  int next_level;
  const Queues *next_q;
  CounterSet *next_cs;
  __device__ __forceinline__ Src src(bool valid, int u, long long, long long) const {
    return Src{valid ? ldcg(sigma + u) : 0.0};
  }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int) const {
    int lv[N];
#pragma unroll
    for (int j = 0; j < N; ++j) lv[j] = valid ? ldcg(level + v[j]) : -2;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      int l = lv[j];
      if (l == -1) {
        l = atomicCAS(level + v[j], -1, next_level);          // Alg. 1 l.10-12
        if (l == -1) {
          in[j] = true;
          l = next_level;
        }
      }
      if (l == next_level) red_add_f64(sigma + v[j], s.su);   // Alg. 1 l.13-15
    }
  }
};

struct BcBwd {
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = false;
  const Queues *next_q = nullptr;
  CounterSet *next_cs = nullptr;
  const int *level;
  const double *sigma;
  double *delta;
  int child_level;
  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int lpt) const {
    double acc = 0.0;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      if (valid && ldcg(level + v[j]) == child_level)
        acc += ldcg(sigma + v[j]);   // = (1 + delta[v]) / sigma[v], Alg. 1 l.21-23 (k_bc_bwd)
    }
    for (int o = lpt >> 1; o > 0; o >>= 1) acc += __shfl_xor_sync(FULL, acc, o);
    if (valid && (lane_id() & (lpt - 1)) == 0 && acc != 0.0) red_add_f64(delta + s.u, ldcg(sigma + s.u) * acc);
  }
};

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_bc_fwd(const __grid_constant__ BcArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BcFwd::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  if ((threadIdx.x & 31) == 0) {
    wsm[warp].cpos = wsm[warp].cend = 0;
    wsm[warp].ndisc = 0;
  }
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x < (int)(sizeof(CounterSet) / sizeof(PaddedCounter)))
      reinterpret_cast<PaddedCounter *>(&ctl->set[(L + 2) % 3])[threadIdx.x].v = 0ull;
    BcFwd f;
    f.flist = a.flist;
    f.flc = &nxt->flc.v;
    f.level = a.level;
    f.sigma = a.sigma;
    f.next_level = L + 1;
    f.next_q = &a.q[(L + 1) & 1];
    f.next_cs = nxt;
    consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, nullptr, &wsm[warp], fsrc[warp], a.vec_ok);
    grid_barrier(&ctl->bar);
    if (classify_deferred(a.off, a.flist, &nxt->flc.v, a.L, a.q[(L + 1) & 1], nxt))
      grid_barrier(&ctl->bar);
    const unsigned long long nF = ldcg(&nxt->nF.v);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      ctl->levels = L + 1;
      ctl->tot_push_expanded += ldcg(&cur->nF.v);
      ctl->tot_push_arcs += ldcg(&cur->arcsF.v);
      ctl->tot_arcs_reached += ldcg(&nxt->arcsF.v);
      if (L < kMaxRec) {
        ctl->rec[L].nF = ldcg(&cur->nF.v);
        ctl->rec[L].discovered = nF;
      }
    }
    if (nF == 0) break;
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
  }
}

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_bc_bwd(const __grid_constant__ BcArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BcBwd::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  Ctl *ctl = a.ctl;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  // deepest level has no children: delta = 0 there; walk levels nlev-2 .. 0
  for (int L = a.nlev - 2, k = 0; L >= 0; --L, ++k) {
    CounterSet *cs = &ctl->set[k % 3];
    __syncthreads();
    if (blockIdx.x == 0 && threadIdx.x < (int)(sizeof(CounterSet) / sizeof(PaddedCounter)))
      reinterpret_cast<PaddedCounter *>(&ctl->set[(k + 2) % 3])[threadIdx.x].v = 0ull;
    // Tiled Partitioning of the level's rows (revisit); no order output on this pass
    Queues qk = a.q[k & 1];
    qk.order = nullptr;
    const long long b = a.seg[L], e = a.seg[L + 1];
    for (long long base = b + gw * 32; base < e; base += nw * 32) {
      const long long i = base + lane;
      const bool act = i < e;
      enqueue_ids(act, act ? ldcg(a.order + i) : 0, a.off, a.L, qk, cs);
    }
    // the children's coefficients, once per vertex: sigma[w] <- (1 + delta[w]) / sigma[w] for w
    // on level L+1 (their delta is final; their sigma is not read again), so the gather below
    // reads one fp64 per child arc instead of two and divides once per vertex, not per arc
    {
      const long long cb = a.seg[L + 1], ce = a.seg[L + 2];
      const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
      const long long nth = (long long)gridDim.x * blockDim.x;
      for (long long i = cb + tid; i < ce; i += nth) {
        const int w = ldcg(a.order + i);
        a.sigma[w] = (1.0 + ldcg(a.delta + w)) / ldcg(a.sigma + w);
      }
    }
    grid_barrier(&ctl->bar);
    BcBwd f;
    f.level = a.level;
    f.sigma = a.sigma;
    f.delta = a.delta;
    f.child_level = L + 1;
    consume_log<VEC>(f, a.L, qk, cs, a.off, a.col, nullptr, &wsm[warp], fsrc[warp], a.vec_ok);
    grid_barrier(&ctl->bar);
  }
  // accumulate the source's dependencies
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long nreach = a.seg[a.nlev];
  for (long long i = tid; i < nreach; i += stride) {
    const int v = ldcg(a.order + i);
    if (v != a.src) a.bc[v] += ldcg(a.delta + v);
  }
}

__global__ void k_bc_seed(BcArgs a) {
  const bool act = threadIdx.x == 0;
  long long b = 0, e = 0;
  if (act) {
    b = a.off[a.src];
    e = a.off[a.src + 1];
    a.level[a.src] = 0;
    a.sigma[a.src] = 1.0;
  }
  Queues q0 = a.q[0];
  enqueue_warp(act, a.src, b, e, a.L, q0, &a.ctl->set[0]);
}

}  // namespace sage

using namespace sage;

extern "C" sage_status sage_bc(sage_graph *g, const int32_t *sources, int64_t n_sources, double *bc_out,
                               sage_stats *st) {
  NvtxRange nvtx_("sage_bc");
  clear_error();
  if (!g || !bc_out || n_sources < 0 || (n_sources > 0 && !sources)) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (g->comm) {
    set_error("BC is single-GPU only");
    return SAGE_E_UNSUPPORTED;
  }
  for (int64_t i = 0; i < n_sources; ++i)
    if (sources[i] < 0 || sources[i] >= g->n) {
      set_error("source %d out of range", sources[i]);
      return SAGE_E_INVALID;
    }
  sage_status s;
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  TraversalState &t = g->ts;
  const long long n = g->n_local;
  double *sigma = nullptr, *delta = nullptr, *acc = nullptr;
  int *order = nullptr;
  unsigned long long *ocnt = nullptr;
  long long *seg = nullptr;
  if ((s = dalloc(g, (void **)&sigma, sizeof(double) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&delta, sizeof(double) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&acc, sizeof(double) * (size_t)n)) != SAGE_OK ||
      (s = dalloc(g, (void **)&order, sizeof(int) * (size_t)(n + 1))) != SAGE_OK ||
      (s = dalloc(g, (void **)&ocnt, sizeof(unsigned long long))) != SAGE_OK ||
      (s = dalloc(g, (void **)&seg, sizeof(long long) * (kMaxRec + 2))) != SAGE_OK)
    return s;
  cudaMemsetAsync(acc, 0, sizeof(double) * (size_t)n, g->stream);
  BcArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.n = n;
  a.L = g->ladder;
  a.q[0] = t.q[0];
  a.q[1] = t.q[1];
  for (int i = 0; i < 2; ++i) {
    a.q[i].order = order;
    a.q[i].order_cnt = ocnt;
  }
  a.ctl = t.ctl;
  a.level = t.level;
  a.sigma = sigma;
  a.delta = delta;
  a.bc = acc;
  a.order = order;
  a.order_cnt = ocnt;
  a.seg = seg;
  a.vec_ok = g->vec_ok ? 1 : 0;
  a.max_levels = kMaxRec;
  a.flist = t.flist;
  const void *ffn = g->vec == 4 ? (const void *)k_bc_fwd<4> : (const void *)k_bc_fwd<1>;
  const void *bfn = g->vec == 4 ? (const void *)k_bc_bwd<4> : (const void *)k_bc_bwd<1>;
  static int grid_f = 0, grid_b = 0;
  const int gf = coop_grid(g, ffn, &grid_f), gb = coop_grid(g, bfn, &grid_b);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, g->stream);
  long long levels_tot = 0, reached_arcs = 0, expanded = 0, arcs = 0;
  std::vector<long long> hseg(kMaxRec + 2);
  Ctl *h = new Ctl;
  for (int64_t k = 0; k < n_sources; ++k) {
    a.src = to_internal_id(g, sources[k]);
    cudaMemsetAsync(t.level, 0xff, sizeof(int32_t) * (size_t)n, g->stream);
    cudaMemsetAsync(sigma, 0, sizeof(double) * (size_t)n, g->stream);
    cudaMemsetAsync(delta, 0, sizeof(double) * (size_t)n, g->stream);
    cudaMemsetAsync(ocnt, 0, sizeof(unsigned long long), g->stream);
    cudaMemsetAsync(t.ctl, 0, sizeof(Ctl), g->stream);
    k_bc_seed<<<1, 32, 0, g->stream>>>(a);
    void *args[] = {&a};
    if ((s = launch_coop(g, ffn, gf, args, "BC forward")) != SAGE_OK) break;
    cudaMemcpyAsync(h, t.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost, g->stream);
    cudaError_t e = cudaStreamSynchronize(g->stream);
    if (e != cudaSuccess) {
      s = cuda_fail(g, e, "BC forward");
      break;
    }
    if (h->status == 1) {
      set_error("BC: more than %d levels", kMaxRec);
      s = SAGE_E_UNSUPPORTED;
      break;
    }
    // level segments of the BFS order: level 0 = the source, level L+1 = discoveries of level L
    const int nl = h->levels;
    hseg[0] = 0;
    hseg[1] = 1;
    for (int L = 0; L < nl; ++L) hseg[L + 2] = hseg[L + 1] + (long long)h->rec[L].discovered;
    levels_tot += nl;
    expanded += (long long)h->tot_push_expanded;
    arcs += (long long)h->tot_push_arcs;
    {
      long long sb = 0, se = 0;
      cudaMemcpy(&sb, g->off + a.src, 8, cudaMemcpyDeviceToHost);
      cudaMemcpy(&se, g->off + a.src + 1, 8, cudaMemcpyDeviceToHost);
      reached_arcs += (long long)h->tot_arcs_reached + (se - sb);
    }
    cudaMemcpyAsync(seg, hseg.data(), sizeof(long long) * (size_t)(nl + 2), cudaMemcpyHostToDevice,
                    g->stream);
    a.nlev = nl;   // levels 0 .. nl-1 hold vertices (the last one discovered nothing)
    cudaMemsetAsync(t.ctl, 0, offsetof(Ctl, rec), g->stream);
    if ((s = launch_coop(g, bfn, gb, args, "BC backward")) != SAGE_OK) break;
  }
  delete h;
  cudaEventRecord(e1, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (s == SAGE_OK && e != cudaSuccess) s = cuda_fail(g, e, "BC");
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (s == SAGE_OK) {
    if (st) {
      memset(st, 0, sizeof(*st));
      st->levels = (int32_t)levels_tot;
      st->push_levels = (int32_t)levels_tot;
      st->vertices_expanded = expanded;
      st->arcs_inspected = 2 * arcs;                 // forward + backward sweeps
      st->edges_traversed = (g->flags & SAGE_F_SYMMETRIC) ? reached_arcs / 2 : reached_arcs;
      st->ms = ms;
      st->kernel_ms = ms;
      // two sweeps of the BFS push model plus 8-B sigma / delta traffic per arc
      st->model_bytes = 2.0 * (20.0 * expanded + 8.0 * arcs) + 16.0 * arcs + 8.0 * n * n_sources;
    }
    s = translate_out_f64(g, acc, bc_out);
    if (s == SAGE_OK) {
      e = cudaStreamSynchronize(g->stream);
      if (e != cudaSuccess) s = cuda_fail(g, e, "BC output");
    }
  }
  dfree(g, sigma);
  dfree(g, delta);
  dfree(g, acc);
  dfree(g, order);
  dfree(g, ocnt);
  dfree(g, seg);
  return s;
}
