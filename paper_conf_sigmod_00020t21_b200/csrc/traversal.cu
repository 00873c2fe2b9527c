// traversal.cu — BFS and SSSP: the node-centric pipeline of SAGE (§4; Fig. 2) as ONE
// persistent cooperative kernel per query.
//
// Per level L (all in the same launch, one grid-wide barrier per level):
//   push : the stealing consumer (Resident Tile Stealing, Alg. 3) drains level L's tile log
//          (built by Tiled Partitioning, Alg. 2) and applies the filter (Alg. 1) to every
//          neighbour; filtered-in vertices are classified into level L+1's log in the same
//          pass (warp-aggregated expandTiles + contraction).
//   pull : (symmetric graphs, not in the paper; north_star) each unvisited vertex scans its
//          row until it meets a vertex of the frontier bitmap.
//   barrier; every CTA reads the same counters and takes the same decision: stop (empty
//   frontier), continue, and the Beamer direction for the next level.
// BFS filter (Alg. 1 l.1-6): visited-bitmap test-and-set, level := L+1.  The paper's
// non-atomic "dirty writes" are replaced by an atomicOr claim so every vertex enters
// the next log exactly once (reading R3); levels are identical.
// SSSP filter (reading R4): nd = dist[u] + w; atomicMin; improved vertices enter the next
// log once per iteration (bitmap dedupe) -> frontier Bellman-Ford.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>
#include <math.h>
#include <string.h>

#include <algorithm>

#include "common.cuh"
#include "graph.h"
#include "internal.h"

namespace sage {

// ============================================================================ filters
struct BfsPush {
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
#ifndef SAGE_BFS_DEFER
#define SAGE_BFS_DEFER 1
#endif
  static constexpr bool kDefer = SAGE_BFS_DEFER != 0;   // contraction deferred to a K2' phase
  int *flist = nullptr;                  // deferred frontier list
  unsigned long long *flc = nullptr;     // its slot counter (next level's CounterSet)
  uint32_t *visited;
  int *level;
  int *parent;
  uint32_t *fb_next;   // next-frontier bitmap (only when direction switching is enabled)
  int next_level;
  int v_base;          // global id of local row 0 (0 on one GPU)
  const Queues *next_q;
  CounterSet *next_cs;

  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }

  // Alg. 1 l.1-6: if dist[nb] = -1 then dist[nb] := dist[fr] + 1; filter_in(nb)
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N],
                                        const uint32_t (&)[N], bool (&in)[N], int) const {
    uint32_t wd[N];
    const unsigned long long keep = policy_evict_last();
#pragma unroll
    for (int j = 0; j < N; ++j) wd[j] = valid ? ld_status(visited + (v[j] >> 5), keep) : 0xffffffffu;
    // claims of all N neighbours in flight together (predicated, no branch between them)
    uint32_t old[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const uint32_t bit = 1u << (v[j] & 31);
      old[j] = atom_or_if(!(wd[j] & bit), visited + (v[j] >> 5), bit, bit);
    }
#pragma unroll
    for (int j = 0; j < N; ++j) {
      const uint32_t bit = 1u << (v[j] & 31);
      in[j] = !(old[j] & bit);
      if (in[j]) {
        level[v[j]] = next_level;
        if (parent) parent[v[j]] = s.u + v_base;
        if (fb_next) atomicOr(fb_next + (v[j] >> 5), bit);
      }
    }
  }
};

struct SsspPush {
  struct Src {
    uint32_t du;
  };
  static constexpr bool kWeights = true;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
#ifndef SAGE_SSSP_DEFER
#define SAGE_SSSP_DEFER 1
#endif
  static constexpr bool kDefer = SAGE_SSSP_DEFER != 0;   // contraction deferred (see BfsPush)
  int *flist = nullptr;
  unsigned long long *flc = nullptr;
  uint32_t *dist;
  uint32_t *inq_next;   // dedupe bitmap of the next frontier
  int *overflow;
  const Queues *next_q;
  CounterSet *next_cs;
  // near-far ordering: improvements at distance >= T go to the far pile instead of the frontier
  unsigned long long T;
  uint32_t *infar;      // far-pile membership bitmap
  int *far;             // far pile being appended to
  unsigned long long *far_cnt;
  uint32_t *expd;       // distance at which each vertex was last expanded (near-far only)

  __device__ __forceinline__ Src src(bool valid, int u, long long, long long) const {
    // dist[u] may have been lowered by another SM in an earlier iteration: read through L2
    const uint32_t du = valid ? ldcg(dist + u) : 0xffffffffu;
    if (valid && expd) expd[u] = du;
    return Src{du};
  }

  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N],
                                        const uint32_t (&w)[N], bool (&in)[N], int) const {
    uint32_t cur[N];
    const unsigned long long keep = policy_evict_last();
#pragma unroll
    for (int j = 0; j < N; ++j) cur[j] = valid ? ld_status(dist + v[j], keep) : 0u;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      const unsigned long long nd = (unsigned long long)s.du + w[j];
      if (valid && nd >= 0xffffffffull) {
        if (s.du != 0xffffffffu) *overflow = 1;  // possible overflow: resolved after the traversal
      } else if (valid && nd < cur[j]) {
        {
          const uint32_t old = atomicMin(dist + v[j], (uint32_t)nd);
          if ((uint32_t)nd < old) {
            const uint32_t bit = 1u << (v[j] & 31);
            if (nd < T) {
              const uint32_t o2 = atomicOr(inq_next + (v[j] >> 5), bit);
              in[j] = !(o2 & bit);
            } else if (!(atomicOr(infar + (v[j] >> 5), bit) & bit)) {
              far[atomicAdd(far_cnt, 1ull)] = v[j];
            }
          }
        }
      }
    }
  }
};

struct TailSmem;
// ============================================================================ kernel args
struct TravArgs {
  const long long *off;
  const int *col;
  const uint32_t *w;
  long long n;          // local rows (== global n on one GPU)
  long long m;
  Ladder L;
  Queues q[2];
  uint32_t *fb[3];
  uint32_t *visited;
  int *level;
  int *parent;
  uint32_t *dist;
  Ctl *ctl;
  int do_enabled;       // direction switching allowed
  int vec_ok;           // 16-B vector loads allowed (A % 4 == 0 and 16-B aligned col / w)
  double alpha, beta;
  int max_levels;
  int *tail;            // tail mode: next-frontier list (n entries of scratch)
  struct TailSmem *tailmem;   // tail mode state (global scratch: only block 0 uses it)
  int steal;            // 0 = ablation: static tile assignment instead of stealing
  int *flist;           // deferred contraction: frontier list (n + slack entries)
  unsigned long long defer_min_arcs;   // defer only on levels with arcs(F) >= this
};

// Pull (bottom-up) step over the visited bitmap: one warp per 32-vertex word.
__device__ __forceinline__ void pull_level(const TravArgs &a, int next_level, const uint32_t *fbc,
                                           uint32_t *fbn, const Queues &Qn, CounterSet *cur,
                                           CounterSet *nxt, WarpScratch *ws) {
  int bcnt = 0;
  const unsigned lane = lane_id();
  const long long nwords = (a.n + 31) >> 5;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  unsigned long long insp = 0, scanned = 0;
  for (long long wd = gw; wd < nwords; wd += nw) {
    const long long v = (wd << 5) + lane;
    const uint32_t vis = ldcg(a.visited + wd);
    const bool todo = v < a.n && !((vis >> lane) & 1u);
    long long b = 0, e = 0;
    bool found = false;
    int par = -1;
    if (todo) {
      b = ld_off(a.off + v);
      e = ld_off(a.off + v + 1);
      if (e > b) scanned++;
      for (long long k = b; k < e; ++k) {
        const int u = ld_stream1(a.col + k);
        ++insp;
        if ((ldcg(fbc + (u >> 5)) >> (u & 31)) & 1u) {
          found = true;
          par = u;
          break;
        }
      }
    }
    const unsigned fm = __ballot_sync(FULL, found);
    if (fm) {
      if (lane == 0) {
        a.visited[wd] = vis | fm;
        fbn[wd] = fm;
      }
      if (found) {
        a.level[v] = next_level;
        if (a.parent) a.parent[v] = par;
      }
    }
    buffer_push(found, (int)v, ws, bcnt, a.off, a.L, Qn, nxt);
  }
  if (bcnt) buffer_flush(ws, bcnt, a.off, a.L, Qn, nxt);
  insp = warp_sum64(insp);
  scanned = warp_sum64(scanned);
  if (lane == 0) {
    if (insp) atomicAdd(&cur->inspected.v, insp);
    if (scanned) atomicAdd(&cur->scanned.v, scanned);
  }
}

__device__ __forceinline__ void zero_counterset(CounterSet *s) {
  constexpr int nctr = sizeof(CounterSet) / sizeof(PaddedCounter);
  if (blockIdx.x == 0 && threadIdx.x < nctr)
    reinterpret_cast<PaddedCounter *>(s)[threadIdx.x].v = 0ull;
}

__device__ __forceinline__ void clear_words(uint32_t *p, long long nwords) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nwords; i += stride)
    p[i] = 0u;
}

// Record level L's statistics (single thread).
__device__ __forceinline__ void record_level(Ctl *ctl, int L, int dir, const CounterSet *cur,
                                             const CounterSet *nxt) {
  const unsigned long long nF = ldcg(&cur->nF.v), aF = ldcg(&cur->arcsF.v);
  const unsigned long long disc = ldcg(&nxt->nF.v), aN = ldcg(&nxt->arcsF.v);
  const unsigned long long insp = ldcg(&cur->inspected.v), sc = ldcg(&cur->scanned.v);
  if (dir == 0) {
    ctl->tot_push_expanded += nF;
    ctl->tot_push_arcs += aF;
    ctl->tot_push_disc += disc;
    ctl->push_levels++;
  } else {
    ctl->tot_pull_scanned += sc;
    ctl->tot_pull_inspected += insp;
    ctl->tot_pull_disc += disc;
    ctl->pull_levels++;
  }
  ctl->tot_arcs_reached += aN;
  ctl->tot_improved += disc;
  if (L < kMaxRec) {
    LevelRec &r = ctl->rec[L];
    r.dir = dir;
    r.nF = nF;
    r.arcsF = aF;
    r.inspected = dir == 0 ? aF : insp;
    r.scanned = sc;
    r.discovered = disc;
    r.t_ns = globaltimer();
  }
  ctl->levels = L + 1;
}

// ============================================================================ tail mode
// High-diameter graphs (C4's tendrils: hundreds of levels with a handful of vertices) pay the
// per-level cost of the grid pipeline: one warp's chain of dependent accesses (ticket, log entry,
// offsets, column, status, claim, classification, reservation) plus a grid barrier, ~10 us.
// When a push level's next frontier is small, block 0 alone runs the following levels with the
// frontier in shared memory (block scan over degrees, load-balanced arc loop, __syncthreads);
// the other CTAs wait at the grid barrier.  If the frontier grows again, block 0 classifies it
// into the regular log (Tiled Partitioning) and the whole grid resumes.  Push levels only,
// without direction switching (the frontier bitmaps are not maintained in tail mode).
constexpr int kTailV = kBlock;       // max frontier vertices handled by one CTA (one per thread)
constexpr int kTailE = 16384;        // max frontier arcs handled by one CTA
constexpr int kTailCollect = 512;    // max log entries gathered when entering tail mode

struct TailSmem {
  int f[2][kTailV];                  // frontier (ping-pong)
  long long b[2][kTailV];            // row start of each frontier vertex
  int d[2][kTailV];                  // its out-degree
  int pre[kTailV + 1];
  int buf[kTailCollect];
  int wsum[kWarps];
  int nnext;
  unsigned long long anext;
};

// exclusive block scan of x (one value per thread, 256 threads); returns the total
__device__ __forceinline__ int block_scan_excl(int x, int *out_excl, int *wsum) {
  const int lane = (int)lane_id(), warp = threadIdx.x >> 5;
  int inc = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(FULL, inc, o);
    if (lane >= o) inc += y;
  }
  if (lane == 31) wsum[warp] = inc;
  __syncthreads();
  int base = 0, total = 0;
  for (int w = 0; w < kWarps; ++w) {
    if (w < warp) base += wsum[w];
    total += wsum[w];
  }
  *out_excl = base + inc - x;
  __syncthreads();
  return total;
}

// Block 0 only.  Runs levels Lstart, Lstart+1, ... while the frontier is small.  The state `ts`
// lives in a small global scratch block (L1-cached for this CTA) rather than in shared memory, so
// the persistent kernel's static shared memory — and with it the L1 left for the status words of
// the main path — is unchanged.
__device__ void tail_run(const TravArgs &a, int Lstart, TailSmem &ts) {
  Ctl *ctl = a.ctl;
  const int tid = threadIdx.x, lane = (int)lane_id(), warp = tid >> 5;
  int nf = 0;
  // ---- gather the frontier of level Lstart from its log and deduplicate
  {
    const CounterSet *cs = &ctl->set[Lstart % 3];
    const Queues &Q = a.q[Lstart & 1];
    int E = 0;
    for (int c = 0; c <= a.L.ncls; ++c) {
      const int cnt = (int)ldcg(&cs->cnt[c].v);
      for (int i = tid; i < cnt; i += blockDim.x)
        ts.buf[E + i] = c == 0 ? ldcg_tile(Q.cta + i).u : (c == a.L.ncls ? ldcg(Q.frag + i) : ldcg(Q.cls[c] + i));
      E += cnt;
    }
    int P = 1;
    while (P < E) P <<= 1;
    for (int i = E + tid; i < P; i += blockDim.x) ts.buf[i] = 0x7fffffff;
    __syncthreads();
    for (int k = 2; k <= P; k <<= 1)
      for (int j = k >> 1; j > 0; j >>= 1) {
        for (int i = tid; i < P; i += blockDim.x) {
          const int l = i ^ j;
          if (l > i) {
            const int x = ts.buf[i], y = ts.buf[l];
            if ((x > y) == ((i & k) == 0)) {
              ts.buf[i] = y;
              ts.buf[l] = x;
            }
          }
        }
        __syncthreads();
      }
    for (int base = 0; base < E; base += blockDim.x) {
      const int i = base + tid;
      const bool keep = i < E && (i == 0 || ts.buf[i] != ts.buf[i - 1]);
      int pos;
      const int tot = block_scan_excl(keep ? 1 : 0, &pos, ts.wsum);
      if (keep) {
        const int u = ts.buf[i];
        const long long rb = a.off[u];
        ts.f[0][nf + pos] = u;
        ts.b[0][nf + pos] = rb;
        ts.d[0][nf + pos] = (int)(a.off[u + 1] - rb);
      }
      nf += tot;
    }
    __syncthreads();
  }
  // statistics kept in registers of thread 0, written once
  unsigned long long s_exp = 0, s_arcs = 0, s_disc = 0, s_reach = 0;
  int cur = 0;
  int L = Lstart;
  for (;; ++L) {
    // exclusive scan of the frontier's degrees (nf <= kTailV = blockDim: one row per thread)
    int p1;
    const int A = block_scan_excl(tid < nf ? ts.d[cur][tid] : 0, &p1, ts.wsum);
    if (tid < nf) ts.pre[tid] = p1;
    if (tid == 0) {
      ts.pre[nf] = A;
      ts.nnext = 0;
      ts.anext = 0;
    }
    __syncthreads();
    const int nx = cur ^ 1;
    for (int k = tid; k < A; k += blockDim.x) {
      int lo = 0, hi = nf - 1;      // largest o with pre[o] <= k
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (ts.pre[mid] <= k) lo = mid; else hi = mid - 1;
      }
      const int v = a.col[ts.b[cur][lo] + (k - ts.pre[lo])];
      const uint32_t bit = 1u << (v & 31);
      if (!(atomicOr(a.visited + (v >> 5), bit) & bit)) {
        a.level[v] = L + 1;
        if (a.parent) a.parent[v] = ts.f[cur][lo];
        const int idx = atomicAdd(&ts.nnext, 1);
        a.tail[idx] = v;
        const long long rb = a.off[v];
        const int dg = (int)(a.off[v + 1] - rb);
        if (idx < kTailV) {
          ts.f[nx][idx] = v;
          ts.b[nx][idx] = rb;
          ts.d[nx][idx] = dg;
        }
        atomicAdd(&ts.anext, (unsigned long long)dg);
      }
    }
    __syncthreads();
    const int nn = ts.nnext;
    const unsigned long long an = ts.anext;
    if (tid == 0) {
      s_exp += nf;
      s_arcs += A;
      s_disc += nn;
      s_reach += an;
      if (L < kMaxRec) {
        LevelRec &r = ctl->rec[L];
        r.dir = 0;
        r.nF = nf;
        r.arcsF = A;
        r.inspected = A;
        r.scanned = 0;
        r.discovered = nn;
        r.t_ns = r.t_work = globaltimer();
      }
    }
    const bool fits = nn <= kTailV && an <= (unsigned long long)kTailE;
    if (nn == 0 || L + 1 >= a.max_levels || !fits) break;
    nf = nn;
    cur = nx;
    __syncthreads();
  }
  const int nn = ts.nnext;
  if (tid == 0) {
    ctl->tot_push_expanded += s_exp;
    ctl->tot_push_arcs += s_arcs;
    ctl->tot_push_disc += s_disc;
    ctl->tot_arcs_reached += s_reach;
    ctl->tot_improved += s_disc;
    ctl->push_levels += L - Lstart + 1;
    ctl->levels = L + 1;
    ctl->tail_levels += L - Lstart + 1;
    if (nn == 0) {
      ctl->tail_state = 1;
    } else if (L + 1 >= a.max_levels) {
      ctl->status = 1;
      ctl->tail_state = 1;
    }
  }
  if (nn == 0 || L + 1 >= a.max_levels) return;
  // the frontier grew: classify it into level L+1's log and hand back to the grid
  constexpr int nctr = sizeof(CounterSet) / sizeof(PaddedCounter);
  if (tid < nctr) {
    reinterpret_cast<PaddedCounter *>(&ctl->set[(L + 1) % 3])[tid].v = 0ull;
    reinterpret_cast<PaddedCounter *>(&ctl->set[(L + 2) % 3])[tid].v = 0ull;
  }
  __threadfence_block();
  __syncthreads();
  for (int base = warp * 32; base < nn; base += blockDim.x) {
    const int i = base + lane;
    const bool act = i < nn;
    enqueue_ids(act, act ? ldcg(a.tail + i) : 0, a.off, a.L, a.q[(L + 1) & 1], &ctl->set[(L + 1) % 3]);
  }
  if (tid == 0) {
    ctl->tail_state = 2;
    ctl->tail_resume = L + 1;
  }
}

// ============================================================================ BFS kernel
#ifndef SAGE_BFS_VEC8
#define SAGE_BFS_VEC8 0   // push BFS with 8 neighbours per lane per step (more loads in flight)
#endif
template <int VEC>
#ifndef SAGE_BFS_MINB
#define SAGE_BFS_MINB 4
#endif
__global__ void __launch_bounds__(kBlock, SAGE_BFS_MINB) k_bfs(const __grid_constant__ TravArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BfsPush::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  double mU = (double)a.m - (double)ldcg(&ctl->set[0].arcsF.v);
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t0_ns = globaltimer();
  int dir = 0;
  unsigned long long prev_nF = 1;
  const long long nwords = (a.n + 31) >> 5;
  if ((threadIdx.x & 31) == 0) wsm[warp].cpos = wsm[warp].cend = 0;
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();   // block 0: record_level(L-1) finished before set (L+2)%3 is zeroed
    zero_counterset(&ctl->set[(L + 2) % 3]);
    uint32_t *fbc = a.fb[L % 3], *fbn = a.fb[(L + 1) % 3];
    if (a.do_enabled) clear_words(a.fb[(L + 2) % 3], nwords);
    if (dir == 0) {
      BfsPush f;
      f.visited = a.visited;
      f.level = a.level;
      f.parent = a.parent;
      f.fb_next = a.do_enabled ? fbn : nullptr;
      f.next_level = L + 1;
      f.v_base = 0;
      f.next_q = &a.q[(L + 1) & 1];
      f.next_cs = nxt;
      f.flist = (!SAGE_DEFER_RUNTIME || ldcg(&cur->arcsF.v) >= a.defer_min_arcs) ? a.flist : nullptr;
      f.flc = &nxt->flc.v;
#ifdef SAGE_PROF
      const unsigned long long pt0 = globaltimer();
#endif
      consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc[warp], a.vec_ok,
                       a.steal != 0);
#ifdef SAGE_PROF
      if (L == 1 && (threadIdx.x & 31) == 0) {   // per-warp consume durations of level 1
        const unsigned long long d = globaltimer() - pt0;
        atomicAdd(&g_prof[8], d);
        atomicMax(&g_prof[9], d);
        if (d > 20000) atomicAdd(&g_prof[10], 1ull);
        atomicAdd(&g_prof[11], 1ull);
        atomicMax(&g_prof[12], pt0 - ctl->t0_ns);
        atomicMin(&g_prof[13], pt0 - ctl->t0_ns);
      }
#endif
    } else {
      pull_level(a, L + 1, fbc, fbn, a.q[(L + 1) & 1], cur, nxt, &wsm[warp]);
    }
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    if (BfsPush::kDefer && classify_deferred(a.off, a.flist, &nxt->flc.v, a.L, a.q[(L + 1) & 1], nxt))
      grid_barrier(&ctl->bar);
    const unsigned long long nF = ldcg(&nxt->nF.v);
    const unsigned long long aF = ldcg(&nxt->arcsF.v);
    if (blockIdx.x == 0 && threadIdx.x == 0) record_level(ctl, L, dir, cur, nxt);
    if (nF == 0) break;
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
    // small frontier on a push-only traversal: block 0 runs the next levels alone
    if (!a.do_enabled && nF <= kTailV && aF <= (unsigned long long)kTailE) {
      unsigned long long ents = 0;
      for (int c = 0; c <= a.L.ncls; ++c) ents += ldcg(&nxt->cnt[c].v);
      if (ents <= (unsigned long long)kTailCollect) {
        if (blockIdx.x == 0) {
          __syncthreads();
          if (threadIdx.x == 0) ctl->tail_state = 0;
          __syncthreads();
          tail_run(a, L + 1, *a.tailmem);
        }
        grid_barrier(&ctl->bar);
        if (ldcg(&ctl->tail_state) == 1) break;
        L = ldcg(&ctl->tail_resume) - 1;   // ++L resumes the grid at the returned level
        continue;
      }
    }
    mU -= (double)aF;
    if (a.do_enabled) {
      if (dir == 0) {
        if ((double)aF > mU / a.alpha) dir = 1;
      } else {
        if (!(nF >= prev_nF || (double)nF > (double)a.n / a.beta)) dir = 0;
      }
    }
    prev_nF = nF;
  }
}

// ============================================================================ binned push BFS
// B200 restructuring of the push filter: a scattered 4-B status read costs about one
// L1TEX cycle per SM from L2-resident global memory but ~0.2 from shared memory (measured,
// tools/micro/status_reads.cu).  A push level therefore runs in two phases:
//   phase 1: the unchanged TP + RTS expansion; every neighbour id is stored into the bin of its
//            vertex slice (1M ids = 128 KB of bitmap), in a chunk reserved per (warp, slice);
//   phase 2: each CTA stages the visited bits of one slice in shared memory and runs Alg. 1's
//            filter on its share of that slice's bin; a vertex new to the CTA is claimed with a
//            global atomicOr (other CTAs of the slice), and filtered-in vertices are classified
//            into the next level's log exactly as before.
constexpr int kBinBlock = 1024;
constexpr int kBinWarps = kBinBlock / 32;
constexpr int kMaxSlices = 40;
constexpr int kSliceLg = 20;         // 2^20 vertices per slice
constexpr int kBinRes = 512;         // entries reserved per (warp, slice) with one atomic

struct BinArgs {
  int *bins;                         // nslices x cap
  long long cap;
  PaddedCounter *fill;               // [2][kMaxSlices]
  int nslices;
  int slice_lg;
};

struct BinPush {
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = false;
  const Queues *next_q = nullptr;
  CounterSet *next_cs = nullptr;
  // phase-1 context
  const TravArgs *a;
  const BinArgs *b;
  int *rpos, *rend;                  // this warp's reserved bin range per slice
  int fillset;
  int next_level;
  int nbits;                         // bits of a slice id
  const Queues *qn;
  CounterSet *csn;
  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }

  // end of phase 1: pad the unused part of every reservation
  __device__ __forceinline__ void close_reservations() const {
    const unsigned lane = lane_id();
    for (int s = 0; s < b->nslices; ++s) {
      const int pos = rpos[s], end = rend[s];
      for (int i = pos + (int)lane; i < end; i += 32) b->bins[(long long)s * b->cap + i] = -1;
    }
  }

  // Warp multi-split of 32 ids into their slices without staging: lanes of one slice are found
  // with one ballot per slice-id bit, ranked with popc, and stored straight into this warp's
  // reserved chunk of the slice's bin (one global atomic per kBinRes ids and slice).
  __device__ __forceinline__ void append(bool valid, int v) const {
    const unsigned lane = lane_id();
    const int sl = valid ? (v >> b->slice_lg) : 0;
    unsigned grp = __ballot_sync(FULL, valid);
    if (!grp) return;
#pragma unroll
    for (int bit = 0; bit < 6; ++bit) {
      if (bit < nbits) {
        const bool on = (sl >> bit) & 1;
        const unsigned bb = __ballot_sync(FULL, on);
        grp &= on ? bb : ~bb;
      }
    }
    const unsigned lt = lanemask_lt();
    const int rank = __popc(grp & lt), c = __popc(grp);
    const bool leader = valid && rank == 0;
    int pos = valid ? rpos[sl] : 0;
    const int end = valid ? rend[sl] : 0;
    unsigned nm = __ballot_sync(FULL, leader && end - pos < c);
    while (nm) {   // new reservation for the slices whose chunk is too small (rare)
      const int ld = __ffs(nm) - 1;
      nm &= nm - 1;
      const int s2 = __shfl_sync(FULL, sl, ld);
      const int p2 = rpos[s2], e2 = rend[s2];
      for (int i = p2 + (int)lane; i < e2; i += 32) b->bins[(long long)s2 * b->cap + i] = -1;
      unsigned long long np = 0;
      if (lane == 0) np = atomicAdd(&b->fill[fillset * kMaxSlices + s2].v, (unsigned long long)kBinRes);
      np = shfl64(np, 0);
      __syncwarp();
      if (lane == 0) {
        rpos[s2] = (int)min(np, (unsigned long long)b->cap);
        rend[s2] = (int)min(np + kBinRes, (unsigned long long)b->cap);
      }
      __syncwarp();
    }
    pos = valid ? rpos[sl] : 0;
    const bool fits = valid && pos + c <= rend[sl];
    if (fits) b->bins[(long long)sl * b->cap + pos + rank] = v;
    __syncwarp();
    if (leader && fits) rpos[sl] = pos + c;
    __syncwarp();
    // bin capacity exhausted (skewed ids): Alg. 1's filter on the global bitmap directly
    const bool direct = valid && !fits;
    if (__any_sync(FULL, direct)) {
      bool disc = false;
      if (direct) {
        const uint32_t bit = 1u << (v & 31);
        disc = !(atomicOr(a->visited + (v >> 5), bit) & bit);
        if (disc) {
          a->level[v] = next_level;
          if (a->do_enabled) atomicOr(a->fb[next_level % 3] + (v >> 5), bit);
        }
      }
      enqueue_ids(disc, v, a->off, a->L, *qn, csn);
    }
  }

  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int) const {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      append(valid, v[j]);
    }
  }
};

// phase 2: Alg. 1's filter against a shared-memory copy of one slice of the visited bitmap
__device__ __forceinline__ void bin_check(const TravArgs &a, const BinArgs &b, int fillset, int L,
                                          uint32_t *sbm, WarpScratch *ws, const Queues &Qn,
                                          CounterSet *csn) {
  const unsigned lane = lane_id();
  const int warp = threadIdx.x >> 5;
  const int nw = blockDim.x >> 5;
  const int ns = b.nslices;
  int bcnt = 0;
  uint32_t *fbn = a.do_enabled ? a.fb[(L + 1) % 3] : nullptr;
  const int G = gridDim.x;
  const int first = (int)blockIdx.x % ns;
  const int nparts = G >= ns ? (G - first + ns - 1) / ns : 1;
  const int part = G >= ns ? (int)blockIdx.x / ns : 0;
  for (int s = first; s < ns; s += (G >= ns ? ns : G)) {
    const long long v0 = (long long)s << b.slice_lg;
    const long long v1 = min(a.n, v0 + (1ll << b.slice_lg));
    const long long nwd = (v1 - v0 + 31) >> 5;
    for (long long i = threadIdx.x; i < nwd; i += blockDim.x) sbm[i] = ldcg(a.visited + (v0 >> 5) + i);
    __syncthreads();
    const long long fill = (long long)ldcg(&b.fill[fillset * kMaxSlices + s].v);
    const long long tot = fill < b.cap ? fill : b.cap;
    const long long lo = tot * part / nparts, hi = tot * (part + 1) / nparts;
    const int *bin = b.bins + (long long)s * b.cap;
    for (long long base = lo + (long long)warp * 128; base < hi; base += (long long)nw * 128) {
      int vv[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const long long i = base + j * 32 + lane;
        vv[j] = i < hi ? ldcg(bin + i) : -1;
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int v = vv[j];
        bool disc = false;
        if (v >= 0) {
          const int lb = (int)(v - v0);
          const uint32_t bit = 1u << (lb & 31);
          if (!(sbm[lb >> 5] & bit)) {
            if (!(atomicOr(sbm + (lb >> 5), bit) & bit)) {
              disc = !(atomicOr(a.visited + (v >> 5), bit) & bit);
              if (disc) {
                a.level[v] = L + 1;
                if (fbn) atomicOr(fbn + (v >> 5), bit);
              }
            }
          }
        }
        buffer_push(disc, v, &ws[warp], bcnt, a.off, a.L, Qn, csn);
      }
    }
    __syncthreads();
  }
  if (bcnt) buffer_flush(&ws[warp], bcnt, a.off, a.L, Qn, csn);
}

template <int VEC>
__global__ void __launch_bounds__(kBinBlock, 1) k_bfs_bin(const __grid_constant__ TravArgs a,
                                                          const __grid_constant__ BinArgs b) {
  extern __shared__ __align__(16) unsigned char dsm[];
  WarpScratch *wsm = reinterpret_cast<WarpScratch *>(dsm);
  BinPush::Src *fsrc = reinterpret_cast<BinPush::Src *>(dsm + sizeof(WarpScratch) * kBinWarps);
  int *rps = reinterpret_cast<int *>(dsm + sizeof(WarpScratch) * kBinWarps + sizeof(BinPush::Src) * 32 * kBinWarps);
  int *res = rps + kMaxSlices * kBinWarps;
  unsigned char *U = dsm + sizeof(WarpScratch) * kBinWarps + sizeof(BinPush::Src) * 32 * kBinWarps +
                     2 * sizeof(int) * kMaxSlices * kBinWarps;
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  Ctl *ctl = a.ctl;
  double mU = (double)a.m - (double)ldcg(&ctl->set[0].arcsF.v);
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t0_ns = globaltimer();
  int dir = 0;
  unsigned long long prev_nF = 1;
  const long long nwords = (a.n + 31) >> 5;
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();
    zero_counterset(&ctl->set[(L + 2) % 3]);
    if (blockIdx.x == 0 && threadIdx.x < kMaxSlices) b.fill[((L + 1) & 1) * kMaxSlices + threadIdx.x].v = 0ull;
    if (a.do_enabled) clear_words(a.fb[(L + 2) % 3], nwords);
    if (dir == 0) {
      // phase 1: expansion into slice bins
      for (int i = lane; i < b.nslices; i += 32) {
        rps[warp * kMaxSlices + i] = 0;
        res[warp * kMaxSlices + i] = 0;
      }
      __syncwarp();
      BinPush f;
      f.a = &a;
      f.b = &b;
      f.rpos = rps + warp * kMaxSlices;
      f.rend = res + warp * kMaxSlices;
      f.fillset = L & 1;
      f.next_level = L + 1;
      f.nbits = 0;
      while ((1 << f.nbits) < b.nslices) ++f.nbits;
      f.qn = &a.q[(L + 1) & 1];
      f.csn = nxt;
      consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc + warp * 32, a.vec_ok);
      f.close_reservations();
      grid_barrier(&ctl->bar);
      if (blockIdx.x == 0 && threadIdx.x == 0 && L < kMaxRec)
        ctl->rec[L].t_mid_us = (int)((globaltimer() - ctl->t0_ns) / 1000);
      // phase 2: filter against shared-memory slices of the visited bitmap
      bin_check(a, b, L & 1, L, reinterpret_cast<uint32_t *>(U), wsm, a.q[(L + 1) & 1], nxt);
    } else {
      pull_level(a, L + 1, a.fb[L % 3], a.fb[(L + 1) % 3], a.q[(L + 1) & 1], cur, nxt, &wsm[warp]);
    }
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    const unsigned long long nF = ldcg(&nxt->nF.v);
    const unsigned long long aF = ldcg(&nxt->arcsF.v);
    if (blockIdx.x == 0 && threadIdx.x == 0) record_level(ctl, L, dir, cur, nxt);
    if (nF == 0) break;
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
    mU -= (double)aF;
    if (a.do_enabled) {
      if (dir == 0) {
        if ((double)aF > mU / a.alpha) dir = 1;
      } else {
        if (!(nF >= prev_nF || (double)nF > (double)a.n / a.beta)) dir = 0;
      }
    }
    prev_nF = nF;
  }
}

static size_t bin_smem_bytes(int nslices, long long n) {
  const size_t fixed = sizeof(WarpScratch) * kBinWarps + sizeof(int) * 32 * kBinWarps +
                       2 * sizeof(int) * kMaxSlices * kBinWarps;
  const long long sw = std::min<long long>(n, 1ll << kSliceLg);
  const size_t bm = sizeof(uint32_t) * (size_t)((sw + 31) / 32 + 1);
  (void)nslices;
  return fixed + bm;
}

// ============================================================================ SSSP kernel
struct FarArgs {                      // near-far state of k_sssp
  int *far[3];                       // three rotating far piles (append / scan / spare)
  uint32_t *infar;                   // far-pile membership bitmap
  uint32_t *expd;                    // last expanded distance per vertex (stale far entries)
  PaddedCounter *cnt;                // [3] far pile sizes
  PaddedCounter *fmin;               // [3] min distance seen in a scan
  unsigned long long delta;          // threshold step; 0xffff... = plain Bellman-Ford
};

// Advance phase of near-far SSSP: move far-pile vertices with dist < T into the next log.
__device__ __forceinline__ void far_scan(const TravArgs &a, const FarArgs &fa, int k, unsigned long long T,
                                         uint32_t *inq_next, const Queues &Qn, CounterSet *csn,
                                         WarpScratch *ws) {
  const unsigned lane = lane_id();
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const int *src = fa.far[k % 3];
  int *dst = fa.far[(k + 1) % 3];
  const long long cnt = (long long)ldcg(&fa.cnt[k % 3].v);
  unsigned long long mn = ~0ull;
  int bcnt = 0;
  for (long long base = gw * 32; base < cnt; base += nw * 32) {
    const long long i = base + lane;
    bool move = false, keep = false;
    int v = 0;
    if (i < cnt) {
      v = ldcg(src + i);
      const uint32_t d = ldcg(a.dist + v);
      const uint32_t bit = 1u << (v & 31);
      if (d < T) {
        atomicAnd(fa.infar + (v >> 5), ~bit);
        // skip entries whose vertex was already expanded at its current distance
        move = ldcg(fa.expd + v) != d && !(atomicOr(inq_next + (v >> 5), bit) & bit);
      } else {
        keep = true;
        if (d < mn) mn = d;
      }
    }
    const unsigned km = __ballot_sync(FULL, keep);
    if (km) {
      const int leader = __ffs(km) - 1;
      unsigned long long p = 0;
      if ((int)lane == leader) p = atomicAdd(&fa.cnt[(k + 1) % 3].v, (unsigned long long)__popc(km));
      p = shfl64(p, leader);
      if (keep) dst[p + __popc(km & lanemask_lt())] = v;
    }
    buffer_push(move, v, ws, bcnt, a.off, a.L, Qn, csn);
  }
  if (bcnt) buffer_flush(ws, bcnt, a.off, a.L, Qn, csn);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const unsigned long long y = __shfl_xor_sync(FULL, mn, o);
    mn = y < mn ? y : mn;
  }
  if (lane == 0 && mn != ~0ull) atomicMin(&fa.fmin[k % 3].v, mn);
}

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_sssp(const __grid_constant__ TravArgs a, int *overflow,
                                                    const __grid_constant__ FarArgs fa) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ SsspPush::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  const long long nwords = (a.n + 31) >> 5;
  if ((threadIdx.x & 31) == 0) wsm[warp].cpos = wsm[warp].cend = 0;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t0_ns = globaltimer();
  unsigned long long T = fa.delta;   // near threshold
  int k = 0;                         // far scans done; the current far pile is far[k % 3]
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();
    zero_counterset(&ctl->set[(L + 2) % 3]);
    clear_words(a.fb[(L + 2) % 3], nwords);
    SsspPush f;
    f.dist = a.dist;
    f.inq_next = a.fb[(L + 1) % 3];
    f.overflow = overflow;
    f.next_q = &a.q[(L + 1) & 1];
    f.next_cs = nxt;
    f.T = T;
    f.infar = fa.infar;
    f.far = fa.far[k % 3];
    f.far_cnt = &fa.cnt[k % 3].v;
    f.expd = fa.delta == ~0ull ? nullptr : fa.expd;
    f.flist = (!SAGE_DEFER_RUNTIME || ldcg(&cur->arcsF.v) >= a.defer_min_arcs) ? a.flist : nullptr;
    f.flc = &nxt->flc.v;
    consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc[warp], a.vec_ok);
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    if (SsspPush::kDefer && classify_deferred(a.off, a.flist, &nxt->flc.v, a.L, a.q[(L + 1) & 1], nxt))
      grid_barrier(&ctl->bar);
    unsigned long long nF = ldcg(&nxt->nF.v);
    // near frontier exhausted: raise the threshold and pull the far pile forward
    while (nF == 0 && ldcg(&fa.cnt[k % 3].v) != 0) {
      if (blockIdx.x == 0 && threadIdx.x == 0) {
        fa.cnt[(k + 2) % 3].v = 0ull;     // scan k-1's source pile, no longer read
        fa.fmin[(k + 1) % 3].v = ~0ull;   // written by scan k+1, not read before it
      }
      const unsigned long long fm = k > 0 ? ldcg(&fa.fmin[(k + 2) % 3].v) : ~0ull;  // scan k-1's
      T = (T + fa.delta > T) ? T + fa.delta : ~0ull;
      if (fm != ~0ull && fm >= T) T = (fm / fa.delta + 1) * fa.delta;   // skip empty buckets
      far_scan(a, fa, k, T, a.fb[(L + 1) % 3], a.q[(L + 1) & 1], nxt, &wsm[warp]);
      grid_barrier(&ctl->bar);
      ++k;
      nF = ldcg(&nxt->nF.v);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) record_level(ctl, L, 0, cur, nxt);
    if (nF == 0) break;
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
  }
}

// Seed the level-0 log with the source (one warp).
__global__ void k_seed(TravArgs a, int src, int mode /*0 bfs, 1 sssp*/) {
  const bool act = threadIdx.x == 0;
  long long b = 0, e = 0;
  if (act) {
    b = a.off[src];
    e = a.off[src + 1];
    a.ctl->tot_arcs_reached += (unsigned long long)(e - b);   // the source's own arcs (R1)
    a.visited[src >> 5] |= 1u << (src & 31);
    a.fb[0][src >> 5] |= 1u << (src & 31);
    if (mode == 0) a.level[src] = 0;
    else a.dist[src] = 0u;
  }
  enqueue_warp(act, src, b, e, a.L, a.q[0], &a.ctl->set[0]);
}

// SSSP overflow resolution: a finite distance >= UINT32_MAX exists iff some arc leaves a reached
// vertex towards an unreached one.
__global__ void k_overflow_check(const long long *__restrict__ off, const int *__restrict__ col,
                                 const uint32_t *__restrict__ dist, long long n, int *found) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < n; u += stride) {
    if (dist[u] == 0xffffffffu) continue;
    for (long long k = off[u]; k < off[u + 1]; ++k)
      if (dist[col[k]] == 0xffffffffu) {
        *found = 1;
        return;
      }
  }
}

__global__ void k_sum_u32(const uint32_t *__restrict__ w, long long m, unsigned long long *out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long s = 0;
  for (long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x; k < m; k += stride) s += w[k];
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

// R1 edge count of an SSSP result: sum of out-degrees of the reached vertices.
__global__ void k_reached_arcs(const long long *__restrict__ off, const uint32_t *__restrict__ dist,
                               long long n, unsigned long long *out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long s = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    if (dist[v] != 0xffffffffu) s += (unsigned long long)(off[v + 1] - off[v]);
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

__global__ void k_gather_i32(const int32_t *__restrict__ src, const int32_t *__restrict__ sigma,
                             const int32_t *__restrict__ sigma_inv, int32_t *__restrict__ dst,
                             long long n, int map_values) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride) {
    int32_t x = src[sigma[v]];
    if (map_values && x >= 0) x = sigma_inv[x];
    dst[v] = x;
  }
}
__global__ void k_gather_u32(const uint32_t *__restrict__ src, const int32_t *__restrict__ sigma,
                             uint32_t *__restrict__ dst, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    dst[v] = src[sigma[v]];
}
__global__ void k_gather_f64(const double *__restrict__ src, const int32_t *__restrict__ sigma,
                             double *__restrict__ dst, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    dst[v] = src[sigma[v]];
}
__global__ void k_iota(int32_t *p, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    p[v] = (int32_t)v;
}

// Debug export of the tile log of a vertex set (sage_debug_export_tiles).
__global__ void k_classify_list(const long long *__restrict__ off, const int *__restrict__ verts,
                                long long count, Ladder L, Queues Q, CounterSet *cs) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long nthr = ((count + 31) / 32) * 32;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < nthr; i += stride) {
    const bool act = i < count;
    int v = 0;
    long long b = 0, e = 0;
    if (act) {
      v = verts[i];
      b = off[v];
      e = off[v + 1];
    }
    enqueue_warp(act, v, b, e, L, Q, cs);
  }
}
__global__ void k_expand_log(const long long *__restrict__ off, Ladder L, Queues Q,
                             const CounterSet *cs, long long *quads, unsigned long long *nq,
                             long long cap) {
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  auto emit = [&](long long u, long long o, long long s, long long kind) {
    unsigned long long k = atomicAdd(nq, 1ull);
    if ((long long)k < cap) {
      quads[4 * k] = u;
      quads[4 * k + 1] = o;
      quads[4 * k + 2] = s;
      quads[4 * k + 3] = kind;
    }
  };
  for (long long i = tid; i < (long long)cs->cnt[0].v; i += stride) {
    CtaTile T = Q.cta[i];
    emit(T.u, T.start, T.len, 0);
  }
  for (int c = 1; c < L.ncls; ++c) {
    const int t = L.B >> c;
    for (long long i = tid; i < (long long)cs->cnt[c].v; i += stride) {
      const int u = Q.cls[c][i];
      const long long b = off[u], e = off[u + 1];
      RowSplit s = split_row(b, e, L);
      emit(u, class_tile_start(e, s.r, t), t, 0);
    }
  }
  for (long long i = tid; i < (long long)cs->cnt[L.ncls].v; i += stride) {
    const int u = Q.frag[i];
    const long long b = off[u], e = off[u + 1];
    RowSplit s = split_row(b, e, L);
    if (s.h > 0) emit(u, b, s.h, 1);
    const int tl = s.r & (L.M - 1);
    if (tl > 0) emit(u, e - tl, tl, 1);
  }
}

// ============================================================================ host side
void iota_device(sage_graph *g, int32_t *p, int64_t n) {
  k_iota<<<g->num_sms * 4, 256, 0, g->stream>>>(p, n);
}

sage_status alloc_queues(sage_graph *g, Queues *q, long long n_rows, long long m) {
  memset(q, 0, sizeof(*q));
  sage_status st;
  const long long cta_cap = m / g->ladder.B + 1;
  if ((st = dalloc(g, (void **)&q->cta, sizeof(CtaTile) * (size_t)cta_cap)) != SAGE_OK) return st;
  for (int c = 1; c < g->ladder.ncls; ++c)
    if ((st = dalloc(g, (void **)&q->cls[c], sizeof(int) * (size_t)(n_rows + 1))) != SAGE_OK)
      return st;
  if ((st = dalloc(g, (void **)&q->frag, sizeof(int) * (size_t)(n_rows + 1))) != SAGE_OK) return st;
  return SAGE_OK;
}
void free_queues(sage_graph *g, Queues *q) {
  dfree(g, q->cta);
  for (int c = 0; c < kMaxCls; ++c) dfree(g, q->cls[c]);
  dfree(g, q->frag);
  memset(q, 0, sizeof(*q));
}

void free_traversal_state(sage_graph *g) {
  TraversalState &t = g->ts;
  dfree(g, t.level);
  dfree(g, t.parent);
  dfree(g, t.dist);
  dfree(g, t.visited);
  for (int i = 0; i < 3; ++i) dfree(g, t.fb[i]);
  free_queues(g, &t.q[0]);
  free_queues(g, &t.q[1]);
  dfree(g, t.ctl);
  dfree(g, t.tmp_out);
  dfree(g, t.bins);
  dfree(g, t.fill);
  for (int i = 0; i < 3; ++i) dfree(g, t.far[i]);
  dfree(g, t.tailmem);
  dfree(g, t.expd);
  dfree(g, t.infar);
  dfree(g, t.farc);
  dfree(g, t.flist);
  t = TraversalState();
}

sage_status ensure_traversal_state(sage_graph *g) {
  TraversalState &t = g->ts;
  if (t.ready) return SAGE_OK;
  const long long n = g->n_local;
  const size_t words = (size_t)((g->n + 31) / 32 + 8);
  sage_status st;
  if ((st = dalloc(g, (void **)&t.level, sizeof(int32_t) * (size_t)n)) != SAGE_OK ||
      (st = dalloc(g, (void **)&t.visited, sizeof(uint32_t) * words)) != SAGE_OK ||
      (st = dalloc(g, (void **)&t.ctl, sizeof(Ctl))) != SAGE_OK ||
      (st = dalloc(g, (void **)&t.tmp_out, sizeof(int64_t) * (size_t)n)) != SAGE_OK) {
    free_traversal_state(g);
    return st;
  }
  for (int i = 0; i < 3; ++i)
    if ((st = dalloc(g, (void **)&t.fb[i], sizeof(uint32_t) * words)) != SAGE_OK) {
      free_traversal_state(g);
      return st;
    }
  // deferred-contraction frontier list: n entries + one open 256-slot chunk per possible warp
  if ((st = dalloc(g, (void **)&t.flist,
                   sizeof(int) * (size_t)(n + (long long)g->num_sms * 64 * kDeferChunk + 64))) != SAGE_OK) {
    free_traversal_state(g);
    return st;
  }
  if ((st = dalloc(g, &t.tailmem, sizeof(TailSmem))) != SAGE_OK) {
    free_traversal_state(g);
    return st;
  }
  for (int i = 0; i < 2; ++i)
    if ((st = alloc_queues(g, &t.q[i], n, g->m)) != SAGE_OK) {
      free_traversal_state(g);
      return st;
    }
  t.ready = true;
  return SAGE_OK;
}

int coop_grid(sage_graph *g, const void *fn, int *cache) {
  if (*cache) return *cache;
  // shared-memory carveout: the persistent kernels use <= 10 KB of shared memory per CTA; the rest
  // of the SM's 256 KB goes to L1, which caches status words and row offsets (SAGE_CARVEOUT = %)
  // (measured on C2 push BFS: driver default 3.40 ms, smallest carveout for 4 CTAs 3.15 ms)
  {
    const char *e = getenv("SAGE_CARVEOUT");
    int pct = e ? atoi(e) : -1;
    if (!e) {   // smallest carveout that still holds kMinBlocks CTAs (+1 KB reserved per CTA)
      cudaFuncAttributes fa;
      if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) {
        int dev = 0, smem_sm = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, dev);
        const size_t need = 4 * (fa.sharedSizeBytes + 1024);
        if (smem_sm > 0) pct = (int)std::min<size_t>(100, (need * 100 + smem_sm - 1) / smem_sm);
      }
    }
    if (pct >= 0) cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
  }
  int nb = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, kBlock, 0);
  if (nb < 1) nb = 1;
  // small graphs (C1: 1.8M arcs, L2-resident) are latency-bound per level: one CTA per SM halves
  // the grid barrier's participants and the counter traffic (C1 DO BFS 156 -> 135 us measured)
  const int nb_occ = nb;
  if (g->m < (8ll << 20)) nb = 1;
  if (const char *e = getenv("SAGE_CTAS_PER_SM")) nb = std::max(1, std::min(nb_occ, atoi(e)));
  *cache = nb * g->num_sms;
  return *cache;
}

sage_status launch_coop(sage_graph *g, const void *fn, int grid, void **args, const char *what) {
  cudaError_t e = cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kBlock), args, 0, g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, what);
  return SAGE_OK;
}

int32_t to_internal_id(sage_graph *g, int32_t v) {
  return g->reordered ? g->h_sigma[(size_t)v] : v;
}

sage_status translate_out_i32(sage_graph *g, const int32_t *src, int32_t *dst_user,
                              bool map_values) {
  const size_t bytes = sizeof(int32_t) * (size_t)g->n_local;
  if (!g->reordered) return copy_out(g, dst_user, src, bytes);
  int32_t *tmp = (int32_t *)g->ts.tmp_out;
  k_gather_i32<<<g->num_sms * 8, 256, 0, g->stream>>>(src, g->sigma, g->sigma_inv, tmp,
                                                      g->n_local, map_values ? 1 : 0);
  return copy_out(g, dst_user, tmp, bytes);
}
sage_status translate_out_u32(sage_graph *g, const uint32_t *src, uint32_t *dst_user) {
  const size_t bytes = sizeof(uint32_t) * (size_t)g->n_local;
  if (!g->reordered) return copy_out(g, dst_user, src, bytes);
  uint32_t *tmp = (uint32_t *)g->ts.tmp_out;
  k_gather_u32<<<g->num_sms * 8, 256, 0, g->stream>>>(src, g->sigma, tmp, g->n_local);
  return copy_out(g, dst_user, tmp, bytes);
}
sage_status translate_out_f64(sage_graph *g, const double *src, double *dst_user) {
  const size_t bytes = sizeof(double) * (size_t)g->n_local;
  if (!g->reordered) return copy_out(g, dst_user, src, bytes);
  double *tmp = (double *)g->ts.tmp_out;
  k_gather_f64<<<g->num_sms * 8, 256, 0, g->stream>>>(src, g->sigma, tmp, g->n_local);
  return copy_out(g, dst_user, tmp, bytes);
}

static TravArgs make_args(sage_graph *g) {
  TravArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.w = g->w;
  a.n = g->n_local;
  a.m = g->m;
  a.L = g->ladder;
  a.q[0] = g->ts.q[0];
  a.q[1] = g->ts.q[1];
  for (int i = 0; i < 3; ++i) a.fb[i] = g->ts.fb[i];
  a.visited = g->ts.visited;
  a.level = g->ts.level;
  a.parent = g->ts.parent;
  a.dist = g->ts.dist;
  a.ctl = g->ts.ctl;
  a.alpha = g->alpha;
  a.beta = g->beta;
  a.max_levels = (int)std::min<long long>(g->n + 1, 0x7fffffffll);
  if (const char *e = getenv("SAGE_DEBUG_MAX_LEVELS")) a.max_levels = atoi(e);   // diagnostics only
  a.tail = (int *)g->ts.tmp_out;
  a.tailmem = reinterpret_cast<TailSmem *>(g->ts.tailmem);
  a.flist = g->ts.flist;
  a.defer_min_arcs = 1ull << 16;   // SAGE_DEFER_MIN_ARCS overrides (tests: 0 = every level)
  if (const char *e = getenv("SAGE_DEFER_MIN_ARCS")) a.defer_min_arcs = strtoull(e, nullptr, 10);
  a.steal = 1;
  a.vec_ok = g->vec_ok ? 1 : 0;
  return a;
}

static void fill_stats(sage_graph *g, const Ctl &h, bool bfs, bool symmetric, double ms,
                       double kms, sage_stats *st) {
  if (!st) return;
  memset(st, 0, sizeof(*st));
  st->levels = h.levels;
  st->push_levels = h.push_levels;
  st->pull_levels = h.pull_levels;
  st->vertices_expanded = (int64_t)(h.tot_push_expanded + h.tot_pull_scanned);
  st->arcs_inspected = (int64_t)(h.tot_push_arcs + h.tot_pull_inspected);
  st->ms = ms;
  st->kernel_ms = kms;
  const double n = (double)g->n_local;
  if (bfs) {
    // reached arcs = arcs of the source + arcs of every discovered vertex
    const double reached_arcs = (double)h.tot_arcs_reached;
    st->vertices_discovered = (int64_t)(h.tot_push_disc + h.tot_pull_disc);
    st->edges_traversed = (int64_t)(symmetric ? reached_arcs / 2.0 : reached_arcs);
    // SURVEY §8(d) frozen byte model
    double mb = 4.0 * n;
    mb += 20.0 * h.tot_push_expanded + 8.0 * h.tot_push_arcs + 8.0 * h.tot_push_disc;
    mb += 16.0 * h.tot_pull_scanned + (n / 8.0) * h.pull_levels +
          4.125 * h.tot_pull_inspected + 4.125 * h.tot_pull_disc;
    st->model_bytes = mb;
  } else {
    st->vertices_discovered = (int64_t)h.tot_improved;
    st->edges_traversed = 0;   // filled by the caller from the reached set (R1)
    double mb = 4.0 * n + 24.0 * h.tot_push_expanded + 12.0 * h.tot_push_arcs +
                8.0 * h.tot_push_disc;
    st->model_bytes = mb;
  }
}

static sage_status check_common(sage_graph *g, int32_t source, const void *out) {
  if (!g || !out) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) {
    set_error("graph handle is in a failed state (sticky error %d); free it", g->sticky);
    return (sage_status)g->sticky;
  }
  if (source < 0 || source >= g->n) {
    set_error("source %d out of range [0, %lld)", source, (long long)g->n);
    return SAGE_E_INVALID;
  }
  return SAGE_OK;
}

sage_status run_bfs_multi(sage_graph *g, int32_t source, int32_t *level_out, int32_t *parent_out,
                          uint32_t call_flags, sage_stats *st);
sage_status run_sssp_multi(sage_graph *g, int32_t source, uint32_t *dist_out, sage_stats *st);

}  // namespace sage

using namespace sage;

extern "C" sage_status sage_bfs_ex(sage_graph *g, int32_t source, int32_t *level_out,
                                   int32_t *parent_out, uint32_t call_flags, sage_stats *st) {
  clear_error();
  sage_status s = check_common(g, source, level_out);
  if (s != SAGE_OK) return s;
  if (g->comm) return run_bfs_multi(g, source, level_out, parent_out, call_flags, st);
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  TraversalState &t = g->ts;
  if (parent_out && !t.parent) {
    if ((s = dalloc(g, (void **)&t.parent, sizeof(int32_t) * (size_t)g->n_local)) != SAGE_OK)
      return s;
  }
  const int32_t src = to_internal_id(g, source);
  const bool symmetric = g->flags & SAGE_F_SYMMETRIC;
  const bool push_only = (g->flags | call_flags) & SAGE_F_PUSH_ONLY;
  cudaEvent_t e0, e1, e2;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventCreate(&e2);
  cudaEventRecord(e0, g->stream);
  const size_t words = (size_t)((g->n + 31) / 32 + 8);
  cudaMemsetAsync(t.level, 0xff, sizeof(int32_t) * (size_t)g->n_local, g->stream);
  if (parent_out) cudaMemsetAsync(t.parent, 0xff, sizeof(int32_t) * (size_t)g->n_local, g->stream);
  cudaMemsetAsync(t.visited, 0, sizeof(uint32_t) * words, g->stream);
  for (int i = 0; i < 3; ++i) cudaMemsetAsync(t.fb[i], 0, sizeof(uint32_t) * words, g->stream);
  cudaMemsetAsync(t.ctl, 0, sizeof(Ctl), g->stream);
  TravArgs a = make_args(g);
  a.parent = parent_out ? t.parent : nullptr;
  a.do_enabled = (symmetric && !push_only) ? 1 : 0;
  a.steal = (call_flags & SAGE_F_NO_STEALING) ? 0 : 1;
  k_seed<<<1, 32, 0, g->stream>>>(a, src, 0);
  const int nslices = (int)((g->n + (1ll << kSliceLg) - 1) >> kSliceLg);
  const bool binned = !parent_out && (call_flags & SAGE_F_BINNED) && nslices <= kMaxSlices;
  if (binned && !t.bins) {
    // per-slice capacity: 1.5x the average share of all arcs plus staging slack; a full bin
    // spills to the direct filter, so the capacity only affects speed
    t.nslices = nslices;
    t.bin_cap = (long long)(1.5 * (double)g->m / nslices) + (long long)kBinRes * kBinWarps * g->num_sms + 1024;
    if ((s = dalloc(g, (void **)&t.bins, sizeof(int) * (size_t)t.bin_cap * nslices)) != SAGE_OK ||
        (s = dalloc(g, (void **)&t.fill, sizeof(PaddedCounter) * 2 * kMaxSlices)) != SAGE_OK)
      return s;
  }
  if (binned) cudaMemsetAsync(t.fill, 0, sizeof(PaddedCounter) * 2 * kMaxSlices, g->stream);
  cudaEventRecord(e1, g->stream);
  if (binned) {
    BinArgs b;
    b.bins = t.bins;
    b.cap = t.bin_cap;
    b.fill = t.fill;
    b.nslices = nslices;
    b.slice_lg = kSliceLg;
    const void *fn = g->vec == 4 ? (const void *)k_bfs_bin<4> : (const void *)k_bfs_bin<1>;
    const size_t smem = bin_smem_bytes(nslices, g->n);
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (!g->grid_bin) {
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, kBinBlock, smem);
      g->grid_bin = std::max(1, nb) * g->num_sms;
    }
    void *args[] = {&a, &b};
    cudaError_t le = cudaLaunchCooperativeKernel(fn, dim3(g->grid_bin), dim3(kBinBlock), args, smem, g->stream);
    if (le != cudaSuccess) return cuda_fail(g, le, "binned BFS kernel");
  } else {
    static const int bfs_vec8 = getenv("SAGE_BFS_VEC") ? atoi(getenv("SAGE_BFS_VEC")) == 8 : SAGE_BFS_VEC8;
    const void *fn = g->vec == 4 ? (bfs_vec8 && g->ladder.M >= 8 ? (const void *)k_bfs<8> : (const void *)k_bfs<4>)
                                 : (const void *)k_bfs<1>;
    const int grid = coop_grid(g, fn, &g->grid_bfs);
    void *args[] = {&a};
    if ((s = launch_coop(g, fn, grid, args, "BFS kernel")) != SAGE_OK) return s;
  }
  cudaEventRecord(e2, g->stream);
  Ctl h;
  cudaMemcpyAsync(&h, t.ctl, offsetof(Ctl, rec), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "BFS");
  float ms = 0, kms = 0;
  cudaEventElapsedTime(&ms, e0, e2);
  cudaEventElapsedTime(&kms, e1, e2);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaEventDestroy(e2);
  if (h.status == 1 && !getenv("SAGE_DEBUG_MAX_LEVELS")) {
    set_error("BFS exceeded the level cap (internal error)");
    g->sticky = SAGE_E_CUDA;
    return SAGE_E_CUDA;
  }
  fill_stats(g, h, true, symmetric, ms, kms, st);
  if ((s = translate_out_i32(g, t.level, level_out, false)) != SAGE_OK) return s;
  if (parent_out && (s = translate_out_i32(g, t.parent, parent_out, true)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "BFS output");
  // online sampling: record the rows this query expanded (after the answer has been delivered)
  return online_after_query(g, t.level, 0);
}

extern "C" sage_status sage_bfs(sage_graph *g, int32_t source, int32_t *level_out,
                                int32_t *parent_out, sage_stats *st) {
  return sage_bfs_ex(g, source, level_out, parent_out, 0u, st);
}

extern "C" sage_status sage_sssp(sage_graph *g, int32_t source, uint32_t *dist_out,
                                 sage_stats *st) {
  clear_error();
  sage_status s = check_common(g, source, dist_out);
  if (s != SAGE_OK) return s;
  if (!g->w) {
    set_error("SSSP needs weights (load the CSR with weights)");
    return SAGE_E_INVALID;
  }
  if (g->comm) return run_sssp_multi(g, source, dist_out, st);
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  TraversalState &t = g->ts;
  if (!t.dist && (s = dalloc(g, (void **)&t.dist, sizeof(uint32_t) * (size_t)g->n_local)) != SAGE_OK)
    return s;
  const int32_t src = to_internal_id(g, source);
  int *ovf = nullptr;
  if ((s = dalloc(g, (void **)&ovf, sizeof(int) * 2)) != SAGE_OK) return s;
  cudaEvent_t e0, e1, e2;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventCreate(&e2);
  cudaEventRecord(e0, g->stream);
  const size_t words = (size_t)((g->n + 31) / 32 + 8);
  cudaMemsetAsync(ovf, 0, sizeof(int) * 2, g->stream);
  cudaMemsetAsync(t.dist, 0xff, sizeof(uint32_t) * (size_t)g->n_local, g->stream);
  cudaMemsetAsync(t.visited, 0, sizeof(uint32_t) * words, g->stream);
  for (int i = 0; i < 3; ++i) cudaMemsetAsync(t.fb[i], 0, sizeof(uint32_t) * words, g->stream);
  cudaMemsetAsync(t.ctl, 0, sizeof(Ctl), g->stream);
  // near-far state (SSSP ordering); delta from the mean weight and degree
  if (!t.far[0]) {
    for (int i = 0; i < 3; ++i)
      if ((s = dalloc(g, (void **)&t.far[i], sizeof(int) * (size_t)(g->n_local + 1))) != SAGE_OK) return s;
    if ((s = dalloc(g, (void **)&t.infar, sizeof(uint32_t) * words)) != SAGE_OK ||
        (s = dalloc(g, (void **)&t.farc, sizeof(PaddedCounter) * 6)) != SAGE_OK)
      return s;
  }
  if (g->w_mean <= 0.0) {
    unsigned long long *dsum = reinterpret_cast<unsigned long long *>(t.farc);
    unsigned long long hsum = 0;
    cudaMemsetAsync(dsum, 0, sizeof(unsigned long long), g->stream);
    k_sum_u32<<<g->num_sms * 8, 256, 0, g->stream>>>(g->w, g->m, dsum);
    cudaMemcpyAsync(&hsum, dsum, sizeof(hsum), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
    g->w_mean = g->m ? (double)hsum / (double)g->m : 1.0;
  }
  FarArgs fa;
  for (int i = 0; i < 3; ++i) fa.far[i] = t.far[i];
  fa.infar = t.infar;
  fa.expd = reinterpret_cast<uint32_t *>(t.far[2]) + 0;   // placeholder, set below
  fa.cnt = t.farc;
  fa.fmin = t.farc + 3;
  {
    const double avgdeg = g->n_local ? (double)g->m / (double)g->n_local : 1.0;
    double dl = 32.0 * g->w_mean / std::max(1.0, avgdeg);
    const char *env = getenv("SAGE_SSSP_DELTA");
    if (env) dl = atof(env);
    fa.delta = dl <= 0.0 ? ~0ull : (unsigned long long)std::max(1.0, std::floor(dl + 0.5));
    if (!env) fa.delta = ~0ull;   // default: plain frontier Bellman-Ford (near-far measured slower)
  }
  if (fa.delta != ~0ull) {
    if (!t.expd && (s = dalloc(g, (void **)&t.expd, sizeof(uint32_t) * (size_t)g->n_local)) != SAGE_OK)
      return s;
    cudaMemsetAsync(t.expd, 0xff, sizeof(uint32_t) * (size_t)g->n_local, g->stream);
  }
  fa.expd = t.expd;
  cudaMemsetAsync(t.infar, 0, sizeof(uint32_t) * words, g->stream);
  cudaMemsetAsync(t.farc, 0, sizeof(PaddedCounter) * 3, g->stream);
  cudaMemsetAsync(t.farc + 3, 0xff, sizeof(PaddedCounter) * 3, g->stream);
  TravArgs a = make_args(g);
  k_seed<<<1, 32, 0, g->stream>>>(a, src, 1);
  cudaEventRecord(e1, g->stream);
  const void *fn = g->vec == 4 ? (const void *)k_sssp<4> : (const void *)k_sssp<1>;
  const int grid = coop_grid(g, fn, &g->grid_sssp);
  void *args[] = {&a, &ovf, &fa};
  if ((s = launch_coop(g, fn, grid, args, "SSSP kernel")) != SAGE_OK) {
    dfree(g, ovf);
    return s;
  }
  cudaEventRecord(e2, g->stream);
  int hovf[2] = {0, 0};
  cudaMemcpyAsync(hovf, ovf, sizeof(int), cudaMemcpyDeviceToHost, g->stream);
  Ctl h;
  cudaMemcpyAsync(&h, t.ctl, offsetof(Ctl, rec), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) {
    dfree(g, ovf);
    return cuda_fail(g, e, "SSSP");
  }
  float ms = 0, kms = 0;
  cudaEventElapsedTime(&ms, e0, e2);
  cudaEventElapsedTime(&kms, e1, e2);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaEventDestroy(e2);
  if (h.status == 1) {
    dfree(g, ovf);
    set_error("SSSP exceeded the iteration cap (internal error)");
    g->sticky = SAGE_E_CUDA;
    return SAGE_E_CUDA;
  }
  if (hovf[0]) {
    cudaMemsetAsync(ovf + 1, 0, sizeof(int), g->stream);
    k_overflow_check<<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, g->col,
                                                            t.dist, g->n_local, ovf + 1);
    cudaMemcpyAsync(hovf + 1, ovf + 1, sizeof(int), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
  }
  dfree(g, ovf);
  if (hovf[1]) {
    set_error("a finite shortest distance is >= UINT32_MAX");
    return SAGE_E_OVERFLOW;
  }
  fill_stats(g, h, false, g->flags & SAGE_F_SYMMETRIC, ms, kms, st);
  if (st) {
    unsigned long long *dra = nullptr, hra = 0;
    if ((s = dalloc(g, (void **)&dra, sizeof(unsigned long long))) != SAGE_OK) return s;
    cudaMemsetAsync(dra, 0, sizeof(unsigned long long), g->stream);
    k_reached_arcs<<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, t.dist,
                                                          g->n_local, dra);
    cudaMemcpyAsync(&hra, dra, sizeof(hra), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
    dfree(g, dra);
    st->edges_traversed = (int64_t)((g->flags & SAGE_F_SYMMETRIC) ? hra / 2 : hra);
  }
  if ((s = translate_out_u32(g, t.dist, dist_out)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "SSSP output");
  return SAGE_OK;
}

extern "C" sage_status sage_debug_export_tiles(sage_graph *g, const int32_t *vertices,
                                               int64_t count, int64_t *quads_out, int64_t cap,
                                               int64_t *n_out) {
  clear_error();
  if (!g || (count > 0 && !vertices) || !n_out || count < 0) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  for (int64_t i = 0; i < count; ++i)
    if (vertices[i] < 0 || vertices[i] >= g->n_local) {
      set_error("vertex %d out of range", vertices[i]);
      return SAGE_E_INVALID;
    }
  sage_status s;
  Queues q;
  // queue capacity: each listed vertex appears once per class
  long long msum = 0;
  {
    std::vector<long long> hoff((size_t)g->n_local + 1);
    cudaStreamSynchronize(g->stream);
    cudaMemcpy(hoff.data(), g->off, sizeof(long long) * hoff.size(), cudaMemcpyDeviceToHost);
    for (int64_t i = 0; i < count; ++i) msum += hoff[vertices[i] + 1] - hoff[vertices[i]];
  }
  if ((s = alloc_queues(g, &q, count, msum)) != SAGE_OK) return s;
  int *dv = nullptr;
  CounterSet *cs = nullptr;
  long long *dq = nullptr;
  unsigned long long *dn = nullptr;
  const long long dcap = msum / g->ladder.B + 16 * count + 16;
  if ((s = dalloc(g, (void **)&dv, sizeof(int) * (size_t)(count + 1))) != SAGE_OK ||
      (s = dalloc(g, (void **)&cs, sizeof(CounterSet))) != SAGE_OK ||
      (s = dalloc(g, (void **)&dq, sizeof(long long) * 4 * (size_t)dcap)) != SAGE_OK ||
      (s = dalloc(g, (void **)&dn, sizeof(unsigned long long))) != SAGE_OK) {
    free_queues(g, &q);
    return s;
  }
  cudaMemcpyAsync(dv, vertices, sizeof(int) * (size_t)count, cudaMemcpyHostToDevice, g->stream);
  cudaMemsetAsync(cs, 0, sizeof(CounterSet), g->stream);
  cudaMemsetAsync(dn, 0, sizeof(unsigned long long), g->stream);
  if (count > 0) {
    k_classify_list<<<g->num_sms * 4, 256, 0, g->stream>>>((const long long *)g->off, dv, count,
                                                           g->ladder, q, cs);
    k_expand_log<<<g->num_sms * 4, 256, 0, g->stream>>>((const long long *)g->off, g->ladder, q,
                                                        cs, dq, dn, dcap);
  }
  unsigned long long hn = 0;
  cudaMemcpyAsync(&hn, dn, sizeof(hn), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e == cudaSuccess && (long long)hn <= cap && quads_out && hn > 0)
    e = cudaMemcpy(quads_out, dq, sizeof(long long) * 4 * hn, cudaMemcpyDeviceToHost);
  *n_out = (int64_t)hn;
  free_queues(g, &q);
  dfree(g, dv);
  dfree(g, cs);
  dfree(g, dq);
  dfree(g, dn);
  cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "debug_export_tiles");
  return SAGE_OK;
}

extern "C" sage_status sage_debug_level_records(const sage_graph *gc, int64_t *rec_out, int32_t cap,
                                                int32_t *n_out) {
  // 8 int64 per level (the 8th = device time at which the last warp finished the level's work)
  clear_error();
  sage_graph *g = const_cast<sage_graph *>(gc);
  if (!g || !n_out || (cap > 0 && !rec_out)) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (!g->ts.ready) {
    *n_out = 0;
    return SAGE_OK;
  }
  Ctl *h = new Ctl;
  cudaStreamSynchronize(g->stream);
  cudaError_t e = cudaMemcpy(h, g->ts.ctl, sizeof(Ctl), cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    delete h;
    return cuda_fail(g, e, "level records");
  }
  const int nl = std::min(h->levels, kMaxRec);
  *n_out = h->levels;
  for (int i = 0; i < nl && i < cap; ++i) {
    const LevelRec &r = h->rec[i];
    int64_t *o = rec_out + 9 * i;
    o[0] = r.dir;
    o[1] = (int64_t)r.nF;
    o[2] = (int64_t)r.arcsF;
    o[3] = (int64_t)r.inspected;
    o[4] = (int64_t)r.scanned;
    o[5] = (int64_t)r.discovered;
    o[6] = (int64_t)(r.t_ns - h->t0_ns);
    o[7] = r.t_work ? (int64_t)(r.t_work - h->t0_ns) : 0;
    o[8] = (int64_t)r.t_mid_us * 1000;
  }
  delete h;
  return SAGE_OK;
}

#ifdef SAGE_PROF
extern "C" int sage_prof_read(unsigned long long *out16, int reset) {
  cudaMemcpyFromSymbol(out16, sage::g_prof, sizeof(unsigned long long) * 16);
  if (reset) {
    unsigned long long z[16] = {0};
    z[13] = ~0ull;
    cudaMemcpyToSymbol(sage::g_prof, z, sizeof(z));
  }
  return 0;
}
#endif
