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
// Hub filter (B200 addition): a push level examines the status of every arc's
// target, and on a scale-free graph most arcs of the heavy levels point at a few high-degree
// vertices that are already visited.  A scattered global status read costs one L1TEX wavefront
// per lane (32 per warp instruction) and holds an L1 line while it waits for L2; a shared-memory
// read of a random byte costs ~4 wavefronts per warp instruction.  Each CTA therefore keeps a
// direct-mapped table of visited hubs in shared memory (slot = v & (T-1), entry = (v >> lgT) + 1,
// 0 = empty) and skips the global read when the slot holds v.  The table only ever holds visited
// vertices, so a hit is exact (visited bits only rise); a miss falls back to Alg. 1's test.
// HT selects (lgT, key bits): 1 = (17, 8) and 2 = (16, 16): 128 KB; 3 = (16, 8) and 4 = (15, 16): 64 KB.
template <int HT> struct HubGeom;
template <> struct HubGeom<0> { static constexpr int lgT = 0, kbits = 0, bytes = 0; };
template <> struct HubGeom<1> { static constexpr int lgT = 17, kbits = 8, bytes = 1 << 17; };
template <> struct HubGeom<2> { static constexpr int lgT = 16, kbits = 16, bytes = 2 << 16; };
template <> struct HubGeom<3> { static constexpr int lgT = 16, kbits = 8, bytes = 1 << 16; };
template <> struct HubGeom<4> { static constexpr int lgT = 15, kbits = 16, bytes = 2 << 15; };
__device__ __forceinline__ uint32_t ld_shared_u8(uint32_t addr) {
  uint32_t r;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(r) : "r"(addr));
  return r;
}
__device__ __forceinline__ uint32_t ld_shared_u16(uint32_t addr) {
  uint32_t r;
  asm volatile("ld.shared.u16 %0, [%1];" : "=r"(r) : "r"(addr));
  return r;
}

template <int HT>
struct BfsPushT {
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
  static constexpr bool kDefer = true;   // contraction deferred to a K2' phase
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
  uint32_t ht = 0;     // shared-memory address of the hub table (HT > 0)
  unsigned long long keep = 0;   // L2 evict_last policy of the status loads (made once per level)
  unsigned long long *nfc = nullptr;   // fused tiling: |F| of the next list, counted at discovery

  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }

  // Alg. 1 l.1-6: if dist[nb] = -1 then dist[nb] := dist[fr] + 1; filter_in(nb)
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N],
                                        const uint32_t (&)[N], bool (&in)[N], int) const {
    bool hit[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      hit[j] = false;
      if constexpr (HT > 0) {
        constexpr int lg = HubGeom<HT>::lgT;
        const uint32_t slot = (uint32_t)v[j] & ((1u << lg) - 1u), k1 = ((uint32_t)v[j] >> lg) + 1u;
        if constexpr (HubGeom<HT>::kbits == 8) hit[j] = ld_shared_u8(ht + slot) == k1;
        else hit[j] = ld_shared_u16(ht + 2u * slot) == k1;
      }
    }
    uint32_t wd[N];
#pragma unroll
    for (int j = 0; j < N; ++j)
      wd[j] = (valid && !hit[j]) ? ld_status(visited + (v[j] >> 5), keep) : 0xffffffffu;
    bool need = false;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      need |= !((wd[j] >> (v[j] & 31)) & 1u);
    }
    // on the heavy levels almost every target is already visited: one vote skips the claims
    if (!__any_sync(FULL, need)) return;
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
  // the same filter for N independent elements per lane, each with its own source and validity
  // (the fused fragment gather: lane k takes elements k, k + 32, ... of the chunk's fragments)
  template <int N>
  __device__ __forceinline__ void visit_each(const bool (&valid)[N], const int (&u)[N], const int (&v)[N],
                                             bool (&in)[N]) const {
    bool hit[N];
#pragma unroll
    for (int j = 0; j < N; ++j) {
      hit[j] = false;
      if constexpr (HT > 0) {
        constexpr int lg = HubGeom<HT>::lgT;
        const uint32_t slot = (uint32_t)v[j] & ((1u << lg) - 1u), k1 = ((uint32_t)v[j] >> lg) + 1u;
        if (valid[j]) {
          if constexpr (HubGeom<HT>::kbits == 8) hit[j] = ld_shared_u8(ht + slot) == k1;
          else hit[j] = ld_shared_u16(ht + 2u * slot) == k1;
        }
      }
    }
    uint32_t wd[N];
#pragma unroll
    for (int j = 0; j < N; ++j)
      wd[j] = (valid[j] && !hit[j]) ? ld_status(visited + (v[j] >> 5), keep) : 0xffffffffu;
    bool need = false;
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      need |= !((wd[j] >> (v[j] & 31)) & 1u);
    }
    if (!__any_sync(FULL, need)) return;
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
        if (parent) parent[v[j]] = u[j] + v_base;
        if (fb_next) atomicOr(fb_next + (v[j] >> 5), bit);
      }
    }
  }
};
using BfsPush = BfsPushT<0>;

struct SsspPush {
  struct Src {
    uint32_t du;
  };
  static constexpr bool kWeights = true;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
  static constexpr bool kDefer = true;   // contraction deferred to the K2' phase (see BfsPush)
  int *flist = nullptr;
  unsigned long long *flc = nullptr;
  uint32_t *dist;
  uint32_t *inq_next;   // dedupe bitmap of the next frontier
  int *overflow;
  const Queues *next_q;
  CounterSet *next_cs;

  __device__ __forceinline__ Src src(bool valid, int u, long long, long long) const {
    // dist[u] may have been lowered by another SM in an earlier iteration: read through L2
    return Src{valid ? ldcg(dist + u) : 0xffffffffu};
  }

  // nd = dist[u] + w(u,v); if nd < dist[v]: dist[v] = nd and v enters the next frontier
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
        const uint32_t old = atomicMin(dist + v[j], (uint32_t)nd);
        if ((uint32_t)nd < old) {
          const uint32_t bit = 1u << (v[j] & 31);
          in[j] = !(atomicOr(inq_next + (v[j] >> 5), bit) & bit);
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
  int *fl[2];           // fused runtime tiling: the frontier list of level L is fl[L & 1]
  int src;              // fused path: the source (query init runs inside the kernel)
  HubIns hub;           // hub filter: global table + insert rule (hub.g null = off)
  unsigned long long hub_min_arcs;   // reload the CTA's table before levels with arcs(F) >= this
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
  int wsum[32];
  int nnext;
  unsigned long long anext;
};

// exclusive block scan of x (one value per thread, <= 1024 threads); returns the total
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
  const int nw = blockDim.x >> 5;
  for (int w = 0; w < nw; ++w) {
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
template <bool FUSED>
__device__ void tail_run(const TravArgs &a, int Lstart, TailSmem &ts) {
  Ctl *ctl = a.ctl;
  const int tid = threadIdx.x, lane = (int)lane_id(), warp = tid >> 5;
  int nf = 0;
  if constexpr (FUSED) {
    // ---- the frontier of level Lstart: its list, compacted by the whole grid before the entry
    //      (bfs_body_fused) into the other list buffer, tail_n entries
    const int *fl = a.fl[(Lstart + 1) & 1];
    const long long fc = (long long)ldcg(&ctl->tail_n);
    if (tid == 0) ts.nnext = 0;
    __syncthreads();
    for (long long i = tid; i < fc; i += blockDim.x) {   // order is free: compact with a counter
      const int u = ldcg(fl + i);
      if (u >= 0) {
        const int pos = atomicAdd(&ts.nnext, 1);
        if (pos < kTailV) {
          const long long rb = a.off[u];
          ts.f[0][pos] = u;
          ts.b[0][pos] = rb;
          ts.d[0][pos] = (int)(a.off[u + 1] - rb);
        }
      }
    }
    __syncthreads();
    nf = ts.nnext < kTailV ? ts.nnext : kTailV;
    __syncthreads();
  } else {
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
  }
  // statistics kept in registers of thread 0, written once
  unsigned long long s_exp = 0, s_arcs = 0, s_disc = 0, s_reach = 0;
  int cur = 0;
  int L = Lstart;
  for (;; ++L) {
    // exclusive scan of the frontier's degrees (nf <= kTailV = blockDim: one row per thread)
    int p1;
    const int A = block_scan_excl(tid < nf ? ts.d[cur][tid] : 0, &p1, ts.wsum);
    if constexpr (FUSED) {
      if (L == Lstart && A > kTailE) {   // the entering frontier is too heavy: the grid runs it
        if (tid == 0) {
          ctl->tail_state = 2;
          ctl->tail_resume = Lstart;
        }
        return;
      }
    }
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
      s_reach += FUSED ? (unsigned long long)A : an;
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
  // the frontier grew: hand level L+1's frontier back to the grid (its list, or its tile log)
  constexpr int nctr = sizeof(CounterSet) / sizeof(PaddedCounter);
  if (tid < nctr) {
    reinterpret_cast<PaddedCounter *>(&ctl->set[(L + 1) % 3])[tid].v = 0ull;
    reinterpret_cast<PaddedCounter *>(&ctl->set[(L + 2) % 3])[tid].v = 0ull;
  }
  __threadfence_block();
  __syncthreads();
  if constexpr (FUSED) {
    int *fl = a.fl[(L + 1) & 1];
    for (int i = tid; i < nn; i += blockDim.x) fl[i] = ldcg(a.tail + i);
    if (tid == 0) {
      ctl->set[(L + 1) % 3].flc.v = (unsigned long long)nn;
      ctl->set[(L + 1) % 3].nF.v = (unsigned long long)nn;
    }
  } else {
    for (int base = warp * 32; base < nn; base += blockDim.x) {
      const int i = base + lane;
      const bool act = i < nn;
      enqueue_ids(act, act ? ldcg(a.tail + i) : 0, a.off, a.L, a.q[(L + 1) & 1], &ctl->set[(L + 1) % 3]);
    }
  }
  if (tid == 0) {
    ctl->tail_state = 2;
    ctl->tail_resume = L + 1;
  }
}

// ============================================================================ BFS kernel
// Load the CTA's hub table from the global one (after the K2' phase that inserted into it).
template <int HT>
__device__ __forceinline__ void hub_load(const TravArgs &a, uint8_t *ht) {
  const uint4 *g4 = reinterpret_cast<const uint4 *>(a.hub.g);
  constexpr int nvec = (1 << HubGeom<HT>::lgT) >> 2;
  constexpr uint32_t km = (1u << HubGeom<HT>::kbits) - 1u;
  for (int i = threadIdx.x; i < nvec; i += blockDim.x) {
    const uint4 p = __ldcg(g4 + i);
    const uint32_t k0 = p.x & km, k1 = p.y & km, k2 = p.z & km, k3 = p.w & km;
    if constexpr (HubGeom<HT>::kbits == 8) {
      reinterpret_cast<uint32_t *>(ht)[i] = k0 | (k1 << 8) | (k2 << 16) | (k3 << 24);
    } else {
      reinterpret_cast<uint2 *>(ht)[i] = make_uint2(k0 | (k1 << 16), k2 | (k3 << 16));
    }
  }
}

// The BFS level loop (one persistent cooperative launch per query).  HT > 0: hub filter on (the
// CTA holds the table in `ht`, HubGeom<HT>::bytes of shared memory).
// Query init (a2, Alg. 1 l.2) inside the persistent kernel for the level-log paths (direction-
// optimising BFS: MODE 0, SSSP: MODE 1): the output (level = -1 / dist = UINT32_MAX), parents, the
// visited bitmap and the three frontier bitmaps, the counters and statistics, then the source
// seeded into level 0's log (Tiled Partitioning of its row) — two grid barriers instead of six
// memsets and a seed launch per call.
template <int MODE>
__device__ __forceinline__ void query_init(const TravArgs &a, int *overflow) {
  Ctl *ctl = a.ctl;
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nth = (long long)gridDim.x * blockDim.x;
  const long long n4 = a.n >> 2;
  int4 *out4 = MODE == 0 ? reinterpret_cast<int4 *>(a.level) : reinterpret_cast<int4 *>(a.dist);
  for (long long i = tid; i < n4; i += nth) {
    out4[i] = make_int4(-1, -1, -1, -1);
    if (MODE == 0 && a.parent) reinterpret_cast<int4 *>(a.parent)[i] = make_int4(-1, -1, -1, -1);
  }
  for (long long i = 4 * n4 + tid; i < a.n; i += nth) {
    if (MODE == 0) a.level[i] = -1;
    else a.dist[i] = 0xffffffffu;
    if (MODE == 0 && a.parent) a.parent[i] = -1;
  }
  const long long words = ((a.n + 31) >> 5) + 8;
  for (long long i = tid; i < words; i += nth) {
    a.visited[i] = 0u;
    a.fb[0][i] = 0u;
    a.fb[1][i] = 0u;
    a.fb[2][i] = 0u;
  }
  if (blockIdx.x == 0) {
    constexpr int nctr = sizeof(CounterSet) / sizeof(PaddedCounter);
    for (int i = threadIdx.x; i < 3 * nctr; i += blockDim.x) reinterpret_cast<PaddedCounter *>(ctl->set)[i].v = 0ull;
    for (int i = threadIdx.x; i < 16; i += blockDim.x) ctl->prof[i] = 0ull;
    if (threadIdx.x == 0) {
      ctl->tot_push_expanded = ctl->tot_push_arcs = ctl->tot_push_disc = 0;
      ctl->tot_pull_scanned = ctl->tot_pull_inspected = ctl->tot_pull_disc = 0;
      ctl->tot_arcs_reached = ctl->tot_improved = ctl->tail_levels = 0;
      ctl->levels = ctl->push_levels = ctl->pull_levels = ctl->status = 0;
      ctl->tail_state = ctl->tail_resume = 0;
      ctl->rec[0].t_work = ctl->rec[0].t_mid = 0;
      if (overflow) overflow[0] = 0;
    }
  }
  grid_barrier(&ctl->bar);
  if (blockIdx.x == 0 && threadIdx.x < 32) {   // seed the source's row into level 0's log (one warp)
    const int src = a.src;
    const bool act = threadIdx.x == 0;
    long long b = 0, e = 0;
    if (act) {
      b = a.off[src];
      e = a.off[src + 1];
      ctl->tot_arcs_reached = (unsigned long long)(e - b);   // the source's own arcs (R1)
      a.visited[src >> 5] = 1u << (src & 31);
      a.fb[0][src >> 5] = 1u << (src & 31);
      if (MODE == 0) a.level[src] = 0;
      else a.dist[src] = 0u;
    }
    enqueue_warp(act, src, b, e, a.L, a.q[0], &ctl->set[0]);
  }
  grid_barrier(&ctl->bar);
}

template <int VEC, int HT>
__device__ __forceinline__ void bfs_body(const TravArgs &a, WarpScratch *wsm, typename BfsPushT<HT>::Src (*fsrc)[32],
                                         uint8_t *ht) {
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t0_ns = globaltimer();
  query_init<0>(a, nullptr);
  double mU = (double)a.m - (double)ldcg(&ctl->set[0].arcsF.v);
  int dir = 0;
  unsigned long long prev_nF = 1;
  const long long nwords = (a.n + 31) >> 5;
  if ((threadIdx.x & 31) == 0) {
    wsm[warp].cpos = wsm[warp].cend = 0;
    wsm[warp].ndisc = 0;
  }
  if constexpr (HT > 0) {   // empty table
    for (int i = threadIdx.x; i < HubGeom<HT>::bytes / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(ht)[i] = 0u;
  }
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();   // block 0: record_level(L-1) finished before set (L+2)%3 is zeroed
    zero_counterset(&ctl->set[(L + 2) % 3]);
    if (blockIdx.x == 0 && threadIdx.x == 0 && L + 1 < kMaxRec) ctl->rec[L + 1].t_work = ctl->rec[L + 1].t_mid = 0;
    uint32_t *fbc = a.fb[L % 3], *fbn = a.fb[(L + 1) % 3];
    if (a.do_enabled) clear_words(a.fb[(L + 2) % 3], nwords);
    if (dir == 0) {
      if constexpr (HT > 0) {
        if (ldcg(&cur->arcsF.v) >= a.hub_min_arcs) {
          hub_load<HT>(a, ht);
          __syncthreads();
        }
      }
      BfsPushT<HT> f;
      f.keep = policy_evict_last();
      f.visited = a.visited;
      f.level = a.level;
      f.parent = a.parent;
      f.fb_next = a.do_enabled ? fbn : nullptr;
      f.next_level = L + 1;
      f.v_base = 0;
      f.next_q = &a.q[(L + 1) & 1];
      f.next_cs = nxt;
      f.flist = a.flist;
      f.flc = &nxt->flc.v;
      if constexpr (HT > 0) f.ht = (uint32_t)__cvta_generic_to_shared(ht);
      consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc[warp], a.vec_ok,
                       a.steal != 0);
    } else {
      pull_level(a, L + 1, fbc, fbn, a.q[(L + 1) & 1], cur, nxt, &wsm[warp]);
    }
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    if (blockIdx.x == 0 && threadIdx.x == 0 && L < kMaxRec) ctl->rec[L].t_mid = globaltimer();
    if (classify_deferred(a.off, a.flist, &nxt->flc.v, a.L, a.q[(L + 1) & 1], nxt, a.hub))
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
          tail_run<false>(a, L + 1, *a.tailmem);
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

// ============================================================================ fused runtime tiling
#ifndef SAGE_FUSED_PACK_SMALL
#define SAGE_FUSED_PACK_SMALL 0   // A/B: 1 = the small-graph fused kernel packs the classes (C1: 207 vs 204 us)
#endif
#ifndef SAGE_FUSED_PACK
#define SAGE_FUSED_PACK 0
#endif
#ifndef SAGE_FUSED_LOGC
#define SAGE_FUSED_LOGC 2   // classes logged for phase B (1 = CTA tiles only; 2 = + the B/2 tiles)
#endif
// Push-only BFS (the configuration of the headline): Tiled Partitioning runs INSIDE the consumer,
// as Alg. 2's runtime tiling does (the expand kernel splits each frontier vertex's
// adjacency list into tiles when it reaches it), instead of as a separate K2' grid phase with its
// own barrier that re-reads every discovered vertex's row offsets twice.  Per level L:
//   phase A: every warp takes 32-entry chunks of the level's frontier list (ticket cur->ftk),
//            loads the rows once, and splits each row (split_row): CTA tiles (>= B) go to the
//            level's CTA-tile log (device-visible, consumed with stealing in phase B); the
//            sub-CTA class tiles t = B/2 .. M are consumed right away by lane groups of t/VEC
//            lanes (tps tiles per warp step, like consume_log); the fragments (< M) by the warp
//            scan-gather.  Filtered-in vertices are appended to level L+1's list.
//   grid barrier;
//   phase B: the CTA tiles (hub rows, the load imbalance Resident Tile Stealing exists for) are
//            consumed by the stealing consumer (consume_log on class 0 only); one more barrier.
// |F| of the next list is counted at discovery; arcs(F) of the level in phase A.  The tile log
// (a3/a4) stays the same decomposition (tests: sage_debug_export_tiles vs the oracle).
// Hub table refresh while a level runs: the frontier's hubs are inserted into the global table as
// phase A reaches them, and every warp copies its 1/(warps per CTA) share of the table into the
// CTA's shared copy every kRefreshChunks chunks.  Entries are single bytes / aligned shorts and
// only ever change from one visited vertex to another (or from empty), so readers need no sync.
constexpr int kRefreshChunks = 16;
template <int HT>
__device__ __forceinline__ void hub_refresh_share(const TravArgs &a, uint32_t ht_s) {
  constexpr int nvec = (1 << HubGeom<HT>::lgT) >> 2;   // 4 slots per uint4 of the global table
  constexpr uint32_t km = (1u << HubGeom<HT>::kbits) - 1u;
  const int nw = blockDim.x >> 5, w = threadIdx.x >> 5;
  const int per = (nvec + nw - 1) / nw;
  const uint4 *g4 = reinterpret_cast<const uint4 *>(a.hub.g);
  for (int i = w * per + (int)lane_id(); i < (w + 1) * per && i < nvec; i += 32) {
    const uint4 p = __ldcg(g4 + i);
    const uint32_t k0 = p.x & km, k1 = p.y & km, k2 = p.z & km, k3 = p.w & km;
    if constexpr (HubGeom<HT>::kbits == 8) {
      asm volatile("st.shared.u32 [%0], %1;" ::"r"(ht_s + 4u * i), "r"(k0 | (k1 << 8) | (k2 << 16) | (k3 << 24)));
    } else {
      asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(ht_s + 8u * i), "r"(k0 | (k1 << 16)), "r"(k2 | (k3 << 16)));
    }
  }
}
template <class F> struct HtOf { static constexpr int value = 0; };
template <int HT> struct HtOf<BfsPushT<HT>> { static constexpr int value = HT; };

// Small frontiers (|F| < kFusedLogAll): one warp per chunk would expand its rows' sub-CTA tiles
// serially; instead phase A only classifies (Tiled Partitioning into the level's log, every class)
// and phase B consumes the whole log with stealing — the latency of a small level is then one
// classification round plus one parallel consume, as with the separate K2' phase.
#ifndef SAGE_LOGALL
#define SAGE_LOGALL 8192
#endif
constexpr unsigned long long kFusedLogAll = SAGE_LOGALL;
template <int VEC, class F>
__device__ __forceinline__ void fused_phase_a(const TravArgs &a, const F &f, CounterSet *cur, const int *fl_in,
                                              const Queues &Q, WarpScratch *ws, typename F::Src *fsrc,
                                              int &bcnt, bool log_all) {
  const unsigned lane = lane_id();
  int chunks = 0;
  const unsigned lt = lanemask_lt();
  const Ladder &L = a.L;
  const unsigned long long pol = policy_evict_first();
  const long long fcount = (long long)ldcg(&cur->flc.v);
  const bool contig_ok = a.vec_ok && (VEC % 4) == 0;
  unsigned long long arcs = 0;
  unsigned hubc = 0;
  for (;;) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(&cur->ftk.v, 32ull);
    base = shfl64(base, 0);
    if ((long long)base >= fcount) break;
    if constexpr (HtOf<F>::value > 0) {
      if (++chunks % kRefreshChunks == 0) hub_refresh_share<HtOf<F>::value>(a, f.ht);
    }
    const long long i = (long long)base + lane;
    const int v = i < fcount ? ldcg(fl_in + i) : -1;
    long long b = 0, e = 0;
    if (v >= 0) ld_row_pair(a.off, v, &b, &e);
    const bool act = v >= 0;
    arcs += act ? (unsigned long long)(e - b) : 0ull;
    hubc += (unsigned)hub_insert(a.hub, v, e - b);
    if (log_all) {   // small frontier: classify every tile into the log; phase B consumes it
      enqueue_warp(act, v, b, e, L, Q, cur, false);
      continue;
    }
    RowSplit s{0, 0, 0, 0};
    if (act) s = split_row(b, e, L);
    // (1) CTA tiles -> the level's CTA-tile log (one reservation atomic per chunk)
    {
      unsigned long long q = act ? (unsigned long long)s.q : 0ull;
      unsigned long long incq = q;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(FULL, incq, o);
        if ((int)lane >= o) incq += y;
      }
      const unsigned long long totq = shfl64(incq, 31);
      if (totq) {
        unsigned long long base0 = 0;
        if (lane == 0) base0 = atomicAdd(&cur->cnt[0].v, totq);
        base0 = shfl64(base0, 0);
        if (q > 0 && q <= SAGE_ENQ_LANEQ) {
          const unsigned long long bs = base0 + incq - q;
          for (unsigned long long j = 0; j < q; ++j) st_tile(Q.cta + bs + j, s.b2 + (long long)j * L.B, v, L.B);
        }
        unsigned hm = __ballot_sync(FULL, q > SAGE_ENQ_LANEQ);
        while (hm) {
          const int src = __ffs(hm) - 1;
          hm &= hm - 1;
          const unsigned long long qs = shfl64(q, src);
          const unsigned long long bs = base0 + shfl64(incq, src) - qs;
          const long long b2 = (long long)shfl64((unsigned long long)s.b2, src);
          const int vv = __shfl_sync(FULL, v, src);
          for (unsigned long long j = lane; j < qs; j += 32) st_tile(Q.cta + bs + j, b2 + (long long)j * L.B, vv, L.B);
        }
      }
    }
    // classes below SAGE_FUSED_LOGC go to the log (phase B) in both forms below
#pragma unroll
    for (int c = 1; c < SAGE_FUSED_LOGC; ++c) {
      if (c >= L.ncls) break;
      const unsigned cm = __ballot_sync(FULL, act && (s.r & (L.B >> c)));
      if (!cm) continue;
      unsigned long long b0 = 0;
      if (lane == 0) b0 = atomicAdd(&cur->cnt[c].v, (unsigned long long)__popc(cm));
      b0 = shfl64(b0, 0);
      if (cm & (1u << lane)) Q.cls[c][b0 + __popc(cm & lt)] = v;
    }
    // small graphs (the 256-thread kernel without the hub table): every class's tiles of the chunk
    // are packed into common warp steps, so a level's dependent column-load chains overlap
    // (latency-bound levels); the hub kernel keeps one class at a time (C2: 3.22 vs 2.52 ms)
    constexpr bool kPack = SAGE_FUSED_PACK || (SAGE_FUSED_PACK_SMALL && HtOf<F>::value == 0);
    bool packed = false;
    if constexpr (kPack) {
    // (2) sub-CTA class tiles, consumed here, all classes of the chunk packed into warp steps: tile
    //     k of class c (t = B >> c elements, lpt = t / VEC lanes) takes lanes [base_c + k * lpt, ..)
    //     of the chunk's lane sequence; classes in descending size keep every group aligned.  A
    //     lane finds its class, tile and owner vertex (nth set bit of the class ballot) and reads
    //     the owner's row end / residual by shuffle; each lane loads VEC consecutive elements.
    if (VEC == 4 && contig_ok && (L.B >> 1) <= 32 * VEC) {
      packed = true;
      int cbase[kMaxCls + 1];
      unsigned cms[kMaxCls];
      int tl = 0;
#pragma unroll
      for (int c = 1; c < kMaxCls; ++c) {
        cms[c] = 0;
        cbase[c] = tl;
        if (c < L.ncls && c >= SAGE_FUSED_LOGC) {
          const int t = L.B >> c;
          cms[c] = __ballot_sync(FULL, act && (s.r & t));
          tl += __popc(cms[c]) * (t / VEC);
        }
      }
      cbase[kMaxCls] = tl;
      const int nst = (tl + 31) >> 5;
      auto load_step = [&](int st, int (&vv)[VEC], int &u_out, bool &valid, int &lg) {
        const int g = st * 32 + (int)lane;
        valid = g < tl;
        int c = 1, cb = cbase[1];
        unsigned m = cms[1];
#pragma unroll
        for (int cc = 2; cc < kMaxCls; ++cc)   // unrolled: the arrays stay in registers
          if (cc < L.ncls && g >= cbase[cc]) {
            c = cc;
            cb = cbase[cc];
            m = cms[cc];
          }
        const int t = L.B >> c;
        const int lgl = L.lgB - c - 2;                 // log2(lanes per tile) = log2(t / 4)
        const int rel = g - cb;
        const int k = rel >> lgl, sl = rel & ((1 << lgl) - 1);
        int owner = 0, kk = k;
#pragma unroll
        for (int sh = 16; sh > 0; sh >>= 1) {
          const int cnt = __popc(m & ((1u << sh) - 1u));
          if (kk >= cnt) {
            kk -= cnt;
            m >>= sh;
            owner += sh;
          }
        }
        owner &= 31;
        const long long eo = (long long)shfl64((unsigned long long)e, owner);
        const int ro = __shfl_sync(FULL, s.r, owner);
        u_out = __shfl_sync(FULL, v, owner);
        const long long start = eo - (long long)(ro & (2 * t - 1));
        int4 c4 = make_int4(0, 0, 0, 0);
        if (valid) c4 = ld_col4(a.col + start + 4ll * sl, pol);
        vv[0] = c4.x; vv[1 % VEC] = c4.y; vv[2 % VEC] = c4.z; vv[3 % VEC] = c4.w;
        lg = 1 << lgl;
      };
      int vn[VEC], un = 0, lgn = 1;
      bool vdn = false;
      if (nst) load_step(0, vn, un, vdn, lgn);
      for (int st = 0; st < nst; ++st) {
        int vv[VEC];
        uint32_t ww[VEC];
#pragma unroll
        for (int j = 0; j < VEC; ++j) {
          vv[j] = vn[j];
          ww[j] = 0u;
        }
        const int u = un, lg = lgn;
        const bool valid = vdn;
        if (st + 1 < nst) load_step(st + 1, vn, un, vdn, lgn);
        typename F::Src sc = f.src(valid, u, 0, 0);
        bool in[VEC];
        f.template visit<VEC>(valid, sc, vv, ww, in, lg);
#pragma unroll
        for (int j = 0; j < VEC; ++j) push_filtered(f, in[j], vv[j], ws, bcnt, a.off, L);
      }
    }
    }
    if (!packed) {
    // (2) sub-CTA class tiles, consumed here: the class members' tile starts and sources are
    //     staged in shared memory, then lane groups of t/VEC lanes take one tile each per step.
    //     Classes below SAGE_FUSED_LOGC are logged for phase B's stealing instead (A/B knob: a
    //     chunk's longest serial work shrinks from 32 x (B-1) to 32 x (B/2^LOGC - 1) elements).
    for (int c = 1; c < L.ncls; ++c) {
      const int t = L.B >> c;
      const unsigned cm = __ballot_sync(FULL, act && (s.r & t));
      if (!cm || c < SAGE_FUSED_LOGC) continue;   // (logged above)
      const int nt = __popc(cm);
      __syncwarp();
      if (cm & (1u << lane)) {
        const int r = __popc(cm & lt);
        ws->hb[r] = class_tile_start(e, s.r, t);
        fsrc[r] = f.src(true, v, b, e);
      }
      __syncwarp();
      const int lpt = (t / VEC) < 32 ? (t / VEC) : 32;
      const int tps = 32 / lpt;
      const int spt = (t / VEC) > 32 ? (t / (32 * VEC)) : 1;
      const int lg_spt = __ffs(spt) - 1;
      const int sub = lane / lpt, sl = lane % lpt;
      const bool contiguous = lpt < 32 && contig_ok;
      const int nst = ((nt + tps - 1) / tps) << lg_spt;
      int vn[VEC];
      uint32_t wn[VEC];
      auto load_step = [&](int st, int (&vv)[VEC], uint32_t (&ww)[VEC]) {
        const int k = ((st >> lg_spt) * tps) + sub;
        const bool valid = k < nt;
        const long long start = ws->hb[valid ? k : 0];
        if (contiguous) {
          const long long p0 = start + (long long)sl * VEC;
#pragma unroll
          for (int qq = 0; qq < (VEC + 3) / 4; ++qq) {
            int4 c4 = make_int4(0, 0, 0, 0);
            if (valid) c4 = ld_col4(a.col + p0 + 4 * qq, pol);
            vv[(4 * qq) % VEC] = c4.x; vv[(4 * qq + 1) % VEC] = c4.y;
            vv[(4 * qq + 2) % VEC] = c4.z; vv[(4 * qq + 3) % VEC] = c4.w;
          }
        } else {
          const long long p0 = start + (long long)(st & (spt - 1)) * (lpt * VEC) + sl;
#pragma unroll
          for (int j = 0; j < VEC; ++j) vv[j] = valid ? ld_col(a.col + p0 + j * lpt, pol) : 0;
        }
#pragma unroll
        for (int j = 0; j < VEC; ++j) ww[j] = 0u;
      };
      load_step(0, vn, wn);
      for (int st = 0; st < nst; ++st) {
        int vv[VEC];
        uint32_t ww[VEC];
#pragma unroll
        for (int j = 0; j < VEC; ++j) {
          vv[j] = vn[j];
          ww[j] = wn[j];
        }
        if (st + 1 < nst) load_step(st + 1, vn, wn);
        const int k = ((st >> lg_spt) * tps) + sub;
        const bool valid = k < nt;
        const typename F::Src sc = fsrc[valid ? k : 0];
        bool in[VEC];
        f.template visit<VEC>(valid, sc, vv, ww, in, lpt);
        bool anyin = false;
#pragma unroll
        for (int j = 0; j < VEC; ++j) anyin |= in[j];
        if (__any_sync(FULL, anyin)) {
#pragma unroll
          for (int j = 0; j < VEC; ++j) push_filtered(f, in[j], vv[j], ws, bcnt, a.off, L);
        }
      }
      __syncwarp();
    }
    }
    // (3) fragments (< M, and the aligned head): warp scan-based gather over the chunk's rows
    {
      int hl = 0, tl = 0;
      long long tb = 0;
      if (act) {
        hl = s.h;
        tl = s.r & (L.M - 1);
        tb = e - tl;
      }
      const int fl = hl + tl;
      int inc = fl;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const int y = __shfl_up_sync(FULL, inc, o);
        if ((int)lane >= o) inc += y;
      }
      const int total = __shfl_sync(FULL, inc, 31);
      if (total) {
        __syncwarp();
        ws->pre[lane] = inc - fl;
        ws->hl[lane] = hl;
        ws->hb[lane] = b;
        ws->tb[lane] = (int)(tb - b);
        fsrc[lane] = f.src(act, v, b, e);
        __syncwarp();
        // FE elements per lane per round (k0 + j * 32 + lane): FE status reads in flight per lane
        constexpr int FE = 4;
        for (int k0 = 0; k0 < total; k0 += 32 * FE) {
          bool kv[FE];
          int vv[FE], uu[FE];
#pragma unroll
          for (int j = 0; j < FE; ++j) {
            const int k = k0 + j * 32 + (int)lane;
            kv[j] = k < total;
            int o = 0;
            if (kv[j]) {   // largest o with pre[o] <= k
              int lo = 0, hi = 31;
#pragma unroll
              for (int it = 0; it < 5; ++it) {
                const int mid = (lo + hi + 1) >> 1;
                if (ws->pre[mid] <= k) lo = mid; else hi = mid - 1;
              }
              o = lo;
            }
            vv[j] = 0;
            uu[j] = fsrc[o].u;
            if (kv[j]) {
              const int idx = k - ws->pre[o];
              const long long pos = ws->hb[o] + (idx < ws->hl[o] ? idx : ws->tb[o] + (idx - ws->hl[o]));
              vv[j] = ld_col(a.col + pos, pol);
            }
          }
          bool in[FE];
          f.template visit_each<FE>(kv, uu, vv, in);
          bool anyin = false;
#pragma unroll
          for (int j = 0; j < FE; ++j) anyin |= in[j];
          if (__any_sync(FULL, anyin)) {
#pragma unroll
            for (int j = 0; j < FE; ++j) push_filtered(f, in[j], vv[j], ws, bcnt, a.off, L);
          }
        }
        __syncwarp();
      }
    }
  }
  arcs = warp_sum64(arcs);
  if (lane == 0 && arcs) atomicAdd(&cur->arcsF.v, arcs);
  const unsigned long long hc = warp_sum64((unsigned long long)hubc);
  if (lane == 0 && hc) atomicAdd(&cur->hubc.v, hc);
}

// level L's record in the fused path: |F| and arcs(F) of the level itself, discoveries = |F_{L+1}|
__device__ __forceinline__ void record_level_fused(Ctl *ctl, int L, const CounterSet *cur, const CounterSet *nxt) {
  const unsigned long long nF = ldcg(&cur->nF.v), aF = ldcg(&cur->arcsF.v), disc = ldcg(&nxt->nF.v);
  ctl->tot_push_expanded += nF;
  ctl->tot_push_arcs += aF;
  ctl->tot_push_disc += disc;
  ctl->push_levels++;
  ctl->tot_arcs_reached += aF;
  ctl->tot_improved += disc;
  if (L < kMaxRec) {
    LevelRec &r = ctl->rec[L];
    r.dir = 0;
    r.nF = nF;
    r.arcsF = aF;
    r.inspected = aF;
    r.scanned = 0;
    r.discovered = disc;
    r.t_ns = globaltimer();
  }
  ctl->levels = L + 1;
}

// Push-only BFS level loop with the fused runtime tiling.
constexpr long long kTailCompactGrid = 2048;   // list slots above which the grid compacts it
constexpr unsigned long long kHubReloadMinChanges = 256;   // reload the CTA's hub table after such levels
// Profiling builds only (tools/level_isolate.sh): the fused kernel stops after level L, so that the
// counter difference of two builds (L and L-1) is level L alone.  Default -1 = off (dead code).
#ifndef SAGE_BFS_STOP_AFTER
#define SAGE_BFS_STOP_AFTER -1
#endif
template <int VEC, int HT>
__device__ __forceinline__ void bfs_body_fused(const TravArgs &a, WarpScratch *wsm,
                                               typename BfsPushT<HT>::Src (*fsrc)[32], uint8_t *ht) {
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  if ((threadIdx.x & 31) == 0) {
    wsm[warp].cpos = wsm[warp].cend = 0;
    wsm[warp].ndisc = 0;
  }
  if constexpr (HT > 0) {
    for (int i = threadIdx.x; i < HubGeom<HT>::bytes / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(ht)[i] = 0u;
  }
  // ---- query init (a2, Alg. 1 l.2) inside the kernel: level = -1 (the source 0), visited = 0 (the
  //      source's bit set), parent = -1, the global hub table and the counters cleared, the source
  //      seeded as level 0's list; one grid barrier instead of six memsets and a seed launch
  {
    const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
    const long long nth = (long long)gridDim.x * blockDim.x;
    const int src = a.src;
    const long long n4 = a.n >> 2;
    for (long long i = tid; i < n4; i += nth) {
      const bool here = (src >> 2) == i;
      const int4 x = make_int4(here && (src & 3) == 0 ? 0 : -1, here && (src & 3) == 1 ? 0 : -1,
                               here && (src & 3) == 2 ? 0 : -1, here && (src & 3) == 3 ? 0 : -1);
      reinterpret_cast<int4 *>(a.level)[i] = x;
      if (a.parent) reinterpret_cast<int4 *>(a.parent)[i] = make_int4(-1, -1, -1, -1);
    }
    for (long long i = 4 * n4 + tid; i < a.n; i += nth) {
      a.level[i] = i == src ? 0 : -1;
      if (a.parent) a.parent[i] = -1;
    }
    const long long words = ((a.n + 31) >> 5) + 8;
    for (long long i = tid; i < words; i += nth) a.visited[i] = i == (src >> 5) ? 1u << (src & 31) : 0u;
    if (a.hub.g)
      for (long long i = tid; i <= (long long)a.hub.mask; i += nth) a.hub.g[i] = 0u;
    if (blockIdx.x == 0) {
      constexpr int nctr = sizeof(CounterSet) / sizeof(PaddedCounter);
      for (int i = threadIdx.x; i < 3 * nctr; i += blockDim.x) reinterpret_cast<PaddedCounter *>(ctl->set)[i].v = 0ull;
      if (threadIdx.x == 0) {
        ctl->tot_push_expanded = ctl->tot_push_arcs = ctl->tot_push_disc = 0;
        ctl->tot_pull_scanned = ctl->tot_pull_inspected = ctl->tot_pull_disc = 0;
        ctl->tot_arcs_reached = ctl->tot_improved = ctl->tail_levels = 0;
        ctl->levels = ctl->push_levels = ctl->pull_levels = ctl->status = 0;
        ctl->tail_state = ctl->tail_resume = 0;
        ctl->rec[0].t_work = ctl->rec[0].t_mid = 0;
        ctl->t0_ns = globaltimer();
      }
      __syncthreads();
      if (threadIdx.x == 0) {
        a.fl[0][0] = src;
        ctl->set[0].flc.v = 1ull;
        ctl->set[0].nF.v = 1ull;
      }
    }
    grid_barrier(&ctl->bar);
  }
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();   // block 0: record of L-1 finished before set (L+2)%3 is zeroed
    if (L > 0) zero_counterset(&ctl->set[(L + 2) % 3]);
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      if (L + 1 < kMaxRec) ctl->rec[L + 1].t_work = ctl->rec[L + 1].t_mid = 0;
      ctl->tail_n = 0;   // (read after this level's barriers)
    }
    BfsPushT<HT> f;
    f.keep = policy_evict_last();
    f.visited = a.visited;
    f.level = a.level;
    f.parent = a.parent;
    f.fb_next = nullptr;
    f.next_level = L + 1;
    f.v_base = 0;
    f.next_q = &a.q[(L + 1) & 1];
    f.next_cs = nxt;
    f.flist = a.fl[(L + 1) & 1];
    f.flc = &nxt->flc.v;
    f.nfc = &nxt->nF.v;
    if constexpr (HT > 0) f.ht = (uint32_t)__cvta_generic_to_shared(ht);
    int bcnt = 0;
    const bool log_all = ldcg(&cur->nF.v) < kFusedLogAll;
    fused_phase_a<VEC>(a, f, cur, a.fl[L & 1], a.q[L & 1], &wsm[warp], fsrc[warp], bcnt, log_all);
    defer_close(&wsm[warp], bcnt, f.flist, f.flc, f.nfc);
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    if (blockIdx.x == 0 && threadIdx.x == 0 && L < kMaxRec) ctl->rec[L].t_mid = globaltimer();
    // phase B: the logged tiles (CTA tiles; every class on a small level), Resident Tile Stealing
    bool logged = ldcg(&cur->cnt[0].v) > 0;
    for (int c = 1; c <= a.L.ncls; ++c)
      if (log_all || c < SAGE_FUSED_LOGC) logged |= ldcg(&cur->cnt[c].v) > 0;
    if constexpr (HT > 0) {   // the CTA's copy of the table with the hubs phase A inserted
      if (ldcg(&cur->hubc.v) >= kHubReloadMinChanges) {
        hub_load<HT>(a, ht);
        __syncthreads();
      }
    }
    if (logged) {
      consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc[warp], a.vec_ok,
                       a.steal != 0);
      grid_barrier(&ctl->bar);
    }
    const unsigned long long nF = ldcg(&nxt->nF.v);
    if (blockIdx.x == 0 && threadIdx.x == 0) record_level_fused(ctl, L, cur, nxt);
    if (nF == 0) break;
    if (SAGE_BFS_STOP_AFTER >= 0 && L >= SAGE_BFS_STOP_AFTER) break;   // profiling build only (below)
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
    // small frontier: block 0 runs the next levels alone (it hands back when arcs(F) is large).
    // Level L+1's list is sparse (a 256-slot chunk per warp that discovered anything: up to ~10^5
    // slots on C1 for a few hundred vertices), so the whole grid compacts it first — block 0
    // alone scanning it cost up to 130 us.
    if (nF <= kTailV) {
      {
        const long long fc = (long long)ldcg(&nxt->flc.v);
        // long lists: the whole grid compacts them (one more grid barrier); short ones: block 0
        const bool grid_wide = fc > kTailCompactGrid;
        const int *src = a.fl[(L + 1) & 1];
        int *dst = a.fl[L & 1];
        const long long tid = grid_wide ? (long long)blockIdx.x * blockDim.x + threadIdx.x : (long long)threadIdx.x;
        const long long nth = grid_wide ? (long long)gridDim.x * blockDim.x : (long long)blockDim.x;
        const unsigned lane = lane_id();
        for (long long base = tid - lane; (grid_wide || blockIdx.x == 0) && base < fc; base += nth) {
          const long long i = base + lane;
          const int u = i < fc ? ldcg(src + i) : -1;
          const unsigned m = __ballot_sync(FULL, u >= 0);
          if (m) {
            int pos = 0;
            if (lane == 0) pos = atomicAdd(&ctl->tail_n, __popc(m));
            pos = __shfl_sync(FULL, pos, 0);
            if (u >= 0) dst[pos + __popc(m & lanemask_lt())] = u;
          }
        }
        if (grid_wide) grid_barrier(&ctl->bar);
        else __syncthreads();
      }
      if (blockIdx.x == 0) {
        __syncthreads();
        if (threadIdx.x == 0) ctl->tail_state = 0;
        __syncthreads();
        tail_run<true>(a, L + 1, *a.tailmem);
      }
      grid_barrier(&ctl->bar);
      if (ldcg(&ctl->tail_state) == 1) break;
      L = ldcg(&ctl->tail_resume) - 1;   // ++L resumes the grid at the returned level
      if (SAGE_BFS_STOP_AFTER >= 0 && L >= SAGE_BFS_STOP_AFTER) break;
      continue;
    }
  }
}

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_bfs_fused(const __grid_constant__ TravArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BfsPush::Src fsrc[kWarps][32];
  bfs_body_fused<VEC, 0>(a, wsm, fsrc, nullptr);
}
template <int VEC, int HT>
__global__ void __launch_bounds__(1024, 1) k_bfs_fused_hub(const __grid_constant__ TravArgs a) {
  __shared__ WarpScratch wsm[32];
  __shared__ typename BfsPushT<HT>::Src fsrc[32][32];
  extern __shared__ __align__(16) uint8_t hub_smem[];
  bfs_body_fused<VEC, HT>(a, wsm, fsrc, hub_smem);
}

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_bfs(const __grid_constant__ TravArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BfsPush::Src fsrc[kWarps][32];
  bfs_body<VEC, 0>(a, wsm, fsrc, nullptr);
}

// Hub-filter variant: one 1024-thread CTA per SM (one table per SM, not per CTA).
constexpr int kHubBlock = 1024;
template <int VEC, int HT>
__global__ void __launch_bounds__(kHubBlock, 1) k_bfs_hub(const __grid_constant__ TravArgs a) {
  __shared__ WarpScratch wsm[kHubBlock / 32];
  __shared__ typename BfsPushT<HT>::Src fsrc[kHubBlock / 32][32];
  extern __shared__ __align__(16) uint8_t hub_smem[];
  bfs_body<VEC, HT>(a, wsm, fsrc, hub_smem);
}

// ============================================================================ SSSP kernel
template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_sssp(const __grid_constant__ TravArgs a, int *overflow) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ SsspPush::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  Ctl *ctl = a.ctl;
  const long long nwords = (a.n + 31) >> 5;
  if ((threadIdx.x & 31) == 0) {
    wsm[warp].cpos = wsm[warp].cend = 0;
    wsm[warp].ndisc = 0;
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) ctl->t0_ns = globaltimer();
  query_init<1>(a, overflow);
  for (int L = 0;; ++L) {
    CounterSet *cur = &ctl->set[L % 3];
    CounterSet *nxt = &ctl->set[(L + 1) % 3];
    __syncthreads();
    zero_counterset(&ctl->set[(L + 2) % 3]);
    if (blockIdx.x == 0 && threadIdx.x == 0 && L + 1 < kMaxRec) ctl->rec[L + 1].t_work = ctl->rec[L + 1].t_mid = 0;
    clear_words(a.fb[(L + 2) % 3], nwords);
    SsspPush f;
    f.dist = a.dist;
    f.inq_next = a.fb[(L + 1) % 3];
    f.overflow = overflow;
    f.next_q = &a.q[(L + 1) & 1];
    f.next_cs = nxt;
    f.flist = a.flist;
    f.flc = &nxt->flc.v;
    consume_log<VEC>(f, a.L, a.q[L & 1], cur, a.off, a.col, a.w, &wsm[warp], fsrc[warp], a.vec_ok);
    if ((threadIdx.x & 31) == 0 && L < kMaxRec) atomicMax(&ctl->rec[L].t_work, globaltimer());
    grid_barrier(&ctl->bar);
    if (classify_deferred(a.off, a.flist, &nxt->flc.v, a.L, a.q[(L + 1) & 1], nxt))
      grid_barrier(&ctl->bar);
    const unsigned long long nF = ldcg(&nxt->nF.v);
    if (blockIdx.x == 0 && threadIdx.x == 0) record_level(ctl, L, 0, cur, nxt);
    if (nF == 0) break;
    if (L + 1 >= a.max_levels) {
      if (blockIdx.x == 0 && threadIdx.x == 0) ctl->status = 1;
      break;
    }
  }
}

// Seed the level-0 log with the source (one warp).

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
  if (t.ev_caller) cudaEventDestroy(t.ev_caller);
  dfree(g, t.visited);
  for (int i = 0; i < 3; ++i) dfree(g, t.fb[i]);
  free_queues(g, &t.q[0]);
  free_queues(g, &t.q[1]);
  dfree(g, t.ctl);
  dfree(g, t.tmp_out);
  dfree(g, t.tailmem);
  dfree(g, t.flist);
  dfree(g, t.hub_g);
  dfree(g, t.flist2);
  for (int i = 0; i < 3; ++i)
    if (t.ev[i]) cudaEventDestroy(t.ev[i]);
  if (t.hctl) {
    cudaStreamSynchronize(g->stream);
    cudaFreeHost(t.hctl);
  }
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
  cudaMemsetAsync(t.ctl, 0, sizeof(Ctl), g->stream);   // the grid barrier starts consistent
  for (int i = 0; i < 3; ++i) cudaEventCreate(&t.ev[i]);
  if (cudaMallocHost((void **)&t.hctl, sizeof(Ctl)) != cudaSuccess) {
    cudaGetLastError();
    free_traversal_state(g);
    set_error("pinned host allocation failed");
    return SAGE_E_NOMEM;
  }
  t.ready = true;
  return SAGE_OK;
}

int coop_grid(sage_graph *g, const void *fn, int *cache, int block, size_t dyn_smem) {
  if (*cache) return *cache;
  // shared-memory carveout: the smallest that still holds the occupancy limit's CTAs (+1 KB
  // reserved per CTA); the rest of the SM's 256 KB goes to L1, which caches status words and row
  // offsets (measured on C2 push BFS: driver default 3.40 ms, smallest carveout 3.15 ms)
  if (dyn_smem) cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn_smem);
  int nb = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, block, dyn_smem);
  if (nb < 1) nb = 1;
  {
    cudaFuncAttributes fa;
    if (cudaFuncGetAttributes(&fa, fn) == cudaSuccess) {
      int smem_sm = 0;
      cudaDeviceGetAttribute(&smem_sm, cudaDevAttrMaxSharedMemoryPerMultiprocessor, g->device);
      const size_t need = (size_t)nb * (fa.sharedSizeBytes + dyn_smem + 1024);
      if (smem_sm > 0) {
        const int pct = (int)std::min<size_t>(100, (need * 100 + smem_sm - 1) / smem_sm);
        cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
      }
    }
  }
  const int nb_occ = nb;
  // small graphs (C1: 1.8M arcs, L2-resident) are latency-bound per level: one CTA per SM halves
  // the grid barrier's participants and the counter traffic (C1 DO BFS 156 -> 135 us measured)
  if (g->m < (8ll << 20)) nb = 1;
  if (g->ctas_per_sm > 0) nb = std::max(1, std::min(nb_occ, g->ctas_per_sm));
  *cache = nb * g->num_sms;
  return *cache;
}

sage_status launch_coop(sage_graph *g, const void *fn, int grid, void **args, const char *what, int block,
                        size_t dyn_smem) {
  cudaError_t e = cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(block), args, dyn_smem, g->stream);
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

// Hub filter (BfsPushT): on graphs with >= 32M arcs the push BFS runs the 1024-thread variant with
// a table of visited hubs per SM.  SAGE_HUB_KB (compile time) = 64 or 128 KB tables; 8-bit keys
// when every key + 1 fits a byte (n <= 255 * T), else 16-bit keys.
#ifndef SAGE_HUB_KB
#define SAGE_HUB_KB 64
#endif
constexpr long long kHubMinGraphArcs = 32ll << 20;
constexpr unsigned long long kHubMinLevelArcs = 4ull << 20;   // reload the tables before such levels
static int hub_mode(const sage_graph *g) {
#ifdef SAGE_NO_HUB
  return 0;
#else
  if (g->vec != 4 || g->hub_filter < 0 || (g->hub_filter == 0 && g->m < kHubMinGraphArcs)) return 0;
  // 8-bit keys hold (v >> lgT) + 1 <= 255, so ids >= 255 << lgT are never inserted (0.4% of the
  // ids at n = 2^24, which keeps C2 on the 2^16-slot byte table)
  if (SAGE_HUB_KB == 128) return g->n <= 256ll << 17 ? 1 : 2;
  return g->n <= 256ll << 16 ? 3 : 4;
#endif
}
static int hub_lgT(int ht) { return ht == 1 ? 17 : ht == 4 ? 15 : 16; }
static int hub_kbits(int ht) { return (ht == 1 || ht == 3) ? 8 : 16; }
static size_t hub_bytes(int ht) { return ht == 1 || ht == 2 ? (128u << 10) : (64u << 10); }

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
  a.tail = (int *)g->ts.tmp_out;
  a.tailmem = reinterpret_cast<TailSmem *>(g->ts.tailmem);
  a.flist = g->ts.flist;
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

// true when p is device memory of the graph's GPU (cudaMalloc / a CUDA tensor), not host memory
static bool is_own_device_ptr(const sage_graph *g, const void *p) {
  if (!p) return false;
  cudaPointerAttributes at;
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return at.type == cudaMemoryTypeDevice && at.device == g->device;
}

// Outputs written in place into caller device buffers: on the library's own (non-blocking) stream
// the writes must follow the caller's earlier work on the legacy default stream (e.g. a torch
// fill of the same buffer); with a caller stream they are ordered by that stream already.
static void order_after_caller(sage_graph *g) {
  if (!g->own_stream) return;
  TraversalState &t = g->ts;
  if (!t.ev_caller && cudaEventCreateWithFlags(&t.ev_caller, cudaEventDisableTiming) != cudaSuccess) {
    cudaGetLastError();
    t.ev_caller = nullptr;
    cudaStreamSynchronize(cudaStreamLegacy);   // fallback: order by a host wait
    return;
  }
  cudaEventRecord(t.ev_caller, cudaStreamLegacy);
  cudaStreamWaitEvent(g->stream, t.ev_caller, 0);
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
  NvtxRange nvtx_("sage_bfs");
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
  const bool do_enabled = symmetric && !push_only;
#ifdef SAGE_NO_FUSED
  const bool fused = false;
#else
  const bool fused = !do_enabled;   // push-only: Tiled Partitioning fused into the consumer
#endif
  // outputs written in place: when the caller's buffers are device memory of this GPU and no ID
  // translation is needed, the kernel initialises and fills them directly (no output copy)
  const bool direct_lv = !g->reordered && !g->online && is_own_device_ptr(g, level_out);
  const bool direct_par = parent_out && !g->reordered && is_own_device_ptr(g, parent_out);
  if (direct_lv || direct_par) order_after_caller(g);
  cudaEvent_t e0 = t.ev[0], e1 = t.ev[1], e2 = t.ev[2];
  cudaEventRecord(e0, g->stream);
  TravArgs a = make_args(g);
  a.parent = parent_out ? t.parent : nullptr;
  if (direct_lv) a.level = level_out;
  if (direct_par) a.parent = parent_out;
  a.do_enabled = do_enabled ? 1 : 0;
  a.steal = (call_flags & SAGE_F_NO_STEALING) ? 0 : 1;
  a.src = src;
  if (const int ht = hub_mode(g)) {
    const int lgT = hub_lgT(ht);
    if (!t.hub_g && (s = dalloc(g, (void **)&t.hub_g, sizeof(uint32_t) << 17)) != SAGE_OK) return s;
    if (!fused) cudaMemsetAsync(t.hub_g, 0, sizeof(uint32_t) << lgT, g->stream);
    a.hub.g = t.hub_g;
    a.hub.lgT = lgT;
    a.hub.mask = (1u << lgT) - 1u;
    a.hub.kbits = hub_kbits(ht);
    a.hub.thr = std::max<long long>(2, 2 * ((g->m + g->n_local - 1) / std::max<long long>(1, g->n_local)));
    a.hub_min_arcs = kHubMinLevelArcs;
  }
  if (fused) {
    if (!t.flist2 && (s = dalloc(g, (void **)&t.flist2,
                                 sizeof(int) * (size_t)(g->n_local + (long long)g->num_sms * 64 * kDeferChunk + 64))) != SAGE_OK)
      return s;
    a.fl[0] = t.flist;
    a.fl[1] = t.flist2;
  }
  cudaEventRecord(e1, g->stream);
  if (fused) {
    const int ht = hub_mode(g);
#ifndef SAGE_FUSED_VEC
#define SAGE_FUSED_VEC 4   // neighbours per lane per step of the fused push BFS (A/B: 8)
#endif
    constexpr int FV = SAGE_FUSED_VEC;
    const void *fn = ht == 1 ? (const void *)k_bfs_fused_hub<FV, 1>
                   : ht == 2 ? (const void *)k_bfs_fused_hub<FV, 2>
                   : ht == 3 ? (const void *)k_bfs_fused_hub<FV, 3>
                   : ht == 4 ? (const void *)k_bfs_fused_hub<FV, 4>
                   : g->vec == 4 ? (const void *)k_bfs_fused<4> : (const void *)k_bfs_fused<1>;
    const int block = ht ? kHubBlock : kBlock;
    const size_t dyn = ht ? hub_bytes(ht) : 0;
    const int grid = coop_grid(g, fn, ht ? &g->grid_bfs_fused_hub : &g->grid_bfs_fused, block, dyn);
    void *args[] = {&a};
    if ((s = launch_coop(g, fn, grid, args, "BFS kernel", block, dyn)) != SAGE_OK) return s;
  } else {
    const int ht = hub_mode(g);
    const void *fn = ht == 1 ? (const void *)k_bfs_hub<4, 1>
                   : ht == 2 ? (const void *)k_bfs_hub<4, 2>
                   : ht == 3 ? (const void *)k_bfs_hub<4, 3>
                   : ht == 4 ? (const void *)k_bfs_hub<4, 4>
                   : g->vec == 4 ? (const void *)k_bfs<4> : (const void *)k_bfs<1>;
    int block = ht ? kHubBlock : kBlock;
    size_t dyn = ht ? hub_bytes(ht) : 0;
#ifdef SAGE_HUB_NOTABLE   // A/B: the 1024-thread configuration without the table (1: same smem, 2: no smem)
    if (ht) {
      fn = (const void *)k_bfs_hub<4, 0>;
      if (SAGE_HUB_NOTABLE == 2) dyn = 0;
    }
#endif
    const int grid = coop_grid(g, fn, ht ? &g->grid_bfs_hub : &g->grid_bfs, block, dyn);
    void *args[] = {&a};
    if ((s = launch_coop(g, fn, grid, args, "BFS kernel", block, dyn)) != SAGE_OK) return s;
    (void)block;
  }
  cudaEventRecord(e2, g->stream);
  // counters and outputs in one stream round trip (one synchronisation per call)
  Ctl &h = *t.hctl;
  cudaMemcpyAsync(&h, t.ctl, offsetof(Ctl, rec), cudaMemcpyDeviceToHost, g->stream);
  if (!direct_lv && (s = translate_out_i32(g, t.level, level_out, false)) != SAGE_OK) return s;
  if (parent_out && !direct_par && (s = translate_out_i32(g, t.parent, parent_out, true)) != SAGE_OK) return s;
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "BFS");
  float ms = 0, kms = 0;
  cudaEventElapsedTime(&ms, e0, e2);
  cudaEventElapsedTime(&kms, e1, e2);
  if (h.status == 1) {
    set_error("BFS exceeded the level cap (internal error)");
    g->sticky = SAGE_E_CUDA;
    return SAGE_E_CUDA;
  }
  fill_stats(g, h, true, symmetric, ms, kms, st);
  // online sampling: record the rows this query expanded (after the answer has been delivered)
  return online_after_query(g, t.level, 0);
}

extern "C" sage_status sage_bfs(sage_graph *g, int32_t source, int32_t *level_out,
                                int32_t *parent_out, sage_stats *st) {
  return sage_bfs_ex(g, source, level_out, parent_out, 0u, st);
}

extern "C" sage_status sage_sssp(sage_graph *g, int32_t source, uint32_t *dist_out,
                                 sage_stats *st) {
  NvtxRange nvtx_("sage_sssp");
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
  // distances written in place when the caller's buffer is device memory of this GPU (no copy)
  const bool direct = !g->reordered && is_own_device_ptr(g, dist_out);
  uint32_t *dd = direct ? dist_out : t.dist;
  if (direct) order_after_caller(g);
  // dist, bitmaps, counters and the seed: query_init<1> inside the kernel
  TravArgs a = make_args(g);
  a.dist = dd;
  a.src = src;
  cudaEventRecord(e1, g->stream);
  const void *fn = g->vec == 4 ? (const void *)k_sssp<4> : (const void *)k_sssp<1>;
  const int grid = coop_grid(g, fn, &g->grid_sssp, kBlock, 0);
  void *args[] = {&a, &ovf};
  if ((s = launch_coop(g, fn, grid, args, "SSSP kernel", kBlock, 0)) != SAGE_OK) {
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
                                                            dd, g->n_local, ovf + 1);
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
    k_reached_arcs<<<g->num_sms * 8, 256, 0, g->stream>>>((const long long *)g->off, dd,
                                                          g->n_local, dra);
    cudaMemcpyAsync(&hra, dra, sizeof(hra), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
    dfree(g, dra);
    st->edges_traversed = (int64_t)((g->flags & SAGE_F_SYMMETRIC) ? hra / 2 : hra);
  }
  if (!direct && (s = translate_out_u32(g, t.dist, dist_out)) != SAGE_OK) return s;
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
  // 9 int64 per level (include/sage.h): dir, |F|, arcs(F), inspected, scanned, discovered,
  // level end, last warp's work end, expansion end (K2' start); times in ns since kernel start
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
    o[8] = r.t_mid ? (int64_t)(r.t_mid - h->t0_ns) : 0;
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
