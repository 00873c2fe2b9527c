// comm.cu — multi-GPU traversal: 1D vertex partition + NCCL frontier exchange.
//
// The paper runs two GPUs with no pre-partitioning and "data ... synchronized after each
// iteration" without naming the mechanism.  Here (north_star): rank r owns the
// contiguous vertex block [vb[r], vb[r+1]) and its out-rows (global column ids); one process per
// GPU; the communicator is created from a unique id the caller broadcasts.  Per BFS level:
//   push : the local stealing consumer expands the local log; owned neighbours are claimed
//          locally, remote ones go to their owner in one of two forms, chosen per level from the
//          global arcs(F) every rank already knows (so all ranks agree without a counts round):
//          sparse (C1a) when arcs(F) < Wp - int32 ids in per-destination lists of capacity
//          arcs(F), which no sender can exceed - else dense (C1b) - the owners' bitmap slices;
//          an all-to-all(v) moves them and the owners apply the received candidates.
//   pull : allgather of the frontier slices (C1c), then every rank scans its own unvisited rows.
//   stats: allreduce of (|F|, arcs(F)) gives termination and the Beamer direction (C1d).
// PageRank: push into a full-length partial y, ncclReduceScatter(sum) to the owners (C1e), plus
// an allreduce of the dangling mass (C1f).
// Global-indexed bitmaps / vectors use a PADDED layout: vertex v of owner r sits at
// r * P + (v - vb[r]) with P = 32 * Wp >= max rows per rank, so every rank's slice is a contiguous
// word range and the exchanges are plain equal-count collectives.
// With dist != NULL and world == 1 the same path runs on a 1-rank communicator (tested on 1 GPU);
// the collectives go through an Xport (xport.h): NCCL, or the test-only loopback transport that
// runs p logical ranks on one GPU so the r > 0 paths are checked against the oracle.
// BFS parents (any valid BFS-tree parent, sage.h): after the traversal every rank allgathers the
// levels, proposes for each target v of its rows the smallest u with level(u) = level(v) - 1, and
// a reduce-scatter(min) hands each owner its answer.
#include <cuda_runtime.h>
#include <nccl.h>
#include <string.h>

#include <algorithm>
#include <vector>

#include "common.cuh"
#include "graph.h"
#include "internal.h"
#include "xport.h"

namespace sage {

constexpr int kMaxRanks = 64;

struct PartMap {
  int p;
  int rank;
  long long P;                    // padded vertices per rank (multiple of 32)
  long long vb[kMaxRanks + 1];    // rank boundaries
};

__device__ __forceinline__ long long pidx(const PartMap &pm, long long v, bool *own) {
  int lo = 0, hi = pm.p;
  while (hi - lo > 1) {
    const int mid = (lo + hi) >> 1;
    if (pm.vb[mid] <= v) lo = mid; else hi = mid;
  }
  *own = lo == pm.rank;
  return (long long)lo * pm.P + (v - pm.vb[lo]);
}

struct Comm {
  Xport *x = nullptr;
  int rank = 0, world = 1;
  std::vector<long long> vb;
  long long Wp = 0;                  // padded words per rank
  long long m_total = 0;
  uint32_t *out = nullptr;           // p*Wp words
  uint32_t *recv = nullptr;          // p*Wp words
  uint32_t *visited = nullptr;       // p*Wp words (own slice authoritative, remote = "sent")
  uint32_t *fb[3] = {nullptr, nullptr, nullptr};
  unsigned long long *stats = nullptr;  // 8 u64
  double *y = nullptr, *yown = nullptr, *dsum = nullptr;
  uint32_t *cand = nullptr, *cown = nullptr;   // SSSP min-exchange buffers (p*P and P)
  uint32_t *sp_send = nullptr, *sp_recv = nullptr;   // sparse exchange: p blocks of (cap + 2) words
  long long sp_words = 0;                            // allocated words of each
  int32_t *glevel = nullptr;         // parents: allgathered levels (p*P, padded layout)
  unsigned long long *hmap = nullptr, *dmap = nullptr;   // mapped pinned stats (16 u64) + device alias
  unsigned long long pub_seq = 0;
  uint32_t *pcand = nullptr, *pown = nullptr;        // parents: p*P proposals, own P after min
  // fused exchange over peer memory (sage_dist.exchange = 0 and every rank mappable): one
  // cudaMalloc'd (IPC-able) region per rank = the BFS inbox bitmap (Wp words) followed by the
  // SSSP candidate minima of the own rows (P words); peers[q] = rank q's region as seen from here
  bool p2p = false;
  uint32_t *inbox = nullptr;
  void *peers[kMaxRanks] = {};
  uint32_t **d_peers = nullptr;                       // device copy of peers (p entries)
  PartMap pm;
};

#define XCHECK(call)                \
  do {                              \
    sage_status s_ = (call);        \
    if (s_ != SAGE_OK) return s_;   \
  } while (0)

// ============================================================================ filters / kernels
struct MultiArgs {
  const long long *off;
  const int *col;
  long long n_local, v_begin;
  Ladder L;
  Queues q[2];
  Ctl *ctl;
  uint32_t *visited;
  uint32_t *fb[3];
  uint32_t *out;
  const uint32_t *recv;
  int *level;
  int do_enabled;
  int vec_ok;
  int lvl;                         // current level L
  PartMap pm;
  uint32_t *const *pin;            // peer form: pin[q] = rank q's region (inbox Wp words, then the
                                   // SSSP minima P words), nullptr = collective form
  uint32_t *sp_send;               // sparse form: p blocks of (sp_cap + 2) words [count, 0, ids...]
  const uint32_t *sp_recv;
  long long sp_cap;                // 0 = dense form this level
  int *flist;                      // deferred contraction: frontier list
  // SSSP (frontier Bellman-Ford across ranks)
  const uint32_t *w;
  uint32_t *dist;                  // own rows' distances
  uint32_t *cand;                  // p*P candidate distances for remote targets (UINT32_MAX = none)
  const uint32_t *cown;            // own slice after the min reduce-scatter
  uint32_t *inq_next;              // own rows: next-frontier dedupe bitmap
  int *overflow;
};

struct BfsPushMulti {
  struct Src {
    int u;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
  static constexpr bool kDefer = true;   // contraction deferred to k_mclassify (see traversal.cu)
  int *flist = nullptr;
  unsigned long long *flc = nullptr;
  const MultiArgs *a;
  uint32_t *fb_next;
  const Queues *next_q;
  CounterSet *next_cs;
  __device__ __forceinline__ Src src(bool, int u, long long, long long) const { return Src{u}; }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int) const {
    const unsigned long long keep = policy_evict_last();
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      if (!valid) continue;
      bool own;
      const long long p = pidx(a->pm, v[j], &own);
      const uint32_t bit = 1u << (p & 31);
      if (ld_status(a->visited + (p >> 5), keep) & bit) continue;
      const uint32_t old = atomicOr(a->visited + (p >> 5), bit);
      if (old & bit) continue;
      if (own) {
        const int lv = (int)(v[j] - a->v_begin);
        a->level[lv] = a->lvl + 1;
        if (fb_next) atomicOr(fb_next + (p >> 5), bit);
        v[j] = lv;                   // enqueue the LOCAL row id
        in[j] = true;
      } else if (a->pin) {          // candidate for its owner: OR into its inbox over NVLink
        const int q = (int)(p / a->pm.P);
        atomicOr(a->pin[q] + ((p >> 5) - (long long)q * (a->pm.P >> 5)), bit);
      } else if (a->sp_cap) {       // candidate for its owner: sparse form (global id)
        const int q = (int)(p / a->pm.P);
        uint32_t *blk = a->sp_send + (long long)q * (a->sp_cap + 2);
        const uint32_t pos = atomicAdd(blk, 1u);
        blk[2 + pos] = (uint32_t)v[j];
      } else {
        atomicOr(a->out + (p >> 5), bit);   // dense form: the owner's bitmap slice
      }
    }
  }
};

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_mpush(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ BfsPushMulti::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  const int L = a.lvl;
  if ((threadIdx.x & 31) == 0) {
    wsm[warp].cpos = wsm[warp].cend = 0;
    wsm[warp].ndisc = 0;
  }
  __syncwarp();
  BfsPushMulti f;
  f.a = &a;
  f.fb_next = a.do_enabled ? a.fb[(L + 1) % 3] : nullptr;
  f.next_q = &a.q[(L + 1) & 1];
  f.next_cs = &a.ctl->set[(L + 1) % 3];
  f.flist = a.flist;
  f.flc = &a.ctl->set[(L + 1) % 3].flc.v;
  consume_log<VEC>(f, a.L, a.q[L & 1], &a.ctl->set[L % 3], a.off, a.col, nullptr, &wsm[warp],
                   fsrc[warp], a.vec_ok);
  if (a.pin) __threadfence_system();   // the peer ORs are performed before the barrier that follows
}

// K2' of the deferred contraction for the vertices k_mpush claimed locally.
__global__ void __launch_bounds__(kBlock) k_mclassify(const __grid_constant__ MultiArgs a) {
  const int L = a.lvl;
  classify_deferred(a.off, a.flist, &a.ctl->set[(L + 1) % 3].flc.v, a.L, a.q[(L + 1) & 1],
                    &a.ctl->set[(L + 1) % 3]);
}

// Owners apply the candidates received from every other rank (dense form: the p - 1 received
// slices; peer form: the own inbox, cleared as it is read for the next level).
__global__ void __launch_bounds__(kBlock) k_mapply(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const int L = a.lvl;
  const long long Wp = a.pm.P >> 5;
  const long long words = (a.n_local + 31) >> 5;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  uint32_t *fbn = a.do_enabled ? a.fb[(L + 1) % 3] : nullptr;
  const Queues &Qn = a.q[(L + 1) & 1];
  CounterSet *csn = &a.ctl->set[(L + 1) % 3];
  int bcnt = 0;
  for (long long base = gw * 32; base < words; base += nw * 32) {
    const long long w = base + lane;
    uint32_t nw_bits = 0;
    if (w < words) {
      uint32_t cand = 0;
      if (a.pin) {
        uint32_t *box = a.pin[a.pm.rank] + w;
        cand = *box;
        if (cand) *box = 0u;
      } else {
        for (int r = 0; r < a.pm.p; ++r)
          if (r != a.pm.rank) cand |= a.recv[(long long)r * Wp + w];
      }
      if (w == words - 1 && (a.n_local & 31)) cand &= (1u << (a.n_local & 31)) - 1u;
      const long long gwd = (long long)a.pm.rank * Wp + w;
      const uint32_t own = a.visited[gwd];
      nw_bits = cand & ~own;
      if (nw_bits) {
        a.visited[gwd] = own | nw_bits;
        if (fbn) fbn[gwd] |= nw_bits;
      }
    }
    while (__any_sync(FULL, nw_bits != 0)) {
      const bool has = nw_bits != 0;
      int lv = 0;
      if (has) {
        const int b = __ffs(nw_bits) - 1;
        nw_bits &= nw_bits - 1;
        lv = (int)(w * 32 + b);
        a.level[lv] = L + 1;
      }
      buffer_push(has, lv, &wsm[warp], bcnt, a.off, a.L, Qn, csn);
    }
  }
  if (bcnt) buffer_flush(&wsm[warp], bcnt, a.off, a.L, Qn, csn);
}

// Sparse form: owners apply the ids received from every other rank.
__global__ void __launch_bounds__(kBlock) k_mapply_sparse(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  const int warp = threadIdx.x >> 5;
  const int L = a.lvl;
  const long long gt = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long nt = (long long)gridDim.x * blockDim.x;
  uint32_t *fbn = a.do_enabled ? a.fb[(L + 1) % 3] : nullptr;
  const Queues &Qn = a.q[(L + 1) & 1];
  CounterSet *csn = &a.ctl->set[(L + 1) % 3];
  const long long blk = a.sp_cap + 2;
  const long long total = (long long)a.pm.p * a.sp_cap;
  int bcnt = 0;
  for (long long base = gt - (gt & 31); base < total; base += nt) {
    const long long i = base + (gt & 31);
    bool in = false;
    int lv = 0;
    if (i < total) {
      const int q = (int)(i / a.sp_cap);
      const long long k = i - (long long)q * a.sp_cap;
      if (q != a.pm.rank && k < (long long)a.sp_recv[(long long)q * blk]) {
        lv = (int)((long long)a.sp_recv[(long long)q * blk + 2 + k] - a.v_begin);
        const long long gp = (long long)a.pm.rank * a.pm.P + lv;
        const uint32_t bit = 1u << (gp & 31);
        if (!(atomicOr(a.visited + (gp >> 5), bit) & bit)) {
          in = true;
          a.level[lv] = L + 1;
          if (fbn) atomicOr(fbn + (gp >> 5), bit);
        }
      }
    }
    buffer_push(in, lv, &wsm[warp], bcnt, a.off, a.L, Qn, csn);
  }
  if (bcnt) buffer_flush(&wsm[warp], bcnt, a.off, a.L, Qn, csn);
}

// Parents after the traversal: for every own row u and arc u->v with level(v) = level(u) + 1,
// propose u (global id) for v in the padded proposal array (smallest wins: atomicMin).
__global__ void k_mparent_propose(const MultiArgs a, const int32_t *glevel, uint32_t *pcand) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < a.n_local; u += stride) {
    const int lu = a.level[u];
    if (lu < 0) continue;
    for (long long k = a.off[u]; k < a.off[u + 1]; ++k) {
      bool own;
      const long long p = pidx(a.pm, a.col[k], &own);
      if (glevel[p] == lu + 1) atomicMin(pcand + p, (uint32_t)(u + a.v_begin));
    }
  }
}
__global__ void k_mparent_final(const int *level, const uint32_t *pown, long long n, int *parent) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    parent[v] = level[v] > 0 ? (int)pown[v] : -1;
}
__global__ void k_fill_u32(uint32_t *p, long long n, uint32_t v) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) p[i] = v;
}

// Pull level over the own rows; the frontier bitmap holds the allgathered global frontier.
__global__ void __launch_bounds__(kBlock) k_mpull(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const int L = a.lvl;
  const long long Wp = a.pm.P >> 5;
  const long long words = (a.n_local + 31) >> 5;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const uint32_t *fbc = a.fb[L % 3];
  uint32_t *fbn = a.fb[(L + 1) % 3];
  const Queues &Qn = a.q[(L + 1) & 1];
  CounterSet *cur = &a.ctl->set[L % 3];
  CounterSet *csn = &a.ctl->set[(L + 1) % 3];
  int bcnt = 0;
  unsigned long long insp = 0, scanned = 0;
  for (long long wd = gw; wd < words; wd += nw) {
    const long long gwd = (long long)a.pm.rank * Wp + wd;
    const long long v = (wd << 5) + lane;
    const uint32_t vis = a.visited[gwd];
    const bool todo = v < a.n_local && !((vis >> lane) & 1u);
    bool found = false;
    if (todo) {
      const long long b = a.off[v], e = a.off[v + 1];
      if (e > b) scanned++;
      for (long long k = b; k < e; ++k) {
        const int u = a.col[k];
        ++insp;
        bool own;
        const long long p = pidx(a.pm, u, &own);
        if ((fbc[p >> 5] >> (p & 31)) & 1u) {
          found = true;
          break;
        }
      }
    }
    const unsigned fm = __ballot_sync(FULL, found);
    if (fm && lane == 0) {
      a.visited[gwd] = vis | fm;
      fbn[gwd] = fm;
    }
    if (found) a.level[v] = L + 1;
    buffer_push(found, (int)v, &wsm[warp], bcnt, a.off, a.L, Qn, csn);
  }
  if (bcnt) buffer_flush(&wsm[warp], bcnt, a.off, a.L, Qn, csn);
  insp = warp_sum64(insp);
  scanned = warp_sum64(scanned);
  if (lane == 0) {
    if (insp) atomicAdd(&cur->inspected.v, insp);
    if (scanned) atomicAdd(&cur->scanned.v, scanned);
  }
}

// ---- multi-GPU SSSP (dense form).  Same filter as the single-GPU SSSP
// (reading R4: nd = dist[u] + w, atomicMin, improved vertices enter the next log once per
// iteration); an improvement of a REMOTE target is an atomicMin into the padded candidate array,
// and one ncclReduceScatter(min) per iteration hands every owner the minimum over all ranks.
struct SsspPushMulti {
  struct Src {
    uint32_t du;
  };
  static constexpr bool kWeights = true;
  static constexpr bool kNeedRow = false;
  static constexpr bool kEnqueue = true;
  const MultiArgs *a;
  const Queues *next_q;
  CounterSet *next_cs;
  __device__ __forceinline__ Src src(bool valid, int u, long long, long long) const {
    return Src{valid ? ldcg(a->dist + u) : 0xffffffffu};
  }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N], const uint32_t (&w)[N],
                                        bool (&in)[N], int) const {
    const unsigned long long keep = policy_evict_last();
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      if (!valid) continue;
      const unsigned long long nd = (unsigned long long)s.du + w[j];
      if (nd >= 0xffffffffull) {
        if (s.du != 0xffffffffu) *a->overflow = 1;   // resolved after the traversal
        continue;
      }
      bool own;
      const long long p = pidx(a->pm, v[j], &own);
      if (own) {
        const int lv = (int)(v[j] - a->v_begin);
        if (nd >= ld_status(a->dist + lv, keep)) continue;
        const uint32_t old = atomicMin(a->dist + lv, (uint32_t)nd);
        if ((uint32_t)nd < old) {
          const uint32_t bit = 1u << (lv & 31);
          in[j] = !(atomicOr(a->inq_next + (lv >> 5), bit) & bit);
          v[j] = lv;                 // enqueue the LOCAL row id
        }
      } else if (nd < ld_status(a->cand + p, keep)) {
        const uint32_t old = atomicMin(a->cand + p, (uint32_t)nd);
        if (a->pin && (uint32_t)nd < old) {   // peer form: cand = the minimum sent so far; improve
          const int q = (int)(p / a->pm.P);   // the owner's minimum over NVLink
          const long long Wp = a->pm.P >> 5;
          atomicMin(a->pin[q] + Wp + (p - (long long)q * a->pm.P), (uint32_t)nd);
        }
      }
    }
  }
};

template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_msssp_push(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ SsspPushMulti::Src fsrc[kWarps][32];
  const int warp = threadIdx.x >> 5;
  const int L = a.lvl;
  SsspPushMulti f;
  f.a = &a;
  f.next_q = &a.q[(L + 1) & 1];
  f.next_cs = &a.ctl->set[(L + 1) % 3];
  consume_log<VEC>(f, a.L, a.q[L & 1], &a.ctl->set[L % 3], a.off, a.col, a.w, &wsm[warp], fsrc[warp],
                   a.vec_ok);
  if (a.pin) __threadfence_system();
}

// Owners apply the minima received for their rows: one warp per 32-row word of the dedupe bitmap.
__global__ void __launch_bounds__(kBlock) k_msssp_apply(const __grid_constant__ MultiArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  const int warp = threadIdx.x >> 5;
  const unsigned lane = lane_id();
  const int L = a.lvl;
  const long long words = (a.n_local + 31) >> 5;
  const long long gw = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const Queues &Qn = a.q[(L + 1) & 1];
  CounterSet *csn = &a.ctl->set[(L + 1) % 3];
  int bcnt = 0;
  for (long long wd = gw; wd < words; wd += nw) {
    const long long v = (wd << 5) + lane;
    bool improved = false;
    if (v < a.n_local) {
      const uint32_t c = a.cown[v];
      if (c < a.dist[v]) {
        a.dist[v] = c;
        improved = true;
      }
    }
    const unsigned im = __ballot_sync(FULL, improved);
    const uint32_t had = a.inq_next[wd];
    if (im && lane == 0) a.inq_next[wd] = had | im;
    const bool enq = improved && !((had >> lane) & 1u);
    buffer_push(enq, (int)v, &wsm[warp], bcnt, a.off, a.L, Qn, csn);
  }
  if (bcnt) buffer_flush(&wsm[warp], bcnt, a.off, a.L, Qn, csn);
}

__global__ void k_msssp_seed(MultiArgs a, long long src_local) {
  const bool act = threadIdx.x == 0;
  long long b = 0, e = 0;
  if (act) {
    b = a.off[src_local];
    e = a.off[src_local + 1];
    a.dist[src_local] = 0u;
  }
  enqueue_warp(act, (int)src_local, b, e, a.L, a.q[0], &a.ctl->set[0]);
}

// reached bitmap of the own rows (padded global layout) for the overflow resolution
__global__ void k_mreached_bits(const uint32_t *__restrict__ dist, long long n_local, uint32_t *bits) {
  const long long words = (n_local + 31) >> 5;
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long wd = (long long)blockIdx.x * blockDim.x + threadIdx.x; wd < words; wd += stride) {
    uint32_t b = 0;
    for (int k = 0; k < 32; ++k) {
      const long long v = (wd << 5) + k;
      if (v < n_local && dist[v] != 0xffffffffu) b |= 1u << k;
    }
    bits[wd] = b;
  }
}
// a finite distance >= UINT32_MAX exists iff a reached vertex has an arc to an unreached one
// (DESIGN.md "SSSP overflow"); `bits` = allgathered reached bitmap (padded layout)
__global__ void k_moverflow_check(const MultiArgs a, const uint32_t *__restrict__ bits, int *found) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long u = (long long)blockIdx.x * blockDim.x + threadIdx.x; u < a.n_local; u += stride) {
    if (a.dist[u] == 0xffffffffu) continue;
    for (long long k = a.off[u]; k < a.off[u + 1]; ++k) {
      bool own;
      const long long p = pidx(a.pm, a.col[k], &own);
      if (!((bits[p >> 5] >> (p & 31)) & 1u)) {
        *found = 1;
        return;
      }
    }
  }
}
__global__ void k_mreached_arcs(const long long *__restrict__ off, const uint32_t *__restrict__ dist,
                                long long n, unsigned long long *out) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long s = 0;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n; v += stride)
    if (dist[v] != 0xffffffffu) s += (unsigned long long)(off[v + 1] - off[v]);
  s = warp_sum64(s);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

__global__ void k_mseed(MultiArgs a, long long src_local) {
  const bool act = threadIdx.x == 0;
  long long b = 0, e = 0;
  if (act) {
    b = a.off[src_local];
    e = a.off[src_local + 1];
    const long long p = (long long)a.pm.rank * a.pm.P + src_local;
    a.visited[p >> 5] |= 1u << (p & 31);
    a.fb[0][p >> 5] |= 1u << (p & 31);
    a.level[src_local] = 0;
  }
  enqueue_warp(act, (int)src_local, b, e, a.L, a.q[0], &a.ctl->set[0]);
}

// stats of the next log -> comm buffer (nF, arcsF, inspected, scanned of the level just run)
__global__ void k_mstats(const Ctl *ctl, int cur, int nxt, unsigned long long *st) {
  if (threadIdx.x == 0) {
    st[0] = ctl->set[nxt].nF.v;
    st[1] = ctl->set[nxt].arcsF.v;
    st[2] = ctl->set[cur].inspected.v;
    st[3] = ctl->set[cur].scanned.v;
    st[4] = ctl->set[cur].nF.v;
    st[5] = ctl->set[cur].arcsF.v;
  }
}

// ---- PageRank
struct PrPushMulti {
  struct Src {
    double c;
  };
  static constexpr bool kWeights = false;
  static constexpr bool kNeedRow = true;
  static constexpr bool kEnqueue = false;
  const Queues *next_q = nullptr;
  CounterSet *next_cs = nullptr;
  const double *x;
  double *y;
  const PartMap *pm;
  __device__ __forceinline__ Src src(bool valid, int u, long long b, long long e) const {
    return Src{(valid && e > b) ? ldcg(x + u) / (double)(e - b) : 0.0};
  }
  template <int N>
  __device__ __forceinline__ void visit(bool valid, const Src &s, int (&v)[N], const uint32_t (&)[N],
                                        bool (&in)[N], int) const {
#pragma unroll
    for (int j = 0; j < N; ++j) {
      in[j] = false;
      if (!valid) continue;
      bool own;
      red_add_f64(y + pidx(*pm, v[j], &own), s.c);
    }
  }
};
struct MprArgs {
  const long long *off;
  const int *col;
  Ladder L;
  Queues q;
  CounterSet *cs;
  const int *dangling;
  long long n_dangling;
  const double *x;
  double *y;
  double *dsum;
  int vec_ok;
  PartMap pm;
};
template <int VEC>
__global__ void __launch_bounds__(kBlock, 4) k_mpr_push(const __grid_constant__ MprArgs a) {
  __shared__ WarpScratch wsm[kWarps];
  __shared__ PrPushMulti::Src fsrc[kWarps][32];
  __shared__ double red[kWarps];
  const int warp = threadIdx.x >> 5;
  PrPushMulti f;
  f.x = a.x;
  f.y = a.y;
  f.pm = &a.pm;
  consume_log<VEC>(f, a.L, a.q, a.cs, a.off, a.col, nullptr, &wsm[warp], fsrc[warp], a.vec_ok);
  const long long tid = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  const long long stride = (long long)gridDim.x * blockDim.x;
  double d = 0.0;
  for (long long i = tid; i < a.n_dangling; i += stride) d += a.x[a.dangling[i]];
  d = warp_sumd(d);
  if (lane_id() == 0) red[warp] = d;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int k = 0; k < kWarps; ++k) s += red[k];
    if (s != 0.0) atomicAdd(a.dsum, s);
  }
}
__global__ void k_mpr_finalize(double *x, const double *yown, long long n_local, double base,
                               double dmp, const double *dsum_global, double N) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  const double add = base + dmp * (*dsum_global) / N;
  for (long long v = (long long)blockIdx.x * blockDim.x + threadIdx.x; v < n_local; v += stride)
    x[v] = add + dmp * yown[v];
}
__global__ void k_fill_f64(double *p, long long n, double v) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) p[i] = v;
}

// ============================================================================ host side
__global__ void k_peer_probe(uint32_t *const *peers, int world, int rank) {
  const int q = threadIdx.x;
  if (q < world && q != rank)
    atomicOr(reinterpret_cast<unsigned long long *>(peers[q]), 1ull << rank);
  __threadfence_system();
}
__global__ void k_peer_check(const unsigned long long *mine, int world, int rank, unsigned long long *bad) {
  const unsigned long long all = world == 64 ? ~0ull : (1ull << world) - 1ull;
  *bad = *mine != (all & ~(1ull << rank)) ? 1ull : 0ull;
}

sage_status init_comm(sage_graph *g, const sage_dist *ds) {
  Comm *c = new Comm();
  g->comm = c;
  c->rank = ds->rank;
  c->world = ds->world;
  if (c->world > kMaxRanks) {
    set_error("at most %d ranks", kMaxRanks);
    return SAGE_E_INVALID;
  }
  sage_status s;
  c->x = make_loopback_xport(g, ds->nccl_unique_id, c->rank, c->world, &s);
  if (!c->x && s == SAGE_OK) c->x = make_nccl_xport(g, ds->nccl_unique_id, c->rank, c->world, &s);
  if (!c->x) return s;
  // every rank's block and arc count
  long long *d = nullptr;
  if ((s = dalloc(g, (void **)&d, sizeof(long long) * 4 * (size_t)(c->world + 1))) != SAGE_OK) return s;
  long long mine[3] = {(long long)g->v_begin, (long long)g->v_end, (long long)g->m};
  cudaMemcpyAsync(d + 3 * c->rank, mine, sizeof(mine), cudaMemcpyHostToDevice, g->stream);
  XCHECK(c->x->allgather(g, d + 3 * c->rank, d, 3 * sizeof(long long)));
  std::vector<long long> all(3 * (size_t)c->world);
  cudaMemcpyAsync(all.data(), d, sizeof(long long) * all.size(), cudaMemcpyDeviceToHost, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  dfree(g, d);
  if (e != cudaSuccess) return cuda_fail(g, e, "comm init");
  c->vb.assign((size_t)c->world + 1, 0);
  long long maxrows = 0;
  for (int r = 0; r < c->world; ++r) {
    if (all[3 * r] != (r == 0 ? 0 : all[3 * (r - 1) + 1])) {
      set_error("rank blocks must cover [0, n) contiguously in rank order");
      return SAGE_E_INVALID;
    }
    c->vb[r] = all[3 * r];
    c->vb[r + 1] = all[3 * r + 1];
    maxrows = std::max(maxrows, all[3 * r + 1] - all[3 * r]);
    c->m_total += all[3 * r + 2];
  }
  if (c->vb[c->world] != g->n) {
    set_error("rank blocks must end at n");
    return SAGE_E_INVALID;
  }
  c->Wp = (maxrows + 31) / 32 + 1;
  memset(&c->pm, 0, sizeof(c->pm));
  c->pm.p = c->world;
  c->pm.rank = c->rank;
  c->pm.P = c->Wp * 32;
  for (int r = 0; r <= c->world; ++r) c->pm.vb[r] = c->vb[r];
  const size_t words = (size_t)c->Wp * (size_t)c->world;
  if ((s = dalloc(g, (void **)&c->out, 4 * words)) != SAGE_OK ||
      (s = dalloc(g, (void **)&c->recv, 4 * words)) != SAGE_OK ||
      (s = dalloc(g, (void **)&c->visited, 4 * words)) != SAGE_OK ||
      (s = dalloc(g, (void **)&c->stats, sizeof(unsigned long long) * 16)) != SAGE_OK)
    return s;
  for (int i = 0; i < 3; ++i)
    if ((s = dalloc(g, (void **)&c->fb[i], 4 * words)) != SAGE_OK) return s;
  if (cudaHostAlloc((void **)&c->hmap, 16 * sizeof(unsigned long long), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer((void **)&c->dmap, c->hmap, 0) != cudaSuccess) {
    cudaGetLastError();
    set_error("mapped pinned host memory unavailable");
    return SAGE_E_NOMEM;
  }
  memset(c->hmap, 0, 16 * sizeof(unsigned long long));
  // the fused push exchange over peer memory (sage_dist.exchange == 0); every rank takes the same
  // decision because peer_map's verdict is collective
  if (c->world > 1 && ds->exchange == 0) {
    cudaError_t e2 = cudaMalloc((void **)&c->inbox, 4 * (size_t)c->Wp * 33);
    if (e2 != cudaSuccess) return cuda_fail(g, e2, "peer inbox");
    cudaMemsetAsync(c->inbox, 0, 4 * (size_t)c->Wp * 33, g->stream);
    s = c->x->peer_map(g, c->inbox, c->peers);
    if (s == SAGE_OK) {
      if ((s = dalloc(g, (void **)&c->d_peers, sizeof(void *) * (size_t)c->world)) != SAGE_OK) return s;
      cudaMemcpyAsync(c->d_peers, c->peers, sizeof(void *) * (size_t)c->world, cudaMemcpyHostToDevice, g->stream);
      // probe before trusting the mapping: every rank ORs its bit into every peer's first word
      // pair, one barrier, every rank checks it holds exactly the others' bits; a collective
      // verdict keeps all ranks on the same form
      k_peer_probe<<<1, 64, 0, g->stream>>>(c->d_peers, c->world, c->rank);
      XCHECK(c->x->barrier(g));
      k_peer_check<<<1, 1, 0, g->stream>>>(reinterpret_cast<const unsigned long long *>(c->inbox), c->world,
                                           c->rank, c->stats);
      XCHECK(c->x->allreduce_sum_u64(g, c->stats, c->stats + 8, 1));
      unsigned long long bad = 0;
      cudaMemcpyAsync(&bad, c->stats + 8, sizeof(bad), cudaMemcpyDeviceToHost, g->stream);
      cudaMemsetAsync(c->inbox, 0, 8, g->stream);
      XCHECK(c->x->barrier(g));
      if ((e2 = cudaStreamSynchronize(g->stream)) != cudaSuccess) return cuda_fail(g, e2, "peer map");
      c->p2p = bad == 0;
      if (!c->p2p) c->x->peer_unmap(c->peers);
    } else if (s == SAGE_E_UNSUPPORTED) {
      clear_error();
    } else {
      return s;
    }
  }
  return SAGE_OK;
}

bool comm_peer_exchange(const sage_graph *g) { return g->comm && g->comm->p2p; }

void free_comm(sage_graph *g) {
  Comm *c = g->comm;
  if (!c) return;
  dfree(g, c->out);
  dfree(g, c->recv);
  dfree(g, c->visited);
  dfree(g, c->stats);
  for (int i = 0; i < 3; ++i) dfree(g, c->fb[i]);
  dfree(g, c->y);
  dfree(g, c->yown);
  dfree(g, c->dsum);
  dfree(g, c->cand);
  dfree(g, c->cown);
  dfree(g, c->sp_send);
  dfree(g, c->sp_recv);
  dfree(g, c->glevel);
  dfree(g, c->pcand);
  dfree(g, c->pown);
  dfree(g, c->d_peers);
  cudaStreamSynchronize(g->stream);
  if (c->p2p) c->x->peer_unmap(c->peers);
  if (c->inbox) cudaFree(c->inbox);
  if (c->hmap) cudaFreeHost(c->hmap);
  delete c->x;
  delete c;
  g->comm = nullptr;
}

// The per-level stats reach the host through mapped pinned memory: a one-warp kernel copies the
// allreduced counters and then a sequence number (after a system-scope fence), and the host spins
// on that number instead of synchronising the stream (no driver round trip per level).
__global__ void k_publish(const unsigned long long *src, int n, volatile unsigned long long *dst,
                          unsigned long long seq) {
  if (threadIdx.x < (unsigned)n) dst[threadIdx.x] = src[threadIdx.x];
  __threadfence_system();
  __syncwarp();
  if (threadIdx.x == 0) dst[15] = seq;
}
static sage_status wait_published(sage_graph *g, unsigned long long *h6, int n) {
  Comm *c = g->comm;
  const unsigned long long seq = ++c->pub_seq;
  k_publish<<<1, 32, 0, g->stream>>>(c->stats + 8, n, c->dmap, seq);
  volatile unsigned long long *hm = c->hmap;
  for (unsigned long long spins = 0; hm[15] != seq; ++spins) {
    if ((spins & 4095) == 4095) {   // the stream failed or is slow: look at it
      const cudaError_t q = cudaStreamQuery(g->stream);
      if (q != cudaSuccess && q != cudaErrorNotReady) return cuda_fail(g, q, "stats");
    }
  }
  for (int i = 0; i < n; ++i) h6[i] = hm[i];
  return SAGE_OK;
}

static sage_status allreduce_stats(sage_graph *g, int L, unsigned long long *h6) {
  Comm *c = g->comm;
  k_mstats<<<1, 32, 0, g->stream>>>(g->ts.ctl, L % 3, (L + 1) % 3, c->stats);
  XCHECK(c->x->allreduce_sum_u64(g, c->stats, c->stats + 8, 6));
  return wait_published(g, h6, 6);
}

sage_status run_bfs_multi(sage_graph *g, int32_t source, int32_t *level_out, int32_t *parent_out,
                          uint32_t call_flags, sage_stats *st) {
  Comm *c = g->comm;
  sage_status s;
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  TraversalState &t = g->ts;
  const bool symmetric = g->flags & SAGE_F_SYMMETRIC;
  const bool do_enabled = symmetric && !((g->flags | call_flags) & SAGE_F_PUSH_ONLY);
  const size_t words = (size_t)c->Wp * (size_t)c->world;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, g->stream);
  cudaMemsetAsync(t.level, 0xff, sizeof(int32_t) * (size_t)g->n_local, g->stream);
  cudaMemsetAsync(c->visited, 0, 4 * words, g->stream);
  cudaMemsetAsync(c->out, 0, 4 * words, g->stream);
  for (int i = 0; i < 3; ++i) cudaMemsetAsync(c->fb[i], 0, 4 * words, g->stream);
  cudaMemsetAsync(t.ctl, 0, offsetof(Ctl, rec), g->stream);
  MultiArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.n_local = g->n_local;
  a.v_begin = g->v_begin;
  a.L = g->ladder;
  a.q[0] = t.q[0];
  a.q[1] = t.q[1];
  a.ctl = t.ctl;
  a.visited = c->visited;
  for (int i = 0; i < 3; ++i) a.fb[i] = c->fb[i];
  a.out = c->out;
  a.recv = c->recv;
  a.level = t.level;
  a.flist = t.flist;
  a.do_enabled = do_enabled ? 1 : 0;
  a.vec_ok = g->vec_ok ? 1 : 0;
  a.pm = c->pm;
  a.pin = c->p2p ? c->d_peers : nullptr;
  if (c->p2p) cudaMemsetAsync(c->inbox, 0, 4 * (size_t)c->Wp, g->stream);   // ordered before any peer OR:
                                                                            // the seed's stats allreduce follows
  if (source >= g->v_begin && source < g->v_end)
    k_mseed<<<1, 32, 0, g->stream>>>(a, (long long)source - g->v_begin);
  // global arcs of the source (level-0 frontier)
  unsigned long long h6[6];
  {
    k_mstats<<<1, 32, 0, g->stream>>>(t.ctl, 2, 0, c->stats);   // set[0] = the seed's log
    XCHECK(c->x->allreduce_sum_u64(g, c->stats, c->stats + 8, 6));
    XCHECK(wait_published(g, h6, 6));
  }
  double mU = (double)c->m_total - (double)h6[1];
  unsigned long long reached_arcs = h6[1];
  unsigned long long aF_cur = h6[1];   // global arcs(F) of the level about to run
  const int grid_push = g->num_sms * 4;
  int dir = 0;
  unsigned long long prev_nF = 1;
  long long push_exp = 0, push_arcs = 0, push_disc = 0, pull_sc = 0, pull_insp = 0, pull_disc = 0;
  int levels = 0, pushL = 0, pullL = 0;
  for (int L = 0;; ++L) {
    cudaMemsetAsync(&t.ctl->set[(L + 2) % 3], 0, sizeof(CounterSet), g->stream);
    if (do_enabled) cudaMemsetAsync(c->fb[(L + 2) % 3], 0, 4 * words, g->stream);
    a.lvl = L;
    if (dir == 0) {
      // exchange form of this level (every rank knows the global arcs(F)): sparse lists of
      // capacity arcs(F) when that is smaller than a dense slice, else the dense slices
      const long long cap = (c->world > 1 && !c->p2p && (long long)aF_cur < c->Wp) ? (long long)aF_cur : 0;
      a.sp_cap = cap;
      if (cap) {
        const long long need = (cap + 2) * c->world;
        if (need > c->sp_words) {
          dfree(g, c->sp_send);
          dfree(g, c->sp_recv);
          c->sp_send = c->sp_recv = nullptr;
          const long long alloc = std::max<long long>(need, 4096);
          if ((s = dalloc(g, (void **)&c->sp_send, 4 * (size_t)alloc)) != SAGE_OK ||
              (s = dalloc(g, (void **)&c->sp_recv, 4 * (size_t)alloc)) != SAGE_OK)
            return s;
          c->sp_words = alloc;
        }
        cudaMemsetAsync(c->sp_send, 0, 4 * (size_t)need, g->stream);
        a.sp_send = c->sp_send;
        a.sp_recv = c->sp_recv;
      }
      if (g->vec == 4) k_mpush<4><<<grid_push, kBlock, 0, g->stream>>>(a);
      else k_mpush<1><<<grid_push, kBlock, 0, g->stream>>>(a);
      k_mclassify<<<grid_push, kBlock, 0, g->stream>>>(a);
      if (c->p2p) {
        // peer form: the candidates are already in the owners' inboxes; one barrier, then apply
        XCHECK(c->x->barrier(g));
        k_mapply<<<grid_push, kBlock, 0, g->stream>>>(a);
      } else if (c->world > 1) {
        std::vector<size_t> off((size_t)c->world + 1);
        const size_t blk = cap ? 4 * (size_t)(cap + 2) : 4 * (size_t)c->Wp;
        for (int r = 0; r <= c->world; ++r) off[(size_t)r] = blk * (size_t)r;
        if (cap) {
          XCHECK(c->x->alltoallv(g, c->sp_send, off.data(), c->sp_recv, off.data()));
          k_mapply_sparse<<<grid_push, kBlock, 0, g->stream>>>(a);
        } else {
          XCHECK(c->x->alltoallv(g, c->out, off.data(), c->recv, off.data()));
          cudaMemsetAsync(c->out, 0, 4 * words, g->stream);
          k_mapply<<<grid_push, kBlock, 0, g->stream>>>(a);
        }
      }
    } else {
      k_mpull<<<grid_push, kBlock, 0, g->stream>>>(a);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(g, e, "multi-GPU level");
    if ((s = allreduce_stats(g, L, h6)) != SAGE_OK) return s;
    const unsigned long long nF = h6[0], aF = h6[1];
    levels = L + 1;
    if (dir == 0) {
      pushL++;
      push_exp += (long long)h6[4];
      push_arcs += (long long)h6[5];
      push_disc += (long long)nF;
    } else {
      pullL++;
      pull_sc += (long long)h6[3];
      pull_insp += (long long)h6[2];
      pull_disc += (long long)nF;
    }
    reached_arcs += aF;
    aF_cur = aF;
    if (nF == 0) break;
    if (L + 1 > g->n) {
      set_error("level cap exceeded");
      return SAGE_E_CUDA;
    }
    mU -= (double)aF;
    int ndir = dir;
    if (do_enabled) {
      if (dir == 0) {
        if ((double)aF > mU / g->alpha) ndir = 1;
      } else {
        if (!(nF >= prev_nF || (double)nF > (double)g->n / g->beta)) ndir = 0;
      }
    }
    if (ndir == 1) {
      // pull needs the global frontier: allgather of every owner's slice of fb[L+1]
      uint32_t *fbn = c->fb[(L + 1) % 3];
      XCHECK(c->x->allgather(g, fbn + (size_t)c->rank * c->Wp, fbn, 4 * (size_t)c->Wp));
    }
    dir = ndir;
    prev_nF = nF;
  }
  cudaEventRecord(e1, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "multi-GPU BFS");
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (st) {
    memset(st, 0, sizeof(*st));
    st->levels = levels;
    st->push_levels = pushL;
    st->pull_levels = pullL;
    st->vertices_expanded = push_exp + pull_sc;
    st->arcs_inspected = push_arcs + pull_insp;
    st->vertices_discovered = push_disc + pull_disc;
    st->edges_traversed = (int64_t)(symmetric ? reached_arcs / 2 : reached_arcs);
    st->ms = ms;
    st->kernel_ms = ms;
    const double n = (double)g->n;
    st->model_bytes = 4.0 * n + 20.0 * push_exp + 8.0 * push_arcs + 8.0 * push_disc + 16.0 * pull_sc +
                      (n / 8.0) * pullL + 4.125 * pull_insp + 4.125 * pull_disc;
  }
  if (parent_out) {
    // any valid parent: allgather the levels (padded layout), propose the smallest u with
    // level(u) = level(v) - 1 for every target v of the own rows, min reduce-scatter to the owners
    const long long P = c->pm.P;
    if (!c->glevel) {
      if ((s = dalloc(g, (void **)&c->glevel, sizeof(int32_t) * (size_t)P * c->world)) != SAGE_OK ||
          (s = dalloc(g, (void **)&c->pcand, sizeof(uint32_t) * (size_t)P * c->world)) != SAGE_OK ||
          (s = dalloc(g, (void **)&c->pown, sizeof(uint32_t) * (size_t)P)) != SAGE_OK)
        return s;
    }
    if (!t.parent && (s = dalloc(g, (void **)&t.parent, sizeof(int32_t) * (size_t)g->n_local)) != SAGE_OK)
      return s;
    int32_t *mine = c->glevel + (size_t)c->rank * P;
    cudaMemsetAsync(mine, 0xff, sizeof(int32_t) * (size_t)P, g->stream);
    cudaMemcpyAsync(mine, t.level, sizeof(int32_t) * (size_t)g->n_local, cudaMemcpyDeviceToDevice, g->stream);
    XCHECK(c->x->allgather(g, mine, c->glevel, sizeof(int32_t) * (size_t)P));
    k_fill_u32<<<grid_push, 256, 0, g->stream>>>(c->pcand, P * c->world, 0xffffffffu);
    k_mparent_propose<<<grid_push, 256, 0, g->stream>>>(a, c->glevel, c->pcand);
    XCHECK(c->x->reduce_scatter_min_u32(g, c->pcand, c->pown, (size_t)P));
    k_mparent_final<<<grid_push, 256, 0, g->stream>>>(t.level, c->pown, g->n_local, t.parent);
    if ((s = copy_out(g, parent_out, t.parent, sizeof(int32_t) * (size_t)g->n_local)) != SAGE_OK) return s;
  }
  if ((s = copy_out(g, level_out, t.level, sizeof(int32_t) * (size_t)g->n_local)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "output");
  return SAGE_OK;
}

// Multi-GPU SSSP: host-sequenced frontier Bellman-Ford iterations.  Per iteration: local push
// (own targets relaxed in place, remote ones into cand) -> ncclReduceScatter(min) of cand to the
// owners (C1e with min instead of sum) -> owners apply and enqueue -> stats allreduce (C1d).
sage_status run_sssp_multi(sage_graph *g, int32_t source, uint32_t *dist_out, sage_stats *st) {
  Comm *c = g->comm;
  sage_status s;
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  TraversalState &t = g->ts;
  if (!t.dist && (s = dalloc(g, (void **)&t.dist, sizeof(uint32_t) * (size_t)g->n_local)) != SAGE_OK)
    return s;
  const long long P = c->pm.P;
  if (!c->cand) {
    if ((s = dalloc(g, (void **)&c->cand, sizeof(uint32_t) * (size_t)P * c->world)) != SAGE_OK ||
        (s = dalloc(g, (void **)&c->cown, sizeof(uint32_t) * (size_t)P)) != SAGE_OK)
      return s;
  }
  int *ovf = nullptr;
  if ((s = dalloc(g, (void **)&ovf, sizeof(int) * 4)) != SAGE_OK) return s;
  const size_t lwords = (size_t)((g->n_local + 31) / 32 + 1);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, g->stream);
  cudaMemsetAsync(ovf, 0, sizeof(int) * 4, g->stream);
  cudaMemsetAsync(t.dist, 0xff, sizeof(uint32_t) * (size_t)g->n_local, g->stream);
  cudaMemsetAsync(c->cand, 0xff, sizeof(uint32_t) * (size_t)P * c->world, g->stream);
  if (c->p2p) cudaMemsetAsync(c->inbox + c->Wp, 0xff, sizeof(uint32_t) * (size_t)P, g->stream);
  for (int i = 0; i < 3; ++i) cudaMemsetAsync(t.fb[i], 0, sizeof(uint32_t) * lwords, g->stream);
  cudaMemsetAsync(t.ctl, 0, offsetof(Ctl, rec), g->stream);
  MultiArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.w = g->w;
  a.n_local = g->n_local;
  a.v_begin = g->v_begin;
  a.L = g->ladder;
  a.q[0] = t.q[0];
  a.q[1] = t.q[1];
  a.ctl = t.ctl;
  a.vec_ok = g->vec_ok ? 1 : 0;
  a.pm = c->pm;
  a.dist = t.dist;
  a.cand = c->cand;
  a.cown = c->p2p ? c->inbox + c->Wp : c->cown;
  a.pin = c->p2p ? c->d_peers : nullptr;
  a.overflow = ovf;
  if (source >= g->v_begin && source < g->v_end)
    k_msssp_seed<<<1, 32, 0, g->stream>>>(a, (long long)source - g->v_begin);
  const int grid = g->num_sms * 4;
  if (c->p2p) XCHECK(c->x->barrier(g));   // every rank's minima reset before any peer update
  unsigned long long h6[6];
  long long exp_ = 0, arcs = 0, impr = 0;
  int iters = 0;
  for (int L = 0;; ++L) {
    cudaMemsetAsync(&t.ctl->set[(L + 2) % 3], 0, sizeof(CounterSet), g->stream);
    cudaMemsetAsync(t.fb[(L + 2) % 3], 0, sizeof(uint32_t) * lwords, g->stream);
    a.lvl = L;
    a.inq_next = t.fb[(L + 1) % 3];
    if (g->vec == 4) k_msssp_push<4><<<grid, kBlock, 0, g->stream>>>(a);
    else k_msssp_push<1><<<grid, kBlock, 0, g->stream>>>(a);
    if (c->p2p) {
      // peer form: the owners' minima were improved in place (monotone, never reset: an entry
      // that does not beat dist is a no-op for k_msssp_apply); one barrier, then apply
      XCHECK(c->x->barrier(g));
    } else {
      XCHECK(c->x->reduce_scatter_min_u32(g, c->cand, c->cown, (size_t)P));
      cudaMemsetAsync(c->cand, 0xff, sizeof(uint32_t) * (size_t)P * c->world, g->stream);
    }
    if (c->world > 1) k_msssp_apply<<<grid, kBlock, 0, g->stream>>>(a);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) {
      dfree(g, ovf);
      return cuda_fail(g, e, "multi-GPU SSSP iteration");
    }
    if ((s = allreduce_stats(g, L, h6)) != SAGE_OK) {
      dfree(g, ovf);
      return s;
    }
    iters = L + 1;
    exp_ += (long long)h6[4];
    arcs += (long long)h6[5];
    impr += (long long)h6[0];
    if (h6[0] == 0) break;
    if (L + 1 > 4 * g->n + 64) {
      dfree(g, ovf);
      set_error("SSSP iteration cap exceeded (internal error)");
      return SAGE_E_CUDA;
    }
  }
  // overflow: any rank saw du + w >= 2^32 -> check reached -> unreached arcs globally
  unsigned long long *red = c->stats;   // reuse: [0] local flag, [8] global
  int hflag = 0;
  cudaMemcpyAsync(&hflag, ovf, sizeof(int), cudaMemcpyDeviceToHost, g->stream);
  cudaStreamSynchronize(g->stream);
  unsigned long long fl[2] = {(unsigned long long)hflag, 0ull};
  cudaMemcpyAsync(red, fl, sizeof(unsigned long long), cudaMemcpyHostToDevice, g->stream);
  XCHECK(c->x->allreduce_sum_u64(g, red, red + 8, 1));
  cudaMemcpyAsync(&fl[1], red + 8, sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream);
  cudaStreamSynchronize(g->stream);
  if (fl[1]) {
    uint32_t *bits = c->visited;   // p*Wp words, padded layout
    k_mreached_bits<<<grid, 256, 0, g->stream>>>(t.dist, g->n_local, bits + (size_t)c->rank * c->Wp);
    XCHECK(c->x->allgather(g, bits + (size_t)c->rank * c->Wp, bits, 4 * (size_t)c->Wp));
    k_moverflow_check<<<grid, 256, 0, g->stream>>>(a, bits, ovf + 1);
    int hf = 0;
    cudaMemcpyAsync(&hf, ovf + 1, sizeof(int), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
    fl[0] = (unsigned long long)hf;
    cudaMemcpyAsync(red, fl, sizeof(unsigned long long), cudaMemcpyHostToDevice, g->stream);
    XCHECK(c->x->allreduce_sum_u64(g, red, red + 8, 1));
    cudaMemcpyAsync(&fl[1], red + 8, sizeof(unsigned long long), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
    if (fl[1]) {
      dfree(g, ovf);
      set_error("a finite shortest distance is >= UINT32_MAX");
      return SAGE_E_OVERFLOW;
    }
  }
  cudaEventRecord(e1, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  dfree(g, ovf);
  if (e != cudaSuccess) return cuda_fail(g, e, "multi-GPU SSSP");
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  // reached arcs (collective on every rank, whether or not this rank asked for stats)
  unsigned long long hra = 0;
  {
    unsigned long long *ra = c->stats;
    cudaMemsetAsync(ra, 0, sizeof(unsigned long long), g->stream);
    k_mreached_arcs<<<grid, 256, 0, g->stream>>>((const long long *)g->off, t.dist, g->n_local, ra);
    XCHECK(c->x->allreduce_sum_u64(g, ra, ra + 8, 1));
    cudaMemcpyAsync(&hra, ra + 8, sizeof(hra), cudaMemcpyDeviceToHost, g->stream);
    cudaStreamSynchronize(g->stream);
  }
  if (st) {
    memset(st, 0, sizeof(*st));
    st->levels = st->push_levels = iters;
    st->vertices_expanded = exp_;
    st->arcs_inspected = arcs;
    st->vertices_discovered = impr;
    st->edges_traversed = (int64_t)((g->flags & SAGE_F_SYMMETRIC) ? hra / 2 : hra);
    st->ms = st->kernel_ms = ms;
    st->model_bytes = 4.0 * (double)g->n + 24.0 * exp_ + 12.0 * arcs + 8.0 * impr;
  }
  if ((s = copy_out(g, dist_out, t.dist, sizeof(uint32_t) * (size_t)g->n_local)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "output");
  return SAGE_OK;
}

sage_status run_pagerank_multi(sage_graph *g, double damping, int32_t iterations, double *rank_out,
                               sage_stats *st) {
  Comm *c = g->comm;
  sage_status s;
  if ((s = ensure_traversal_state(g)) != SAGE_OK) return s;
  if ((s = ensure_pagerank_log(g)) != SAGE_OK) return s;
  const long long P = c->pm.P;
  if (!c->y) {
    if ((s = dalloc(g, (void **)&c->y, sizeof(double) * (size_t)P * c->world)) != SAGE_OK ||
        (s = dalloc(g, (void **)&c->yown, sizeof(double) * (size_t)P)) != SAGE_OK ||
        (s = dalloc(g, (void **)&c->dsum, sizeof(double) * 2)) != SAGE_OK)
      return s;
  }
  PageRankState &p = g->pr;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, g->stream);
  const int grid = g->num_sms * 4;
  k_fill_f64<<<grid, 256, 0, g->stream>>>(p.x, g->n_local, 1.0 / (double)g->n);
  MprArgs a;
  memset(&a, 0, sizeof(a));
  a.off = (const long long *)g->off;
  a.col = g->col;
  a.L = g->ladder;
  a.q = p.q;
  a.cs = p.cs;
  a.dangling = p.dangling;
  a.n_dangling = p.n_dangling;
  a.x = p.x;
  a.y = c->y;
  a.dsum = c->dsum;
  a.vec_ok = g->vec_ok ? 1 : 0;
  a.pm = c->pm;
  const double N = (double)g->n;
  for (int it = 0; it < iterations; ++it) {
    cudaMemsetAsync(c->y, 0, sizeof(double) * (size_t)P * c->world, g->stream);
    cudaMemsetAsync(c->dsum, 0, sizeof(double), g->stream);
    cudaMemsetAsync(&p.cs[0].tk, 0, sizeof(p.cs[0].tk), g->stream);
    if (g->vec == 4) k_mpr_push<4><<<grid, kBlock, 0, g->stream>>>(a);
    else k_mpr_push<1><<<grid, kBlock, 0, g->stream>>>(a);
    XCHECK(c->x->reduce_scatter_sum_f64(g, c->y, c->yown, (size_t)P));
    XCHECK(c->x->allreduce_sum_f64(g, c->dsum, c->dsum + 1, 1));
    k_mpr_finalize<<<grid, 256, 0, g->stream>>>(p.x, c->yown, g->n_local, (1.0 - damping) / N, damping,
                                                c->dsum + 1, N);
  }
  cudaEventRecord(e1, g->stream);
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "multi-GPU PageRank");
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (st) {
    memset(st, 0, sizeof(*st));
    st->levels = st->push_levels = iterations;
    st->edges_traversed = st->arcs_inspected = (int64_t)iterations * c->m_total;
    st->ms = st->kernel_ms = ms;
    st->model_bytes = (double)iterations * (40.0 * (double)g->n_local + 12.0 * (double)g->m);
  }
  if ((s = copy_out(g, rank_out, p.x, sizeof(double) * (size_t)g->n_local)) != SAGE_OK) return s;
  e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "output");
  return SAGE_OK;
}

}  // namespace sage

extern "C" sage_status sage_nccl_unique_id(void *out128) {
  sage::clear_error();
  if (!out128) {
    sage::set_error("null argument");
    return SAGE_E_INVALID;
  }
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) {
    sage::set_error("ncclGetUniqueId: %s", ncclGetErrorString(r));
    return SAGE_E_NCCL;
  }
  memcpy(out128, &id, sizeof(id));
  return SAGE_OK;
}
