// common.cuh — device-side building blocks shared by the SAGE kernels (sm_100a).
//
// Product code (libsage.so).  Shares nothing with oracle/ (the CPU checker).
//
//  * Tile geometry of Tiled Partitioning (Alg. 2; §5.1; Fig. 3):
//    a row [b, e) is split into an optional head fragment that brings b to a multiple of the
//    alignment A (tile alignment, reading R14), q = floor(rest/B) "CTA" tiles of B
//    elements, one tile per set bit t in B/2 .. M of the residual r = rest mod B (the binary
//    partition of P:257, residual kept at the row end, Alg. 2 l.14-16, R12), and a tail
//    fragment of r mod M elements (< MIN_TILE_SIZE, Alg. 2 l.32).  Closed form used by every
//    consumer: the class-t tile of the row is [e - (r & (2t-1)), + t).
//  * Resident tile log (Alg. 3 l.2-7): per class c (tile size B >> c) a queue.
//    Class 0 entries are explicit (start, vertex) CTA tiles (Alg. 3's (node, offset, size));
//    classes 1..ncls-1 and the fragment queue hold vertex ids, the offset being implied by the
//    closed form above (4 B per entry instead of 16).
//  * The warp-aggregated enqueue (contraction) classifies a newly filtered-in vertex into
//    the next level's log in the same pass (expandTiles fused with filter_in).
#pragma once
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <type_traits>
#include <stdint.h>

namespace sage {

namespace cg = cooperative_groups;

constexpr unsigned FULL = 0xffffffffu;
constexpr int kMaxCls = 13;          // B/M <= 4096 -> at most 13 tile classes
constexpr int kQueues = kMaxCls + 1; // + fragment queue
constexpr int kBlock = 256;          // threads per CTA of the persistent kernels
constexpr int kWarps = kBlock / 32;

struct CtaTile {       // explicit CTA-class tile (Alg. 3's (node, offset, size) triple)
  long long start;     // first arc index
  int u;               // source vertex (local row index)
  int len;             // == B
};

struct Ladder {        // tile ladder (sage_options)
  int B, M, A;         // CTA tile, MIN_TILE_SIZE, alignment (elements; 0 = paper mode)
  int lgB;             // log2(B)
  int ncls;            // number of tile classes = log2(B/M) + 1 (class c has size B >> c)
};

struct Queues {        // one resident tile log (one level's, or the all-V log of PageRank)
  CtaTile *cta;        // class 0
  int *cls[kMaxCls];   // cls[c], 1 <= c < ncls
  int *frag;           // fragment queue (vertex ids)
  int *order;          // optional: every enqueued vertex is also appended here (BC's BFS order)
  unsigned long long *order_cnt;
};

// One counter per 128-B line: every warp of the grid hits these with atomics, and counters that
// share a line serialise on the same L2 slice.
struct alignas(128) PaddedCounter {
  unsigned long long v;
  unsigned long long pad[15];
};
struct CounterSet {                      // counters of one log (rotated over 3 levels)
  PaddedCounter cnt[kQueues];            // entries per queue (index ncls = fragment queue)
  PaddedCounter tk[kQueues];             // stealing tickets per queue
  PaddedCounter nF, arcsF;               // |F| and arcs(F) of the vertices enqueued here
  PaddedCounter inspected;               // pull: arcs inspected while consuming this level
  PaddedCounter scanned;                 // pull: unvisited non-isolated vertices scanned
  PaddedCounter flc;                     // deferred contraction: frontier-list slots reserved
  PaddedCounter ftk;                     // fused tiling: frontier-list chunk tickets
  PaddedCounter hubc;                    // fused tiling: hub-table slots changed in this level
};

struct LevelRec {                        // per-level record (first kMaxRec levels)
  int dir;                               // 0 push, 1 pull
  int pad_;
  unsigned long long nF, arcsF, inspected, scanned, discovered;
  unsigned long long t_ns;               // %globaltimer at the end of the level
  unsigned long long t_work;             // %globaltimer when the last warp finished its work
  unsigned long long t_mid;              // %globaltimer after the expansion's grid barrier (K2' start)
};
constexpr int kMaxRec = 4096;

struct alignas(128) GridBar {
  unsigned int count;
  unsigned int pad0[31];
  unsigned int gen;
  unsigned int pad1[31];
};
struct Ctl {                             // control block of one query (device memory)
  CounterSet set[3];
  unsigned long long tot_push_expanded, tot_push_arcs, tot_push_disc;
  unsigned long long tot_pull_scanned, tot_pull_inspected, tot_pull_disc;
  unsigned long long tot_arcs_reached;   // sum of out-degrees of reached / enqueued vertices
  int levels, push_levels, pull_levels;
  int status;                            // 0 ok, 1 iteration cap hit, 2 possible overflow
  double D[3];                           // PageRank dangling mass (rotated)
  unsigned long long tot_improved;
  unsigned long long t0_ns;              // %globaltimer at kernel start
  GridBar bar;                           // grid barrier of the persistent kernel
  unsigned long long prof[16];           // SAGE_PROF builds: per-phase cycle sums
  int tail_state;                        // tail mode: 1 = traversal finished, 2 = resume grid mode
  int tail_n;                            // fused tail entry: vertices of the compacted list
  int tail_resume;                       // tail mode: level at which the grid resumes
  unsigned long long tail_levels;        // levels run in tail mode (diagnostic)
  LevelRec rec[kMaxRec];
};

// ------------------------------------------------------------------------------------------
// Loads.  col / w / off are read-only for the lifetime of every kernel -> non-coherent path,
// streaming (no L1 allocation) for the column stream.  Data produced inside a persistent
// kernel (queues, counters) is read through L2 (ld.cg).
__device__ __forceinline__ int4 ld_stream4(const int *p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ld_stream4u(const uint32_t *p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ int ld_stream1(const int *p) {
  int r;
  asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream1u(const uint32_t *p) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
// row offsets: read-only, re-read by the K2' passes and the consumer's metadata round -> L1-
// allocating non-coherent loads (round 1 A/B: L1::evict_last equal, L1::no_allocate +3%)
__device__ __forceinline__ long long ld_off(const long long *p) { return __ldg(p); }
__device__ __forceinline__ void ld_row_pair(const long long *off, int v, long long *b, long long *e) {
  *b = ld_off(off + v);
  *e = ld_off(off + v + 1);
}

// L2 cache policies: the column / weight stream is read once per level -> evict_first; the
// status words (visited bitmap, dist) are re-read at random all level long -> evict_last.
// SAGE_COL_POLICY (A/B builds only): 0 = evict_first (default), 1 = evict_normal, 2 = evict_first
// on half of the lines (fractional 0.5, the rest evict_unchanged)
#ifndef SAGE_COL_POLICY
#define SAGE_COL_POLICY 0
#endif
__device__ __forceinline__ unsigned long long policy_evict_first() {
  unsigned long long p;
#if SAGE_COL_POLICY == 1
  asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(p));
#elif SAGE_COL_POLICY == 2
  asm volatile("createpolicy.fractional.L2::evict_first.L2::evict_unchanged.b64 %0, 0.5;" : "=l"(p));
#else
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
#endif
  return p;
}
__device__ __forceinline__ unsigned long long policy_evict_last() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ int ld_col(const int *p, unsigned long long pol) {
  int r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;"
               : "=r"(r) : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ int4 ld_col4(const int *p, unsigned long long pol) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint4 ld_col4u(const uint32_t *p, unsigned long long pol) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint32_t ld_colu(const uint32_t *p, unsigned long long pol) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;"
               : "=r"(r) : "l"(p), "l"(pol));
  return r;
}
// status word load (kept in L2; a stale read is harmless for the visited bitmap: bits only go
// 0 -> 1 within a kernel and the atomicOr claim decides).  Status loads' L1 policy: 2 = L1::evict_last (default; hub status words stay in L1, measured
// 2.767 -> 2.742 ms on C2 push BFS), 1 = L1::no_allocate (2.786), 0 = default allocation
#ifndef SAGE_STATUS_L1
#define SAGE_STATUS_L1 2
#endif
// small-log class split (`consume_log`): the classes run concurrently while every class needs at
// most SAGE_SPLIT_K grabs per warp of its group (A/B knob)
#ifndef SAGE_SPLIT_K
#define SAGE_SPLIT_K 1
#endif
// medium logs: proportional class split while the log holds <= SAGE_SPLIT_PROP elements per warp
// (0 = off; big logs measured 2x slower with it)
#ifndef SAGE_SPLIT_PROP
#define SAGE_SPLIT_PROP 0
#endif
// stealing ticket batches (`consume_log`): grabs per warp per class, column elements per grab
#ifndef SAGE_TK_GRABS
#define SAGE_TK_GRABS 2
#endif
#ifndef SAGE_TK_ELEMS
#define SAGE_TK_ELEMS 4096
#endif

__device__ __forceinline__ uint32_t ld_status(const uint32_t *p, unsigned long long pol) {
  uint32_t r;
#if defined(SAGE_STATUS_L1) && SAGE_STATUS_L1 == 1
  asm volatile("ld.global.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
#elif defined(SAGE_STATUS_L1) && SAGE_STATUS_L1 == 2
  asm volatile("ld.global.L1::evict_last.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
#else
  asm volatile("ld.global.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
#endif
  return r;
}
// Predicated atomicOr: issues the atomic only when `pred`; otherwise returns `dflt`.  Written as
// one predicated instruction (no branch) so a lane's several claims are in flight together.
__device__ __forceinline__ uint32_t atom_or_if(bool pred, uint32_t *p, uint32_t bits, uint32_t dflt) {
  uint32_t r = dflt;
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %3, 0;\n\t@q atom.global.or.b32 %0, [%1], %2;\n\t}"
               : "+r"(r) : "l"(p), "r"(bits), "r"((uint32_t)pred));
  return r;
}
// fp64 add without a return value.  atomicAdd(double *) whose result is unused can still come out
// as a returning ATOMG (it did in the PageRank push filter); red.global.add.f64 is the REDG form.
__device__ __forceinline__ void red_add_f64(double *p, double v) {
  asm volatile("red.global.add.f64 [%0], %1;" ::"l"(p), "d"(v) : "memory");
}
template <class T> __device__ __forceinline__ T ldcg(const T *p) { return __ldcg(p); }
__device__ __forceinline__ CtaTile ldcg_tile(const CtaTile *p) {
  longlong2 v = __ldcg(reinterpret_cast<const longlong2 *>(p));
  CtaTile t;
  t.start = v.x;
  t.u = (int)(v.y & 0xffffffffll);
  t.len = (int)(v.y >> 32);
  return t;
}
__device__ __forceinline__ void st_tile(CtaTile *p, long long start, int u, int len) {
  longlong2 v;
  v.x = start;
  v.y = (long long)(unsigned)u | ((long long)len << 32);
  *reinterpret_cast<longlong2 *>(p) = v;
}

__device__ __forceinline__ unsigned long long globaltimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ unsigned long long shfl64(unsigned long long v, int src) {
  return __shfl_sync(FULL, v, src);
}
__device__ __forceinline__ unsigned long long warp_sum64(unsigned long long v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}
__device__ __forceinline__ double warp_sumd(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(FULL, v, o);
  return v;
}

// ------------------------------------------------------------------------------------------
// Grid-wide barrier of the persistent kernels (launched cooperatively, so every CTA is
// resident).  Waiting CTA leaders back off with __nanosleep instead of hammering the flag's L2
// line, which would slow down the warps still working on a small level.
__device__ __forceinline__ unsigned ld_acquire_gpu(const unsigned *p) {
  unsigned v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(unsigned *p, unsigned v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// CTA-interleaved warp rank: rank r is warp r / gridDim.x of CTA r % gridDim.x, so a level with
// fewer work units than warps (the first `grabs` ranks take one each) spreads them over every SM
// instead of packing them into the first few CTAs (C2 level 1: 354 CTA tiles went to 11 SMs).
#ifndef SAGE_WARP_RANK_LINEAR
#define SAGE_WARP_RANK_LINEAR 0   // A/B: 1 = rank r is warp r % (warps per CTA) of CTA r / (warps per CTA)
#endif
__device__ __forceinline__ long long warp_rank() {
  if (SAGE_WARP_RANK_LINEAR) return ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  return (long long)(threadIdx.x >> 5) * gridDim.x + blockIdx.x;
}

__device__ __forceinline__ void grid_barrier(GridBar *b) {
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned g = ld_acquire_gpu(&b->gen);
    __threadfence();
    if (atomicAdd(&b->count, 1u) == gridDim.x - 1) {
      b->count = 0;
      __threadfence();
      st_release_gpu(&b->gen, g + 1);
    } else {
      unsigned ns = 32;
      while (ld_acquire_gpu(&b->gen) == g) {
        __nanosleep(ns);
        if (ns < 512) ns <<= 1;
      }
    }
    __threadfence();
  }
  __syncthreads();
}

// ------------------------------------------------------------------------------------------
// Row split of Tiled Partitioning (see header comment).
struct RowSplit {
  long long b2;  // first element after the head fragment
  long long q;   // number of CTA tiles
  int r;         // residual after the CTA tiles (< B)
  int h;         // head-fragment length (< A)
};
__device__ __forceinline__ RowSplit split_row(long long b, long long e, const Ladder &L) {
  RowSplit s;
  long long d = e - b;
  int h = 0;
  if (L.A > 0) {
    h = (int)((L.A - (b & (L.A - 1))) & (L.A - 1));
    if (h > d) h = (int)d;
  }
  s.h = h;
  s.b2 = b + h;
  long long rest = e - s.b2;
  s.q = rest >> L.lgB;
  s.r = (int)(rest & (L.B - 1));
  return s;
}
// start of the class-t tile of a row ending at e with residual r (requires r & t)
__device__ __forceinline__ long long class_tile_start(long long e, int r, int t) {
  return e - (long long)(r & (2 * t - 1));
}

// ------------------------------------------------------------------------------------------
// Warp-aggregated enqueue = expandTiles (Alg. 3 l.2-7) of the vertices filtered in by this warp.
// Every lane of the warp must call it (convergent).  `active` lanes carry vertex v with row
// [b, e).  Appends v's tiles to the log Q, counting in cs, and accumulates |F| and arcs(F).
// All queue reservations of one call are issued in ONE parallel round of atomics (lane c reserves
// for queue c), so a call costs a single atomic latency whatever the number of classes.
__device__ __forceinline__ void enqueue_warp(bool active, int v, long long b, long long e,
                                             const Ladder &L, const Queues &Q, CounterSet *cs,
                                             bool count_f = true) {
  const unsigned am = __ballot_sync(FULL, active);
  if (!am) return;
  const unsigned lane = lane_id();
  const unsigned lt = lanemask_lt();
  RowSplit s{0, 0, 0, 0};
  if (active) s = split_row(b, e, L);
  // heavy vertices: exclusive scan of their CTA-tile counts
  unsigned long long q = active ? (unsigned long long)s.q : 0ull;
  unsigned long long incq = q;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    unsigned long long y = __shfl_up_sync(FULL, incq, o);
    if ((int)lane >= o) incq += y;
  }
  const unsigned long long totq = shfl64(incq, 31);
  unsigned long long deg = active ? (unsigned long long)(e - b) : 0ull;
  deg = warp_sum64(deg);
  // class ballots; lane c keeps the ballot of queue c (c = 1..ncls-1 tiles, ncls = fragments)
  unsigned cm[kQueues];
  unsigned mine_mask = 0;
#pragma unroll
  for (int c = 1; c < kQueues; ++c) {
    cm[c] = 0;
    if (c < L.ncls) cm[c] = __ballot_sync(FULL, active && (s.r & (L.B >> c)));
    else if (c == L.ncls) cm[c] = __ballot_sync(FULL, active && (s.h > 0 || (s.r & (L.M - 1)) != 0));
    if ((int)lane == c) mine_mask = cm[c];
  }
  // one parallel round of reservations
  unsigned long long mybase = 0;
  if (lane == 0) {
    if (totq) mybase = atomicAdd(&cs->cnt[0].v, totq);
  } else if ((int)lane <= L.ncls) {
    if (mine_mask) mybase = atomicAdd(&cs->cnt[lane].v, (unsigned long long)__popc(mine_mask));
  } else if (lane == 29) {
    if (Q.order) mybase = atomicAdd(Q.order_cnt, (unsigned long long)__popc(am));
  } else if (lane == 30) {
    if (count_f) atomicAdd(&cs->nF.v, (unsigned long long)__popc(am));
  } else if (lane == 31) {
    if (deg && count_f) atomicAdd(&cs->arcsF.v, deg);
  }
  if (Q.order) {
    const unsigned long long ob = shfl64(mybase, 29);
    if (active) Q.order[ob + __popc(am & lt)] = v;
  }
  // sub-CTA classes and fragments
#pragma unroll
  for (int c = 1; c < kQueues; ++c) {
    if (c > L.ncls) break;
    const unsigned long long base = shfl64(mybase, c);
    if (cm[c] & (1u << lane)) {
      int *qp = (c == L.ncls) ? Q.frag : Q.cls[c];
      qp[base + __popc(cm[c] & lt)] = v;
    }
  }
  // CTA class: cooperative write of every heavy vertex's q explicit tiles.
  if (totq) {
    const unsigned long long base0 = shfl64(mybase, 0);
#ifndef SAGE_ENQ_LANEQ
#define SAGE_ENQ_LANEQ 16
#endif
    // vertices with few CTA tiles write them from their own lane; the warp writes the rest
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
      for (unsigned long long j = lane; j < qs; j += 32)
        st_tile(Q.cta + bs + j, b2 + (long long)j * L.B, vv, L.B);
    }
  }
}

// Two-pass form of enqueue_warp for a warp that classifies many 32-vertex groups (the K2' phase):
// enqueue_count accumulates what the groups need (lane 0: CTA tiles, lane c: entries of queue c,
// lane 29: order-list entries; nF / arcs warp-uniform), the warp reserves everything with ONE
// round of atomics, and enqueue_write writes each group at the running bases (no atomics).
__device__ __forceinline__ void enqueue_count(bool active, long long b, long long e, const Ladder &L,
                                              unsigned long long &tot, unsigned long long &nf,
                                              unsigned long long &arcs) {
  const unsigned am = __ballot_sync(FULL, active);
  if (!am) return;
  const unsigned lane = lane_id();
  RowSplit s{0, 0, 0, 0};
  if (active) s = split_row(b, e, L);
  const unsigned long long totq = warp_sum64(active ? (unsigned long long)s.q : 0ull);
  arcs += warp_sum64(active ? (unsigned long long)(e - b) : 0ull);
  nf += (unsigned long long)__popc(am);
#pragma unroll
  for (int c = 1; c < kQueues; ++c) {
    unsigned cm = 0;
    if (c < L.ncls) cm = __ballot_sync(FULL, active && (s.r & (L.B >> c)));
    else if (c == L.ncls) cm = __ballot_sync(FULL, active && (s.h > 0 || (s.r & (L.M - 1)) != 0));
    if ((int)lane == c) tot += (unsigned long long)__popc(cm);
  }
  if (lane == 0) tot += totq;
  if (lane == 29) tot += (unsigned long long)__popc(am);
}
__device__ __forceinline__ void enqueue_write(bool active, int v, long long b, long long e, const Ladder &L,
                                              const Queues &Q, unsigned long long &run) {
  const unsigned am = __ballot_sync(FULL, active);
  if (!am) return;
  const unsigned lane = lane_id();
  const unsigned lt = lanemask_lt();
  RowSplit s{0, 0, 0, 0};
  if (active) s = split_row(b, e, L);
  unsigned long long q = active ? (unsigned long long)s.q : 0ull;
  unsigned long long incq = q;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    unsigned long long y = __shfl_up_sync(FULL, incq, o);
    if ((int)lane >= o) incq += y;
  }
  const unsigned long long totq = shfl64(incq, 31);
  if (Q.order) {
    const unsigned long long ob = shfl64(run, 29);
    if (active) Q.order[ob + __popc(am & lt)] = v;
    if (lane == 29) run += (unsigned long long)__popc(am);
  }
#pragma unroll
  for (int c = 1; c < kQueues; ++c) {
    if (c > L.ncls) break;
    unsigned cm;
    if (c < L.ncls) cm = __ballot_sync(FULL, active && (s.r & (L.B >> c)));
    else cm = __ballot_sync(FULL, active && (s.h > 0 || (s.r & (L.M - 1)) != 0));
    const unsigned long long base = shfl64(run, c);
    if (cm & (1u << lane)) {
      int *qp = (c == L.ncls) ? Q.frag : Q.cls[c];
      qp[base + __popc(cm & lt)] = v;
    }
    if ((int)lane == c) run += (unsigned long long)__popc(cm);
  }
  if (totq) {
    const unsigned long long base0 = shfl64(run, 0);
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
      for (unsigned long long j = lane; j < qs; j += 32)
        st_tile(Q.cta + bs + j, b2 + (long long)j * L.B, vv, L.B);
    }
    if (lane == 0) run += totq;
  }
}

// enqueue_warp for vertex ids only: loads the rows first (one round of loads for the warp).
// Not inlined: it is the cold path of the consumer (once per 32 filtered-in vertices) and
// inlining it at every call site multiplies the kernel's code size (I-cache misses).
static __device__ __noinline__ void enqueue_ids(bool active, int v, const long long *__restrict__ off,
                                            const Ladder &L, const Queues &Q, CounterSet *cs) {
  long long b = 0, e = 0;
  if (active) ld_row_pair(off, v, &b, &e);
  enqueue_warp(active, v, b, e, L, Q, cs);
}

// Per-warp shared scratch: the fragment gather's tables and the buffer of filtered-in vertices
// (contraction is batched: 32 vertices per enqueue call, not one call per discovery).
struct WarpScratch {
  int pre[32];
  int hl[32];
  long long hb[32];
  int tb[32];          // fragment gather: tail start - head start (a row's length fits 31 bits)
  int buf[64];
  long long cpos, cend;   // deferred contraction: the warp's open chunk of the frontier list
  unsigned long long ndisc;   // deferred contraction: vertices appended since the last close
};

#ifdef SAGE_PROF
__device__ unsigned long long g_prof[16];
#define PROF_T(x) long long x = clock64()
#define PROF_ADD(i, v) if (lane_id() == 0) atomicAdd(&g_prof[i], (unsigned long long)(v))
#else
#define PROF_T(x)
#define PROF_ADD(i, v)
#endif

// ---- deferred contraction (filters with kDefer and a non-null flist; the kernels leave flist null
// on small levels, where the second grid barrier would cost more than the enqueue stalls it
// saves): a filtered-in vertex is only appended
// to a plain frontier list (32-slot groups inside 256-slot chunks reserved per warp, -1 = empty
// slot); Tiled Partitioning of the list into the next level's log runs as its own grid phase after
// the level (K2' before K3', Fig. 2), where every warp classifies with all its loads in flight,
// instead of stalling the consumer warp for an enqueue round trip every 32 discoveries.
template <class F, class = void> struct DeferTrait { static constexpr bool value = false; };
template <class F> struct DeferTrait<F, std::void_t<decltype(F::kDefer)>> {
  static constexpr bool value = F::kDefer;
};
constexpr int kDeferChunk = 256;
__device__ __forceinline__ void defer_group(int x, WarpScratch *ws, int *list, unsigned long long *lc) {
  const unsigned lane = lane_id();
  long long pos = 0;
  if (lane == 0) {
    pos = ws->cpos;
    if (pos >= ws->cend) {
      pos = (long long)atomicAdd(lc, (unsigned long long)kDeferChunk);
      ws->cend = pos + kDeferChunk;
    }
    ws->cpos = pos + 32;
  }
  pos = (long long)shfl64((unsigned long long)pos, 0);
  list[pos + lane] = x;
}
__device__ __forceinline__ void defer_push(bool in, int v, WarpScratch *ws, int &cnt, int *list,
                                           unsigned long long *lc) {
  const unsigned m = __ballot_sync(FULL, in);
  if (!m) return;
  const unsigned lane = lane_id();
  if (in) ws->buf[cnt + __popc(m & lanemask_lt())] = v;
  cnt += __popc(m);
  if (lane == 0) ws->ndisc += (unsigned long long)__popc(m);
  if (cnt >= 32) {
    __syncwarp();
    const int x = ws->buf[lane];
    const int y = ws->buf[32 + lane];
    __syncwarp();
    cnt -= 32;
    if ((int)lane < cnt) ws->buf[lane] = y;
    __syncwarp();
    defer_group(x, ws, list, lc);
  }
}
// last partial group, then -1 over the rest of the open chunk; leaves the chunk state reset.
// nfc (optional): the vertices appended since the last close are added to it (|F| of the list).
__device__ __forceinline__ void defer_close(WarpScratch *ws, int &cnt, int *list, unsigned long long *lc,
                                            unsigned long long *nfc = nullptr) {
  __syncwarp();
  const unsigned lane = lane_id();
  if (cnt) {
    const int x = (int)lane < cnt ? ws->buf[lane] : -1;
    __syncwarp();
    defer_group(x, ws, list, lc);
    cnt = 0;
  }
  __syncwarp();
  const long long p0 = ws->cpos, p1 = ws->cend;
  for (long long i = p0 + lane; i < p1; i += 32) list[i] = -1;
  __syncwarp();
  if (lane == 0) {
    if (nfc && ws->ndisc) atomicAdd(nfc, ws->ndisc);
    ws->ndisc = 0;
    ws->cpos = ws->cend = 0;
  }
  __syncwarp();
}

// K2' of the deferred contraction: Tiled Partitioning of the frontier list (32-slot groups, -1 =
// empty) into the next level's log; every warp takes groups grid-stride with the next group's ids
// and rows loaded before the current enqueue.  Returns whether the list was non-empty (then the
// caller must barrier before reading the log's counters).  Must stay inlined (an out-of-line call
// cost k_bfs its register allocation).
// Hub table inserts (BFS, DESIGN.md §5 "hub filter"): every classified vertex of degree >= thr is
// offered to slot v & mask of a global direct-mapped table with atomicMax of (degree, key + 1), so
// a slot ends up holding the highest-degree VISITED vertex mapped to it (visited bits only rise).
// 0 = empty slot; a vertex whose key + 1 does not fit the key field is never inserted.
struct HubIns {
  uint32_t *g = nullptr;   // T packed entries (0 = empty); null = no table
  uint32_t mask = 0;       // T - 1
  int lgT = 0;             // key = v >> lgT
  int kbits = 0;           // key field bits (8 or 16); degree in the upper 32 - kbits bits
  long long thr = 0;       // minimum degree of an inserted vertex
};
// returns 1 when the slot changed (the caller counts changes to decide when to reload)
__device__ __forceinline__ int hub_insert(const HubIns &h, int v, long long deg) {
  if (h.g && v >= 0 && deg >= h.thr) {
    const uint32_t k1 = ((uint32_t)v >> h.lgT) + 1u;
    if (k1 >> h.kbits) return 0;
    const unsigned long long dmax = (1ull << (32 - h.kbits)) - 1;
    const uint32_t d = (uint32_t)((unsigned long long)deg < dmax ? (unsigned long long)deg : dmax);
    const uint32_t nv = (d << h.kbits) | k1;
    return atomicMax(h.g + ((uint32_t)v & h.mask), nv) < nv ? 1 : 0;
  }
  return 0;
}

__device__ __forceinline__ bool classify_deferred(const long long *__restrict__ off, const int *flist,
                                                  const unsigned long long *flc, const Ladder &L,
                                                  const Queues &Q, CounterSet *cs,
                                                  const HubIns &hub = HubIns()) {
  const unsigned long long fl = ldcg(flc);
  if (!fl) return false;
  const unsigned lane = threadIdx.x & 31;
  const long long gw = warp_rank();
  const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
  const long long first = gw * 32, step = nw * 32;
  // pass A: what this warp's groups need (next group's ids and rows loaded ahead)
  unsigned long long tot = 0, nf = 0, arcs = 0;
  {
    long long base = first;
    int v = base < (long long)fl ? ldcg(flist + base + lane) : -1;
    long long b = 0, e = 0;
    if (v >= 0) ld_row_pair(off, v, &b, &e);
    while (base < (long long)fl) {
      const long long nb = base + step;
      const int v2 = nb < (long long)fl ? ldcg(flist + nb + lane) : -1;
      long long b2 = 0, e2 = 0;
      if (v2 >= 0) ld_row_pair(off, v2, &b2, &e2);
      enqueue_count(v >= 0, b, e, L, tot, nf, arcs);
      hub_insert(hub, v, e - b);
      base = nb;
      v = v2;
      b = b2;
      e = e2;
    }
  }
  if (nf == 0) return true;
  // one round of reservations for all of them
  unsigned long long run = 0;
  if (lane == 0 || ((int)lane <= L.ncls)) {
    if (tot) run = atomicAdd(&cs->cnt[lane].v, tot);
  } else if (lane == 29) {
    if (Q.order && tot) run = atomicAdd(Q.order_cnt, tot);
  } else if (lane == 30) {
    atomicAdd(&cs->nF.v, nf);
  } else if (lane == 31) {
    if (arcs) atomicAdd(&cs->arcsF.v, arcs);
  }
  // pass B: the same groups again (rows now in L1/L2), written at the running bases
  {
    long long base = first;
    int v = base < (long long)fl ? ldcg(flist + base + lane) : -1;
    long long b = 0, e = 0;
    if (v >= 0) ld_row_pair(off, v, &b, &e);
    while (base < (long long)fl) {
      const long long nb = base + step;
      const int v2 = nb < (long long)fl ? ldcg(flist + nb + lane) : -1;
      long long b2 = 0, e2 = 0;
      if (v2 >= 0) ld_row_pair(off, v2, &b2, &e2);
      enqueue_write(v >= 0, v, b, e, L, Q, run);
      base = nb;
      v = v2;
      b = b2;
      e = e2;
    }
  }
  return true;
}

// Append the lanes' filtered-in vertices to the warp buffer; flush full batches of 32.
__device__ __forceinline__ void buffer_push(bool in, int v, WarpScratch *ws, int &cnt,
                                            const long long *__restrict__ off, const Ladder &L,
                                            const Queues &Q, CounterSet *cs) {
  const unsigned m = __ballot_sync(FULL, in);
  if (!m) return;
  const unsigned lane = lane_id();
  if (in) ws->buf[cnt + __popc(m & lanemask_lt())] = v;
  cnt += __popc(m);
  if (cnt >= 32) {
    PROF_T(tf0);
    __syncwarp();
    const int x = ws->buf[lane];
    const int y = ws->buf[32 + lane];
    __syncwarp();
    cnt -= 32;
    if ((int)lane < cnt) ws->buf[lane] = y;
    __syncwarp();
    enqueue_ids(true, x, off, L, Q, cs);
    PROF_T(tf1);
    PROF_ADD(0, tf1 - tf0);
    PROF_ADD(1, 1);
  }
}
__device__ __forceinline__ void buffer_flush(WarpScratch *ws, int &cnt,
                                             const long long *__restrict__ off, const Ladder &L,
                                             const Queues &Q, CounterSet *cs) {
  __syncwarp();
  const unsigned lane = lane_id();
  const bool in = (int)lane < cnt;
  const int x = in ? ws->buf[lane] : 0;
  __syncwarp();
  cnt = 0;
  enqueue_ids(in, x, off, L, Q, cs);
}

// ------------------------------------------------------------------------------------------
// The stealing consumer (Resident Tile Stealing, Alg. 3 l.9-17).  Every warp of the
// persistent grid takes batches of tiles of one class from a device-wide ticket counter, so any
// SM consumes any tile; classes are drained largest first.  A tile of t elements is covered by
// t/VEC lanes (the paper's one-neighbour-per-thread tile, each lane carrying VEC neighbours).
// Lane sl of a tile's group reads elements sl, sl + g, sl + 2g, ... (g = group width): every
// load instruction is coalesced, and the 32 neighbours a warp checks at once are CONSECUTIVE
// entries of a row, so on a sorted hub row their status words share L1/L2 lines.
// Fragments (< M) are consumed by a warp scan-based gather ([30]): 32 fragment vertices
// per round, lane k takes the k-th element of their concatenation.
//
// Filter policy F provides:
//   struct Src;                                    per-source-vertex context
//   Src src(bool valid, int u, long long b, long long e);   (b,e = row of u when needed)
//   template<int N> void visit(bool valid, const Src&, int (&v)[N], const uint32_t (&w)[N],
//                              bool (&in)[N], int lpt); marks the neighbours filtered in (and may
//                              rewrite v[j] to the row id to enqueue, e.g. global -> local);
//                              lpt = lanes sharing the tile (aligned groups of the warp)
//   kWeights (load weights), kNeedRow (src needs the row for CTA tiles), kEnqueue (contraction)
//   Queues *next_q; CounterSet *next_cs;             where filtered-in vertices go
// steal = false (ablation of Resident Tile Stealing, Fig. 10): tiles are dealt to warps
// statically, round robin in batch units, instead of through the device-wide tickets.
// Contraction of a filtered-in vertex: deferred (frontier list) or immediate (warp buffer -> log).
#ifndef SAGE_DEFER_RUNTIME
#define SAGE_DEFER_RUNTIME 0   // 1: small levels contract immediately (measured slower: the second path costs k_bfs 130 B of spills)
#endif
template <class F>
__device__ __forceinline__ void push_filtered(const F &f, bool in, int v, WarpScratch *ws, int &cnt,
                                              const long long *__restrict__ off, const Ladder &L) {
  if constexpr (DeferTrait<F>::value) {
    if (!SAGE_DEFER_RUNTIME || f.flist) {
      defer_push(in, v, ws, cnt, f.flist, f.flc);
      return;
    }
  }
  buffer_push(in, v, ws, cnt, off, L, *f.next_q, f.next_cs);
}
// Filters may carry `nfc`: where the deferred contraction counts |F| of the list it appends to
// (the fused runtime tiling of push BFS, traversal.cu); others count in the K2' phase.
template <class F, class = void> struct NfcOf {
  __device__ __forceinline__ static unsigned long long *get(const F &) { return nullptr; }
};
template <class F> struct NfcOf<F, std::void_t<decltype(F::nfc)>> {
  __device__ __forceinline__ static unsigned long long *get(const F &f) { return f.nfc; }
};
template <class F>
__device__ __forceinline__ void close_filtered(const F &f, WarpScratch *ws, int &cnt,
                                               const long long *__restrict__ off, const Ladder &L) {
  if constexpr (DeferTrait<F>::value) {
    if (!SAGE_DEFER_RUNTIME || f.flist) {
      defer_close(ws, cnt, f.flist, f.flc, NfcOf<F>::get(f));
      return;
    }
  }
  if (cnt) buffer_flush(ws, cnt, off, L, *f.next_q, f.next_cs);
}

// Column-prefetch depth of a filter (F::kPrefetch, default 1 step ahead).
template <class F, class = void> struct PrefetchDepth { static constexpr int value = 1; };
template <class F> struct PrefetchDepth<F, std::void_t<decltype(F::kPrefetch)>> {
  static constexpr int value = F::kPrefetch;
};

template <int VEC, class F>
__device__ __forceinline__ void consume_log(const F &f, const Ladder &L, const Queues &Q,
                                            CounterSet *cs, const long long *__restrict__ off,
                                            const int *__restrict__ col,
                                            const uint32_t *__restrict__ w, WarpScratch *ws,
                                            typename F::Src *fsrc, bool vec_ok, bool steal = true) {
  const unsigned lane = lane_id();
  const unsigned long long pol = policy_evict_first();
  const long long gwarp = warp_rank();
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  // all queue sizes in one round of loads (lane c holds cnt[c])
  const unsigned long long my_cnt = (int)lane <= L.ncls ? ldcg(&cs->cnt[lane].v) : 0ull;
  // Small logs (every class fits in one grab per warp of a 1/(ncls+1) share of the grid): the
  // classes are consumed CONCURRENTLY by disjoint warp groups (group = rank mod (ncls+1)) instead
  // of one after another by the same warps — a small level's latency is then the longest class's
  // dependent chain (ticket -> log entry -> row -> columns -> status -> claim), not their sum.
  // (Splitting big logs in proportion to their classes' elements was measured 2x slower on C2
  // SSSP / PageRank / BC: the groups finish far apart.)
  const int G = L.ncls + 1;
  long long rank = gwarp, nranks = nwarps;
  int group = -1;
  {
    unsigned long long need = 0;
    if ((int)lane < L.ncls) {
      const int t = L.B >> lane;
      const int tps = 32 / ((t / VEC) < 32 ? (t / VEC) : 32);
      need = (my_cnt + tps - 1) / tps;
    } else if ((int)lane == L.ncls) {
      need = (my_cnt + 31) / 32;
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const unsigned long long y = __shfl_xor_sync(FULL, need, o);
      need = y > need ? y : need;
    }
    const long long per = nwarps / G;
    if (steal && per >= 1 && need <= (unsigned long long)per * SAGE_SPLIT_K) {
      group = (int)(gwarp % G);
      rank = gwarp / G;
      nranks = per;
      if (rank >= per) group = G;   // the remainder warps take nothing (but still close below)
    } else if (steal && SAGE_SPLIT_PROP && nwarps >= 2 * G) {
      // medium logs (a few hundred elements per warp in all): the classes still run concurrently,
      // each with a share of the warps proportional to its elements (fragments ~4 per entry)
      unsigned long long wk = 0;
      if ((int)lane < L.ncls) wk = my_cnt * (unsigned long long)(L.B >> lane);
      else if ((int)lane == L.ncls) wk = my_cnt * 4ull;
      const unsigned long long tot = warp_sum64(wk);
      if (tot > 0 && tot <= (unsigned long long)nwarps * SAGE_SPLIT_PROP) {
        const unsigned long long spare = (unsigned long long)(nwarps - G);
        const unsigned long long share = wk ? 1ull + (unsigned long long)((double)spare * (double)wk / (double)tot) : 0ull;
        unsigned long long incl = share;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const unsigned long long y = __shfl_up_sync(FULL, incl, o);
          if ((int)lane >= o) incl += y;
        }
        const unsigned m = __ballot_sync(FULL, (int)lane <= L.ncls && incl <= (unsigned long long)gwarp);
        group = __popc(m);   // the class whose share holds this rank (G = none: idle remainder)
        if (group < G) {
          rank = gwarp - (long long)(shfl64(incl, group) - shfl64(share, group));
          nranks = (long long)shfl64(share, group);
        }
      }
    }
  }
  int bcnt = 0;   // warp-uniform fill of ws->buf
  for (int c = 0; c < L.ncls; ++c) {
    if (group >= 0 && c != group) continue;
    const int t = L.B >> c;
    const unsigned long long count = shfl64(my_cnt, c);
    if (count == 0) continue;
    const int lpt = (t / VEC) < 32 ? (t / VEC) : 32;  // lanes per tile
    const int tps = 32 / lpt;                           // tiles per warp step
    const int spt = (t / VEC) > 32 ? (t / (32 * VEC)) : 1;  // steps per tile
    // adaptive ticket batch: ~2 grabs per warp, <= 16 KB of columns per grab; warps beyond the
    // number of grabs skip the class (no ticket traffic on small levels)
    unsigned long long batch = (count + SAGE_TK_GRABS * nranks - 1) / (SAGE_TK_GRABS * nranks);
    const unsigned long long bmax = (SAGE_TK_ELEMS / t) > (unsigned)tps ? (SAGE_TK_ELEMS / t) : tps;
    if (batch > bmax) batch = bmax;
    batch = ((batch + tps - 1) / tps) * tps;
    const unsigned long long grabs = (count + batch - 1) / batch;
    if ((unsigned long long)rank >= grabs) continue;
    const int sub = lane / lpt, sl = lane % lpt;
    const bool contiguous = lpt < 32 && vec_ok && (VEC % 4) == 0;
    const int lg_spt = __ffs(spt) - 1;
    // stealing: the ticket of the NEXT batch is taken when a batch starts, so the ticket atomic's
    // round trip overlaps the batch (a ticket beyond `count` just ends the loop)
    unsigned long long tk_next = 0;
    if (steal && lane == 0) tk_next = atomicAdd(&cs->tk[c].v, batch);
    for (unsigned long long rr = 0;; ++rr) {
      unsigned long long base = 0;
      if (steal) {
        base = shfl64(tk_next, 0);
        if (base < count && lane == 0) tk_next = atomicAdd(&cs->tk[c].v, batch);
      } else {
        base = ((unsigned long long)rank + rr * (unsigned long long)nranks) * batch;
      }
      if (base >= count) break;
      const unsigned long long end = (base + batch < count) ? base + batch : count;
      // log entries of the batch's next 32-tile group, loaded while the current group's steps run
      // (the metadata chain of a group is then offsets -> start only)
      int pf_u = 0;
      long long pf_start = 0;
      if ((unsigned long long)lane < end - base) {
        if (c == 0) {
          const CtaTile T = ldcg_tile(Q.cta + base + lane);
          pf_u = T.u;
          pf_start = T.start;
        } else {
          pf_u = ldcg(Q.cls[c] + base + lane);
        }
      }
      for (unsigned long long r0 = base; r0 < end; r0 += 32) {
        // ---- metadata round: lane k resolves tile r0 + k (log entry -> row -> tile start and
        //      the filter's per-source context) in ONE round of loads for up to 32 tiles; the
        //      steps below read them from shared memory.
        const int nt = (end - r0) < 32ull ? (int)(end - r0) : 32;
        {
          const bool mv = (int)lane < nt;
          long long start = 0, rb = 0, re = 0;
          int u = 0;
          if (mv) {
            u = pf_u;
            if (c == 0) {
              start = pf_start;
              if (F::kNeedRow) {
                rb = ld_off(off + u);
                re = ld_off(off + u + 1);
              }
            } else {
              rb = ld_off(off + u);
              re = ld_off(off + u + 1);
              RowSplit s = split_row(rb, re, L);
              start = class_tile_start(re, s.r, t);
            }
          }
          const unsigned long long r1 = r0 + 32;
          if (r1 + lane < end) {
            if (c == 0) {
              const CtaTile T = ldcg_tile(Q.cta + r1 + lane);
              pf_u = T.u;
              pf_start = T.start;
            } else {
              pf_u = ldcg(Q.cls[c] + r1 + lane);
            }
          }
          const typename F::Src sc = f.src(mv, u, rb, re);
          __syncwarp();
          ws->hb[lane] = start;
          fsrc[lane] = sc;
          __syncwarp();
        }
        // ---- steps: step st covers tile k = (st / spt) * tps + sub, sub-step st % spt.  The
        //      column loads of step st + 1 are issued before the filter of step st runs, so
        //      the column stream's latency hides behind the status reads.
        const int nst = ((nt + tps - 1) / tps) << lg_spt;
        int vn[VEC];
        uint32_t wn[VEC];
        auto load_step = [&](int st, int (&v)[VEC], uint32_t (&ww)[VEC]) {
          const int k = ((st >> lg_spt) * tps) + sub;
          const bool valid = k < nt;
          const long long start = ws->hb[valid ? k : 0];
          if (contiguous) {
            const long long p0 = start + (long long)sl * VEC;
#pragma unroll
            for (int q = 0; q < (VEC + 3) / 4; ++q) {
              int4 c4 = make_int4(0, 0, 0, 0);
              uint4 w4 = make_uint4(0, 0, 0, 0);
              if (valid) {
                c4 = ld_col4(col + p0 + 4 * q, pol);
                if (F::kWeights) w4 = ld_col4u(w + p0 + 4 * q, pol);
              }
              v[(4 * q) % VEC] = c4.x; v[(4 * q + 1) % VEC] = c4.y;
              v[(4 * q + 2) % VEC] = c4.z; v[(4 * q + 3) % VEC] = c4.w;
              ww[(4 * q) % VEC] = w4.x; ww[(4 * q + 1) % VEC] = w4.y;
              ww[(4 * q + 2) % VEC] = w4.z; ww[(4 * q + 3) % VEC] = w4.w;
            }
          } else {
            const long long p0 = start + (long long)(st & (spt - 1)) * (lpt * VEC) + sl;
#pragma unroll
            for (int j = 0; j < VEC; ++j) {
              v[j] = valid ? ld_col(col + p0 + j * lpt, pol) : 0;
              ww[j] = (valid && F::kWeights) ? ld_colu(w + p0 + j * lpt, pol) : 0u;
            }
          }
        };
        if constexpr (PrefetchDepth<F>::value > 1) {
          // filters with little work per step (PageRank: VEC fp64 atomics, no status reads) keep
          // the column loads of the next PD steps in flight
          constexpr int PD = PrefetchDepth<F>::value;
          int vq[PD][VEC];
          uint32_t wq[PD][VEC];
#pragma unroll
          for (int r = 0; r < PD; ++r)
            if (r < nst) load_step(r, vq[r], wq[r]);
          for (int st0 = 0; st0 < nst; st0 += PD) {
#pragma unroll
            for (int r = 0; r < PD; ++r) {
              const int st = st0 + r;
              if (st < nst) {
                int v[VEC];
                uint32_t ww[VEC];
#pragma unroll
                for (int j = 0; j < VEC; ++j) {
                  v[j] = vq[r][j];
                  ww[j] = wq[r][j];
                }
                if (st + PD < nst) load_step(st + PD, vq[r], wq[r]);
                const int k = ((st >> lg_spt) * tps) + sub;
                const bool valid = k < nt;
                const typename F::Src sc = fsrc[valid ? k : 0];
                bool in[VEC];
                f.template visit<VEC>(valid, sc, v, ww, in, lpt);
              }
            }
          }
          __syncwarp();
          continue;
        }
        load_step(0, vn, wn);
        for (int st = 0; st < nst; ++st) {
          PROF_T(tv0);
          int v[VEC];
          uint32_t ww[VEC];
#pragma unroll
          for (int j = 0; j < VEC; ++j) {
            v[j] = vn[j];
            ww[j] = wn[j];
          }
          if (st + 1 < nst) load_step(st + 1, vn, wn);
          const int k = ((st >> lg_spt) * tps) + sub;
          const bool valid = k < nt;
          const typename F::Src sc = fsrc[valid ? k : 0];
          bool in[VEC];
          f.template visit<VEC>(valid, sc, v, ww, in, lpt);
          PROF_T(tv1);
          PROF_ADD(2, tv1 - tv0);
          PROF_ADD(4, 1);
          if constexpr (F::kEnqueue) {
            bool anyin = false;
#pragma unroll
            for (int j = 0; j < VEC; ++j) anyin |= in[j];
            if (__any_sync(FULL, anyin)) {   // most steps of a heavy level find nothing new
#pragma unroll
              for (int j = 0; j < VEC; ++j)
                push_filtered(f, in[j], v[j], ws, bcnt, off, L);
            }
          }
        }
        __syncwarp();
      }
    }
  }
  // ---- fragments: warp scan-based gather
  const unsigned long long fcount = shfl64(my_cnt, L.ncls);
  const unsigned long long fgrabs = (fcount + 31) / 32;
  unsigned long long frr = 0;
  for (;;) {
    if (fcount == 0 || (group >= 0 && group != L.ncls) || (unsigned long long)rank >= fgrabs) break;
    unsigned long long base = 0;
    if (steal) {
      if (lane == 0) base = atomicAdd(&cs->tk[L.ncls].v, 32ull);
      base = shfl64(base, 0);
    } else {
      base = ((unsigned long long)rank + frr++ * (unsigned long long)nranks) * 32ull;
    }
    if (base >= fcount) break;
    const bool valid = base + lane < fcount;
    int u = 0, hl = 0, tl = 0;
    long long hb = 0, tb = 0, rb = 0, re = 0;
    if (valid) {
      u = ldcg(Q.frag + base + lane);
      rb = ld_off(off + u);
      re = ld_off(off + u + 1);
      RowSplit s = split_row(rb, re, L);
      hb = rb;
      hl = s.h;
      tl = s.r & (L.M - 1);
      tb = re - tl;
    }
    const typename F::Src sc = f.src(valid, u, rb, re);
    int fl = hl + tl;
    int inc = fl;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int y = __shfl_up_sync(FULL, inc, o);
      if ((int)lane >= o) inc += y;
    }
    const int total = __shfl_sync(FULL, inc, 31);
    ws->pre[lane] = inc - fl;
    ws->hl[lane] = hl;
    ws->hb[lane] = hb;
    ws->tb[lane] = (int)(tb - hb);
    fsrc[lane] = sc;
    __syncwarp();
    for (int k0 = 0; k0 < total; k0 += 32) {
      const int k = k0 + (int)lane;
      const bool kv = k < total;
      int o = 0;
      if (kv) {   // largest o with pre[o] <= k
        int lo = 0, hi = 31;
#pragma unroll
        for (int it = 0; it < 5; ++it) {
          int mid = (lo + hi + 1) >> 1;
          if (ws->pre[mid] <= k) lo = mid; else hi = mid - 1;
        }
        o = lo;
      }
      int vv[1] = {0};
      uint32_t w1[1] = {0u};
      const typename F::Src so = fsrc[o];
      if (kv) {
        const int idx = k - ws->pre[o];
        const long long pos = ws->hb[o] + (idx < ws->hl[o] ? idx : ws->tb[o] + (idx - ws->hl[o]));
        vv[0] = ld_col(col + pos, pol);
        if (F::kWeights) w1[0] = ld_colu(w + pos, pol);
      }
      bool in[1];
      f.template visit<1>(kv, so, vv, w1, in, 1);
      if constexpr (F::kEnqueue) {
        push_filtered(f, in[0], vv[0], ws, bcnt, off, L);
      }
    }
    __syncwarp();
  }
  if constexpr (F::kEnqueue) {
    close_filtered(f, ws, bcnt, off, L);
  }
}

}  // namespace sage
