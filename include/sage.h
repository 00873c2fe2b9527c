/* sage.h — C ABI of the B200-native SAGE hot path (libsage.so).
 *
 * SAGE = Sha, Li, Tan, "Self-adaptive Graph Traversal on GPUs", SIGMOD'21.  "P:NNN" below is
 * line NNN of the paper text; section / algorithm / table names are given beside it.
 *
 * What the library computes:
 *   frontier-driven, node-centric traversal of a plain CSR graph with no preprocessing
 *   (P:35-38), for BFS (Alg. 1 l.1-6), integer-weight SSSP
 *   (named at P:235) and PageRank (Alg. 1 l.26-29), with the per-iteration
 *   neighbour expansion split at runtime into tiles (Tiled Partitioning, Alg. 2)
 *   that are logged in device memory and consumed by a persistent kernel that every SM steals
 *   from (Resident Tile Stealing, Alg. 3), push/pull direction switching on symmetric
 *   graphs, and Sampling-based Reordering (§6, Alg. 4, Fig. 5).
 *
 * Conventions (all entry points):
 *   * extern "C"; every function returns sage_status and never aborts the process.
 *   * Synchronous: on return every output is complete (the call synchronises its stream).
 *   * Pointers are host or device memory.  Inputs are detected with SAGE_F_DEVICE_PTRS; output
 *     buffers are classified with cudaPointerGetAttributes (host pageable / pinned / device).
 *   * Results are always in the caller's ORIGINAL vertex IDs, also after sage_reorder.
 *   * Errors: invalid arguments -> SAGE_E_INVALID and nothing is modified; CUDA / NCCL failures
 *     -> SAGE_E_CUDA / SAGE_E_NCCL and are sticky (the handle may then only be freed).
 *     sage_last_error() gives a thread-local message for the last failing call.
 *   * There is no CPU fallback: without a usable GPU every compute call returns
 *     SAGE_E_UNSUPPORTED.
 *   * A handle is not thread-safe; distinct handles may be used from distinct threads.
 */
#ifndef SAGE_H_
#define SAGE_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct sage_graph sage_graph; /* opaque; owned by the library until sage_free */

typedef enum {
  SAGE_OK = 0,
  SAGE_E_INVALID = 1,     /* bad argument / failed CSR validation; graph unchanged            */
  SAGE_E_NOMEM = 2,       /* device allocation failed                                          */
  SAGE_E_CUDA = 3,        /* CUDA runtime error (sticky)                                       */
  SAGE_E_NCCL = 4,        /* NCCL error (sticky)                                               */
  SAGE_E_OVERFLOW = 5,    /* a finite shortest distance is >= UINT32_MAX                       */
  SAGE_E_UNSUPPORTED = 6  /* no GPU, or a feature not available for this graph / build        */
} sage_status;

enum {
  SAGE_F_SYMMETRIC = 1u,   /* caller asserts the CSR is symmetric -> pull (bottom-up) steps allowed */
  SAGE_F_DEVICE_PTRS = 2u, /* row_offsets / col_indices / weights are device pointers               */
  SAGE_F_BORROW = 4u,      /* with DEVICE_PTRS: use the caller arrays in place (no copy); the caller
                              keeps them alive and unmodified until sage_free                      */
  SAGE_F_NO_VALIDATE = 8u, /* skip the validation pass of sage_load_csr                              */
  SAGE_F_HOST_COLUMNS = 128u, /* out-of-core: col_indices /
                              weights (host arrays) stay in pinned, mapped host memory and the
                              kernels read them zero-copy over the host link; with SAGE_F_BORROW
                              the caller's pages are registered in place, otherwise copied into
                              library-owned pinned memory.  A tile alignment of 32 (128 B) keeps
                              every tile request line-aligned.  sage_reorder is unsupported.     */
  SAGE_F_PUSH_ONLY = 16u,  /* disable direction switching: every level is the paper's push
                              expansion (Alg. 2/3).  Can also be set per call (sage_bfs_ex).     */
                           /* 32u: reserved (an experimental binned push level of round 1, removed;
                              DESIGN.md §5 keeps its measurements)                                */
  SAGE_F_NO_STEALING = 64u /* per call (sage_bfs_ex; sage_pagerank_ex push form, which then also
                              skips the windowed form), ablation (Fig. 10): tiles are
                              dealt to warps statically instead of through Resident Tile Stealing */
};

/* Multi-GPU description (1D vertex partition).  NULL in sage_csr = single GPU.
 * Non-NULL selects the NCCL path (also with world == 1: a 1-rank communicator).  On that path
 * sage_bfs (parents included), sage_sssp and sage_pagerank are collective (every rank calls them with
 * the same arguments; outputs hold the rank's own rows); sage_reorder / sage_bc return
 * SAGE_E_UNSUPPORTED.  Multi-GPU SSSP exchanges candidate distances of
 * remote targets with one ncclReduceScatter(min) per Bellman-Ford iteration.                   */
typedef struct {
  int32_t rank, world;         /* this process's rank and the number of ranks                    */
  const void *nccl_unique_id;  /* 128-byte ncclUniqueId created by rank 0 and broadcast by the
                                  caller (e.g. torch.distributed); required when world > 1       */
  int64_t v_begin, v_end;      /* global vertex block [v_begin, v_end) owned by this rank; ranks
                                  cover [0, n) contiguously in rank order                       */
  int32_t exchange;            /* push-BFS frontier exchange: 0 = automatic - over
                                  peer memory (the push kernel ORs each remote candidate into its
                                  owner's inbox bitmap through NVLink, then one stream-ordered
                                  barrier) when every rank can map every other rank's memory with
                                  native atomics, else the collectives; 1 = collectives only (the
                                  sparse / dense all-to-all(v)).  All ranks must pass the same value. */
} sage_dist;

/* Tile ladder used by every kernel and by the reorder's sample (Alg. 2; readings
 * R9-R14 of DESIGN.md).  NULL = defaults.                                                      */
typedef struct {
  int32_t tile_cta;  /* B: largest ("CTA") tile, power of two in [1, 4096]; default 256   */
  int32_t tile_min;  /* M: MIN_TILE_SIZE, power of two in [1, B]; default 8 (Fig. 3)        */
  int32_t align;     /* A: tile alignment in elements: 0 = paper mode (no head fragment),
                        else a power of two in [1, 64]; default 4 (16 B, one int4 load)          */
  double alpha;      /* Beamer push->pull threshold: pull when arcs(F) > arcs(unvisited)/alpha; 15 */
  double beta;       /* pull->push threshold: push when |F| < n/beta; default 18                     */
  int32_t ctas_per_sm; /* resident CTAs per SM of the persistent kernels; 0 = automatic (the
                        occupancy limit, one CTA per SM on graphs under 8M arcs)                  */
  int32_t hub_filter;  /* push BFS hub filter (a shared-memory table of visited
                        high-degree vertices skips their status reads; results identical):
                        0 = automatic (graphs with >= 32M arcs), 1 = always, -1 = never        */
} sage_options;

/* CSR input of sage_load_csr (Fig. 1: u_offset / v arrays).                         */
typedef struct {
  int64_t n;                     /* GLOBAL vertex count, 0 < n < 2^31                              */
  int64_t m;                     /* LOCAL arc count; must equal row_offsets[n_local]                */
  const int64_t *row_offsets;    /* n_local + 1 entries, row_offsets[0] = 0, non-decreasing, every
                                    row shorter than 2^31 arcs.
                                    n_local = v_end - v_begin (multi-GPU) or n                     */
  const int32_t *col_indices;    /* m entries, GLOBAL ids in [0, n); rows need not be sorted       */
  const uint32_t *weights;       /* m entries >= 1, or NULL (SSSP then returns SAGE_E_INVALID)     */
  uint32_t flags;                /* SAGE_F_*                                                        */
  void *cuda_stream;             /* cudaStream_t used by every call on this graph; NULL = a stream
                                    owned by the library                                            */
  const sage_options *opts;      /* NULL = defaults                                                 */
  const sage_dist *dist;         /* NULL = single GPU                                               */
} sage_csr;

/* Per-call statistics; every field is filled on SAGE_OK (SURVEY §8(d) byte model).           */
typedef struct {
  int32_t levels;              /* BFS levels / SSSP iterations / PR iterations executed            */
  int32_t push_levels, pull_levels;
  int64_t edges_traversed;     /* R1: directed = sum of out(v) over reached v; symmetric = that/2;
                                  PageRank = iterations * m                                          */
  int64_t arcs_inspected;      /* arcs whose target status was examined (push: all arcs of F)      */
  int64_t vertices_expanded;   /* sum over levels of |F|                                            */
  int64_t vertices_discovered; /* BFS: reached vertices; SSSP: improvements that entered a frontier */
  double ms;                   /* device time of the traversal kernels (CUDA events on the graph's
                                  stream; excludes output D2H and ID translation)                 */
  double model_bytes;          /* algorithmic bytes of the frozen model of SURVEY §8(d)             */
  double kernel_ms;            /* device time of the dominant (persistent) kernel alone             */
} sage_stats;

typedef struct {
  int32_t sector_width;        /* S: node ids per sector (R17); power of two; default 8             */
  const int32_t *candidates;   /* optional (host) list of ORIGINAL vertex ids allowed to move, in
                                  every round (Fig. 5's "only consider node-8"); NULL = all   */
  int64_t n_candidates;
} sage_reorder_opts;

/* ---------------------------------------------------------------------------------------------
 * sage_load_csr — load (copy or borrow) a CSR graph onto the current CUDA device and validate it
 * ("after loading ... immediately respond to queries"; no preprocessing: no transpose, no
 * partitioning, no reordering).  Validation (unless SAGE_F_NO_VALIDATE): row_offsets[0] = 0,
 * non-decreasing, row_offsets[n_local] = m, 0 <= col < n, weights >= 1.  On failure *out is NULL.
 * Multi-GPU (dist->world > 1): collective over the ranks; creates the NCCL communicator.       */
sage_status sage_load_csr(const sage_csr *in, sage_graph **out);

/* Create a 128-byte NCCL unique id (rank 0 calls it and broadcasts the bytes to every rank).   */
sage_status sage_nccl_unique_id(void *out128);

/* Free the handle and every library-owned device array.  NULL is a no-op.                     */
sage_status sage_free(sage_graph *g);

/* BFS from `source` (global id): level_out[v] = hop distance, -1 = unreachable (Alg. 1 l.2,
 * P:112).  level_out has n entries (n_local multi-GPU, the rank's slice).  parent_out (nullable)
 * receives a valid BFS-tree parent (-1 for the source and for unreachable vertices).
 * Direction switching is used iff the graph is SAGE_F_SYMMETRIC and not SAGE_F_PUSH_ONLY.
 * Output buffers may be host or device memory (caller-owned; written before the call returns).
 * Device buffers of the graph's GPU are written IN PLACE by the kernel when no ID translation
 * applies (not reordered); those writes follow the caller's earlier work on the graph's stream
 * (sage_csr.cuda_stream) or, without one, on the legacy default stream.  On an error the
 * contents of the output buffers are unspecified.                                              */
sage_status sage_bfs(sage_graph *g, int32_t source, int32_t *level_out, int32_t *parent_out,
                     sage_stats *st);

/* sage_bfs with a per-call flag word (SAGE_F_PUSH_ONLY honoured).                              */
sage_status sage_bfs_ex(sage_graph *g, int32_t source, int32_t *level_out, int32_t *parent_out,
                        uint32_t call_flags, sage_stats *st);

/* Integer-weight SSSP ("iteratively update neighbors' distances"; reading R4): frontier
 * Bellman-Ford with atomicMin.  dist_out[v] = shortest distance, UINT32_MAX = unreachable.
 * Requires weights.  A finite distance >= UINT32_MAX -> SAGE_E_OVERFLOW (dist_out unspecified).
 * dist_out: host or device memory, written in place like sage_bfs's outputs.                  */
sage_status sage_sssp(sage_graph *g, int32_t source, uint32_t *dist_out, sage_stats *st);

/* PageRank, push form of Alg. 1 l.26-29 over the resident all-V tile log;
 * readings R5-R7: x0 = 1/N, x <- (1-d)/N + d*(A^T D^-1 x + dangling/N), fixed `iterations`,
 * fp64.  rank_out has n doubles summing to 1.  damping in [0, 1), iterations >= 0.             */
sage_status sage_pagerank(sage_graph *g, double damping, int32_t iterations, double *rank_out,
                          sage_stats *st);

/* sage_pagerank with a per-call flag word.  On a SAGE_F_SYMMETRIC graph the default form is the
 * pull (gather) form over the same resident log — y_v = sum of x_u / out(u) over v's row, fp32
 * contributions and fp64 accumulation (reading R7), one fp64 atomic per tile lane group instead
 * of one per arc; SAGE_F_PUSH_ONLY (graph or call) selects the paper's push form (Alg. 1
 * l.26-29).  Directed graphs always use push.                                                  */
sage_status sage_pagerank_ex(sage_graph *g, double damping, int32_t iterations, double *rank_out,
                             uint32_t call_flags, sage_stats *st);

/* Betweenness Centrality contributions (Alg. 1 l.8-24): for
 * every source s in `sources` (host array, original ids) a forward push BFS counting shortest
 * paths (sigma, fp64) and a backward dependency accumulation by decreasing level (delta, fp64);
 * bc_out[v] = sum over the sources of delta_s(v), v != s (Brandes; no normalisation — an
 * undirected graph counts every pair in both directions).  At most 4096 levels per source.
 * Single GPU.                                                                                  */
sage_status sage_bc(sage_graph *g, const int32_t *sources, int64_t n_sources, double *bc_out,
                    sage_stats *st);

/* `rounds` rounds of Sampling-based Reordering (§6; readings R17-R25): relabels the
 * vertices in place (the CSR is rewritten, rows sorted, weights moved with their arcs) and
 * composes the permutation; later queries still speak original ids.  Single GPU only.         */
sage_status sage_reorder(sage_graph *g, int32_t rounds, const sage_reorder_opts *opt,
                         sage_stats *st);

/* Online Sampling-based Reordering: §6's "the sampling is performed along
 * with the tile access" with the sampling threshold |E|, reading R19b.
 * enable != 0 starts recording: every later single-GPU sage_bfs / sage_bfs_ex call records the rows
 * of the vertices it reached (one occurrence each) and every sage_pagerank / sage_pagerank_ex call
 * records every non-empty row `iterations` times, as per-vertex occurrence counts under the current
 * labels.  When the recorded row lengths since the last round reach `threshold` (<= 0: |E| = m),
 * one reorder round (stages 1-3 + swap matching + relabel, exactly sage_reorder's round) runs on
 * that weighted sample right after the query that crossed the threshold has written its answer;
 * the counts then restart.  Answers always use original ids.  enable == 0 stops recording.
 * sector_width as in sage_reorder_opts (0 = 8).  Single GPU, device-resident columns only
 * (SAGE_E_UNSUPPORTED otherwise).                                                              */
sage_status sage_online_reorder(sage_graph *g, int32_t enable, int32_t sector_width, int64_t threshold);

/* Online reordering progress: rounds run, label swaps applied, recorded row lengths pending.   */
sage_status sage_online_reorder_info(const sage_graph *g, int64_t *rounds, int64_t *swaps, int64_t *pending);

/* Objective of §6 on the current labels: the sum over the tile sample (every tile of
 * every vertex under the graph's ladder, readings R19/R20) of the number of distinct sectors
 * floor(label / sector_width) among the tile's members.  Lower = better locality.              */
sage_status sage_reorder_objective(sage_graph *g, int32_t sector_width, int64_t *out);

/* new_id_of_old[v] = current label of original vertex v (n entries; identity before reorder). */
sage_status sage_get_permutation(const sage_graph *g, int32_t *new_id_of_old);

/* Copy the CURRENT (possibly reordered) CSR to caller buffers (host or device): off n+1,
 * col m, w m (w may be NULL).  Used to check the relabelled graph's isomorphism.             */
sage_status sage_get_csr(const sage_graph *g, int64_t *off_out, int32_t *col_out, uint32_t *w_out);

/* Graph sizes: any pointer may be NULL.  *flags = the load flags | 0x100 (rows sorted) | 0x200
 * (reordered) | 0x400 (multi-GPU: the push exchange runs over peer memory, sage_dist.exchange)
 * | 0x800 (push PageRank runs the windowed form: chosen at the first push PageRank call when most
 * arcs stay near their source, e.g. web graphs in crawl order).               */
sage_status sage_graph_info(const sage_graph *g, int64_t *n, int64_t *m, int64_t *n_local,
                            int64_t *v_begin, uint32_t *flags);

/* Test entry point (not part of the release ABI): the resident tile log of `count` vertices
 * (host ids, current labels) as (vertex, offset, size, kind) quadruples, kind 0 = tile,
 * 1 = fragment, produced by the same device classifier the traversal kernels use (Alg. 3
 * l.2-7).  triples_out holds 4*cap int64 (host); *n_out = number of quadruples.  If cap is too
 * small nothing is written and *n_out is the required count.                                   */
sage_status sage_debug_export_tiles(sage_graph *g, const int32_t *vertices, int64_t count,
                                    int64_t *quads_out, int64_t cap, int64_t *n_out);

/* Test entry point: stages 1-3 of one reorder round on the current labels, without relabelling:
 * per vertex (current labels) loc1, target sector, loc3 (int64, n each) and mover flag (uint8, n),
 * host buffers.  candidates: optional ORIGINAL ids allowed to move.                              */
sage_status sage_debug_reorder_stages(sage_graph *g, int32_t sector_width, const int32_t *candidates,
                                      int64_t n_candidates, int64_t *loc1_out, int64_t *target_out,
                                      int64_t *loc3_out, uint8_t *mover_out);

/* Diagnostic entry point: per-level records of the last BFS / SSSP query on this graph, 9 int64 per
 * level (rec_out must hold 9 * cap int64): direction (0 push, 1 pull), |F|, arcs(F), arcs
 * inspected, vertices scanned (pull), vertices discovered, device time since the kernel started
 * at the end of the level (ns), the time at which the last warp finished the level's work,
 * before the grid barrier (ns), and the end of the level's expansion phase before Tiled
 * Partitioning of the next frontier (ns; 0 when not recorded).
 * Writes min(levels, cap) records to host memory; *n_out = number of levels (<= 4096 kept).     */
sage_status sage_debug_level_records(const sage_graph *g, int64_t *rec_out, int32_t cap,
                                     int32_t *n_out);

/* Test entry point (not part of the release ABI): a 128-byte id that, passed as
 * sage_dist.nccl_unique_id by `world` graphs loaded in ONE process on ONE GPU (one host thread
 * per rank, every rank loaded before any collective call), replaces NCCL by a loopback transport
 * (stream-ordered device copies / reductions between the ranks' buffers; xport.h).  It exists so
 * the multi-GPU path's remote-owner code (r > 0, padded indexing, the apply kernels, the sparse
 * and dense exchanges) is checked against the oracle on a single-GPU test pool.  The group lives
 * until its last graph is freed.                                                               */
sage_status sage_debug_loopback_id(int32_t world, void *out128);

/* Thread-local message of the last failing call on this thread ("" if none).                   */
const char *sage_last_error(void);

/* Library version string.                                                                      */
const char *sage_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SAGE_H_ */
