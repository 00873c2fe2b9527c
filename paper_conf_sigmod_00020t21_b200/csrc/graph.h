// graph.h — host-side state of a loaded graph (the opaque sage_graph of include/sage.h).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "common.cuh"
#include "sage.h"

namespace sage {

// Thread-local error message + status helpers (capi.cu).
void set_error(const char *fmt, ...);
void clear_error();

struct DeviceBuf {          // a library-owned device allocation
  void *p = nullptr;
  size_t bytes = 0;
};

struct Comm;                // multi-GPU communicator (comm.cu); null on one GPU

struct TraversalState {     // per-query scratch, allocated on first use and kept
  bool ready = false;
  int32_t *level = nullptr;       // BFS levels (int32, -1 = unvisited), n_local
  int32_t *parent = nullptr;      // BFS parents (allocated on first parent request)
  uint32_t *dist = nullptr;       // SSSP distances, n_local
  cudaEvent_t ev_caller = nullptr;   // orders in-place output writes after the caller's stream
  uint32_t *visited = nullptr;    // visited bitmap, ceil(n/32) words (+ padding)
  uint32_t *fb[3] = {nullptr, nullptr, nullptr};  // frontier bitmaps (rotated), pull + SSSP dedupe
  Queues q[2];                    // double-buffered per-level tile logs
  Ctl *ctl = nullptr;             // device control block
  int32_t *tmp_out = nullptr;     // ID-translation scratch (n_local)
  void *tailmem = nullptr;        // BFS tail mode state (global scratch)
  int *flist = nullptr;           // BFS deferred contraction: frontier list
  uint32_t *hub_g = nullptr;      // BFS hub filter: global table of visited hubs (T packed entries)
  int *flist2 = nullptr;          // BFS fused tiling: the second frontier list (levels alternate)
  cudaEvent_t ev[3] = {nullptr, nullptr, nullptr};   // per-call timing events (created once)
  Ctl *hctl = nullptr;            // pinned host copy of the control block
};

struct PageRankState {      // the all-V resident tile log (built once, reused)
  bool valid = false;
  Queues q;
  unsigned long long cnt[kQueues] = {0};
  int32_t *dangling = nullptr;    // vertices with out-degree 0
  long long n_dangling = 0;
  double *x = nullptr, *y = nullptr;
  void *c = nullptr;              // pull form: x_u / out(u) (fp32, or fp64 when damping > 0.9)
  size_t c_bytes = 0;
  CounterSet *cs = nullptr;       // device copy of the log's counters (+ rotating tickets)
  int win = -1;                   // windowed push chosen for this graph (-1 = not measured yet)
  double locality = 0.0;          // sampled fraction of arcs within the window's halo of their source
};

}  // namespace sage

struct sage_graph {
  int64_t n = 0;              // global vertex count
  int64_t n_local = 0;        // rows owned here
  int64_t v_begin = 0, v_end = 0;
  int64_t m = 0;              // local arcs
  uint32_t flags = 0;
  int device = 0;
  int num_sms = 0;
  cudaStream_t stream = nullptr;
  bool own_stream = false;
  int64_t *off = nullptr;     // device, n_local + 1
  int32_t *col = nullptr;     // device, m
  uint32_t *w = nullptr;      // device, m or null
  bool own_off = false, own_col = false, own_w = false;
  bool host_columns = false;          // SAGE_F_HOST_COLUMNS: col / w are mapped pinned host memory
  void *host_registered[2] = {nullptr, nullptr};   // caller pages registered in place (col, w)
  void *host_owned[2] = {nullptr, nullptr};        // library-owned pinned copies (col, w)
  bool rows_sorted = false;
  int64_t max_degree = 0;
  int64_t max_indeg = -1;     // max in-degree (lazily, for the reorder's counter width; -1 = unknown)
  int64_t n_isolated = 0;
  sage::Ladder ladder{};
  double alpha = 15.0, beta = 18.0;
  int ctas_per_sm = 0;        // sage_options.ctas_per_sm (0 = automatic)
  int hub_filter = 0;         // sage_options.hub_filter (0 auto, 1 on, -1 off)
  int vec = 4;                // neighbours per lane per step (4; 1 when tile_min < 4)
  bool vec_ok = true;         // sub-warp tiles use 16-B loads (align % 4 == 0, aligned arrays)
  // reordering: sigma[v_orig] = current label; sigma_inv[label] = v_orig (null = identity)
  int32_t *sigma = nullptr, *sigma_inv = nullptr;
  bool reordered = false;
  std::vector<int32_t> h_sigma;   // host copy of sigma (source-id translation)
  int sticky = 0;             // sticky SAGE_E_CUDA / SAGE_E_NCCL
  sage::TraversalState ts;
  sage::PageRankState pr;
  sage::Comm *comm = nullptr;
  // online sampling (sage_online_reorder): per-vertex occurrence counts, recorded row lengths
  bool online = false;
  int online_lgS = 3;
  long long online_thr = 0, online_pending = 0, online_rounds = 0, online_movers = 0, online_swaps = 0;
  uint32_t *samp_w = nullptr;
  unsigned long long *samp_acc = nullptr;
  int grid_bfs = 0, grid_bfs_hub = 0, grid_bfs_fused = 0, grid_bfs_fused_hub = 0, grid_sssp = 0, grid_pr = 0, grid_pr_pull = 0, grid_pr_pull64 = 0, grid_pr_win = 0;   // persistent grid sizes
};
