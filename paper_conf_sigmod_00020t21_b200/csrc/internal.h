// internal.h — host functions shared between the .cu files of libsage.so (not exported).
#pragma once
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "graph.h"

namespace sage {

// NVTX range over one C-ABI call (SURVEY §5 tracing): visible in Nsight Systems / ncu --nvtx;
// header-only NVTX v3, a no-op without an attached tool.
struct NvtxRange {
  explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
  NvtxRange(const NvtxRange &) = delete;
  NvtxRange &operator=(const NvtxRange &) = delete;
};

sage_status cuda_fail(sage_graph *g, cudaError_t e, const char *what);
bool is_device_ptr(const void *p);
sage_status dalloc(sage_graph *g, void **p, size_t bytes);
void dfree(sage_graph *g, void *p);
sage_status copy_out(sage_graph *g, void *dst, const void *src_dev, size_t bytes);
void iota_device(sage_graph *g, int32_t *p, int64_t n);

// traversal.cu
sage_status ensure_traversal_state(sage_graph *g);
void free_traversal_state(sage_graph *g);
sage_status alloc_queues(sage_graph *g, Queues *q, long long n_rows, long long m);
void free_queues(sage_graph *g, Queues *q);
// gather out[v] = src[sigma[v]] for the caller's original ids (identity when not reordered)
sage_status translate_out_i32(sage_graph *g, const int32_t *src, int32_t *dst_user, bool map_values);
sage_status translate_out_u32(sage_graph *g, const uint32_t *src, uint32_t *dst_user);
sage_status translate_out_f64(sage_graph *g, const double *src, double *dst_user);
int32_t to_internal_id(sage_graph *g, int32_t v);

// pagerank.cu
void free_pagerank_state(sage_graph *g);
sage_status online_after_query(sage_graph *g, const int32_t *level_internal, int32_t pr_iters);
sage_status ensure_pagerank_log(sage_graph *g);

// comm.cu (multi-GPU)
sage_status init_comm(sage_graph *g, const sage_dist *ds);
void free_comm(sage_graph *g);
bool comm_peer_exchange(const sage_graph *g);   // the push exchange runs over peer memory

// cooperative persistent launch helper
sage_status launch_coop(sage_graph *g, const void *fn, int grid, void **args, const char *what,
                        int block = kBlock, size_t dyn_smem = 0);
int coop_grid(sage_graph *g, const void *fn, int *cache, int block = kBlock, size_t dyn_smem = 0);

}  // namespace sage
