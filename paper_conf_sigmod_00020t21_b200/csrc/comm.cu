// comm.cu — multi-GPU (1D vertex partition + NCCL frontier exchange).
// Placeholder until the exchange lands: multi-GPU handles are refused explicitly.
#include "graph.h"
#include "internal.h"

namespace sage {

struct Comm {};

sage_status init_comm(sage_graph *, const sage_dist *) {
  set_error("multi-GPU (world > 1) is not available in this build");
  return SAGE_E_UNSUPPORTED;
}
void free_comm(sage_graph *g) { g->comm = nullptr; }

sage_status run_bfs_multi(sage_graph *, int32_t, int32_t *, int32_t *, uint32_t, sage_stats *) {
  return SAGE_E_UNSUPPORTED;
}
sage_status run_sssp_multi(sage_graph *, int32_t, uint32_t *, sage_stats *) {
  return SAGE_E_UNSUPPORTED;
}
sage_status run_pagerank_multi(sage_graph *, double, int32_t, double *, sage_stats *) {
  return SAGE_E_UNSUPPORTED;
}

}  // namespace sage
