// reorder.cu — Sampling-based Reordering (§6).  Placeholder until the GPU stages land.
#include "graph.h"
#include "internal.h"

using namespace sage;

extern "C" sage_status sage_reorder(sage_graph *g, int32_t rounds, const sage_reorder_opts *opt,
                                    sage_stats *st) {
  (void)g; (void)rounds; (void)opt; (void)st;
  set_error("sage_reorder is not available in this build yet");
  return SAGE_E_UNSUPPORTED;
}
