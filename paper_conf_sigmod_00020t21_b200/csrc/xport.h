// xport.h — collective transport of the multi-GPU path (comm.cu), one object per rank.
//
// The multi-GPU level loop needs six collectives on device buffers, all enqueued
// on the graph's stream.  Two implementations:
//   * NCCL (the product): ncclAllGather / ncclAllReduce / ncclReduceScatter and grouped
//     ncclSend/ncclRecv for the all-to-all(v), one process per GPU over NVLink / NVSwitch; peer
//     memory through CUDA IPC handles exchanged over NCCL (the push BFS's fused exchange);
//   * loopback (TEST ONLY): p logical ranks in one process on ONE GPU, one host thread per rank,
//     collectives done with stream-ordered device copies / reduction kernels between the ranks'
//     buffers.  It lets the single-GPU test pool run the r > 0 code paths (remote owners, padded
//     indexing, the apply kernels) against the oracle.  It is reachable only through an id made by
//     sage_debug_loopback_id(), never through a product flag.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include "sage.h"

struct sage_graph;

namespace sage {

struct Xport {
  int rank = 0, world = 1;
  virtual ~Xport() {}
  // recv = world * bytes, rank order; send may alias recv + rank * bytes
  virtual sage_status allgather(sage_graph *g, const void *send, void *recv, size_t bytes) = 0;
  virtual sage_status allreduce_sum_u64(sage_graph *g, const unsigned long long *send, unsigned long long *recv,
                                        size_t n) = 0;
  virtual sage_status allreduce_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) = 0;
  // send = world * n (block q goes to rank q), recv = n
  virtual sage_status reduce_scatter_min_u32(sage_graph *g, const uint32_t *send, uint32_t *recv, size_t n) = 0;
  virtual sage_status reduce_scatter_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) = 0;
  // bytes [soff[q], soff[q+1]) of send go to rank q and arrive at [roff[me_q], ...) of q's recv;
  // soff / roff are host arrays of world + 1 byte offsets (the counts must agree pairwise)
  virtual sage_status alltoallv(sage_graph *g, const void *send, const size_t *soff, void *recv,
                                const size_t *roff) = 0;
  // Peer memory (collective call): every rank exposes `mine` (a cudaMalloc'd buffer); on return
  // peers[q] is a pointer this rank's kernels may load / store / atomically update in rank q's
  // buffer (peers[rank] = mine).  SAGE_E_UNSUPPORTED on EVERY rank when any rank cannot map any
  // other's memory with native atomics (the caller then keeps the collective exchange).
  virtual sage_status peer_map(sage_graph *g, void *mine, void **peers) = 0;
  virtual void peer_unmap(void **peers) = 0;
  // Stream-ordered barrier: work enqueued on any rank's stream before it completes (its peer
  // writes included) before work enqueued on any rank's stream after it starts.
  virtual sage_status barrier(sage_graph *g) = 0;
};

// NCCL transport from a 128-byte ncclUniqueId.
Xport *make_nccl_xport(sage_graph *g, const void *id128, int rank, int world, sage_status *st);
// Loopback transport if id128 was made by sage_debug_loopback_id (else nullptr).
Xport *make_loopback_xport(sage_graph *g, const void *id128, int rank, int world, sage_status *st);

}  // namespace sage
