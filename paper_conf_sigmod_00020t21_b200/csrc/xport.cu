// xport.cu — the two collective transports of xport.h: NCCL (product) and loopback (tests).
#include <cuda_runtime.h>
#include <nccl.h>
#include <string.h>

#include <atomic>
#include <condition_variable>
#include <mutex>
#include <vector>

#include "graph.h"
#include "internal.h"
#include "xport.h"

namespace sage {

// ============================================================================ NCCL
static sage_status nccl_fail(sage_graph *g, ncclResult_t r, const char *what) {
  set_error("%s: %s", what, ncclGetErrorString(r));
  if (g) g->sticky = SAGE_E_NCCL;
  return SAGE_E_NCCL;
}
#define XN(call, what)                                   \
  do {                                                   \
    ncclResult_t r_ = (call);                            \
    if (r_ != ncclSuccess) return nccl_fail(g, r_, what); \
  } while (0)

struct NcclXport : Xport {
  ncclComm_t nc = nullptr;
  ~NcclXport() override {
    if (nc) ncclCommDestroy(nc);
    if (scratch) cudaFree(scratch);
  }
  sage_status allgather(sage_graph *g, const void *send, void *recv, size_t bytes) override {
    XN(ncclAllGather(send, recv, bytes, ncclUint8, nc, g->stream), "ncclAllGather");
    return SAGE_OK;
  }
  sage_status allreduce_sum_u64(sage_graph *g, const unsigned long long *send, unsigned long long *recv,
                                size_t n) override {
    XN(ncclAllReduce(send, recv, n, ncclUint64, ncclSum, nc, g->stream), "ncclAllReduce");
    return SAGE_OK;
  }
  sage_status allreduce_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) override {
    XN(ncclAllReduce(send, recv, n, ncclFloat64, ncclSum, nc, g->stream), "ncclAllReduce");
    return SAGE_OK;
  }
  sage_status reduce_scatter_min_u32(sage_graph *g, const uint32_t *send, uint32_t *recv, size_t n) override {
    XN(ncclReduceScatter(send, recv, n, ncclUint32, ncclMin, nc, g->stream), "ncclReduceScatter(min)");
    return SAGE_OK;
  }
  sage_status reduce_scatter_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) override {
    XN(ncclReduceScatter(send, recv, n, ncclFloat64, ncclSum, nc, g->stream), "ncclReduceScatter(sum)");
    return SAGE_OK;
  }
  sage_status alltoallv(sage_graph *g, const void *send, const size_t *soff, void *recv,
                        const size_t *roff) override {
    const char *s = static_cast<const char *>(send);
    char *r = static_cast<char *>(recv);
    // own block: a local copy
    if (soff[rank + 1] > soff[rank])
      cudaMemcpyAsync(r + roff[rank], s + soff[rank], soff[rank + 1] - soff[rank], cudaMemcpyDeviceToDevice,
                      g->stream);
    XN(ncclGroupStart(), "ncclGroupStart");
    for (int q = 0; q < world; ++q) {
      if (q == rank) continue;
      if (soff[q + 1] > soff[q])
        XN(ncclSend(s + soff[q], soff[q + 1] - soff[q], ncclUint8, q, nc, g->stream), "ncclSend");
      if (roff[q + 1] > roff[q])
        XN(ncclRecv(r + roff[q], roff[q + 1] - roff[q], ncclUint8, q, nc, g->stream), "ncclRecv");
    }
    XN(ncclGroupEnd(), "ncclGroupEnd");
    return SAGE_OK;
  }
  unsigned long long *scratch = nullptr;   // barrier word + IPC handle exchange (device)
  sage_status ensure_scratch(sage_graph *g) {
    if (scratch) return SAGE_OK;
    const cudaError_t e = cudaMalloc((void **)&scratch, 64 + (size_t)world * sizeof(cudaIpcMemHandle_t));
    if (e != cudaSuccess) return cuda_fail(g, e, "xport scratch");
    cudaMemsetAsync(scratch, 0, 64, g->stream);
    return SAGE_OK;
  }
  sage_status barrier(sage_graph *g) override {
    sage_status s = ensure_scratch(g);
    if (s != SAGE_OK) return s;
    XN(ncclAllReduce(scratch, scratch + 1, 1, ncclUint64, ncclSum, nc, g->stream), "ncclAllReduce(barrier)");
    return SAGE_OK;
  }
  sage_status peer_map(sage_graph *g, void *mine, void **peers) override {
    sage_status s = ensure_scratch(g);
    if (s != SAGE_OK) return s;
    for (int q = 0; q < world; ++q) peers[q] = nullptr;
    peers[rank] = mine;
    // every rank's IPC handle, then every rank's verdict (all ranks must agree on the form)
    cudaIpcMemHandle_t h;
    memset(&h, 0, sizeof(h));
    unsigned long long fail = cudaIpcGetMemHandle(&h, mine) != cudaSuccess;
    cudaGetLastError();
    char *hs = reinterpret_cast<char *>(scratch + 8);
    std::vector<cudaIpcMemHandle_t> all((size_t)world);
    cudaMemcpyAsync(hs + rank * sizeof(h), &h, sizeof(h), cudaMemcpyHostToDevice, g->stream);
    XN(ncclAllGather(hs + rank * sizeof(h), hs, sizeof(h), ncclUint8, nc, g->stream), "ncclAllGather(ipc)");
    cudaMemcpyAsync(all.data(), hs, sizeof(h) * (size_t)world, cudaMemcpyDeviceToHost, g->stream);
    cudaError_t e = cudaStreamSynchronize(g->stream);
    if (e != cudaSuccess) return cuda_fail(g, e, "peer handle exchange");
    int dev = 0;
    cudaGetDevice(&dev);
    for (int q = 0; q < world && !fail; ++q) {
      if (q == rank) continue;
      if (cudaIpcOpenMemHandle(&peers[q], all[(size_t)q], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        peers[q] = nullptr;
        fail = 1;
        break;
      }
      cudaPointerAttributes at;
      int atom = 0;
      if (cudaPointerGetAttributes(&at, peers[q]) != cudaSuccess || at.device == dev ||
          cudaDeviceGetP2PAttribute(&atom, cudaDevP2PAttrNativeAtomicSupported, dev, at.device) != cudaSuccess ||
          !atom)
        fail = 1;
      cudaGetLastError();
    }
    cudaMemcpyAsync(scratch + 2, &fail, sizeof(fail), cudaMemcpyHostToDevice, g->stream);
    XN(ncclAllReduce(scratch + 2, scratch + 3, 1, ncclUint64, ncclSum, nc, g->stream), "ncclAllReduce(peer)");
    unsigned long long nfail = 0;
    cudaMemcpyAsync(&nfail, scratch + 3, sizeof(nfail), cudaMemcpyDeviceToHost, g->stream);
    e = cudaStreamSynchronize(g->stream);
    if (e != cudaSuccess) return cuda_fail(g, e, "peer verdict");
    if (nfail) {
      peer_unmap(peers);
      peers[rank] = mine;
      return SAGE_E_UNSUPPORTED;
    }
    return SAGE_OK;
  }
  void peer_unmap(void **peers) override {
    for (int q = 0; q < world; ++q)
      if (q != rank && peers[q]) {
        cudaIpcCloseMemHandle(peers[q]);
        peers[q] = nullptr;
      }
  }
};

Xport *make_nccl_xport(sage_graph *g, const void *id128, int rank, int world, sage_status *st) {
  NcclXport *x = new NcclXport();
  x->rank = rank;
  x->world = world;
  ncclUniqueId id;
  memcpy(&id, id128, sizeof(id));
  ncclResult_t r = ncclCommInitRank(&x->nc, world, id, rank);
  if (r != ncclSuccess) {
    *st = nccl_fail(g, r, "ncclCommInitRank");
    x->nc = nullptr;
    delete x;
    return nullptr;
  }
  *st = SAGE_OK;
  return x;
}

// ============================================================================ loopback (tests)
static const char kLoopMagic[16] = "SAGE-LOOPBACK-1";

constexpr int kLoopMax = 64;
struct LoopSlot {
  const void *send = nullptr;
  void *recv = nullptr;
  const size_t *soff = nullptr, *roff = nullptr;
  cudaEvent_t ready = nullptr, done = nullptr;
  void *peer = nullptr;
};
struct LoopGroup {
  int world = 0;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  unsigned long long gen = 0;
  LoopSlot slot[kLoopMax];
  std::atomic<int> refs{0};
  void barrier() {
    std::unique_lock<std::mutex> lk(mu);
    const unsigned long long g0 = gen;
    if (++arrived == world) {
      arrived = 0;
      ++gen;
      cv.notify_all();
    } else {
      cv.wait(lk, [&] { return gen != g0; });
    }
  }
};

struct PtrSet {
  const void *p[kLoopMax];
};
template <class T, int OP>   // OP 0 = sum, 1 = min
__global__ void k_loop_reduce(PtrSet src, int world, size_t off, T *dst, size_t n) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    T a = static_cast<const T *>(src.p[0])[off + i];
    for (int q = 1; q < world; ++q) {
      const T b = static_cast<const T *>(src.p[q])[off + i];
      a = OP == 0 ? (T)(a + b) : (b < a ? b : a);
    }
    dst[i] = a;
  }
}

struct LoopXport : Xport {
  LoopGroup *grp = nullptr;
  ~LoopXport() override {
    LoopSlot &s = grp->slot[rank];
    if (s.ready) cudaEventDestroy(s.ready);
    if (s.done) cudaEventDestroy(s.done);
    s.ready = s.done = nullptr;
    if (--grp->refs == 0) delete grp;
  }
  // publish this rank's buffers, wait for every rank's, run `part` on this rank's stream, then
  // wait until every rank has finished reading (stream-ordered through events)
  template <class F>
  sage_status run(sage_graph *g, const void *send, void *recv, const size_t *soff, const size_t *roff, F part) {
    LoopSlot &me = grp->slot[rank];
    me.send = send;
    me.recv = recv;
    me.soff = soff;
    me.roff = roff;
    cudaEventRecord(me.ready, g->stream);
    grp->barrier();
    for (int q = 0; q < world; ++q) cudaStreamWaitEvent(g->stream, grp->slot[q].ready, 0);
    part();
    cudaEventRecord(me.done, g->stream);
    grp->barrier();
    for (int q = 0; q < world; ++q) cudaStreamWaitEvent(g->stream, grp->slot[q].done, 0);
    grp->barrier();   // no rank may destroy its events (sage_free) while another still waits on them
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_fail(g, e, "loopback collective");
    return SAGE_OK;
  }
  PtrSet sends() const {
    PtrSet ps;
    for (int q = 0; q < world; ++q) ps.p[q] = grp->slot[q].send;
    return ps;
  }
  int grid(sage_graph *g) const { return g->num_sms * 4; }
  sage_status allgather(sage_graph *g, const void *send, void *recv, size_t bytes) override {
    return run(g, send, recv, nullptr, nullptr, [&] {
      for (int q = 0; q < world; ++q)
        if (q != rank || grp->slot[q].send != static_cast<char *>(recv) + (size_t)rank * bytes)
          cudaMemcpyAsync(static_cast<char *>(recv) + (size_t)q * bytes, grp->slot[q].send, bytes,
                          cudaMemcpyDeviceToDevice, g->stream);
    });
  }
  sage_status allreduce_sum_u64(sage_graph *g, const unsigned long long *send, unsigned long long *recv,
                                size_t n) override {
    return run(g, send, recv, nullptr, nullptr, [&] {
      k_loop_reduce<unsigned long long, 0><<<grid(g), 256, 0, g->stream>>>(sends(), world, 0, recv, n);
    });
  }
  sage_status allreduce_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) override {
    return run(g, send, recv, nullptr, nullptr, [&] {
      k_loop_reduce<double, 0><<<grid(g), 256, 0, g->stream>>>(sends(), world, 0, recv, n);
    });
  }
  sage_status reduce_scatter_min_u32(sage_graph *g, const uint32_t *send, uint32_t *recv, size_t n) override {
    return run(g, send, recv, nullptr, nullptr, [&] {
      k_loop_reduce<uint32_t, 1><<<grid(g), 256, 0, g->stream>>>(sends(), world, (size_t)rank * n, recv, n);
    });
  }
  sage_status reduce_scatter_sum_f64(sage_graph *g, const double *send, double *recv, size_t n) override {
    return run(g, send, recv, nullptr, nullptr, [&] {
      k_loop_reduce<double, 0><<<grid(g), 256, 0, g->stream>>>(sends(), world, (size_t)rank * n, recv, n);
    });
  }
  sage_status alltoallv(sage_graph *g, const void *send, const size_t *soff, void *recv,
                        const size_t *roff) override {
    return run(g, send, recv, soff, roff, [&] {
      for (int q = 0; q < world; ++q) {
        const LoopSlot &s = grp->slot[q];
        const size_t b = s.soff[rank + 1] - s.soff[rank];
        if (b) cudaMemcpyAsync(static_cast<char *>(recv) + roff[q], static_cast<const char *>(s.send) + s.soff[rank],
                               b, cudaMemcpyDeviceToDevice, g->stream);
      }
    });
  }
  // one device: every rank's buffer is directly addressable
  sage_status peer_map(sage_graph *, void *mine, void **peers) override {
    grp->slot[rank].peer = mine;
    grp->barrier();
    for (int q = 0; q < world; ++q) peers[q] = grp->slot[q].peer;
    grp->barrier();
    return SAGE_OK;
  }
  void peer_unmap(void **) override {}
  sage_status barrier(sage_graph *g) override {
    return run(g, nullptr, nullptr, nullptr, nullptr, [] {});
  }
};

Xport *make_loopback_xport(sage_graph *g, const void *id128, int rank, int world, sage_status *st) {
  const char *id = static_cast<const char *>(id128);
  *st = SAGE_OK;
  if (memcmp(id, kLoopMagic, sizeof(kLoopMagic)) != 0) return nullptr;
  LoopGroup *grp = nullptr;
  memcpy(&grp, id + 16, sizeof(grp));
  if (!grp || grp->world != world || world > kLoopMax) {
    set_error("loopback id does not match world %d", world);
    *st = SAGE_E_INVALID;
    return nullptr;
  }
  LoopXport *x = new LoopXport();
  x->rank = rank;
  x->world = world;
  x->grp = grp;
  grp->refs++;
  LoopSlot &s = grp->slot[rank];
  cudaEventCreateWithFlags(&s.ready, cudaEventDisableTiming);
  cudaEventCreateWithFlags(&s.done, cudaEventDisableTiming);
  (void)g;
  *st = SAGE_OK;
  return x;
}

}  // namespace sage

// Test entry point (include/sage.h): a 128-byte id for `world` logical ranks of ONE process on
// ONE GPU (loopback collectives).  Every rank must load its block with this id (one host thread
// per rank) before any rank calls a collective; the group lives until its last graph is freed.
extern "C" sage_status sage_debug_loopback_id(int32_t world, void *out128) {
  sage::clear_error();
  if (!out128 || world < 1 || world > sage::kLoopMax) {
    sage::set_error("world must be in [1, %d] and out128 non-null", sage::kLoopMax);
    return SAGE_E_INVALID;
  }
  sage::LoopGroup *grp = new sage::LoopGroup();
  grp->world = world;
  char *o = static_cast<char *>(out128);
  memset(o, 0, 128);
  memcpy(o, sage::kLoopMagic, sizeof(sage::kLoopMagic));
  memcpy(o + 16, &grp, sizeof(grp));
  return SAGE_OK;
}
