// capi.cu — the C ABI of include/sage.h: graph load + validation, free, info, outputs, errors.
//
// sage_load_csr follows the paper's problem statement: the CSR is loaded once and then
// queried with no preprocessing — the only pass over the input is validation.
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <string>

#include "graph.h"
#include "internal.h"

namespace sage {

static thread_local std::string g_last_error;

void set_error(const char *fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_last_error = buf;
}
void clear_error() { g_last_error.clear(); }

sage_status cuda_fail(sage_graph *g, cudaError_t e, const char *what) {
  set_error("%s: %s", what, cudaGetErrorString(e));
  if (g) g->sticky = SAGE_E_CUDA;
  return SAGE_E_CUDA;
}

bool is_device_ptr(const void *p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Library-owned stream-ordered memory pool per device.  Freed blocks stay mapped in the pool
// (release threshold = unlimited), so a load / free / load cycle does not re-map gigabytes.
static cudaMemPool_t pool_for(int dev) {
  static cudaMemPool_t pools[64] = {};
  if (dev < 0 || dev >= 64) return nullptr;
  if (!pools[dev]) {
    cudaMemPoolProps props = {};
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t p = nullptr;
    if (cudaMemPoolCreate(&p, &props) != cudaSuccess) {
      cudaGetLastError();
      return nullptr;
    }
    unsigned long long thr = ~0ull;
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = p;
  }
  return pools[dev];
}

sage_status dalloc(sage_graph *g, void **p, size_t bytes) {
  *p = nullptr;
  if (bytes == 0) bytes = 16;
  cudaMemPool_t pool = pool_for(g->device);
  cudaError_t e = pool ? cudaMallocFromPoolAsync(p, bytes, pool, g->stream)
                       : cudaMallocAsync(p, bytes, g->stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    *p = nullptr;
    set_error("device allocation of %zu bytes failed: %s", bytes, cudaGetErrorString(e));
    return SAGE_E_NOMEM;
  }
  return SAGE_OK;
}
void dfree(sage_graph *g, void *p) {
  if (p) cudaFreeAsync(p, g->stream);
}

sage_status copy_out(sage_graph *g, void *dst, const void *src_dev, size_t bytes) {
  if (bytes == 0) return SAGE_OK;
  cudaError_t e = cudaMemcpyAsync(dst, src_dev, bytes, cudaMemcpyDefault, g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "output copy");
  return SAGE_OK;
}

// ------------------------------------------------------------------------------------------
// Validation kernels (one streaming pass over off and col/w).
struct ValidateOut {
  unsigned long long bad_off, bad_col, bad_w, unsorted, isolated, max_deg;
};

__global__ void k_validate_rows(const long long *__restrict__ off, long long n_local, long long m,
                                uint32_t *__restrict__ rowstart, ValidateOut *out) {
  long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
  long long stride = (long long)gridDim.x * blockDim.x;
  unsigned long long bad = 0, iso = 0, mx = 0;
  for (; i < n_local; i += stride) {
    long long b = off[i], e = off[i + 1];
    if (e < b || b < 0 || e > m || e - b > 0x7fffffffll) { bad++; continue; }
    if (e == b) iso++;
    else if (rowstart) atomicOr(rowstart + (b >> 5), 1u << (b & 31));
    unsigned long long d = (unsigned long long)(e - b);
    if (d > mx) mx = d;
  }
  if (bad) atomicAdd(&out->bad_off, bad);
  if (iso) atomicAdd(&out->isolated, iso);
  if (mx) atomicMax(&out->max_deg, mx);
}

// One streaming pass over col (and w): 4 consecutive elements per thread per step (16-B loads
// when aligned), rows-sorted check against the row-start bitmap built by k_validate_rows.
__global__ void k_validate_arcs(const int *__restrict__ col, const uint32_t *__restrict__ w,
                                long long m, long long n, const uint32_t *__restrict__ rowstart,
                                ValidateOut *out) {
  const long long stride = 4ll * gridDim.x * blockDim.x;
  unsigned long long bc = 0, bw = 0, us = 0;
  const bool vec = ((uintptr_t)col % 16) == 0 && (!w || ((uintptr_t)w % 16) == 0);
  for (long long k0 = 4ll * ((long long)blockIdx.x * blockDim.x + threadIdx.x); k0 < m; k0 += stride) {
    int c[5];
    uint32_t ww[4] = {1u, 1u, 1u, 1u};
    if (vec && k0 + 4 <= m) {
      const int4 c4 = __ldg(reinterpret_cast<const int4 *>(col + k0));
      c[0] = c4.x; c[1] = c4.y; c[2] = c4.z; c[3] = c4.w;
      if (w) {
        const uint4 w4 = __ldg(reinterpret_cast<const uint4 *>(w + k0));
        ww[0] = w4.x; ww[1] = w4.y; ww[2] = w4.z; ww[3] = w4.w;
      }
    } else {
      for (int j = 0; j < 4; ++j) {
        c[j] = k0 + j < m ? __ldg(col + k0 + j) : 0;
        if (w && k0 + j < m) ww[j] = __ldg(w + k0 + j);
      }
    }
    c[4] = k0 + 4 < m ? __ldg(col + k0 + 4) : 0;
    // bits k0+1 .. k0+4 of the row-start bitmap (may straddle two words)
    const long long b1 = k0 + 1;
    unsigned long long rs = __ldg(rowstart + (b1 >> 5));
    if (((b1 & 31) + 4) > 32) rs |= (unsigned long long)__ldg(rowstart + (b1 >> 5) + 1) << 32;
    rs >>= (b1 & 31);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const long long k = k0 + j;
      if (k >= m) break;
      if (c[j] < 0 || c[j] >= n) bc++;
      if (ww[j] == 0) bw++;
      if (k + 1 < m && !((rs >> j) & 1ull) && c[j + 1] <= c[j]) us++;
    }
  }
  if (bc) atomicAdd(&out->bad_col, bc);
  if (bw) atomicAdd(&out->bad_w, bw);
  if (us) atomicAdd(&out->unsorted, us);
}

static int ilog2(long long x) {
  int r = 0;
  while ((1ll << r) < x) ++r;
  return r;
}
static bool is_pow2(long long x) { return x > 0 && (x & (x - 1)) == 0; }

static sage_status make_ladder(const sage_options *o, sage_graph *g) {
  int B = 256, M = 8, A = 4, cps = 0, hub = 0;
  double alpha = 15.0, beta = 18.0;
  if (o) {
    B = o->tile_cta;
    M = o->tile_min;
    A = o->align;
    alpha = o->alpha;
    beta = o->beta;
    cps = o->ctas_per_sm;
    hub = o->hub_filter;
  }
  if (hub < -1 || hub > 1) {
    set_error("hub_filter must be -1, 0 or 1");
    return SAGE_E_INVALID;
  }
  if (cps < 0 || cps > 32) {
    set_error("ctas_per_sm must be in [0, 32]");
    return SAGE_E_INVALID;
  }
  if (!is_pow2(B) || B > 4096) {
    set_error("tile_cta must be a power of two in [1, 4096]");
    return SAGE_E_INVALID;
  }
  if (!is_pow2(M) || M > B || (B / M) > 4096) {
    set_error("tile_min must be a power of two in [1, tile_cta] with tile_cta/tile_min <= 4096");
    return SAGE_E_INVALID;
  }
  if (A < 0 || A > 64 || (A > 0 && !is_pow2(A))) {
    set_error("align must be 0 or a power of two <= 64");
    return SAGE_E_INVALID;
  }
  if (!(alpha > 0) || !(beta > 0)) {
    set_error("alpha and beta must be > 0");
    return SAGE_E_INVALID;
  }
  g->ladder.B = B;
  g->ladder.M = M;
  g->ladder.A = A;
  g->ladder.lgB = ilog2(B);
  g->ladder.ncls = ilog2(B / M) + 1;
  g->alpha = alpha;
  g->beta = beta;
  g->ctas_per_sm = cps;
  g->hub_filter = hub;
  return SAGE_OK;
}

void free_traversal_state(sage_graph *g);
void free_pagerank_state(sage_graph *g);

static void destroy(sage_graph *g) {
  if (!g) return;
  free_traversal_state(g);
  free_pagerank_state(g);
  free_comm(g);
  if (g->own_off) dfree(g, g->off);
  if (g->own_col) dfree(g, g->col);
  if (g->own_w) dfree(g, g->w);
  cudaStreamSynchronize(g->stream);
  for (int i = 0; i < 2; ++i) {
    if (g->host_registered[i]) cudaHostUnregister(g->host_registered[i]);
    if (g->host_owned[i]) cudaFreeHost(g->host_owned[i]);
  }
  dfree(g, g->sigma);
  dfree(g, g->sigma_inv);
  dfree(g, g->samp_w);
  dfree(g, g->samp_acc);
  cudaStreamSynchronize(g->stream);
  if (g->own_stream) cudaStreamDestroy(g->stream);
  delete g;
}

}  // namespace sage

using namespace sage;

extern "C" {

const char *sage_last_error(void) { return g_last_error.c_str(); }
const char *sage_version(void) { return "sage-b200 0.1 (sm_100a)"; }

sage_status sage_load_csr(const sage_csr *in, sage_graph **out) {
  NvtxRange nvtx_("sage_load_csr");
  clear_error();
  if (!out) {
    set_error("out is NULL");
    return SAGE_E_INVALID;
  }
  *out = nullptr;
  if (!in || !in->row_offsets || (in->m > 0 && !in->col_indices)) {
    set_error("null CSR argument");
    return SAGE_E_INVALID;
  }
  if (in->n <= 0 || in->n >= (1ll << 31) || in->m < 0) {
    set_error("n must be in (0, 2^31) and m >= 0 (n=%lld m=%lld)", (long long)in->n,
              (long long)in->m);
    return SAGE_E_INVALID;
  }
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    set_error("no CUDA device: the SAGE library has no CPU fallback");
    return SAGE_E_UNSUPPORTED;
  }
  const uint32_t flags = in->flags;
  const bool devptrs = flags & SAGE_F_DEVICE_PTRS;
  const bool borrow = devptrs && (flags & SAGE_F_BORROW);
  int64_t v_begin = 0, v_end = in->n;
  const sage_dist *ds = in->dist;
  if (ds) {
    if (ds->world < 1 || ds->rank < 0 || ds->rank >= ds->world || !ds->nccl_unique_id || ds->v_begin < 0 ||
        ds->v_end < ds->v_begin || ds->v_end > in->n) {
      set_error("invalid sage_dist");
      return SAGE_E_INVALID;
    }
    v_begin = ds->v_begin;
    v_end = ds->v_end;
  }
  const int64_t n_local = v_end - v_begin;

  sage_graph *g = new sage_graph();
  g->n = in->n;
  g->n_local = n_local;
  g->v_begin = v_begin;
  g->v_end = v_end;
  g->m = in->m;
  g->flags = flags;
  cudaGetDevice(&g->device);
  cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device);
  if (in->cuda_stream) {
    g->stream = (cudaStream_t)in->cuda_stream;
  } else {
    cudaStreamCreateWithFlags(&g->stream, cudaStreamNonBlocking);
    g->own_stream = true;
    if (devptrs) {
      // device inputs were produced on the caller's (legacy default) stream: order the copy,
      // the validation pass and every later read of borrowed arrays after that work
      cudaEvent_t ev;
      if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) == cudaSuccess) {
        cudaEventRecord(ev, cudaStreamLegacy);
        cudaStreamWaitEvent(g->stream, ev, 0);
        cudaEventDestroy(ev);
      }
    }
  }
  sage_status st = make_ladder(in->opts, g);
  if (st != SAGE_OK) {
    destroy(g);
    return st;
  }

  // host-side checks that need no device pass
  if (!devptrs) {
    if (in->row_offsets[0] != 0 || in->row_offsets[n_local] != in->m) {
      set_error("row_offsets[0] must be 0 and row_offsets[n_local] must equal m");
      destroy(g);
      return SAGE_E_INVALID;
    }
  }

  // copy or borrow
  const size_t offb = sizeof(int64_t) * (size_t)(n_local + 1);
  const size_t colb = sizeof(int32_t) * (size_t)in->m;
  if (flags & SAGE_F_HOST_COLUMNS) {
    // out-of-core (NEXT #4): columns / weights stay in pinned host memory and the
    // kernels read them zero-copy over PCIe / C2C; offsets and all per-vertex state are on the GPU
    if (devptrs) {
      set_error("SAGE_F_HOST_COLUMNS needs host input arrays");
      destroy(g);
      return SAGE_E_INVALID;
    }
    if ((st = dalloc(g, (void **)&g->off, offb)) != SAGE_OK) {
      destroy(g);
      return st;
    }
    g->own_off = true;
    cudaMemcpyAsync(g->off, in->row_offsets, offb, cudaMemcpyHostToDevice, g->stream);
    const void *hsrc[2] = {in->col_indices, in->weights};
    for (int i = 0; i < 2; ++i) {
      if (!hsrc[i] || !colb) continue;
      void *h = nullptr;
      cudaError_t e;
      if (flags & SAGE_F_BORROW) {   // register the caller's pages in place
        h = const_cast<void *>(hsrc[i]);
        e = cudaHostRegister(h, colb, cudaHostRegisterMapped | cudaHostRegisterReadOnly);
        if (e == cudaSuccess) g->host_registered[i] = h;
      } else {                       // library-owned pinned copy
        e = cudaHostAlloc(&h, colb + 16, cudaHostAllocMapped);
        if (e == cudaSuccess) {
          g->host_owned[i] = h;
          memcpy(h, hsrc[i], colb);
        }
      }
      void *d = nullptr;
      if (e == cudaSuccess) e = cudaHostGetDevicePointer(&d, h, 0);
      if (e != cudaSuccess) {
        cuda_fail(nullptr, e, "host-resident columns");
        destroy(g);
        return SAGE_E_CUDA;
      }
      if (i == 0) g->col = (int32_t *)d;
      else g->w = (uint32_t *)d;
    }
    g->host_columns = true;
  } else if (borrow) {
    g->off = const_cast<int64_t *>(in->row_offsets);
    g->col = const_cast<int32_t *>(in->col_indices);
    g->w = const_cast<uint32_t *>(in->weights);
  } else {
    if ((st = dalloc(g, (void **)&g->off, offb)) != SAGE_OK ||
        (st = dalloc(g, (void **)&g->col, colb + 16)) != SAGE_OK) {
      destroy(g);
      return st;
    }
    g->own_off = g->own_col = true;
    if (in->weights) {
      if ((st = dalloc(g, (void **)&g->w, colb + 16)) != SAGE_OK) {
        destroy(g);
        return st;
      }
      g->own_w = true;
    }
    cudaMemcpyKind kind = devptrs ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
    cudaError_t e = cudaMemcpyAsync(g->off, in->row_offsets, offb, kind, g->stream);
    if (e == cudaSuccess && colb)
      e = cudaMemcpyAsync(g->col, in->col_indices, colb, kind, g->stream);
    if (e == cudaSuccess && in->weights && colb)
      e = cudaMemcpyAsync(g->w, in->weights, colb, kind, g->stream);
    if (e != cudaSuccess) {
      cuda_fail(nullptr, e, "CSR copy");
      destroy(g);
      return SAGE_E_CUDA;
    }
  }
  g->vec = g->ladder.M >= 4 ? 4 : 1;   // neighbours per lane per step (tiles of >= 4 elements)
  g->vec_ok = g->vec == 4 && g->ladder.A >= 4 && ((uintptr_t)g->col % 16) == 0 &&
              (!g->w || ((uintptr_t)g->w % 16) == 0);

  // validation + stats pass
  {
    ValidateOut *vo = nullptr;
    uint32_t *rowstart = nullptr;
    if ((st = dalloc(g, (void **)&vo, sizeof(ValidateOut))) != SAGE_OK) {
      destroy(g);
      return st;
    }
    cudaMemsetAsync(vo, 0, sizeof(ValidateOut), g->stream);
    const bool validate = !(flags & SAGE_F_NO_VALIDATE);
    if (validate && in->m > 0) {
      size_t rsb = sizeof(uint32_t) * (size_t)((in->m + 32) / 32 + 1);
      if ((st = dalloc(g, (void **)&rowstart, rsb)) != SAGE_OK) {
        dfree(g, vo);
        destroy(g);
        return st;
      }
      cudaMemsetAsync(rowstart, 0, rsb, g->stream);
    }
    int grid = g->num_sms * 8;
    k_validate_rows<<<grid, 256, 0, g->stream>>>((const long long *)g->off, n_local, in->m,
                                                 rowstart, vo);
    if (validate && in->m > 0)
      k_validate_arcs<<<grid, 256, 0, g->stream>>>(g->col, g->w, in->m, in->n, rowstart, vo);
    ValidateOut h{};
    long long first = -1, last = -1;
    cudaMemcpyAsync(&h, vo, sizeof(h), cudaMemcpyDeviceToHost, g->stream);
    cudaMemcpyAsync(&first, g->off, 8, cudaMemcpyDeviceToHost, g->stream);
    cudaMemcpyAsync(&last, g->off + n_local, 8, cudaMemcpyDeviceToHost, g->stream);
    cudaError_t e = cudaStreamSynchronize(g->stream);
    dfree(g, vo);
    dfree(g, rowstart);
    if (e == cudaSuccess) e = cudaGetLastError();
    if (e != cudaSuccess) {
      cuda_fail(nullptr, e, "validation");
      destroy(g);
      return SAGE_E_CUDA;
    }
    if (validate) {
      if (first != 0 || last != in->m || h.bad_off) {
        set_error("row_offsets invalid (off[0]=%lld off[n]=%lld m=%lld, %llu bad rows)", first,
                  last, (long long)in->m, h.bad_off);
        destroy(g);
        return SAGE_E_INVALID;
      }
      if (h.bad_col) {
        set_error("%llu column indices out of [0, n)", h.bad_col);
        destroy(g);
        return SAGE_E_INVALID;
      }
      if (h.bad_w) {
        set_error("%llu weights are 0 (weights must be >= 1)", h.bad_w);
        destroy(g);
        return SAGE_E_INVALID;
      }
      g->rows_sorted = h.unsorted == 0;
    }
    g->max_degree = (int64_t)h.max_deg;
    g->n_isolated = (int64_t)h.isolated;
  }
  if (ds) {
    st = init_comm(g, ds);
    if (st != SAGE_OK) {
      destroy(g);
      return st;
    }
  }
  *out = g;
  return SAGE_OK;
}

sage_status sage_free(sage_graph *g) {
  clear_error();
  destroy(g);
  return SAGE_OK;
}

sage_status sage_graph_info(const sage_graph *g, int64_t *n, int64_t *m, int64_t *n_local,
                            int64_t *v_begin, uint32_t *flags) {
  if (!g) {
    set_error("graph is NULL");
    return SAGE_E_INVALID;
  }
  if (n) *n = g->n;
  if (m) *m = g->m;
  if (n_local) *n_local = g->n_local;
  if (v_begin) *v_begin = g->v_begin;
  if (flags) *flags = g->flags | (g->rows_sorted ? 0x100u : 0u) | (g->reordered ? 0x200u : 0u) |
                    (comm_peer_exchange(g) ? 0x400u : 0u) | (g->pr.win == 1 ? 0x800u : 0u);
  return SAGE_OK;
}

sage_status sage_get_permutation(const sage_graph *gc, int32_t *new_id_of_old) {
  clear_error();
  sage_graph *g = const_cast<sage_graph *>(gc);
  if (!g || !new_id_of_old) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  if (g->sigma) {
    sage_status st = copy_out(g, new_id_of_old, g->sigma, sizeof(int32_t) * (size_t)g->n);
    if (st != SAGE_OK) return st;
  } else {
    if (is_device_ptr(new_id_of_old)) {
      iota_device(g, new_id_of_old, g->n);
    } else {
      cudaStreamSynchronize(g->stream);
      for (int64_t i = 0; i < g->n; ++i) new_id_of_old[i] = (int32_t)i;
    }
  }
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "get_permutation");
  return SAGE_OK;
}

sage_status sage_get_csr(const sage_graph *gc, int64_t *off_out, int32_t *col_out,
                         uint32_t *w_out) {
  clear_error();
  sage_graph *g = const_cast<sage_graph *>(gc);
  if (!g || !off_out || (g->m > 0 && !col_out)) {
    set_error("null argument");
    return SAGE_E_INVALID;
  }
  if (g->sticky) return (sage_status)g->sticky;
  sage_status st = copy_out(g, off_out, g->off, sizeof(int64_t) * (size_t)(g->n_local + 1));
  if (st == SAGE_OK) st = copy_out(g, col_out, g->col, sizeof(int32_t) * (size_t)g->m);
  if (st == SAGE_OK && w_out && g->w) st = copy_out(g, w_out, g->w, sizeof(uint32_t) * (size_t)g->m);
  if (st != SAGE_OK) return st;
  cudaError_t e = cudaStreamSynchronize(g->stream);
  if (e != cudaSuccess) return cuda_fail(g, e, "get_csr");
  return SAGE_OK;
}

}  // extern "C"
