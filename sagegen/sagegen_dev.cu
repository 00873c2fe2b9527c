// sagegen_dev.cu — per-rank DEVICE generation of the Graph500 Kronecker/RMAT inputs
// (TEST / BENCH INFRASTRUCTURE, like sagegen.cpp; holds none of SAGE's arithmetic).
//
// "Generated on device per rank: every rank regenerates all tuples and keeps
// arcs whose source it owns (count pass -> offsets -> fill pass -> segmented sort -> dedupe)."
// The tuple stream, the quadrant draws and the ID scramble are the SAME functions as sg_rmat in
// sagegen.cpp (counter-based splitmix64 keyed by (seed, tuple, level group)), so the rows
// [v_begin, v_end) produced here equal rows [v_begin, v_end) of sagegen.rmat(...) exactly
// (tests/test_gpu_sagegen_dev.py pins that at small scales).  Weights follow sg_weights.
//
// C ABI (device pointers, the caller's stream):
//   sgd_rmat_build(scale, ef, seed, A, B, C, symmetric, v_begin, v_end, stream, &handle, &m_local)
//   sgd_rmat_take(handle, off_out[n_local+1], col_out[m_local], stream)   (frees the handle)
//   sgd_weights(n_local, v_begin, off, col, seed, wmax, w_out, stream)
//   sgd_free(handle)
#include <cuda_runtime.h>
#include <stdint.h>

#include <cub/cub.cuh>
#include <thrust/iterator/transform_iterator.h>

namespace {

__device__ __forceinline__ uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__host__ __device__ __forceinline__ uint64_t hmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t hash3(uint64_t seed, uint64_t a, uint64_t b) {
  return mix64(mix64(seed ^ mix64(a + 0x632BE59BD9B4E019ull)) + b);
}

struct Perm {   // sg_perm_pow2's constants for (bits, seed)
  uint64_t mask, k1, k2, c1;
  int s1, s2;
};
static Perm make_perm(int bits, uint64_t seed) {
  Perm p;
  p.mask = (bits >= 64) ? ~0ull : ((1ull << bits) - 1);
  p.k1 = hmix64(seed ^ 0x1111) | 1ull;
  p.k2 = hmix64(seed ^ 0x2222) | 1ull;
  p.c1 = hmix64(seed ^ 0x3333);
  p.s1 = bits / 2 + 1;
  p.s2 = bits / 3 + 1;
  return p;
}
__device__ __forceinline__ uint64_t perm(uint64_t x, const Perm &p) {
  x = (x * p.k1) & p.mask;
  x ^= (x >> p.s1);
  x = (x * p.k2 + p.c1) & p.mask;
  x ^= (x >> p.s2);
  x = (x * p.k1) & p.mask;
  return x & p.mask;
}

struct Gen {
  int scale;
  long long t;          // tuples
  uint64_t seed;
  uint32_t tA, tAB, tABC;
  Perm pm;
  int symmetric;
  long long vb, ve;     // owned rows
};

__device__ __forceinline__ void tuple(const Gen &g, long long i, uint64_t &u, uint64_t &v) {
  u = 0;
  v = 0;
  for (int grp = 0; grp * 4 < g.scale; ++grp) {
    const uint64_t r = hash3(g.seed, (uint64_t)i, (uint64_t)grp);
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int l = grp * 4 + j;
      if (l >= g.scale) break;
      const uint32_t q = (uint32_t)((r >> (16 * j)) & 0xFFFF);
      const uint64_t ub = (q >= g.tAB) ? 1 : 0;
      const uint64_t vbit = ((q >= g.tA && q < g.tAB) || q >= g.tABC) ? 1 : 0;
      u |= ub << l;
      v |= vbit << l;
    }
  }
  u = perm(u, g.pm);
  v = perm(v, g.pm);
}

// pass 1: raw per-row arc counts of the owned rows (self-loops dropped, duplicates kept)
__global__ void k_count(Gen g, unsigned long long *cnt) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < g.t; i += stride) {
    uint64_t u, v;
    tuple(g, i, u, v);
    if (u == v) continue;
    if ((long long)u >= g.vb && (long long)u < g.ve) atomicAdd(cnt + (u - g.vb), 1ull);
    if (g.symmetric && (long long)v >= g.vb && (long long)v < g.ve) atomicAdd(cnt + (v - g.vb), 1ull);
  }
}
// pass 2: fill (cursor = a copy of the raw offsets)
__global__ void k_fill(Gen g, unsigned long long *cur, int *col) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < g.t; i += stride) {
    uint64_t u, v;
    tuple(g, i, u, v);
    if (u == v) continue;
    if ((long long)u >= g.vb && (long long)u < g.ve) col[atomicAdd(cur + (u - g.vb), 1ull)] = (int)v;
    if (g.symmetric && (long long)v >= g.vb && (long long)v < g.ve) col[atomicAdd(cur + (v - g.vb), 1ull)] = (int)u;
  }
}
// distinct entries per sorted row
__global__ void k_uniq_count(const long long *off, const int *col, long long n, long long *deg) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride) {
    long long d = 0;
    for (long long k = off[r]; k < off[r + 1]; ++k) d += (k == off[r] || col[k] != col[k - 1]);
    deg[r] = d;
  }
}
__global__ void k_uniq_copy(const long long *off0, const int *col0, const long long *off, int *col, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride) {
    long long o = off[r];
    for (long long k = off0[r]; k < off0[r + 1]; ++k)
      if (k == off0[r] || col0[k] != col0[k - 1]) col[o++] = col0[k];
  }
}
// bnd[k] = first row r with off[r] >= k * chunk (bnd[nb-1] = n)
__global__ void k_bounds(const long long *off, long long n, long long chunk, long long *bnd, long long nb) {
  const long long k = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= nb) return;
  if (k == nb - 1) {
    bnd[k] = n;
    return;
  }
  long long lo = 0, hi = n;   // first r in [0, n] with off[r] >= k * chunk
  while (lo < hi) {
    const long long mid = (lo + hi) >> 1;
    if (off[mid] >= k * chunk) hi = mid; else lo = mid + 1;
  }
  bnd[k] = lo;
}
struct Rel {   // offset relative to a chunk's first item
  long long base;
  __host__ __device__ __forceinline__ int operator()(long long x) const { return (int)(x - base); }
};
__global__ void k_u64_to_i64(const unsigned long long *a, long long *b, long long n) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) b[i] = (long long)a[i];
}
__global__ void k_weights(long long n, long long vb, const long long *off, const int *col, uint64_t seed,
                          uint32_t wmax, uint32_t *w) {
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long r = (long long)blockIdx.x * blockDim.x + threadIdx.x; r < n; r += stride)
    for (long long k = off[r]; k < off[r + 1]; ++k) {
      uint64_t a = (uint64_t)(r + vb), b = (uint64_t)col[k];
      if (a > b) {
        const uint64_t x = a;
        a = b;
        b = x;
      }
      w[k] = 1u + (uint32_t)(hash3(seed, a, b) % wmax);
    }
}

struct Handle {
  long long n = 0, m = 0;
  long long *off = nullptr;   // n + 1
  int *col = nullptr;         // m
};

int grid_for(cudaStream_t) {
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  return sms * 8;
}

}  // namespace

extern "C" {

int sgd_rmat_build(int scale, int edgefactor, uint64_t seed, double A, double B, double C, int symmetric,
                   long long v_begin, long long v_end, void *stream_p, void **handle_out, long long *m_out) {
  cudaStream_t st = (cudaStream_t)stream_p;
  if (scale < 1 || scale > 31 || v_begin < 0 || v_end < v_begin || v_end > (1ll << scale)) return 1;
  Gen g;
  g.scale = scale;
  g.t = (long long)edgefactor << scale;
  g.seed = seed;
  g.tA = (uint32_t)llround(A * 65536.0);
  g.tAB = (uint32_t)llround((A + B) * 65536.0);
  g.tABC = (uint32_t)llround((A + B + C) * 65536.0);
  g.pm = make_perm(scale, hmix64(seed ^ 0xABCDEF12345ull));
  g.symmetric = symmetric;
  g.vb = v_begin;
  g.ve = v_end;
  const long long n = v_end - v_begin;
  const int grid = grid_for(st);
  unsigned long long *cnt = nullptr, *cur = nullptr;
  long long *off0 = nullptr, *deg = nullptr;
  int *col0 = nullptr, *col1 = nullptr;
  Handle *h = new Handle();
  h->n = n;
  cudaError_t e = cudaMallocAsync((void **)&cnt, sizeof(unsigned long long) * (n + 1), st);
  if (e == cudaSuccess) e = cudaMemsetAsync(cnt, 0, sizeof(unsigned long long) * (n + 1), st);
  if (e == cudaSuccess) k_count<<<grid, 256, 0, st>>>(g, cnt);
  // exclusive scan -> raw offsets
  void *tmp = nullptr;
  size_t tb = 0;
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&cur, sizeof(unsigned long long) * (n + 1), st);
  if (e == cudaSuccess) cub::DeviceScan::ExclusiveSum(nullptr, tb, cnt, cur, n + 1, st);
  if (e == cudaSuccess) e = cudaMallocAsync(&tmp, tb, st);
  if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(tmp, tb, cnt, cur, n + 1, st);
  unsigned long long m0 = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&m0, cur + n, sizeof(m0), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&off0, sizeof(long long) * (n + 1), st);
  if (e == cudaSuccess) k_u64_to_i64<<<grid, 256, 0, st>>>(cur, off0, n + 1);
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&col0, sizeof(int) * (m0 + 1), st);
  if (e == cudaSuccess) k_fill<<<grid, 256, 0, st>>>(g, cur, col0);
  // sort every row; CUB takes int item / segment counts, so rows are sorted in chunks of at most
  // kChunk items (row boundaries found by binary search on the raw offsets)
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&col1, sizeof(int) * (m0 + 1), st);
  if (e == cudaSuccess) {
    constexpr long long kChunk = 1ll << 29;   // + one row of any realistic size < 2^31
    const long long nb = (long long)(m0 / kChunk) + 2;
    long long *bnd = nullptr;
    e = cudaMallocAsync((void **)&bnd, sizeof(long long) * nb, st);
    if (e == cudaSuccess) k_bounds<<<(int)((nb + 255) / 256), 256, 0, st>>>(off0, n, kChunk, bnd, nb);
    long long *hb = new long long[nb];
    if (e == cudaSuccess) e = cudaMemcpyAsync(hb, bnd, sizeof(long long) * nb, cudaMemcpyDeviceToHost, st);
    if (e == cudaSuccess) e = cudaStreamSynchronize(st);
    for (long long k = 0; e == cudaSuccess && k + 1 < nb; ++k) {
      const long long rb = hb[k], re = hb[k + 1];
      if (re <= rb) continue;
      long long ib = 0, ie = 0;
      cudaMemcpy(&ib, off0 + rb, sizeof(long long), cudaMemcpyDeviceToHost);
      cudaMemcpy(&ie, off0 + re, sizeof(long long), cudaMemcpyDeviceToHost);
      if (ie <= ib) continue;
      Rel rel{ib};
      auto obeg = thrust::make_transform_iterator(off0 + rb, rel);
      auto oend = thrust::make_transform_iterator(off0 + rb + 1, rel);
      void *t2 = nullptr;
      size_t b2 = 0;
      cub::DeviceSegmentedSort::SortKeys(nullptr, b2, col0 + ib, col1 + ib, (int)(ie - ib), (int)(re - rb), obeg, oend, st);
      e = cudaMallocAsync(&t2, b2, st);
      if (e == cudaSuccess)
        e = cub::DeviceSegmentedSort::SortKeys(t2, b2, col0 + ib, col1 + ib, (int)(ie - ib), (int)(re - rb), obeg, oend, st);
      cudaFreeAsync(t2, st);
    }
    delete[] hb;
    cudaFreeAsync(bnd, st);
  }
  // dedupe
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&deg, sizeof(long long) * (n + 1), st);
  if (e == cudaSuccess) e = cudaMemsetAsync(deg, 0, sizeof(long long) * (n + 1), st);
  if (e == cudaSuccess) k_uniq_count<<<grid, 256, 0, st>>>(off0, col1, n, deg);
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&h->off, sizeof(long long) * (n + 1), st);
  if (e == cudaSuccess) {
    void *t3 = nullptr;
    size_t b3 = 0;
    cub::DeviceScan::ExclusiveSum(nullptr, b3, deg, h->off, n + 1, st);
    e = cudaMallocAsync(&t3, b3, st);
    if (e == cudaSuccess) e = cub::DeviceScan::ExclusiveSum(t3, b3, deg, h->off, n + 1, st);
    cudaFreeAsync(t3, st);
  }
  long long m = 0;
  if (e == cudaSuccess) e = cudaMemcpyAsync(&m, h->off + n, sizeof(m), cudaMemcpyDeviceToHost, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess) e = cudaMallocAsync((void **)&h->col, sizeof(int) * (m + 1), st);
  if (e == cudaSuccess) k_uniq_copy<<<grid, 256, 0, st>>>(off0, col1, h->off, h->col, n);
  cudaFreeAsync(cnt, st);
  cudaFreeAsync(cur, st);
  cudaFreeAsync(tmp, st);
  cudaFreeAsync(off0, st);
  cudaFreeAsync(col0, st);
  cudaFreeAsync(col1, st);
  cudaFreeAsync(deg, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    cudaFreeAsync(h->off, st);
    cudaFreeAsync(h->col, st);
    delete h;
    return 2;
  }
  h->m = m;
  *handle_out = h;
  *m_out = m;
  return 0;
}

int sgd_rmat_take(void *handle, long long *off_out, int *col_out, void *stream_p) {
  cudaStream_t st = (cudaStream_t)stream_p;
  Handle *h = (Handle *)handle;
  cudaError_t e = cudaMemcpyAsync(off_out, h->off, sizeof(long long) * (h->n + 1), cudaMemcpyDeviceToDevice, st);
  if (e == cudaSuccess && h->m)
    e = cudaMemcpyAsync(col_out, h->col, sizeof(int) * h->m, cudaMemcpyDeviceToDevice, st);
  cudaFreeAsync(h->off, st);
  cudaFreeAsync(h->col, st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  delete h;
  return e == cudaSuccess ? 0 : 2;
}

void sgd_free(void *handle) {
  Handle *h = (Handle *)handle;
  if (!h) return;
  cudaFree(h->off);
  cudaFree(h->col);
  delete h;
}

int sgd_weights(long long n, long long v_begin, const long long *off, const int *col, uint64_t seed,
                uint32_t wmax, uint32_t *w, void *stream_p) {
  cudaStream_t st = (cudaStream_t)stream_p;
  k_weights<<<grid_for(st), 256, 0, st>>>(n, v_begin, off, col, seed, wmax, w);
  return cudaStreamSynchronize(st) == cudaSuccess ? 0 : 2;
}

}  // extern "C"
