// Microbenchmark: throughput of scattered 4-B status reads on B200 from (a) global memory
// (2 MB array, L2 resident), (b) distributed shared memory of a 16-CTA cluster (128 KB per CTA),
// (c) the CTA's own shared memory.  Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cooperative_groups.h>
#include <cstdio>
#include <cstdint>
namespace cg = cooperative_groups;

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
constexpr int ITER = 256;

__global__ void k_global(const uint32_t *__restrict__ bm, uint32_t words, uint32_t *out) {
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < ITER; ++i) {
    x = hsh(x + i);
    s += bm[x & (words - 1)];
  }
  if (s == 0x12345678) out[0] = s;
}

__global__ void __cluster_dims__(16, 1, 1) k_dsmem(uint32_t words_per_cta, uint32_t *out) {
  extern __shared__ uint32_t sm[];
  cg::cluster_group cl = cg::this_cluster();
  for (uint32_t i = threadIdx.x; i < words_per_cta; i += blockDim.x) sm[i] = i * 2654435761u;
  cl.sync();
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < ITER; ++i) {
    x = hsh(x + i);
    uint32_t r = (x >> 24) & 15, w = x & (words_per_cta - 1);
    const uint32_t *p = cl.map_shared_rank(sm, r);
    s += p[w];
  }
  cl.sync();
  if (s == 0x12345678) out[0] = s;
}

__global__ void k_smem(uint32_t words_per_cta, uint32_t *out) {
  extern __shared__ uint32_t sm[];
  for (uint32_t i = threadIdx.x; i < words_per_cta; i += blockDim.x) sm[i] = i * 2654435761u;
  __syncthreads();
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
#pragma unroll 8
  for (int i = 0; i < ITER; ++i) {
    x = hsh(x + i);
    s += sm[x & (words_per_cta - 1)];
  }
  if (s == 0x12345678) out[0] = s;
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t *bm, *out;
  const uint32_t words = 1u << 19;  // 2 MB
  cudaMalloc(&bm, words * 4); cudaMemset(bm, 1, words * 4); cudaMalloc(&out, 64);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms;
  // (a) global, 8 CTAs x 256 per SM
  for (int rep = 0; rep < 2; ++rep) {
    int grid = sms * 8, blk = 256;
    cudaEventRecord(a); k_global<<<grid, blk>>>(bm, words, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    double loads = (double)grid * blk * ITER;
    printf("global  2MB: %.1f Gloads/s  (%.3f loads/cycle/SM @1.965GHz)\n", loads / ms / 1e6, loads / (ms * 1e-3) / sms / 1.965e9);
  }
  // (b) DSMEM cluster 16, 128 KB per CTA, 1 CTA per SM of 1024 threads
  uint32_t wpc = 32768;  // 128 KB
  cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeMaxDynamicSharedMemorySize, wpc * 4);
  cudaFuncSetAttribute(k_dsmem, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int rep = 0; rep < 2; ++rep) {
    int grid = (sms / 16) * 16, blk = 1024;
    cudaEventRecord(a); k_dsmem<<<grid, blk, wpc * 4>>>(wpc, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaError_t e = cudaGetLastError();
    cudaEventElapsedTime(&ms, a, b);
    double loads = (double)grid * blk * ITER;
    printf("dsmem c16  : %.1f Gloads/s  (%.3f loads/cycle/SM) err=%s\n", loads / ms / 1e6, loads / (ms * 1e-3) / grid / 1.965e9, cudaGetErrorString(e));
  }
  cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, wpc * 4);
  for (int rep = 0; rep < 2; ++rep) {
    int grid = sms, blk = 1024;
    cudaEventRecord(a); k_smem<<<grid, blk, wpc * 4>>>(wpc, out); cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
    double loads = (double)grid * blk * ITER;
    printf("smem local : %.1f Gloads/s  (%.3f loads/cycle/SM)\n", loads / ms / 1e6, loads / (ms * 1e-3) / sms / 1.965e9);
  }
  return 0;
}
