// Microbenchmark: same-address 64-bit atomicAdd WITH return (queue reservation) from many warps on
// B200, vs. per-warp distinct addresses.  Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a
#include <cstdio>
#include <cstdint>
__global__ void k_same(unsigned long long *ctr, int iters, int stride, unsigned long long *sink) {
  if ((threadIdx.x & 31) != 0) return;
  const int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  unsigned long long acc = 0;
  unsigned long long *p = ctr + (long long)(w % 8) * stride;   // 8 counters, `stride` u64 apart
  for (int i = 0; i < iters; ++i) acc += atomicAdd(p, 1ull + (acc & 1));
  if (acc == 12345) sink[0] = acc;
}
int main() {
  unsigned long long *ctr, *sink;
  cudaMalloc(&ctr, 1 << 20); cudaMalloc(&sink, 64);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  int grids[] = {50, 148, 592};
  for (int stride : {0, 16}) for (int gsz : grids) {
    int iters = 64;
    cudaMemset(ctr, 0, 1 << 20);
    k_same<<<gsz, 256>>>(ctr, iters, stride, sink);
    cudaEventRecord(a);
    k_same<<<gsz, 256>>>(ctr, iters, stride, sink);
    cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    double ops = (double)gsz * 8 * iters;
    printf("stride %2d grid %4d: %.1f us, %.2f ns per atomic (all warps), %.1f ns per atomic per counter\n",
           stride, gsz, ms * 1e3, ms * 1e6 / ops, ms * 1e6 / (ops / (stride ? 8 : 1)));
  }
  return 0;
}
