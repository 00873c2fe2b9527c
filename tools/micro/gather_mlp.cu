// Microbenchmark: scattered 4-B loads from an L2-resident array (2 MB, like C2's visited bitmap)
// vs L1 size (unused dynamic shared memory per CTA shrinks L1), load flavour and loads in flight.
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o gather_mlp gather_mlp.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
template <int FL>
__device__ __forceinline__ uint32_t ld(const uint32_t *p) {
  uint32_t r;
  if (FL == 0) asm volatile("ld.global.u32 %0, [%1];" : "=r"(r) : "l"(p));
  if (FL == 1) asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(r) : "l"(p));
  if (FL == 2) asm volatile("ld.global.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  if (FL == 3) asm volatile("ld.global.L1::evict_last.u32 %0, [%1];" : "=r"(r) : "l"(p));
  if (FL == 4) asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
constexpr int ITER = 128;
template <int FL, int K>
__global__ void k_gather(const uint32_t *__restrict__ bm, uint32_t mask, uint32_t *out) {
  extern __shared__ uint32_t pad[];
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
  for (int i = 0; i < ITER; ++i) {
    uint32_t v[K];
#pragma unroll
    for (int k = 0; k < K; ++k) { x = hsh(x + k); v[k] = ld<FL>(bm + (x & mask)); }
#pragma unroll
    for (int k = 0; k < K; ++k) s += v[k];
  }
  if (s == 0x12345678) { out[0] = s; pad[0] = s; }
}

template <int FL, int K>
void run(const uint32_t *bm, uint32_t words, uint32_t *out, int sms, int blk, int cps, int dyn_kb) {
  auto fn = k_gather<FL, K>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn_kb * 1024);
  // smallest carveout that holds the dynamic shared memory (+1 KB reserved): L1 = 256 KB - carveout
  const int pct = dyn_kb == 0 ? 0 : (int)(((dyn_kb + 1) * 100 + 227) / 228);
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct > 100 ? 100 : pct);
  int nb = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, fn, blk, dyn_kb * 1024);
  int use = cps < nb ? cps : nb;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a);
    fn<<<sms * use, blk, dyn_kb * 1024>>>(bm, words - 1, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
  }
  double loads = (double)sms * use * blk * ITER * K;
  printf("flavour %d K %2d blk %4d ctas/sm %d dyn %3d KB: %6.1f Gloads/s = %.3f /SM-cycle @1.965  (%s)\n", FL, K,
         blk, use, dyn_kb, loads / ms / 1e6, loads / (ms * 1e-3) / sms / 1.965e9,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t *bm, *out;
  const uint32_t words = 1u << 19;  // 2 MB
  cudaMalloc(&bm, words * 4); cudaMemset(bm, 1, words * 4); cudaMalloc(&out, 64);
  if (getenv("MLP_SWEEP")) {   // loads in flight per thread at the fused BFS's L1 (64 KB table + 35 KB static)
    run<3, 1>(bm, words, out, sms, 1024, 1, 100);
    run<3, 2>(bm, words, out, sms, 1024, 1, 100);
    run<3, 4>(bm, words, out, sms, 1024, 1, 100);
    run<3, 8>(bm, words, out, sms, 1024, 1, 100);
    run<3, 16>(bm, words, out, sms, 1024, 1, 100);
    run<3, 4>(bm, words, out, sms, 512, 2, 100);
    return 0;
  }
  for (int dyn : {0, 16, 48, 80, 112, 144, 176, 208}) {
    run<0, 8>(bm, words, out, sms, 1024, 1, dyn);
    run<3, 8>(bm, words, out, sms, 1024, 1, dyn);
  }
  // 256-thread CTAs, 4 per SM (the k_bfs configuration)
  run<0, 4>(bm, words, out, sms, 256, 4, 0);
  run<3, 4>(bm, words, out, sms, 256, 4, 0);
  run<0, 8>(bm, words, out, sms, 256, 4, 0);
  return 0;
}
