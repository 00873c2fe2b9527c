// Microbenchmark: scattered 32-bit atomicOr (with return) on an L2-resident 2 MB array vs plain
// scattered loads, at two L1 sizes (does an in-flight atomic hold an L1 line like a load miss?).
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o atom_mlp atom_mlp.cu
#include <cstdio>
#include <cstdint>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
constexpr int ITER = 64;
template <int OP, int K>
__global__ void k_op(uint32_t *bm, uint32_t mask, uint32_t *out) {
  extern __shared__ uint32_t pad[];
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
  for (int i = 0; i < ITER; ++i) {
    uint32_t v[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      x = hsh(x + k);
      uint32_t *p = bm + (x & mask);
      if (OP == 0) asm volatile("ld.global.u32 %0, [%1];" : "=r"(v[k]) : "l"(p));
      if (OP == 1) v[k] = atomicOr(p, 1u << (x >> 27));
      if (OP == 2) { asm volatile("red.global.or.b32 [%0], %1;" ::"l"(p), "r"(1u << (x >> 27))); v[k] = 0; }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) s += v[k];
  }
  if (s == 0x12345678) { out[0] = s; pad[0] = s; }
}
template <int OP, int K>
void run(uint32_t *bm, uint32_t words, uint32_t *out, int sms, int dyn_kb) {
  auto fn = k_op<OP, K>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn_kb * 1024);
  const int pct = dyn_kb == 0 ? 0 : (int)(((dyn_kb + 1) * 100 + 227) / 228);
  cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, pct > 100 ? 100 : pct);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a);
    fn<<<sms, 1024, dyn_kb * 1024>>>(bm, words - 1, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
  }
  double ops = (double)sms * 1024 * ITER * K;
  printf("op %d (0 ld, 1 atom.or, 2 red.or) K %d dyn %3d KB: %6.1f Gops/s = %.3f /SM-cycle  (%s)\n", OP, K, dyn_kb,
         ops / ms / 1e6, ops / (ms * 1e-3) / sms / 1.965e9, cudaGetErrorString(cudaGetLastError()));
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t *bm, *out;
  const uint32_t words = 1u << 19;
  cudaMalloc(&bm, words * 4); cudaMemset(bm, 0, words * 4); cudaMalloc(&out, 64);
  for (int dyn : {0, 112, 208}) {
    run<0, 4>(bm, words, out, sms, dyn);
    run<1, 4>(bm, words, out, sms, dyn);
    run<2, 4>(bm, words, out, sms, dyn);
    run<1, 8>(bm, words, out, sms, dyn);
  }
  // small array (hot words): 4 KB
  run<1, 4>(bm, 1024, out, sms, 0);
  run<0, 4>(bm, 1024, out, sms, 0);
  return 0;
}
