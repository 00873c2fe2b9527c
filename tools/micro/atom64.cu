// Microbenchmark: random 64-bit atomic adds without return (fp64 vs u64) on an L2-resident (2 MB)
// and a DRAM-resident (512 MB) array: is an integer (fixed-point) accumulation faster at L2?
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o atom64 atom64.cu
#include <cstdio>
#include <cstdint>
#include <cstdlib>

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
constexpr int ITER = 64;
template <int OP, int K>
__global__ void k_op(void *buf, uint32_t mask, int local) {
  uint32_t x = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t base = x * 64;
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int k = 0; k < K; ++k) {
      x = hsh(x + k);
      const uint32_t idx = local ? ((base + (x & 63)) & mask) : (x & mask);
      if (OP == 0) atomicAdd(static_cast<double *>(buf) + idx, 1.0);
      if (OP == 1) atomicAdd(static_cast<unsigned long long *>(buf) + idx, 1ull);
      if (OP == 2) asm volatile("red.global.add.u64 [%0], %1;" ::"l"(static_cast<unsigned long long *>(buf) + idx), "l"(1ull));
    }
  }
}
template <int OP, int K>
void run(void *buf, uint32_t words, int sms, int local, const char *what) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a);
    k_op<OP, K><<<sms * 2, 1024>>>(buf, words - 1, local);
    cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
  }
  double ops = (double)sms * 2 * 1024 * ITER * K;
  printf("%-34s op %d (0 f64 atomicAdd, 1 u64 atomicAdd, 2 red.add.u64): %7.1f Gops/s  (%s)\n", what, OP, ops / ms / 1e6,
         cudaGetErrorString(cudaGetLastError()));
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  void *buf;
  const uint32_t big = 1u << 26;   // 512 MB of 8-byte words
  cudaMalloc(&buf, (size_t)big * 8); cudaMemset(buf, 0, (size_t)big * 8);
  if (getenv("SIZE_SWEEP")) {   // footprint sweep: 2, 8, 16, 32, 64, 128 MB (fp64 atomicAdd = REDG when unused)
    const char *names[] = {"2 MB", "8 MB", "16 MB", "32 MB", "64 MB", "128 MB", "512 MB"};
    int i = 0;
    for (uint32_t words : {1u << 18, 1u << 20, 1u << 21, 1u << 22, 1u << 23, 1u << 24, big}) run<0, 4>(buf, words, sms, 0, names[i++]);
    return 0;
  }
  for (uint32_t words : {1u << 18, big}) {
    const char *w = words == big ? "512 MB random" : "2 MB random";
    run<0, 4>(buf, words, sms, 0, w); run<1, 4>(buf, words, sms, 0, w); run<2, 4>(buf, words, sms, 0, w);
  }
  run<0, 4>(buf, big, sms, 1, "512 MB, 64-word windows per thread");
  run<1, 4>(buf, big, sms, 1, "512 MB, 64-word windows per thread");
  return 0;
}
