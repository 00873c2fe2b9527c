// Microbenchmark: scattered 4-B loads from a bitmap replicated across a thread-block cluster's
// distributed shared memory (each CTA holds 1/CS of it) vs the same loads from an L2-resident
// global array.  Question: can a cluster-resident copy of the visited bitmap (2 MB at C2) serve
// the push filter's status reads faster than L1/L2 (~1 load per SM-cycle, gather_mlp.cu)?
// Build: nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o dsmem_gather dsmem_gather.cu
#include <cstdio>
#include <cstdint>
#include <cooperative_groups.h>
namespace cg = cooperative_groups;

__device__ __forceinline__ uint32_t hsh(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16; return x;
}
constexpr int ITER = 128;

// MODE 0: DSMEM random (rank = x % CS), 1: own smem only, 2: global (L2-resident 2 MB)
template <int MODE, int K>
__global__ void k_gather(const uint32_t *__restrict__ bm, uint32_t words_per_cta, int cs, uint32_t *out) {
  extern __shared__ uint32_t sm[];
  for (uint32_t i = threadIdx.x; i < words_per_cta; i += blockDim.x) sm[i] = hsh(i) | 1u;
  if (MODE == 0) cg::this_cluster().sync(); else __syncthreads();
  const uint32_t base = (uint32_t)__cvta_generic_to_shared(sm);
  uint32_t s = 0, x = blockIdx.x * blockDim.x + threadIdx.x;
  const uint32_t wmask = words_per_cta - 1;
  for (int i = 0; i < ITER; ++i) {
    uint32_t v[K];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      x = hsh(x + k);
      if (MODE == 0) {
        const uint32_t rank = (x >> 24) % (uint32_t)cs, la = base + 4u * (x & wmask);
        uint32_t ra;
        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(la), "r"(rank));
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v[k]) : "r"(ra));
      } else if (MODE == 1) {
        asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v[k]) : "r"(base + 4u * (x & wmask)));
      } else {
        v[k] = __ldcg(bm + (x & ((1u << 19) - 1u)));
      }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) s += v[k];
  }
  if (MODE == 0) cg::this_cluster().sync();
  if (s == 0x12345678) out[0] = s;
}

template <int MODE, int K>
void run(const uint32_t *bm, uint32_t *out, int sms, int blk, int cs, int kb) {
  auto fn = k_gather<MODE, K>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kb * 1024);
  if (cs > 8) cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = MODE == 0 ? cs : 1;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.blockDim = dim3(blk);
  cfg.dynamicSmemBytes = kb * 1024;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int ncl = 0;
  cfg.gridDim = dim3(cs * 64);
  cudaOccupancyMaxActiveClusters(&ncl, fn, &cfg);
  int nctas = MODE == 0 ? ncl * cs : sms;
  if (MODE != 0) ncl = sms;
  cfg.gridDim = dim3(nctas);
  const uint32_t wpc = (uint32_t)(kb * 1024 / 4);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  float ms = 0;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a);
    cudaLaunchKernelEx(&cfg, fn, bm, wpc, cs, out);
    cudaEventRecord(b); cudaEventSynchronize(b);
    cudaEventElapsedTime(&ms, a, b);
  }
  double loads = (double)nctas * blk * ITER * K;
  printf("mode %d K %2d blk %4d cluster %2d smem %3d KB: active clusters %3d (%3d CTAs): %7.1f Gloads/s = %.3f /SM-cycle (%s)\n",
         MODE, K, blk, cs, kb, ncl, nctas, loads / ms / 1e6, loads / (ms * 1e-3) / nctas / 1.965e9,
         cudaGetErrorString(cudaGetLastError()));
}

int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint32_t *bm, *out;
  cudaMalloc(&bm, 4u << 19); cudaMemset(bm, 1, 4u << 19); cudaMalloc(&out, 64);
  run<2, 8>(bm, out, sms, 1024, 1, 0);
  run<1, 8>(bm, out, sms, 1024, 1, 128);
  for (int cs : {2, 4, 8, 16})
    for (int kb : {64, 128}) {
      run<0, 4>(bm, out, sms, 1024, cs, kb);
      run<0, 8>(bm, out, sms, 1024, cs, kb);
    }
  run<0, 8>(bm, out, sms, 512, 16, 128);
  run<0, 16>(bm, out, sms, 1024, 16, 128);
  return 0;
}
