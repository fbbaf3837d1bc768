// Microbenchmark: tcgen05.mma issue rate with operands resident in shared
// memory (no TMA), one CTA per SM, all 148 SMs busy.  Measures the cycles of
// one "k-block" (4 MMAs of K = 16 + one commit) for the engine's operand
// layouts: A K-major or MN-major, B K-major or MN-major, N = 256 / 128.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_eurosys_ohlks22_b200/csrc \
//        -o tools/mma_probe tools/mma_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <stdint.h>

#include "tc_common.cuh"

using namespace ooo::tc;

__global__ void __launch_bounds__(128, 1) probe(int iters, int bn, int a_mn, int b_mn, int wait_each,
                                                long long *out, int bm) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t sa = smem_u32(smem), sb = sa + 16384, bar = sa + 16384 + 32768;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tslot)),
                 "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = tslot;
  if (threadIdx.x == 0) {
    const uint32_t ID = (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) | ((b_mn ? 1u : 0u) << 16) |
                        ((uint32_t)(bn >> 3) << 17) | ((uint32_t)(bm >> 4) << 24);
    long long t0 = clock64();
    uint32_t ph = 0;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const uint64_t ad = a_mn ? sdesc(sa + kk * 2048, 8192, 1024) : sdesc(sa + kk * 32, 16, 1024);
        const uint64_t bd = b_mn ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
        umma_bf16(tmem + (uint32_t)((it & 1) * 256), ad, bd, ID, (it | kk) != 0 ? 1u : 0u);
      }
      if (wait_each || it == iters - 1) {
        umma_commit(bar);
        while (!mbar_try_wait(bar, ph)) {
        }
        ph ^= 1;
      }
    }
    long long t1 = clock64();
    out[blockIdx.x] = (t1 - t0);
  }
  fence_before();
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
}

int main() {
  long long *d;
  cudaMalloc(&d, 148 * 8);
  const int smem = 16384 + 32768 + 64 + 1024;
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 4000;
  struct C { int bn, a_mn, b_mn, wait, bm; const char *name; } cs[] = {
      {256, 0, 1, 0, 128, "F   (A K-major, B MN-major) N=256"},
      {256, 0, 0, 0, 128, "dO  (A K-major, B K-major)  N=256"},
      {256, 1, 1, 0, 128, "dW  (A MN-major, B MN-major) N=256"},
      {128, 0, 1, 0, 128, "F   N=128"},
      {64, 0, 1, 0, 128, "F   N=64"},
      {64, 0, 0, 0, 128, "dO  N=64"},
      {32, 0, 0, 0, 128, "dO  N=32"},
      {256, 0, 0, 0, 64, "dO  M=64 N=256"},
      {64, 0, 0, 0, 64, "dO  M=64 N=64"},
      {64, 0, 1, 0, 64, "F   M=64 N=64"},
      {256, 0, 1, 1, 128, "F   N=256, commit+wait each k-block"},
      {64, 0, 1, 1, 128, "F   N=64, commit+wait each k-block"},
  };
  for (auto &c : cs) {
    probe<<<148, 128, smem>>>(iters, c.bn, c.a_mn, c.b_mn, c.wait, d, c.bm);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double m = 0;
    for (int i = 0; i < 148; ++i) m += h[i];
    m /= 148;
    const double flop = 2.0 * c.bm * c.bn * 64;   // per k-block per SM
    printf("%-40s %7.1f cycles per 64-deep k-block (%s); ideal %5.0f at 8192 FLOP/clk/SM\n", c.name, m / iters,
           cudaGetErrorString(e), flop / 8192);
  }
  return 0;
}
