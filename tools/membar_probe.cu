// Microbenchmark: cost of a release (fence.acq_rel.gpu / red.release.gpu /
// mbarrier.arrive.release.cluster) against its relaxed form, issued by one
// thread while the other warps of the CTA stream global stores (and, mode 5,
// after the thread's own 16 stores).  DESIGN.md §8, profiles/r02_membar_probe.log.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/membar_probe tools/membar_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void probe(uint4 *buf, size_t per_warp, int *flag, long long *out, int mode, int storers) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  __shared__ volatile int stop;
  if (threadIdx.x == 0) stop = 0;
  __syncthreads();
  if (warp == 0) {
    if (lane == 0) {
      __shared__ __align__(8) unsigned long long bar;
      const uint32_t ba = (uint32_t)__cvta_generic_to_shared(&bar);
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(ba), "r"((1 << 20) - 1) : "memory");
      uint32_t bc;
      asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(bc) : "r"(ba));
      uint4 *own = buf + (size_t)blockIdx.x * 32 * per_warp;
      long long acc = 0;
      for (int i = 0; i < 64; ++i) {
        if (mode == 5)
          for (int j = 0; j < 16; ++j) own[(i * 16 + j) % per_warp] = make_uint4(i, j, i, j);
        long long t0 = clock64();
        if (mode == 0 || mode == 5) asm volatile("fence.acq_rel.gpu;" ::: "memory");
        else if (mode == 1) asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(flag + blockIdx.x) : "memory");
        else if (mode == 2) asm volatile("red.relaxed.gpu.global.add.s32 [%0], 1;" ::"l"(flag + blockIdx.x) : "memory");
        else if (mode == 3) asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(bc) : "memory");
        else asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(bc) : "memory");
        long long t1 = clock64();
        acc += t1 - t0;
        __nanosleep(200);
      }
      out[blockIdx.x] = acc / 64;
      stop = 1;
    }
  } else if (warp <= storers) {
    uint4 *p = buf + ((size_t)blockIdx.x * 32 + warp) * per_warp;
    size_t i = lane;
    while (!stop) {
      p[i % per_warp] = make_uint4(i, i, i, i);
      i += 32;
    }
  }
}

int main() {
  const int blocks = 148, threads = 256;
  const size_t per_warp = 1 << 16;   // 1 MiB per warp
  uint4 *buf; int *flag; long long *out;
  cudaMalloc(&buf, (size_t)blocks * 32 * per_warp * sizeof(uint4));
  cudaMalloc(&flag, blocks * 4);
  cudaMalloc(&out, blocks * 8);
  const char *names[6] = {"fence.acq_rel.gpu", "red.release.gpu", "red.relaxed.gpu",
                          "mbar.arrive.release.cluster", "mbar.arrive.relaxed.cluster", "own stores+fence.acq_rel"};
  for (int mode = 0; mode < 6; ++mode)
    for (int storers : {0, 7}) {
      probe<<<blocks, threads>>>(buf, per_warp, flag, out, mode, storers);
      cudaDeviceSynchronize();
      long long h[blocks];
      cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
      double m = 0; for (int b = 0; b < blocks; ++b) m += h[b]; m /= blocks;
      printf("%-28s storing warps %d : %8.0f cycles per op\n", names[mode], storers, m);
    }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
