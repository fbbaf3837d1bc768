// Microbenchmark: TMEM read-out throughput (tcgen05.ld) of one 128-lane x
// 256-column fp32 accumulator (128 KiB) per CTA, one CTA per SM, for
// different warp counts and load widths.  Prints cycles per accumulator.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_eurosys_ohlks22_b200/csrc \
//        -o tools/tmem_probe tools/tmem_probe.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <stdint.h>

#include "tc_common.cuh"

using namespace ooo::tc;

__device__ __forceinline__ void ld16(uint32_t a, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(a));
}
__device__ __forceinline__ void ldw() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// NW warps (multiple of 4); warp w reads lane quarter w & 3, columns split
// between the NW/4 warps of a quarter; W = columns per tcgen05.ld (16 or 32).
template <int NW, int W, int INFLIGHT>
__global__ void __launch_bounds__(NW * 32, 1) rd(int reps, long long *cyc, float *sink) {
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tslot)), "r"(256)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = tslot;
  const int q = warp & 3, h = warp >> 2;
  constexpr int PER = NW / 4;                 // warps per quarter
  constexpr int COLS = 256 / PER;             // columns per warp
  const uint32_t tb = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(h * COLS);
  float acc = 0.f;
  long long t0 = clock64();
  for (int r = 0; r < reps; ++r) {
    for (int c = 0; c < COLS; c += W * INFLIGHT) {
      if (W == 32) {
        uint32_t a[INFLIGHT][32];
#pragma unroll
        for (int f = 0; f < INFLIGHT; ++f) tmem_ld32_issue(tb + c + f * 32, a[f]);
        ldw();
#pragma unroll
        for (int f = 0; f < INFLIGHT; ++f)
#pragma unroll
          for (int i = 0; i < 32; ++i) acc += __uint_as_float(a[f][i]);
      } else {
        uint32_t a[INFLIGHT][16];
#pragma unroll
        for (int f = 0; f < INFLIGHT; ++f) ld16(tb + c + f * 16, a[f]);
        ldw();
#pragma unroll
        for (int f = 0; f < INFLIGHT; ++f)
#pragma unroll
          for (int i = 0; i < 16; ++i) acc += __uint_as_float(a[f][i]);
      }
    }
    asm volatile("bar.sync 1, %0;" ::"n"(NW * 32) : "memory");
  }
  if (threadIdx.x == 0) cyc[blockIdx.x] = clock64() - t0;
  if (acc == 1.2345f) sink[threadIdx.x] = acc;
  fence_before();
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256) : "memory");
}

template <int NW, int W, int INF>
void run(const char *name, long long *d, float *s) {
  const int reps = 200;
  rd<NW, W, INF><<<148, NW * 32>>>(reps, d, s);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  double m = 0;
  for (int i = 0; i < 148; ++i) m += h[i];
  m /= 148 * reps;
  printf("%-32s %7.0f cycles per 128x256 fp32 accumulator = %5.1f B/cycle  (%s)\n", name, m, 131072.0 / m,
         cudaGetErrorString(e));
}

int main() {
  long long *d;
  float *s;
  cudaMalloc(&d, 148 * 8);
  cudaMalloc(&s, 4096);
  run<4, 32, 1>("4 warps, x32, 1 in flight", d, s);
  run<4, 32, 2>("4 warps, x32, 2 in flight", d, s);
  run<4, 32, 4>("4 warps, x32, 4 in flight", d, s);
  run<8, 32, 1>("8 warps, x32, 1 in flight", d, s);
  run<8, 32, 2>("8 warps, x32, 2 in flight", d, s);
  run<8, 16, 4>("8 warps, x16, 4 in flight", d, s);
  run<16, 32, 1>("16 warps, x32, 1 in flight", d, s);
  run<16, 32, 2>("16 warps, x32, 2 in flight", d, s);
  return 0;
}
