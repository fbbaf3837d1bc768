// HBM-bound elementwise kernels of the backward pass (sm_100a):
//   seed (BK4): the loss-gradient op dO_{L+1} ("T(dO_{L+1}) = 0"):
//               dZ_L = dY * act_L'(Z_L), plus per-row-block column sums (db_L
//               partials).  16-B vector loads/stores, coalesced along d.
//   pack (BK5): deterministic reduction of dW split-K partials and db
//               partials, scaled by 1/N (rank average, §5.1 P:176-180,
//               reading Q9), rounded to the gradient bucket's dtype.
// Both sum in a fixed order, so results do not depend on scheduling.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace ooo {
namespace ew {

__device__ __forceinline__ float act_grad_f(int act, float z) {
  if (act == ACT_DSTORED) return z;   // the Z store holds act'(Z) (engine path)
  if (act == ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == ACT_GELU)
    return 0.5f * (1.f + erff(z * 0.70710678118654752f)) +
           z * 0.39894228040143268f * expf(-0.5f * z * z);
  return 1.f;
}

template <typename T> struct V;
template <> struct V<__nv_bfloat16> {
  static constexpr int N = 8;
  __device__ static void load(const void *p, float (&f)[8]) {
    uint4 u = __ldg(reinterpret_cast<const uint4 *>(p));
    const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      f[2 * j] = __uint_as_float(w[j] << 16);
      f[2 * j + 1] = __uint_as_float(w[j] & 0xFFFF0000u);
    }
  }
  __device__ static void store(void *p, float (&f)[8]) {   // rounds f in place (RNE)
    uint32_t w[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * j], f[2 * j + 1]);
      w[j] = *reinterpret_cast<uint32_t *>(&h);
      f[2 * j] = __low2float(h);
      f[2 * j + 1] = __high2float(h);
    }
    *reinterpret_cast<uint4 *>(p) = make_uint4(w[0], w[1], w[2], w[3]);
  }
  __device__ static void store_scalar(void *p, float f) {
    *reinterpret_cast<__nv_bfloat16 *>(p) = __float2bfloat16_rn(f);
  }
};
template <> struct V<float> {
  static constexpr int N = 4;
  __device__ static void load(const void *p, float (&f)[4]) {
    float4 u = __ldg(reinterpret_cast<const float4 *>(p));
    f[0] = u.x; f[1] = u.y; f[2] = u.z; f[3] = u.w;
  }
  __device__ static void store(void *p, float (&f)[4]) {
    *reinterpret_cast<float4 *>(p) = make_float4(f[0], f[1], f[2], f[3]);
  }
  __device__ static void store_scalar(void *p, float f) { *reinterpret_cast<float *>(p) = f; }
};

// grid (ceil(M / bm), ceil(N / (32 * VEC))), block (32, kSeedTY): kSeedTY
// row lanes so that each thread has bm / kSeedTY rows, all loaded at once
constexpr int kSeedTY = 32;
template <typename T>
__global__ void __launch_bounds__(32 * kSeedTY) seed_kernel(const T *__restrict__ dy, const T *__restrict__ z,
                                                   int act, T *__restrict__ dz,
                                                   float *__restrict__ dbpart, int M, int N, int bm) {
  constexpr int VEC = V<T>::N;
  // the engine launched after the seed may start its prologue now (it reads
  // dZ_L only after griddepcontrol.wait, i.e. after this grid completes)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  __shared__ float red[kSeedTY][32 * VEC];
  const int tx = threadIdx.x, ty = threadIdx.y;
  const int col = (blockIdx.y * 32 + tx) * VEC;
  const int r0 = blockIdx.x * bm;
  float sum[VEC];
#pragma unroll
  for (int j = 0; j < VEC; ++j) sum[j] = 0.f;
  if (col < N) {
    // batches of U rows: all U loads in flight before the first use (the
    // kernel is HBM-latency bound otherwise: one 16-B load per thread in flight)
    constexpr int U = 4;
    const int rend = min(r0 + bm, M);
    for (int rb = r0 + ty; rb < rend; rb += kSeedTY * U) {
      float g[U][VEC], zz[U][VEC];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int r = rb + kSeedTY * u;
        if (r < rend) {
          V<T>::load(dy + (size_t)r * N + col, g[u]);
          if (act != ACT_ID) V<T>::load(z + (size_t)r * N + col, zz[u]);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int r = rb + kSeedTY * u;
        if (r < rend) {
          if (act != ACT_ID) {
#pragma unroll
            for (int j = 0; j < VEC; ++j) g[u][j] *= act_grad_f(act, zz[u][j]);
          }
          V<T>::store(dz + (size_t)r * N + col, g[u]);   // rounds g to the storage dtype
#pragma unroll
          for (int j = 0; j < VEC; ++j) sum[j] += g[u][j];   // rows in increasing order (fixed)
        }
      }
    }
  }
#pragma unroll
  for (int j = 0; j < VEC; ++j) red[ty][tx * VEC + j] = sum[j];
  __syncthreads();
  if (ty < VEC && col < N) {   // row lane ty sums column col + ty over the kSeedTY lanes
    float s = 0.f;
#pragma unroll
    for (int r = 0; r < kSeedTY; ++r) s += red[r][tx * VEC + ty];     // fixed order
    dbpart[(size_t)blockIdx.x * N + col + ty] = s;
  }
}

template <typename T>
__global__ void __launch_bounds__(256) pack_kernel(const float *__restrict__ wpart, int S,
                                                   long long wvec, T *__restrict__ wout,
                                                   const float *__restrict__ dbpart, int R, int N,
                                                   T *__restrict__ dbout, float alpha) {
  const long long total = wvec + N;
  const long long stride = (long long)gridDim.x * blockDim.x;
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += stride) {
    if (t < wvec) {
      const long long e = t * 4;
      const long long count = wvec * 4;
      float4 acc = __ldg(reinterpret_cast<const float4 *>(wpart + e));
      for (int s = 1; s < S; ++s) {                                  // fixed order
        float4 p = __ldg(reinterpret_cast<const float4 *>(wpart + (long long)s * count + e));
        acc.x += p.x; acc.y += p.y; acc.z += p.z; acc.w += p.w;
      }
      if (sizeof(T) == 2) {
        __nv_bfloat162 a = __floats2bfloat162_rn(acc.x * alpha, acc.y * alpha);
        __nv_bfloat162 b = __floats2bfloat162_rn(acc.z * alpha, acc.w * alpha);
        uint2 u = make_uint2(*reinterpret_cast<uint32_t *>(&a), *reinterpret_cast<uint32_t *>(&b));
        *reinterpret_cast<uint2 *>(wout + e) = u;
      } else {
        *reinterpret_cast<float4 *>(wout + e) =
            make_float4(acc.x * alpha, acc.y * alpha, acc.z * alpha, acc.w * alpha);
      }
    } else {
      const int n = (int)(t - wvec);
      float s = 0.f;
      for (int r = 0; r < R; ++r) s += dbpart[(size_t)r * N + n];    // fixed order
      V<T>::store_scalar(dbout + n, s * alpha);
    }
  }
}

inline cudaLaunchConfig_t cfg_for(dim3 grid, dim3 block, const LaunchCtx &ctx, cudaLaunchAttribute *attr) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.stream = ctx.stream;
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = ctx.priority;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cfg;
}

}  // namespace ew

cudaError_t launch_seed(bool bf16, const void *dy, const void *z, int act, void *dz, float *dbpart,
                        int M, int N, int bm, const LaunchCtx &ctx, int *grid_ctas) {
  const int vec = bf16 ? 8 : 4;
  dim3 grid((M + bm - 1) / bm, (N + 32 * vec - 1) / (32 * vec), 1);
  if (grid_ctas) *grid_ctas = grid.x * grid.y;
  cudaLaunchAttribute attr[1];
  cudaLaunchConfig_t cfg = ew::cfg_for(grid, dim3(32, ew::kSeedTY, 1), ctx, attr);
  if (bf16)
    return cudaLaunchKernelEx(&cfg, ew::seed_kernel<__nv_bfloat16>,
                              static_cast<const __nv_bfloat16 *>(dy), static_cast<const __nv_bfloat16 *>(z),
                              act, static_cast<__nv_bfloat16 *>(dz), dbpart, M, N, bm);
  return cudaLaunchKernelEx(&cfg, ew::seed_kernel<float>, static_cast<const float *>(dy),
                            static_cast<const float *>(z), act, static_cast<float *>(dz), dbpart, M, N, bm);
}

cudaError_t launch_pack(bool bf16, const float *wpart, int S, long long wcount, void *wout,
                        const float *dbpart, int R, int N, void *dbout, float alpha,
                        const LaunchCtx &ctx, int *grid_ctas) {
  const long long wvec = wpart ? wcount / 4 : 0;
  const long long total = wvec + N;
  long long blocks = (total + 255) / 256;
  if (blocks > 148 * 8) blocks = 148 * 8;
  if (blocks < 1) blocks = 1;
  if (grid_ctas) *grid_ctas = (int)blocks;
  cudaLaunchAttribute attr[1];
  cudaLaunchConfig_t cfg = ew::cfg_for(dim3((unsigned)blocks, 1, 1), dim3(256, 1, 1), ctx, attr);
  if (bf16)
    return cudaLaunchKernelEx(&cfg, ew::pack_kernel<__nv_bfloat16>, wpart, S, wvec,
                              static_cast<__nv_bfloat16 *>(wout), dbpart, R, N,
                              static_cast<__nv_bfloat16 *>(dbout), alpha);
  return cudaLaunchKernelEx(&cfg, ew::pack_kernel<float>, wpart, S, wvec, static_cast<float *>(wout),
                            dbpart, R, N, static_cast<float *>(dbout), alpha);
}

// Emulated all-reduce (single-GPU measurement aid, OOO_EMULATE_AR_N): one
// thread holds the comm stream for `ns` nanoseconds (the modelled ring
// all-reduce time of a bucket), so the engine's F_i gate on the bucket's
// all-reduce flag sees a realistic completion time.  No data is moved.
namespace ew {
__global__ void delay_kernel(unsigned long long ns) {
  unsigned long long t0, t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  do {
    __nanosleep(200);
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  } while (t - t0 < ns);
}
}  // namespace ew

cudaError_t launch_delay(unsigned long long ns, cudaStream_t stream) {
  ew::delay_kernel<<<1, 1, 0, stream>>>(ns);
  return cudaGetLastError();
}

}  // namespace ooo
