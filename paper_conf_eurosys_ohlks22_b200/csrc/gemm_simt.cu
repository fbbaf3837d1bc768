// fp32 SIMT GEMMs with the fused epilogues of kernels.h (EpiArgs), for the fp32
// mode (BASELINE config 0: 4-layer MLP width 256, batch 32).  Exact fp32 FFMA:
// TF32 tensor cores would round operands to 10 mantissa bits and miss the
// 1e-4 fp32 parity bar (reading Q10).  The fp32 config is launch-bound (each
// GEMM is ~2 MFLOP), so a plain 64x64x16 register-blocked tile is enough.
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace ooo {
namespace simt {

constexpr int BM = kSimtBM;   // 64
constexpr int BN = 64;
constexpr int BK = 16;
constexpr int kThreads = 256;

__device__ __forceinline__ float act_f(int act, float z) {
  if (act == ACT_RELU) return z > 0.f ? z : 0.f;
  if (act == ACT_GELU) return z * 0.5f * (1.f + erff(z * 0.70710678118654752f));
  return z;
}
__device__ __forceinline__ float act_grad_f(int act, float z) {
  if (act == ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == ACT_GELU)
    return 0.5f * (1.f + erff(z * 0.70710678118654752f)) +
           z * 0.39894228040143268f * expf(-0.5f * z * z);
  return 1.f;
}

template <int EPI>
__global__ void __launch_bounds__(kThreads) gemm_simt_kernel(const SimtOperands op, const EpiArgs a) {
  __shared__ float As[BK][BM + 1];
  __shared__ float Bs[BK][BN + 1];
  __shared__ float red[16][BN + 1];
  const int tid = threadIdx.x;
  const int tx = tid & 15, ty = tid >> 4;
  const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
  const int nkb = (a.K + BK - 1) / BK;
  const int kb0 = blockIdx.z * a.kb_per_split;
  int kb1 = kb0 + a.kb_per_split;
  if (kb1 > nkb) kb1 = nkb;
  float acc[4][4];
#pragma unroll
  for (int i = 0; i < 4; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;

  for (int kb = kb0; kb < kb1; ++kb) {
    const int k0 = kb * BK;
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const int e = tid + r * kThreads;            // 0..1023
      // A tile: 64 (m) x 16 (k)
      {
        int mm, kk;
        if (op.sak == 1) { kk = e % BK; mm = e / BK; } else { mm = e % BM; kk = e / BM; }
        const int gm = m0 + mm, gk = k0 + kk;
        As[kk][mm] = (gm < a.M && gk < a.K) ? op.A[(long long)gm * op.sam + (long long)gk * op.sak] : 0.f;
      }
      // B tile: 16 (k) x 64 (n)
      {
        int kk, nn;
        if (op.sbn == 1) { nn = e % BN; kk = e / BN; } else { kk = e % BK; nn = e / BK; }
        const int gk = k0 + kk, gn = n0 + nn;
        Bs[kk][nn] = (gk < a.K && gn < a.N) ? op.B[(long long)gk * op.sbk + (long long)gn * op.sbn] : 0.f;
      }
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) av[i] = As[kk][ty + 16 * i];
#pragma unroll
      for (int j = 0; j < 4; ++j) bv[j] = Bs[kk][tx + 16 * j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    __syncthreads();
  }

  float colsum[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int m = m0 + ty + 16 * i;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx + 16 * j;
      if (m >= a.M || n >= a.N) continue;
      const long long o = (long long)m * a.ldc + n;
      float v = acc[i][j];
      if (EPI == EPI_FWD) {
        v += static_cast<const float *>(a.bias)[n];
        if (a.z_out) static_cast<float *>(a.z_out)[o] = v;
        static_cast<float *>(a.x_out)[o] = act_f(a.act, v);
      } else if (EPI == EPI_DGRAD) {
        if (a.act != ACT_ID) v *= act_grad_f(a.act, static_cast<const float *>(a.zin)[o]);
        static_cast<float *>(a.x_out)[o] = v;
        colsum[j] += v;                              // rows in fixed order i = 0..3
      } else {
        if (a.splits == 1) static_cast<float *>(a.x_out)[o] = v * a.alpha;
        else a.fpart[(long long)blockIdx.z * a.M * a.ldc + o] = v;
      }
    }
  }
  if (EPI == EPI_DGRAD && a.dbpart) {
#pragma unroll
    for (int j = 0; j < 4; ++j) red[ty][tx + 16 * j] = colsum[j];
    __syncthreads();
    if (tid < BN) {
      const int n = n0 + tid;
      if (n < a.N) {
        float s = 0.f;
        for (int r = 0; r < 16; ++r) s += red[r][tid];   // fixed order
        a.dbpart[(long long)blockIdx.x * a.N + n] = s;
      }
    }
  }
}

}  // namespace simt

cudaError_t launch_gemm_simt(int epi, const SimtOperands &ops, const EpiArgs &args,
                             const LaunchCtx &ctx, int *grid_ctas) {
  dim3 grid((args.M + simt::BM - 1) / simt::BM, (args.N + simt::BN - 1) / simt::BN, args.splits);
  if (grid_ctas) *grid_ctas = grid.x * grid.y * grid.z;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = dim3(simt::kThreads, 1, 1);
  cfg.stream = ctx.stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = ctx.priority;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  switch (epi) {
    case EPI_FWD: return cudaLaunchKernelEx(&cfg, simt::gemm_simt_kernel<EPI_FWD>, ops, args);
    case EPI_DGRAD: return cudaLaunchKernelEx(&cfg, simt::gemm_simt_kernel<EPI_DGRAD>, ops, args);
    case EPI_WGRAD: return cudaLaunchKernelEx(&cfg, simt::gemm_simt_kernel<EPI_WGRAD>, ops, args);
  }
  return cudaErrorInvalidValue;
}

}  // namespace ooo
