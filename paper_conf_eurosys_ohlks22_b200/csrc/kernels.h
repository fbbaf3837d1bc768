// Internal interface between the scheduler (ooo_api.cpp) and the sm_100a
// kernels.  Not part of the public ABI (include/ooo.h).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace ooo {

enum Act : int { ACT_ID = 0, ACT_RELU = 1, ACT_GELU = 2,
                 // backward only: the Z store holds act'(Z) (the engine's F_i
                 // epilogue stores gelu'(Z_i) instead of Z_i), act' = stored value
                 ACT_DSTORED = 3 };
enum Epi : int { EPI_FWD = 0, EPI_DGRAD = 1, EPI_WGRAD = 2 };

// Row-block height of the bias-gradient partials written by the dX epilogue
// and the seed kernel: one fp32 row of column sums per block of rows.
constexpr int kTcBM = 128;     // tcgen05 path (bf16)
constexpr int kSimtBM = 64;    // SIMT path (fp32)

// Epilogue arguments of the per-layer fp32 SIMT GEMMs (the bf16 engine has its
// own task descriptors, engine.h).
//   FWD  : v = acc + bias[n];  z_out[m][n] = st(v) (optional);
//          x_out[m][n] = st(act(ld(st(v))))                       (layer forward F_i)
//   DGRAD: v = acc * act'(zin[m][n]) (act' = 1 for ACT_ID, zin unused);
//          x_out[m][n] = st(v);  dbpart[m / BM][n] = sum over the
//          block's rows of ld(st(v)) (optional)                    (dO_i, fused act-grad + bias-grad)
//   WGRAD: splits == 1: x_out[m][n] = st(acc * alpha)  (the gradient bucket)
//          splits  > 1: fpart[z][m][n] = acc           (deterministic split-K)   (dW_i)
// st() = round to the storage dtype (bf16 RNE or fp32), ld() = widen to fp32.
struct EpiArgs {
  int M, N, K;            // output M x N, reduction length K
  int kb_per_split;       // K blocks (of 64) per split (gridDim.z splits)
  int splits;
  int act;                // FWD: act_i; DGRAD: act_{i-1}
  int ldc;                // leading dimension of outputs / zin (elements)
  float alpha;            // WGRAD scale (1/N)
  const void *bias;       // FWD
  const void *zin;        // DGRAD
  void *z_out;            // FWD (may be null)
  void *x_out;            // FWD / DGRAD / WGRAD(splits == 1)
  float *fpart;           // WGRAD(splits > 1)
  float *dbpart;          // DGRAD (may be null)
};

struct LaunchCtx {
  cudaStream_t stream;
  int priority;
  bool pdl = false;   // programmatic dependent launch (the kernel must griddepcontrol.wait)
};

// ---- fp32 SIMT GEMM (gemm_simt.cu): generic strides.
//   A(m, k) = A[m * sam + k * sak];  B(k, n) = B[k * sbk + n * sbn]
struct SimtOperands {
  const float *A; long long sam, sak;
  const float *B; long long sbk, sbn;
};
cudaError_t launch_gemm_simt(int epi, const SimtOperands &ops, const EpiArgs &args,
                             const LaunchCtx &ctx, int *grid_ctas);

// ---- elementwise (ew.cu)
// seed (dO_{L+1}): dz[m][n] = st(ld(dy[m][n]) * act'(ld(z[m][n]))); dbpart[m/bm][n] = column sums.
cudaError_t launch_seed(bool bf16, const void *dy, const void *z, int act, void *dz, float *dbpart,
                        int M, int N, int bm, const LaunchCtx &ctx, int *grid_ctas);
// pack (BK5): wout[e] = st(alpha * sum_s wpart[s][e]) for e < wcount (if wpart != null);
//             dbout[n] = st(alpha * sum_r dbpart[r][n]).  Fixed summation order.
cudaError_t launch_delay(unsigned long long ns, cudaStream_t stream);   // emulated all-reduce
cudaError_t launch_pack(bool bf16, const float *wpart, int S, long long wcount, void *wout,
                        const float *dbpart, int R, int N, void *dbout, float alpha,
                        const LaunchCtx &ctx, int *grid_ctas);

}  // namespace ooo
