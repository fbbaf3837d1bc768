// Standalone probe of the tcgen05 GEMM kernel (tuning aid, not the product):
// compiles gemm_tc.cu with OOO_TRACE, runs one forward-type GEMM
// (M x K) * (K x N) on synthetic data and prints per-CTA phase times from
// %globaltimer stamps: prologue, PDL wait, first TMA arrival, last MMA issue,
// first accumulator ready, epilogue end, exit.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DOOO_TRACE \
//        -I include tools/gemm_probe.cu -o /tmp/gemm_probe && /tmp/gemm_probe M N K [BN] [epi]
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include <algorithm>
#include <vector>

#include "../paper_conf_eurosys_ohlks22_b200/csrc/gemm_tc.cu"

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                  const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static void make_map(EncodeTiledFn enc, CUtensorMap *m, void *ptr, uint64_t inner, uint64_t outer,
                     uint32_t bi, uint32_t bo) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {inner * 2};
  cuuint32_t box[2] = {bi, bo};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, ptr, dims, strides, box, es,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    printf("encode failed %d\n", (int)r);
    exit(1);
  }
}

int main(int argc, char **argv) {
  int M = argc > 1 ? atoi(argv[1]) : 4096;
  int N = argc > 2 ? atoi(argv[2]) : 768;
  int K = argc > 3 ? atoi(argv[3]) : 768;
  int BN = argc > 4 ? atoi(argv[4]) : 192;
  int ctas_max = argc > 5 ? atoi(argv[5]) : 148;
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  EncodeTiledFn enc = (EncodeTiledFn)fn;
  __nv_bfloat16 *X, *W, *b, *Y;
  cudaMalloc(&X, (size_t)M * K * 2);
  cudaMalloc(&W, (size_t)K * N * 2);
  cudaMalloc(&b, (size_t)N * 2);
  cudaMalloc(&Y, (size_t)M * N * 2);
  cudaMemset(X, 0, (size_t)M * K * 2);
  cudaMemset(W, 0, (size_t)K * N * 2);
  cudaMemset(b, 0, (size_t)N * 2);
  CUtensorMap tA, tB;
  make_map(enc, &tA, X, K, M, 64, 128);
  make_map(enc, &tB, W, N, K, 64, 64);
  CUtensorMap tY;
  make_map(enc, &tY, Y, N, M, 64, 32);
  ooo::gemm_tc_init();
  ooo::EpiArgs a = {};
  a.M = M; a.N = N; a.K = K;
  a.kb_per_split = (K + 63) / 64; a.splits = 1;
  a.act = 0; a.ldc = N; a.alpha = 1.f; a.bias = b; a.x_out = Y;
  int units = ((M + 127) / 128) * ((N + BN - 1) / BN);
  int ctas = std::min(units, ctas_max);
  unsigned long long *tr;
  cudaMalloc(&tr, (size_t)ctas * 8 * 8);
  cudaMemset(tr, 0, (size_t)ctas * 8 * 8);
  cudaStream_t st;
  cudaStreamCreate(&st);
  ooo::LaunchCtx ctx{st, 0, false};
  // warm up (no trace)
  for (int i = 0; i < 5; ++i) ooo::launch_gemm_tc(ooo::EPI_FWD, BN, &tA, &tB, &tY, &tY, a, ctas, ctx);
  cudaStreamSynchronize(st);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, st);
  for (int i = 0; i < 20; ++i) ooo::launch_gemm_tc(ooo::EPI_FWD, BN, &tA, &tB, &tY, &tY, a, ctas, ctx);
  cudaEventRecord(e1, st);
  cudaStreamSynchronize(st);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  printf("M=%d N=%d K=%d BN=%d ctas=%d units=%d: %.2f us/launch (back to back), %.1f TFLOP/s\n", M, N, K,
         BN, ctas, units, ms * 1e3 / 20, 2.0 * M * N * K / (ms / 20 * 1e-3) / 1e12);
  cudaMemcpyToSymbol(ooo::tc::g_trace, &tr, sizeof(tr));
  cudaEventRecord(e0, st);
  ooo::launch_gemm_tc(ooo::EPI_FWD, BN, &tA, &tB, &tY, &tY, a, ctas, ctx);
  cudaEventRecord(e1, st);
  cudaError_t err = cudaStreamSynchronize(st);
  cudaEventElapsedTime(&ms, e0, e1);
  printf("traced launch: %.2f us (%s)\n", ms * 1e3, cudaGetErrorString(err));
  std::vector<unsigned long long> h((size_t)ctas * 8);
  cudaMemcpy(h.data(), tr, h.size() * 8, cudaMemcpyDeviceToHost);
  unsigned long long t0 = ~0ull, tend = 0;
  for (int c = 0; c < ctas; ++c) {
    t0 = std::min(t0, h[c * 8]);
    tend = std::max(tend, h[c * 8 + 7]);
  }
  const char *names[8] = {"entry", "prologue", "pdl", "first_tma", "last_mma", "acc0_ready", "epi_end", "exit"};
  printf("span first-entry -> last-exit: %.2f us\n", (tend - t0) / 1e3);
  for (int s = 0; s < 8; ++s) {
    std::vector<double> v;
    for (int c = 0; c < ctas; ++c)
      if (h[c * 8 + s]) v.push_back((h[c * 8 + s] - t0) / 1e3);
    std::sort(v.begin(), v.end());
    if (v.empty()) continue;
    printf("  %-11s min %7.2f  med %7.2f  max %7.2f us\n", names[s], v.front(), v[v.size() / 2], v.back());
  }
  return 0;
}
