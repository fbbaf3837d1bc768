// Microbenchmark: TMA -> shared ring -> tcgen05.mma pipeline of one
// 128 x 256 tile per CTA (cta_group::1), operands L2-resident, all 148 SMs.
// Measures cycles per 64-deep k-block for the engine's operand layouts and a
// few pipeline variants (stages, B K-major vs MN-major).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_eurosys_ohlks22_b200/csrc \
//        -o tools/pipe_probe tools/pipe_probe.cu -lcuda
#include <cuda.h>
#include <cstdio>
#include <cuda_runtime.h>
#include <stdint.h>

#include "tc_common.cuh"

using namespace ooo::tc;

constexpr int kA = 16384, kBmax = 32768;

__global__ void __launch_bounds__(128, 1)
    probe(const __grid_constant__ CUtensorMap mA, const __grid_constant__ CUtensorMap mB, int nkb, int stages,
          int b_mn, int mt, int nt, long long *out) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t base = smem_u32(smem);
  const int STAGE = kA + kBmax;
  const uint32_t bars = base + stages * STAGE;   // full[stages], empty[stages], done
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(bars + 8 * s, 1);
      mbar_init(bars + 8 * (stages + s), 1);
    }
    mbar_init(bars + 16 * stages, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tslot)),
                 "r"(256)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = tslot;
  const int m0 = (blockIdx.x % mt) * 128, n0 = ((blockIdx.x / mt) % nt) * 256;
  long long t0 = clock64();
  if (warp == 0 && lane == 0) {
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      if (kb >= stages) mbar_wait(bars + 8 * (stages + s), ((kb / stages) - 1) & 1);
      const uint32_t sa = base + s * STAGE, sb = sa + kA, fb = bars + 8 * s;
      mbar_expect_tx(fb, kA + kBmax);
      tma_load_2d(sa, &mA, fb, kb * 64, m0);                       // A: box {64 K, 128 M}
      if (b_mn) {
        for (int c = 0; c < 4; ++c) tma_load_2d(sb + 8192 * c, &mB, fb, n0 + 64 * c, kb * 64);   // {64 N, 64 K}
      } else {
        tma_load_2d(sb, &mB, fb, kb * 64, n0);                     // B K-major: box {64 K, 256 N}
      }
    }
  } else if (warp == 1 && lane == 0) {
    const uint32_t ID = (1u << 4) | (1u << 7) | (1u << 10) | ((b_mn ? 1u : 0u) << 16) | ((uint32_t)(256 >> 3) << 17) |
                        ((uint32_t)(128 >> 4) << 24);
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      mbar_wait(bars + 8 * s, (kb / stages) & 1);
      fence_after();
      const uint32_t sa = base + s * STAGE, sb = sa + kA;
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const uint64_t ad = sdesc(sa + kk * 32, 16, 1024);
        const uint64_t bd = b_mn ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
        umma_bf16(tmem, ad, bd, ID, (kb | kk) != 0 ? 1u : 0u);
      }
      umma_commit(bars + 8 * (stages + s));
    }
    umma_commit(bars + 16 * stages);
    mbar_wait(bars + 16 * stages, 0);
    out[blockIdx.x] = clock64() - t0;
  }
  fence_before();
  __syncthreads();
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256) : "memory");
}

// CTA-pair variant (cluster of 2, cta_group::2, M = 256): each CTA loads its
// 128 rows of A and half of B (128 columns) per k-block; the leader's one
// thread issues the M = 256 MMAs and multicasts the commits.
__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
  uint32_t o;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
  return o;
}
template <bool kGlobalMaps>
__global__ void __launch_bounds__(320, 1)
    probe2(const __grid_constant__ CUtensorMap mAp, const __grid_constant__ CUtensorMap mBp, const CUtensorMap *gmaps,
           int nkb, int stages, int mt, int nt, long long *out, int poll_mode, int kpass, int nmode) {
  const CUtensorMap &mA = kGlobalMaps ? gmaps[0] : mAp;
  const CUtensorMap &mB = kGlobalMaps ? gmaps[1] : mBp;
  if (kGlobalMaps && threadIdx.x == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mB)) : "memory");
  }
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t base = smem_u32(smem);
  const int STAGE = 16384 + 16384;
  const uint32_t bars = base + stages * STAGE;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cta_rank();
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) {
      mbar_init(bars + 8 * s, 1);
      mbar_init(bars + 8 * (stages + s), 1);
    }
    mbar_init(bars + 16 * stages, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tslot)),
                 "r"(256)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  fence_before();
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  fence_after();
  const uint32_t tmem = tslot;
  const int pair = blockIdx.x >> 1;
  const int m0 = (pair % mt) * 256 + 128 * rank;
  const int n0 = (nmode ? pair % nt : (pair / mt) % nt) * 256 + 128 * rank;
  const int kwrap = kpass > 0 ? kpass : nkb;   // k-blocks per pass over a K-range that fits L2
  const uint32_t Lfull = mapa(bars, 0);
  long long t0 = clock64();
  unsigned long long g0;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
  if (warp == 0 && lane == 0) {
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      if (kb >= stages) mbar_wait(bars + 8 * (stages + s), ((kb / stages) - 1) & 1);
      const uint32_t sa = base + s * STAGE, sb = sa + 16384, fb = Lfull + 8 * s;
      if (blockIdx.x == 0 && kb < 16) out[200 + kb] = clock64() - t0;
      if (rank == 0) mbar_expect_tx(bars + 8 * s, 2 * STAGE);
      asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
                   " [%0], [%1, {%3, %4}], [%2];" ::"r"(sa), "l"(&mA), "r"(fb), "r"((kb % kwrap) * 64), "r"(m0) : "memory");
      for (int c = 0; c < 2; ++c)
        asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
                     " [%0], [%1, {%3, %4}], [%2];" ::"r"(sb + 8192 * c), "l"(&mB), "r"(fb), "r"(n0 + 64 * c),
                     "r"((kb % kwrap) * 64) : "memory");
    }
  } else if (warp == 1 && lane == 0 && rank == 0) {
    const uint32_t ID = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | ((uint32_t)(256 >> 3) << 17) |
                        ((uint32_t)(256 >> 4) << 24);
    for (int kb = 0; kb < nkb; ++kb) {
      const int s = kb % stages;
      mbar_wait(bars + 8 * s, (kb / stages) & 1);
      fence_after();
      const uint32_t sa = base + s * STAGE, sb = sa + 16384;
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        const uint64_t ad = sdesc(sa + kk * 32, 16, 1024);
        const uint64_t bd = sdesc(sb + kk * 2048, 8192, 1024);
        asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                     "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem),
                     "l"(ad), "l"(bd), "r"(ID), "r"((kb | kk) != 0 ? 1u : 0u));
      }
      asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                   ::"r"(bars + 8 * (stages + s)), "h"((unsigned short)3) : "memory");
    }
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                 ::"r"(bars + 16 * stages), "h"((unsigned short)3) : "memory");
    mbar_wait(bars + 16 * stages, 0);
    out[pair] = clock64() - t0;
    unsigned long long g1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
    out[74 + pair] = (long long)(g1 - g0);
  }
  if (warp == 1 && lane == 0 && rank == 1) mbar_wait(bars + 16 * stages, 0);
  if (warp >= 2) {   // idle warps waiting for the end (like epilogue warps waiting for an accumulator)
    if (poll_mode == 1) {
      while (!mbar_try_wait(bars + 16 * stages, 0)) {
      }
    } else if (poll_mode == 2) {
      while (!mbar_try_wait(bars + 16 * stages, 0)) __nanosleep(200);
    }
  }
  fence_before();
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256) : "memory");
}

typedef CUresult (*Enc)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *, const cuuint64_t *,
                        const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static CUtensorMap map2d(Enc enc, void *p, uint64_t inner, uint64_t outer, uint32_t bi, uint32_t bo) {
  CUtensorMap m;
  cuuint64_t dims[2] = {inner, outer}, str[1] = {inner * 2};
  cuuint32_t box[2] = {bi, bo}, es[2] = {1, 1};
  CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, p, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) printf("encode failed %d\n", (int)r);
  return m;
}

int main() {
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  Enc enc = (Enc)fn;
  const int M = 2048, N = 2048, K = 8192;
  void *A, *Bmn, *Bk;
  cudaMalloc(&A, (size_t)M * K * 2);
  cudaMalloc(&Bmn, (size_t)K * N * 2);   // [K][N]
  cudaMalloc(&Bk, (size_t)N * K * 2);    // [N][K]
  cudaMemset(A, 0, (size_t)M * K * 2);
  cudaMemset(Bmn, 0, (size_t)K * N * 2);
  cudaMemset(Bk, 0, (size_t)N * K * 2);
  CUtensorMap mA = map2d(enc, A, K, M, 64, 128);
  CUtensorMap mBmn = map2d(enc, Bmn, N, K, 64, 64);
  CUtensorMap mBk = map2d(enc, Bk, K, N, 64, 256);
  long long *d;
  cudaMalloc(&d, 300 * 8);
  const int nkb = K / 64;
  for (int stages : {2, 3, 4}) {
    for (int b_mn : {1, 0}) {
      const int smem = stages * (kA + kBmax) + 16 * stages + 8 + 1024;
      cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      probe<<<148, 128, smem>>>(mA, b_mn ? mBmn : mBk, nkb, stages, b_mn, M / 128, N / 256, d);
      cudaError_t e = cudaDeviceSynchronize();
      long long h[148];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      double m = 0;
      for (int i = 0; i < 148; ++i) m += h[i];
      m /= 148;
      printf("stages %d  B %s : %7.1f cycles per k-block (ideal 512)  [%s]\n", stages, b_mn ? "MN-major" : "K-major ",
             m / nkb, cudaGetErrorString(e));
    }
  }
  // CTA pairs
  CUtensorMap mA2 = map2d(enc, A, K, M, 64, 128);
  CUtensorMap hm[2] = {mA2, mBmn};
  CUtensorMap *gm;
  cudaMalloc(&gm, sizeof(hm));
  cudaMemcpy(gm, hm, sizeof(hm), cudaMemcpyHostToDevice);
  for (int variant = 0; variant < 4; ++variant)
  for (int stages : {6}) {
    const int poll_mode = variant >= 2 ? variant - 1 : 0;   // 0 none, 1 spin, 2 sleep
    const int smem = stages * 32768 + 16 * stages + 8 + 1024;
    cudaFuncSetAttribute(probe2<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaFuncSetAttribute(probe2<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(148, 1, 1);
    cfg.blockDim = dim3(variant >= 2 ? 320 : 128, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (variant != 1) cudaLaunchKernelEx(&cfg, probe2<false>, mA2, mBmn, (const CUtensorMap *)gm, nkb, stages, M / 256, N / 256, d, poll_mode, 0, 0);
    else cudaLaunchKernelEx(&cfg, probe2<true>, mA2, mBmn, (const CUtensorMap *)gm, nkb, stages, M / 256, N / 256, d, poll_mode, 0, 0);
    cudaError_t e = cudaDeviceSynchronize();
    long long h[148];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    double m = 0, ns = 0;
    for (int i = 0; i < 74; ++i) { m += h[i]; ns += h[74 + i]; }
    m /= 74;
    ns /= 74;
    printf("   (%.3f us per k-block, clock %.0f MHz)\n", ns / 1e3 / nkb, m / ns * 1e3);
    long long pk[16];
    cudaMemcpy(pk, d + 200, sizeof(pk), cudaMemcpyDeviceToHost);
    printf("   producer issue clocks kb0..15:");
    for (int i = 0; i < 16; ++i) printf(" %lld", pk[i]);
    printf("\n");
    const char *vn[4] = {"params, no pollers", "global maps, no pollers", "params, 8 spinning waiters", "params, 8 sleeping waiters"};
    printf("pair  stages %d  %s : %7.1f cycles per k-block (ideal 512)  [%s]\n", stages, vn[variant], m / nkb,
           cudaGetErrorString(e));
  }
  // ---- L2 sharing experiment: 74 pairs, K = 1024 per pass (operands fit L2), 128 k-blocks
  {
    const int M2 = 74 * 256, N2 = 74 * 256, K2 = 1024;
    void *A2, *B2;
    cudaMalloc(&A2, (size_t)M2 * K2 * 2);
    cudaMalloc(&B2, (size_t)K2 * N2 * 2);
    cudaMemset(A2, 0, (size_t)M2 * K2 * 2);
    cudaMemset(B2, 0, (size_t)K2 * N2 * 2);
    CUtensorMap a2 = map2d(enc, A2, K2, M2, 64, 128);
    CUtensorMap b2 = map2d(enc, B2, N2, K2, 64, 64);
    struct Case { int mt, nt, nmode; const char *name; };
    const Case cases[] = {{8, 8, 0, "A shared by ~9 pairs, B by ~9"},
                          {25, 3, 0, "A shared by 3, B by 25 (engine hxh chain)"},
                          {74, 1, 0, "A distinct, B shared by all"},
                          {74, 74, 1, "A and B distinct per pair"},
                          {1, 1, 0, "A and B shared by all 74"}};
    const int stages = 6, nkb2 = 128;
    const int smem = stages * 32768 + 16 * stages + 8 + 1024;
    cudaFuncSetAttribute(probe2<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    for (const Case &c : cases) {
      for (int rep = 0; rep < 2; ++rep) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(148, 1, 1);
        cfg.blockDim = dim3(128, 1, 1);
        cfg.dynamicSmemBytes = smem;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 2;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, probe2<false>, a2, b2, (const CUtensorMap *)gm, nkb2, stages, c.mt, c.nt, d, 0, K2 / 64,
                           c.nmode);
        cudaError_t e = cudaDeviceSynchronize();
        long long h[148];
        cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
        double m = 0, ns = 0;
        for (int i = 0; i < 74; ++i) { m += h[i]; ns += h[74 + i]; }
        m /= 74;
        ns /= 74;
        if (rep == 1)
          printf("sharing: %-44s %7.1f cycles/kb  %.3f us/kb  -> %.1f TB/s into SMs  [%s]\n", c.name, m / nkb2,
                 ns / 1e3 / nkb2, 74.0 * 65536 / (ns / nkb2) / 1e3, cudaGetErrorString(e));
      }
    }
  }
  return 0;
}
