// tcgen05 / TMEM / TMA bf16 GEMMs for the three per-layer contractions of
// ooo backprop (sm_100a):
//   F_i   (EPI_FWD)  : Z_i = X_i W_i + b_i, X_{i+1} = act_i(Z_i)
//   dO_i  (EPI_DGRAD): dZ_{i-1} = (dZ_i W_i^T) * act'_{i-1}(Z_{i-1}),
//                      + per-128-row column sums (bias-grad partials)
//   dW_i  (EPI_WGRAD): dW_i = X_i^T dZ_i (deterministic split-K)
// The paper keeps dO_i and dW_i as separate ops so they can be reordered
// (§7, tf.group removal; §4.1: the two GEMMs share only their
// smaller inputs, so splitting them costs little locality).
//
// Structure (one 128 x BN output tile per CTA, non-persistent so that stream
// priorities act at CTA-dispatch granularity):
//   warp 0 lane 0 : TMA producer, STAGES-deep smem ring (128B swizzle)
//   warp 1        : TMEM allocator; lane 0 issues tcgen05.mma (M=128, N=BN, K=16)
//   warps 2..5    : epilogue -- tcgen05.ld 32x32b.x32 -> registers -> fused
//                   bias / activation / act-grad / bias-grad / scale -> global
// Operand majors: A K-major (X_i, dZ_i as A of F_i / dO_i) or MN-major
// (X_i^T as A of dW_i); B MN-major (W_i in F_i, dZ_i in dW_i) or K-major
// (W_i^T in dO_i).  16-bit types allow MN-major operands directly, so no
// transpose kernels are needed.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"

namespace ooo {
namespace tc {

constexpr int BM = 128;
constexpr int BK = 64;                 // 64 bf16 = 128 B = one swizzle row
constexpr int A_BYTES = BM * BK * 2;   // 16 KiB
constexpr int kThreads = 192;

template <int BN> struct Cfg {
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES = (BN == 64) ? 8 : (BN == 128 ? 6 : 4);
  static constexpr int RING = STAGE * STAGES;
  static constexpr int TMEM_COLS = BN < 32 ? 32 : BN;
  // ring | full[STAGES] | empty[STAGES] | accum | tmem slot | db scratch [4][BN]
  static constexpr int BAR_OFF = RING;
  static constexpr int SLOT_OFF = BAR_OFF + (2 * STAGES + 1) * 8;
  static constexpr int RED_OFF = (SLOT_OFF + 16 + 15) / 16 * 16;
  static constexpr int SMEM = RED_OFF + 4 * BN * 4 + 1024;   // + alignment slack
};

// ----------------------------------------------------------------- PTX
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  while (!mbar_try_wait(bar, parity)) {
  }
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tma_prefetch(const CUtensorMap *map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
__device__ __forceinline__ void fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void umma_bf16(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                          uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   bar)
               : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// UMMA shared-memory descriptor, SWIZZLE_128B (layout type 2), version 1.
//   K-major : rows of 128 B (64 K-elements), 8-row groups 1024 B apart (SBO).
//   MN-major: 64-element MN chunks LBO apart, 8-row K groups 1024 B apart (SBO).
__device__ __forceinline__ uint64_t sdesc(uint32_t addr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((addr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFF) << 32) | (1ull << 46) | (2ull << 61);
}

// Instruction descriptor, kind::f16: D fp32, A/B bf16, M = 128, N = BN.
template <int BN, bool A_MN, bool B_MN>
__device__ __forceinline__ constexpr uint32_t idesc() {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((A_MN ? 1u : 0u) << 15) |
         ((B_MN ? 1u : 0u) << 16) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

// ------------------------------------------------------------ epilogue math
__device__ __forceinline__ float act_f(int act, float z) {
  if (act == ACT_RELU) return z > 0.f ? z : 0.f;
  if (act == ACT_GELU) return z * 0.5f * (1.f + erff(z * 0.70710678118654752f));
  return z;
}
__device__ __forceinline__ float act_grad_f(int act, float z) {
  if (act == ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == ACT_GELU)
    return 0.5f * (1.f + erff(z * 0.70710678118654752f)) +
           z * 0.39894228040143268f * __expf(-0.5f * z * z);
  return 1.f;
}
__device__ __forceinline__ float bf_lo(uint32_t u) { return __uint_as_float(u << 16); }
__device__ __forceinline__ float bf_hi(uint32_t u) { return __uint_as_float(u & 0xFFFF0000u); }
__device__ __forceinline__ uint32_t pack_bf2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);   // RNE
  return *reinterpret_cast<uint32_t *>(&h);
}
// load 32 consecutive bf16 (64 B, 16-B aligned) as fp32
__device__ __forceinline__ void ld_bf16x32(const __nv_bfloat16 *p, float (&f)[32]) {
  const uint4 *q = reinterpret_cast<const uint4 *>(p);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint4 u = __ldg(q + j);
    f[8 * j + 0] = bf_lo(u.x); f[8 * j + 1] = bf_hi(u.x);
    f[8 * j + 2] = bf_lo(u.y); f[8 * j + 3] = bf_hi(u.y);
    f[8 * j + 4] = bf_lo(u.z); f[8 * j + 5] = bf_hi(u.z);
    f[8 * j + 6] = bf_lo(u.w); f[8 * j + 7] = bf_hi(u.w);
  }
}
// store 32 fp32 as bf16 (RNE) and return the rounded values in f
__device__ __forceinline__ void st_bf16x32(__nv_bfloat16 *p, float (&f)[32]) {
  uint4 *q = reinterpret_cast<uint4 *>(p);
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    uint4 u;
    u.x = pack_bf2(f[8 * j + 0], f[8 * j + 1]);
    u.y = pack_bf2(f[8 * j + 2], f[8 * j + 3]);
    u.z = pack_bf2(f[8 * j + 4], f[8 * j + 5]);
    u.w = pack_bf2(f[8 * j + 6], f[8 * j + 7]);
    q[j] = u;
  }
}
__device__ __forceinline__ void round_bf16x32(float (&f)[32]) {
#pragma unroll
  for (int j = 0; j < 32; ++j) f[j] = __bfloat162float(__float2bfloat16_rn(f[j]));
}
// Column sums over the 32 lanes of a warp: on return lane l holds the sum of
// column l (fixed butterfly order -> deterministic).
__device__ __forceinline__ float warp_colsum32(float (&v)[32], int lane) {
#pragma unroll
  for (int off = 16; off >= 1; off >>= 1) {
    const bool upper = (lane & off) != 0;
#pragma unroll
    for (int j = 0; j < off; ++j) {
      float send = upper ? v[j] : v[j + off];
      float keep = upper ? v[j + off] : v[j];
      v[j] = keep + __shfl_xor_sync(0xffffffffu, send, off);
    }
  }
  return v[0];
}

// ------------------------------------------------------------------ kernel
template <int BN, bool A_MN, bool B_MN, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const EpiArgs args) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                              ~static_cast<uintptr_t>(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar_full = sbase + C::BAR_OFF;
  const uint32_t bar_empty = bar_full + 8 * C::STAGES;
  const uint32_t bar_accum = bar_empty + 8 * C::STAGES;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + C::SLOT_OFF);
  float *red = reinterpret_cast<float *>(smem + C::RED_OFF);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int m0 = blockIdx.x * BM;
  const int n0 = blockIdx.y * BN;
  const int nkb_total = (args.K + BK - 1) / BK;
  const int kb_begin = blockIdx.z * args.kb_per_split;
  int kb_end = kb_begin + args.kb_per_split;
  if (kb_end > nkb_total) kb_end = nkb_total;
  const int nkb = kb_end - kb_begin;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_empty + 8 * s, 1);
    }
    mbar_init(bar_accum, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"((uint32_t)C::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      for (int kb = 0; kb < nkb; ++kb) {
        const int s = kb % C::STAGES;
        if (kb >= C::STAGES) mbar_wait(bar_empty + 8 * s, ((kb / C::STAGES) - 1) & 1);
        const uint32_t fb = bar_full + 8 * s;
        mbar_expect_tx(fb, C::STAGE);
        const uint32_t sa = sbase + s * C::STAGE;
        const uint32_t sb = sa + A_BYTES;
        const int k0 = (kb_begin + kb) * BK;
        if (!A_MN) {
          tma_load_2d(sa, &tmA, fb, k0, m0);                 // box {64 K, 128 M}
        } else {
          tma_load_2d(sa, &tmA, fb, m0, k0);                 // box {64 M, 64 K}
          tma_load_2d(sa + 8192, &tmA, fb, m0 + 64, k0);
        }
        if (!B_MN) {
          tma_load_2d(sb, &tmB, fb, k0, n0);                 // box {64 K, BN N}
        } else {
#pragma unroll
          for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + 8192 * j, &tmB, fb, n0 + 64 * j, k0);
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
    if (lane == 0) {
      constexpr uint32_t ID = idesc<BN, A_MN, B_MN>();
      for (int kb = 0; kb < nkb; ++kb) {
        const int s = kb % C::STAGES;
        mbar_wait(bar_full + 8 * s, (kb / C::STAGES) & 1);
        fence_after();
        const uint32_t sa = sbase + s * C::STAGE;
        const uint32_t sb = sa + A_BYTES;
#pragma unroll
        for (int kk = 0; kk < BK / 16; ++kk) {
          const uint64_t ad = A_MN ? sdesc(sa + kk * 2048, 8192, 1024) : sdesc(sa + kk * 32, 16, 1024);
          const uint64_t bd = B_MN ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
          umma_bf16(tmem, ad, bd, ID, (kb | kk) != 0 ? 1u : 0u);
        }
        umma_commit(bar_empty + 8 * s);     // smem slot free once these MMAs retire
      }
      umma_commit(bar_accum);               // accumulator complete
    }
    __syncwarp();
  } else {
    // ===================== epilogue (warps 2..5) =====================
    const int q = warp & 3;                  // TMEM lane quarter this warp may access
    const int row = m0 + q * 32 + lane;
    const bool row_ok = row < args.M;
    if (nkb > 0) {
      mbar_wait(bar_accum, 0);
      fence_after();
    }
#pragma unroll 1
    for (int c = 0; c < BN / 32; ++c) {
      const int col0 = n0 + c * 32;
      if (col0 >= args.N) break;             // warp-uniform (N % 64 == 0)
      float v[32];
      if (nkb > 0) {
        uint32_t r[32];
        tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(c * 32), r);
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = __uint_as_float(r[j]);
      } else {
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = 0.f;
      }
      const size_t off = (size_t)row * args.ldc + col0;
      if (EPI == EPI_FWD) {
        float bias[32];
        ld_bf16x32(reinterpret_cast<const __nv_bfloat16 *>(args.bias) + col0, bias);
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] += bias[j];
        round_bf16x32(v);                                    // Z_i storage point
        if (row_ok && args.z_out)
          st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.z_out) + off, v);
        if (args.act != ACT_ID) {
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = act_f(args.act, v[j]);
        }
        if (row_ok) st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
      } else if (EPI == EPI_DGRAD) {
        if (args.act != ACT_ID) {
          float z[32];
          if (row_ok) {
            ld_bf16x32(reinterpret_cast<const __nv_bfloat16 *>(args.zin) + off, z);
          } else {
#pragma unroll
            for (int j = 0; j < 32; ++j) z[j] = 0.f;
          }
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] *= act_grad_f(args.act, z[j]);
        }
        round_bf16x32(v);                                    // dZ_{i-1} storage point
        if (!row_ok) {
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = 0.f;
        }
        if (row_ok) st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
        if (args.dbpart) {
          const float s = warp_colsum32(v, lane);           // lane l: column col0 + l
          red[q * BN + c * 32 + lane] = s;
        }
      } else {  // EPI_WGRAD
        if (args.splits == 1) {
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] *= args.alpha;
          if (row_ok) st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
        } else if (row_ok) {
          float4 *dst = reinterpret_cast<float4 *>(args.fpart + (size_t)blockIdx.z * args.M * args.ldc + off);
#pragma unroll
          for (int j = 0; j < 8; ++j) dst[j] = make_float4(v[4 * j], v[4 * j + 1], v[4 * j + 2], v[4 * j + 3]);
        }
      }
    }
    if (EPI == EPI_DGRAD && args.dbpart) {
      // sum the four row quarters in fixed order q = 0..3 (deterministic)
      asm volatile("bar.sync 1, 128;" ::: "memory");
      const int t = threadIdx.x - 64;                        // 0..127
      for (int cc = t; cc < BN; cc += 128) {
        const int col = n0 + cc;
        if (col < args.N) {
          const float s = ((red[cc] + red[BN + cc]) + red[2 * BN + cc]) + red[3 * BN + cc];
          args.dbpart[(size_t)blockIdx.x * args.N + col] = s;
        }
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"((uint32_t)C::TMEM_COLS)
                 : "memory");
  }
}

template <int BN, bool A_MN, bool B_MN, int EPI>
cudaError_t launch_one(const CUtensorMap *tmA, const CUtensorMap *tmB, const EpiArgs &args,
                       dim3 grid, const LaunchCtx &ctx) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.dynamicSmemBytes = Cfg<BN>::SMEM;
  cfg.stream = ctx.stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = ctx.priority;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, gemm_tc_kernel<BN, A_MN, B_MN, EPI>, *tmA, *tmB, args);
}

template <int BN, bool A_MN, bool B_MN, int EPI>
cudaError_t set_attr() {
  return cudaFuncSetAttribute(gemm_tc_kernel<BN, A_MN, B_MN, EPI>,
                              cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<BN>::SMEM);
}

}  // namespace tc

int gemm_tc_smem_bytes(int bn) {
  switch (bn) {
    case 64: return tc::Cfg<64>::SMEM;
    case 128: return tc::Cfg<128>::SMEM;
    case 256: return tc::Cfg<256>::SMEM;
  }
  return -1;
}

#define OOO_TC_ALL(X)                                                   \
  X(64, false, true, EPI_FWD) X(128, false, true, EPI_FWD) X(256, false, true, EPI_FWD) \
  X(64, false, false, EPI_DGRAD) X(128, false, false, EPI_DGRAD) X(256, false, false, EPI_DGRAD) \
  X(64, true, true, EPI_WGRAD) X(128, true, true, EPI_WGRAD) X(256, true, true, EPI_WGRAD)

cudaError_t gemm_tc_init() {
  cudaError_t e = cudaSuccess;
#define OOO_SET(BN, AM, BMJ, EP) \
  if (e == cudaSuccess) e = tc::set_attr<BN, AM, BMJ, EP>();
  OOO_TC_ALL(OOO_SET)
#undef OOO_SET
  return e;
}

cudaError_t launch_gemm_tc(int epi, int bn, const CUtensorMap *tmA, const CUtensorMap *tmB,
                           const EpiArgs &args, dim3 grid, const LaunchCtx &ctx) {
#define OOO_DISPATCH(BN, AM, BMJ, EP) \
  if (epi == EP && bn == BN) return tc::launch_one<BN, AM, BMJ, EP>(tmA, tmB, args, grid, ctx);
  OOO_TC_ALL(OOO_DISPATCH)
#undef OOO_DISPATCH
  return cudaErrorInvalidValue;
}

}  // namespace ooo
