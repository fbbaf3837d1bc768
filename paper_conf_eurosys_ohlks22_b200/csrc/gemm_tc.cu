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
// Persistent, warp-specialised kernel: each CTA walks output tiles
// t = blockIdx.x, blockIdx.x + gridDim.x, ... (128 x BN tiles, optional
// split-K units), so the prologue (barrier init, TMEM alloc, descriptor
// prefetch) is paid once per CTA and the epilogue of tile j overlaps the
// mainloop of tile j+1 through a double-buffered TMEM accumulator:
//   warp 0 lane 0 : TMA producer, STAGES-deep smem ring (128B swizzle)
//   warp 1        : TMEM allocator (2 x BN columns); lane 0 issues
//                   tcgen05.mma (M=128, N=BN, K=16) into accumulator j&1
//   warps 2..5    : epilogue -- tcgen05.ld 32x32b.x32 -> registers -> fused
//                   bias / activation / act-grad / bias-grad / scale -> global
// Programmatic dependent launch: every thread waits (griddepcontrol.wait)
// for the previous kernel in the stream only after its prologue, and the
// next kernel is released (launch_dependents) right away, so back-to-back
// layer kernels overlap their launch + prologue with the predecessor's tail.
// Operand majors: A K-major (X_i, dZ_i as A of F_i / dO_i) or MN-major
// (X_i^T as A of dW_i); B MN-major (W_i in F_i, dZ_i in dW_i) or K-major
// (W_i^T in dO_i).  16-bit types allow MN-major operands directly, so no
// transpose kernels are needed.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "kernels.h"
#include "tc_common.cuh"

namespace ooo {
namespace tc {

#ifdef OOO_TRACE
// Debug-only phase timestamps (tools/gemm_probe.cu): [cta][8] globaltimer ns.
__device__ unsigned long long *g_trace = nullptr;
__device__ __forceinline__ void trace(int slot) {
  if (g_trace) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_trace[blockIdx.x * 8 + slot] = t;
  }
}
#else
__device__ __forceinline__ void trace(int) {}
#endif

constexpr int kThreads = 192;

template <int BN> struct Cfg {
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STG_BYTES = 4 * 4096;                 // 4 epilogue warps x (32 rows x 128 B)
  static constexpr int STAGES_RAW = (kSmemBudget - 1024 - STG_BYTES - 6 * 1024) / STAGE;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  static constexpr int RING = STAGE * STAGES;
  static constexpr int TMEM_COLS = (2 * BN <= 64) ? 64 : (2 * BN <= 128 ? 128 : (2 * BN <= 256 ? 256 : 512));
  // ring | staging [4][4 KiB] | full[S] | empty[S] | tfull[2] | tempty[2] | tmem slot | bias[BN] | red[4][BN]
  static constexpr int STG_OFF = RING;                       // 1024-aligned (STAGE % 1024 == 0)
  static constexpr int BAR_OFF = STG_OFF + STG_BYTES;
  static constexpr int SLOT_OFF = BAR_OFF + (2 * STAGES + 4) * 8;
  static constexpr int BIAS_OFF = (SLOT_OFF + 16 + 15) / 16 * 16;
  static constexpr int RED_OFF = BIAS_OFF + BN * 4;
  static constexpr int SMEM = RED_OFF + 4 * BN * 4 + 1024;   // + alignment slack
  static_assert(SMEM <= kSmemBudget, "smem budget");
  static_assert(STAGE % 1024 == 0, "stage alignment");
};

struct TileIdx {
  int m0, n0, split, kb_begin, nkb;
};
__device__ __forceinline__ TileIdx decode(int t, int mt, int nt, int BN, const EpiArgs &a) {
  TileIdx r;
  const int per = mt * nt;
  r.split = t / per;
  const int rem = t - r.split * per;
  r.m0 = (rem % mt) * BM;
  r.n0 = (rem / mt) * BN;
  const int nkb_total = (a.K + BK - 1) / BK;
  r.kb_begin = r.split * a.kb_per_split;
  int kb_end = r.kb_begin + a.kb_per_split;
  if (kb_end > nkb_total) kb_end = nkb_total;
  r.nkb = kb_end - r.kb_begin;
  return r;
}

// ------------------------------------------------------------------ kernel
// tmA, tmB: operand loads.  tmZ / tmX: bf16 output stores (Z_i and X_{i+1}
// for F_i; dZ_{i-1} or dX for dO_i; the gradient bucket for dW_i with one
// split).  Split-K partials (fp32) use direct vector stores.
template <int BN, bool A_MN, bool B_MN, int EPI>
__global__ void __launch_bounds__(kThreads, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmZ, const __grid_constant__ CUtensorMap tmX,
                   const EpiArgs args) {
  using C = Cfg<BN>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                              ~static_cast<uintptr_t>(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar_full = sbase + C::BAR_OFF;
  const uint32_t bar_empty = bar_full + 8 * C::STAGES;
  const uint32_t bar_tfull = bar_empty + 8 * C::STAGES;
  const uint32_t bar_tempty = bar_tfull + 16;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + C::SLOT_OFF);
  float *bias_s = reinterpret_cast<float *>(smem + C::BIAS_OFF);
  float *red = reinterpret_cast<float *>(smem + C::RED_OFF);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const int mt = (args.M + BM - 1) / BM;
  const int nt = (args.N + BN - 1) / BN;
  const int units = mt * nt * args.splits;
  constexpr bool kWeightB = (EPI != EPI_WGRAD);   // B = W_i: not written by the previous kernel
  if (threadIdx.x == 0) trace(0);

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_empty + 8 * s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(bar_tfull + 8 * a, 1);
      mbar_init(bar_tempty + 8 * a, 4);    // one arrive per epilogue warp
    }
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
  if (threadIdx.x == 0) trace(1);

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      // Weights do not depend on the previous kernel: start streaming the
      // first tile's B operand before the programmatic-dependency wait.
      int pre = 0;
      if (kWeightB && (int)blockIdx.x < units) {
        const TileIdx t0 = decode(blockIdx.x, mt, nt, BN, args);
        pre = t0.nkb < C::STAGES ? t0.nkb : C::STAGES;
        for (int kb = 0; kb < pre; ++kb) {
          const uint32_t fb = bar_full + 8 * kb;
          mbar_expect_tx(fb, C::STAGE);
          const uint32_t sb = sbase + kb * C::STAGE + A_BYTES;
          const int k0 = (t0.kb_begin + kb) * BK;
          if (!B_MN) {
            tma_load_2d(sb, &tmB, fb, k0, t0.n0);
          } else {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + 8192 * j, &tmB, fb, t0.n0 + 64 * j, k0);
          }
        }
      }
      pdl_wait();
      pdl_launch_dependents();
      if (threadIdx.x == 0) trace(2);
      int it = 0;
      for (int t = blockIdx.x; t < units; t += gridDim.x) {
        const TileIdx ti = decode(t, mt, nt, BN, args);
        for (int kb = 0; kb < ti.nkb; ++kb, ++it) {
          const int s = it % C::STAGES;
          const bool b_done = it < pre;
          if (it >= C::STAGES) mbar_wait(bar_empty + 8 * s, ((it / C::STAGES) - 1) & 1);
          const uint32_t fb = bar_full + 8 * s;
          if (!b_done) mbar_expect_tx(fb, C::STAGE);
          const uint32_t sa = sbase + s * C::STAGE;
          const uint32_t sb = sa + A_BYTES;
          const int k0 = (ti.kb_begin + kb) * BK;
          if (!A_MN) {
            tma_load_2d(sa, &tmA, fb, k0, ti.m0);                 // box {64 K, 128 M}
          } else {
            tma_load_2d(sa, &tmA, fb, ti.m0, k0);                 // box {64 M, 64 K}
            tma_load_2d(sa + 8192, &tmA, fb, ti.m0 + 64, k0);
          }
          if (!b_done) {
            if (!B_MN) {
              tma_load_2d(sb, &tmB, fb, k0, ti.n0);               // box {64 K, BN N}
            } else {
#pragma unroll
              for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + 8192 * j, &tmB, fb, ti.n0 + 64 * j, k0);
            }
          }
        }
      }
    } else {
      pdl_wait();
      pdl_launch_dependents();
    }
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
    pdl_wait();
    pdl_launch_dependents();
    if (lane == 0) {
      constexpr uint32_t ID = idesc<BN, A_MN, B_MN>();
      int it = 0, j = 0;
      for (int t = blockIdx.x; t < units; t += gridDim.x, ++j) {
        const TileIdx ti = decode(t, mt, nt, BN, args);
        const int acc = j & 1;
        if (j >= 2) mbar_wait(bar_tempty + 8 * acc, ((j >> 1) - 1) & 1);   // epilogue drained it
        fence_after();
        const uint32_t dtm = tmem + (uint32_t)(acc * BN);
        for (int kb = 0; kb < ti.nkb; ++kb, ++it) {
          const int s = it % C::STAGES;
          mbar_wait(bar_full + 8 * s, (it / C::STAGES) & 1);
          if (it == 0) trace(3);
          fence_after();
          const uint32_t sa = sbase + s * C::STAGE;
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            const uint64_t ad = A_MN ? sdesc(sa + kk * 2048, 8192, 1024) : sdesc(sa + kk * 32, 16, 1024);
            const uint64_t bd = B_MN ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
            umma_bf16(dtm, ad, bd, ID, (kb | kk) != 0 ? 1u : 0u);
          }
          umma_commit(bar_empty + 8 * s);     // smem slot free once these MMAs retire
        }
        umma_commit(bar_tfull + 8 * acc);     // accumulator complete
      }
      trace(4);
    }
    __syncwarp();
  } else {
    // ===================== epilogue (warps 2..5) =====================
    pdl_wait();
    pdl_launch_dependents();
    const int q = warp & 3;                  // TMEM lane quarter this warp may access
    const int et = threadIdx.x - 64;         // 0..127
    const uint32_t stg = sbase + C::STG_OFF + q * 4096;
    int j = 0;
    for (int t = blockIdx.x; t < units; t += gridDim.x, ++j) {
      const TileIdx ti = decode(t, mt, nt, BN, args);
      const int acc = j & 1;
      const int row0 = ti.m0 + q * 32;
      const int row = row0 + lane;
      const bool row_ok = row < args.M;
      if (EPI == EPI_FWD) {
        // stage the tile's bias in smem while the MMAs run
        epi_bar();                                           // previous tile done reading bias_s
        for (int c = et; c < BN; c += 128) {
          const int n = ti.n0 + c;
          bias_s[c] = n < args.N ? __bfloat162float(reinterpret_cast<const __nv_bfloat16 *>(args.bias)[n]) : 0.f;
        }
        epi_bar();
      }
      const bool have = ti.nkb > 0;
      if (have) {
        mbar_wait(bar_tfull + 8 * acc, (j >> 1) & 1);
        fence_after();
      }
      if (et == 0 && j == 0) trace(5);
      const __nv_bfloat16 *zrow =
          reinterpret_cast<const __nv_bfloat16 *>(args.zin) + (size_t)row * args.ldc + ti.n0;
      const bool need_z = (EPI == EPI_DGRAD) && args.act != ACT_ID && row_ok;
      uint4 zraw[8];
      if (need_z) {
        ld_raw32(zrow, *reinterpret_cast<uint4(*)[4]>(&zraw[0]));
        ld_raw32(zrow + 32, *reinterpret_cast<uint4(*)[4]>(&zraw[4]));
      }
#pragma unroll 1
      for (int c = 0; c < BN / 64; ++c) {
        const int col0 = ti.n0 + c * 64;
        if (col0 >= args.N) break;             // warp-uniform (N % 64 == 0)
        float v[64];
        if (have) {
          uint32_t r[32];
          const uint32_t ta = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * BN + c * 64);
          tmem_ld32(ta, r);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
          tmem_ld32(ta + 32, r);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[32 + i] = __uint_as_float(r[i]);
        } else {
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = 0.f;
        }
        if (EPI == EPI_FWD) {
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = __bfloat162float(__float2bfloat16_rn(v[i] + bias_s[c * 64 + i]));
          if (args.z_out) stage_store(&tmZ, stg, lane, v, col0, row0);     // Z_i storage point
          if (args.act != ACT_ID) {
#pragma unroll
            for (int i = 0; i < 64; ++i) v[i] = act_f(args.act, v[i]);
          }
          stage_store(&tmX, stg, lane, v, col0, row0);                       // X_{i+1}
        } else if (EPI == EPI_DGRAD) {
          if (args.act != ACT_ID) {
            float z[64];
            if (need_z) {
              unpack_bf16x32(*reinterpret_cast<uint4(*)[4]>(&zraw[0]), *reinterpret_cast<float(*)[32]>(&z[0]));
              unpack_bf16x32(*reinterpret_cast<uint4(*)[4]>(&zraw[4]), *reinterpret_cast<float(*)[32]>(&z[32]));
              if (c + 1 < BN / 64 && col0 + 64 < args.N) {                  // prefetch next chunk
                ld_raw32(zrow + (c + 1) * 64, *reinterpret_cast<uint4(*)[4]>(&zraw[0]));
                ld_raw32(zrow + (c + 1) * 64 + 32, *reinterpret_cast<uint4(*)[4]>(&zraw[4]));
              }
            } else {
#pragma unroll
              for (int i = 0; i < 64; ++i) z[i] = 0.f;
            }
#pragma unroll
            for (int i = 0; i < 64; ++i) v[i] *= act_grad_f(args.act, z[i]);
          }
#pragma unroll
          for (int i = 0; i < 64; ++i) v[i] = row_ok ? __bfloat162float(__float2bfloat16_rn(v[i])) : 0.f;
          stage_store(&tmX, stg, lane, v, col0, row0);                       // dZ_{i-1} storage point
          if (args.dbpart) {
            float* h0 = reinterpret_cast<float(*)>(&v[0]);
            const float s0 = warp_colsum32(*reinterpret_cast<float(*)[32]>(h0), lane);
            const float s1 = warp_colsum32(*reinterpret_cast<float(*)[32]>(h0 + 32), lane);
            red[q * BN + c * 64 + lane] = s0;
            red[q * BN + c * 64 + 32 + lane] = s1;
          }
        } else {  // EPI_WGRAD
          if (args.splits == 1) {
#pragma unroll
            for (int i = 0; i < 64; ++i) v[i] *= args.alpha;
            stage_store(&tmX, stg, lane, v, col0, row0);                     // gradient bucket
          } else if (row_ok) {
            float4 *dst = reinterpret_cast<float4 *>(args.fpart + (size_t)ti.split * args.M * args.ldc +
                                                     (size_t)row * args.ldc + col0);
#pragma unroll
            for (int i = 0; i < 16; ++i) dst[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
          }
        }
      }
      // accumulator buffer may be reused by the MMA warp
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(bar_tempty + 8 * acc);
      if (EPI == EPI_DGRAD && args.dbpart) {
        // sum the four row quarters in fixed order q = 0..3 (deterministic)
        epi_bar();
        for (int cc = et; cc < BN; cc += 128) {
          const int col = ti.n0 + cc;
          if (col < args.N) {
            const float s = ((red[cc] + red[BN + cc]) + red[2 * BN + cc]) + red[3 * BN + cc];
            args.dbpart[(size_t)(ti.m0 / BM) * args.N + col] = s;
          }
        }
        epi_bar();
      }
    }
    if (lane == 0) tma_store_wait_all();     // bulk stores complete before the grid retires
    __syncwarp();
  }
  if (threadIdx.x == 64) trace(6);
  fence_before();
  __syncthreads();
  if (threadIdx.x == 0) trace(7);
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem),
                 "r"((uint32_t)C::TMEM_COLS)
                 : "memory");
  }
}

template <int BN, bool A_MN, bool B_MN, int EPI>
cudaError_t launch_one(const CUtensorMap *tmA, const CUtensorMap *tmB, const CUtensorMap *tmZ,
                       const CUtensorMap *tmX, const EpiArgs &args, int ctas, const LaunchCtx &ctx) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(ctas, 1, 1);
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.dynamicSmemBytes = Cfg<BN>::SMEM;
  cfg.stream = ctx.stream;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = ctx.priority;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = ctx.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, gemm_tc_kernel<BN, A_MN, B_MN, EPI>, *tmA, *tmB, *tmZ, *tmX, args);
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
    case 192: return tc::Cfg<192>::SMEM;
    case 256: return tc::Cfg<256>::SMEM;
  }
  return -1;
}

#define OOO_TC_BN(X, AM, BMJ, EP) X(64, AM, BMJ, EP) X(128, AM, BMJ, EP) X(192, AM, BMJ, EP) X(256, AM, BMJ, EP)
#define OOO_TC_ALL(X) \
  OOO_TC_BN(X, false, true, EPI_FWD) OOO_TC_BN(X, false, false, EPI_DGRAD) OOO_TC_BN(X, true, true, EPI_WGRAD)

cudaError_t gemm_tc_init() {
  cudaError_t e = cudaSuccess;
#define OOO_SET(BN, AM, BMJ, EP) \
  if (e == cudaSuccess) e = tc::set_attr<BN, AM, BMJ, EP>();
  OOO_TC_ALL(OOO_SET)
#undef OOO_SET
  return e;
}

cudaError_t launch_gemm_tc(int epi, int bn, const CUtensorMap *tmA, const CUtensorMap *tmB,
                           const CUtensorMap *tmZ, const CUtensorMap *tmX, const EpiArgs &args, int ctas,
                           const LaunchCtx &ctx) {
#define OOO_DISPATCH(BN, AM, BMJ, EP) \
  if (epi == EP && bn == BN) return tc::launch_one<BN, AM, BMJ, EP>(tmA, tmB, tmZ, tmX, args, ctas, ctx);
  OOO_TC_ALL(OOO_DISPATCH)
#undef OOO_DISPATCH
  return cudaErrorInvalidValue;
}

}  // namespace ooo
