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

namespace ooo {
namespace tc {

constexpr int BM = 128;
constexpr int BK = 64;                 // 64 bf16 = 128 B = one swizzle row
constexpr int A_BYTES = BM * BK * 2;   // 16 KiB
constexpr int kThreads = 192;
constexpr int kSmemBudget = 227 * 1024;

template <int BN> struct Cfg {
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE = A_BYTES + B_BYTES;
  static constexpr int STAGES_RAW = (kSmemBudget - 8 * 1024) / STAGE;
  static constexpr int STAGES = STAGES_RAW > 8 ? 8 : STAGES_RAW;
  static constexpr int RING = STAGE * STAGES;
  static constexpr int TMEM_COLS = (2 * BN <= 64) ? 64 : (2 * BN <= 128 ? 128 : (2 * BN <= 256 ? 256 : 512));
  // ring | full[S] | empty[S] | tfull[2] | tempty[2] | tmem slot | bias[BN] f32 | red[4][BN] f32
  static constexpr int BAR_OFF = RING;
  static constexpr int SLOT_OFF = BAR_OFF + (2 * STAGES + 4) * 8;
  static constexpr int BIAS_OFF = (SLOT_OFF + 16 + 15) / 16 * 16;
  static constexpr int RED_OFF = BIAS_OFF + BN * 4;
  static constexpr int SMEM = RED_OFF + 4 * BN * 4 + 1024;   // + alignment slack
  static_assert(SMEM <= kSmemBudget, "smem budget");
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
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
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
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

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
__device__ __forceinline__ void unpack_bf16x32(const uint4 (&u)[4], float (&f)[32]) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    f[8 * j + 0] = bf_lo(u[j].x); f[8 * j + 1] = bf_hi(u[j].x);
    f[8 * j + 2] = bf_lo(u[j].y); f[8 * j + 3] = bf_hi(u[j].y);
    f[8 * j + 4] = bf_lo(u[j].z); f[8 * j + 5] = bf_hi(u[j].z);
    f[8 * j + 6] = bf_lo(u[j].w); f[8 * j + 7] = bf_hi(u[j].w);
  }
}
__device__ __forceinline__ void ld_raw32(const __nv_bfloat16 *p, uint4 (&u)[4]) {
  const uint4 *q = reinterpret_cast<const uint4 *>(p);
#pragma unroll
  for (int j = 0; j < 4; ++j) u[j] = __ldg(q + j);
}
// store 32 fp32 as bf16 (RNE)
__device__ __forceinline__ void st_bf16x32(__nv_bfloat16 *p, const float (&f)[32]) {
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
  // everything above overlaps the previous kernel's tail (PDL)
  pdl_wait();
  pdl_launch_dependents();

  if (warp == 0) {
    // ===================== TMA producer =====================
    if (lane == 0) {
      int it = 0;
      for (int t = blockIdx.x; t < units; t += gridDim.x) {
        const TileIdx ti = decode(t, mt, nt, BN, args);
        for (int kb = 0; kb < ti.nkb; ++kb, ++it) {
          const int s = it % C::STAGES;
          if (it >= C::STAGES) mbar_wait(bar_empty + 8 * s, ((it / C::STAGES) - 1) & 1);
          const uint32_t fb = bar_full + 8 * s;
          mbar_expect_tx(fb, C::STAGE);
          const uint32_t sa = sbase + s * C::STAGE;
          const uint32_t sb = sa + A_BYTES;
          const int k0 = (ti.kb_begin + kb) * BK;
          if (!A_MN) {
            tma_load_2d(sa, &tmA, fb, k0, ti.m0);                 // box {64 K, 128 M}
          } else {
            tma_load_2d(sa, &tmA, fb, ti.m0, k0);                 // box {64 M, 64 K}
            tma_load_2d(sa + 8192, &tmA, fb, ti.m0 + 64, k0);
          }
          if (!B_MN) {
            tma_load_2d(sb, &tmB, fb, k0, ti.n0);                 // box {64 K, BN N}
          } else {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_2d(sb + 8192 * j, &tmB, fb, ti.n0 + 64 * j, k0);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ===================== MMA issuer =====================
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
    }
    __syncwarp();
  } else {
    // ===================== epilogue (warps 2..5) =====================
    const int q = warp & 3;                  // TMEM lane quarter this warp may access
    const int et = threadIdx.x - 64;         // 0..127
    int j = 0;
    for (int t = blockIdx.x; t < units; t += gridDim.x, ++j) {
      const TileIdx ti = decode(t, mt, nt, BN, args);
      const int acc = j & 1;
      const int row = ti.m0 + q * 32 + lane;
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
      uint4 zraw[4];
      const __nv_bfloat16 *zrow =
          reinterpret_cast<const __nv_bfloat16 *>(args.zin) + (size_t)row * args.ldc + ti.n0;
      const bool need_z = (EPI == EPI_DGRAD) && args.act != ACT_ID && row_ok;
      if (need_z) ld_raw32(zrow, zraw);
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        const int col0 = ti.n0 + c * 32;
        if (col0 >= args.N) break;             // warp-uniform (N % 32 == 0)
        float v[32];
        if (have) {
          uint32_t r[32];
          tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * BN + c * 32), r);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
        }
        const size_t off = (size_t)row * args.ldc + col0;
        if (EPI == EPI_FWD) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] += bias_s[c * 32 + i];
          round_bf16x32(v);                                    // Z_i storage point
          if (row_ok && args.z_out)
            st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.z_out) + off, v);
          if (args.act != ACT_ID) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = act_f(args.act, v[i]);
          }
          if (row_ok) st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
        } else if (EPI == EPI_DGRAD) {
          if (args.act != ACT_ID) {
            float z[32];
            if (need_z) {
              unpack_bf16x32(zraw, z);
              if (c + 1 < BN / 32 && col0 + 32 < args.N) ld_raw32(zrow + (c + 1) * 32, zraw);  // prefetch
            } else {
#pragma unroll
              for (int i = 0; i < 32; ++i) z[i] = 0.f;
            }
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] *= act_grad_f(args.act, z[i]);
          }
          round_bf16x32(v);                                    // dZ_{i-1} storage point
          if (row_ok) {
            st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] = 0.f;
          }
          if (args.dbpart) {
            const float s = warp_colsum32(v, lane);           // lane l: column col0 + l
            red[q * BN + c * 32 + lane] = s;
          }
        } else {  // EPI_WGRAD
          if (args.splits == 1) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] *= args.alpha;
            if (row_ok) st_bf16x32(reinterpret_cast<__nv_bfloat16 *>(args.x_out) + off, v);
          } else if (row_ok) {
            float4 *dst = reinterpret_cast<float4 *>(args.fpart + (size_t)ti.split * args.M * args.ldc + off);
#pragma unroll
            for (int i = 0; i < 8; ++i) dst[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
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
                       int ctas, const LaunchCtx &ctx) {
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
                           const EpiArgs &args, int ctas, const LaunchCtx &ctx) {
#define OOO_DISPATCH(BN, AM, BMJ, EP) \
  if (epi == EP && bn == BN) return tc::launch_one<BN, AM, BMJ, EP>(tmA, tmB, args, ctas, ctx);
  OOO_TC_ALL(OOO_DISPATCH)
#undef OOO_DISPATCH
  return cudaErrorInvalidValue;
}

}  // namespace ooo
