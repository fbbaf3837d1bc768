// Shared sm_100a device helpers (PTX wrappers for mbarrier / TMA / tcgen05 /
// PDL, UMMA descriptors, epilogue math) used by engine.cu (the persistent
// dataflow kernel of the bf16 path).
#pragma once
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
constexpr int kSmemBudget = 227 * 1024;

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
// L2 prefetch of one 2-D box (no shared memory, no barrier: a hint).
__device__ __forceinline__ void tma_prefetch_l2_2d(const CUtensorMap *map, int c0, int c1) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(c0), "r"(c1)
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
// Split form for software pipelining: issue the load, do other work, then
// wait.  The wait names the destination registers as read-write operands so
// that the compiler cannot move their uses above it.
__device__ __forceinline__ void tmem_ld32_issue(uint32_t taddr, uint32_t (&r)[32]) {
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
}
__device__ __forceinline__ void tmem_ld_wait(uint32_t (&r)[32]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]),
                 "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]),
                 "+r"(r[14]), "+r"(r[15]), "+r"(r[16]), "+r"(r[17]), "+r"(r[18]), "+r"(r[19]),
                 "+r"(r[20]), "+r"(r[21]), "+r"(r[22]), "+r"(r[23]), "+r"(r[24]), "+r"(r[25]),
                 "+r"(r[26]), "+r"(r[27]), "+r"(r[28]), "+r"(r[29]), "+r"(r[30]), "+r"(r[31])
               :
               : "memory");
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
__device__ __forceinline__ uint32_t idesc_rt(int bn, bool a_mn, bool b_mn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) | ((b_mn ? 1u : 0u) << 16) |
         ((uint32_t)(bn >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

// ------------------------------------------------------------ epilogue math
// Phi(z) (standard normal CDF) and e^{-z^2/2} with one exponential:
// erf(x) = 1 - t (a1 + t (a2 + ...)) e^{-x^2}, t = 1 / (1 + p x), x = |z| / sqrt(2)
// (Abramowitz & Stegun 7.1.26, |error| <= 1.5e-7 -- three orders below the
// bf16 rounding applied to every GELU output).  Branch-free, unlike erff.
__device__ __forceinline__ void gauss_cdf_exp(float z, float &Phi, float &ez) {
  const float x = fabsf(z) * 0.70710678118654752f;
  float t;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(t) : "f"(fmaf(0.3275911f, x, 1.f)));   // 1 ulp, no slow path
  const float poly =
      t * fmaf(t, fmaf(t, fmaf(t, fmaf(t, 1.061405429f, -1.453152027f), 1.421413741f), -0.284496736f),
               0.254829592f);
  ez = __expf(-0.5f * z * z);
  const float erf_abs = fmaf(-poly, ez, 1.f);
  Phi = 0.5f * (1.f + copysignf(erf_abs, z));
}
__device__ __forceinline__ float act_f(int act, float z) {
  if (act == ACT_RELU) return z > 0.f ? z : 0.f;
  if (act == ACT_GELU) {
    float Phi, ez;
    gauss_cdf_exp(z, Phi, ez);
    return z * Phi;                                   // gelu(z) = z Phi(z)
  }
  return z;
}
__device__ __forceinline__ float act_grad_f(int act, float z) {
  if (act == ACT_DSTORED) return z;                   // z already holds act'(Z)
  if (act == ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == ACT_GELU) {
    float Phi, ez;
    gauss_cdf_exp(z, Phi, ez);
    return fmaf(z * 0.39894228040143268f, ez, Phi);   // gelu'(z) = Phi(z) + z phi(z)
  }
  return 1.f;
}
// Whole-chunk activation / activation-gradient with the act switch hoisted
// out of the element loop (act must be a register value, not a param-space
// reference: the asm memory clobbers elsewhere would force a reload per element).
__device__ __forceinline__ void act_chunk32(int act, float (&v)[32]) {
  if (act == ACT_GELU) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      float Phi, ez;
      gauss_cdf_exp(v[i], Phi, ez);
      v[i] *= Phi;
    }
  } else if (act == ACT_RELU) {
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = fmaxf(v[i], 0.f);
  }
}
// GELU of a chunk, also returning gelu'(z) = Phi(z) + z phi(z) in d (the
// derivative the backward multiplies by; shares Phi and e^{-z^2/2}).
__device__ __forceinline__ void gelu_and_grad_chunk32(float (&v)[32], float (&d)[32]) {
#pragma unroll
  for (int i = 0; i < 32; ++i) {
    float Phi, ez;
    gauss_cdf_exp(v[i], Phi, ez);
    d[i] = fmaf(v[i] * 0.39894228040143268f, ez, Phi);
    v[i] *= Phi;
  }
}
__device__ __forceinline__ void act_grad_mul_chunk32(int act, float (&v)[32], const float (&z)[32]) {
  if (act == ACT_DSTORED) {
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] *= z[i];
  } else if (act == ACT_GELU) {
#pragma unroll
    for (int i = 0; i < 32; ++i) {
      float Phi, ez;
      gauss_cdf_exp(z[i], Phi, ez);
      v[i] *= fmaf(z[i] * 0.39894228040143268f, ez, Phi);
    }
  } else if (act == ACT_RELU) {
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = z[i] > 0.f ? v[i] : 0.f;
  }
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
// RNE to bf16 and back, two values per F2FP.PACK_AB (the scalar
// __float2bfloat16_rn compiles to the slower F2F.BF16.F32 on sm_100).
__device__ __forceinline__ void round_bf16x32(float (&f)[32]) {
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    const uint32_t u = pack_bf2(f[2 * j], f[2 * j + 1]);
    f[2 * j] = __uint_as_float(u << 16);
    f[2 * j + 1] = __uint_as_float(u & 0xFFFF0000u);
  }
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

// --------------------------------------------------------- TMA store helpers
__device__ __forceinline__ void tma_store_2d(const CUtensorMap *map, uint32_t src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}
__device__ __forceinline__ void tma_store_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}
__device__ __forceinline__ void tma_store_wait_all() {
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}
// Stage one warp's 32 rows x 64 columns (bf16) into a 4 KiB 128B-swizzled
// buffer (16-B chunk c of row r at chunk c ^ (r & 7): conflict-free) and let
// one lane issue the TMA bulk store of box {64 cols, 32 rows} at (col0, row0).
// Rows >= M and columns >= N are clipped by the TMA unit.
__device__ __forceinline__ void stage_store(const CUtensorMap *map, uint32_t buf, int lane,
                                            const float (&v)[64], int col0, int row0) {
  if (lane == 0) tma_store_wait_read();    // previous store finished reading the buffer
  __syncwarp();
  const uint32_t rbase = buf + lane * 128;
#pragma unroll
  for (int c = 0; c < 8; ++c) {
    const uint32_t a = rbase + ((c ^ (lane & 7)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a),
                 "r"(pack_bf2(v[8 * c + 0], v[8 * c + 1])), "r"(pack_bf2(v[8 * c + 2], v[8 * c + 3])),
                 "r"(pack_bf2(v[8 * c + 4], v[8 * c + 5])), "r"(pack_bf2(v[8 * c + 6], v[8 * c + 7]))
                 : "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
  if (lane == 0) tma_store_2d(map, buf, col0, row0);
}
#ifndef OOO_STG256
#define OOO_STG256 1   // 32-B global stores (STG.256), 2 lanes per 64-B row segment (0: 16-B stores)
#endif
// Read back a warp's 32 x 32 bf16 transpose buffer (row r at buf + 64 r,
// 16-B chunk c at (c ^ ((r >> 1) & 3)) << 4) and store it row-major.
__device__ __forceinline__ void readback_store32(__nv_bfloat16 *g, int ldc, uint32_t buf, int lane, int col0,
                                                 int row0, int M) {
#if OOO_STG256
  const int c = (lane & 1) * 2;
#pragma unroll
  for (int k = 0; k < 2; ++k) {
    const int r = (lane >> 1) + 16 * k;
    uint32_t x0, y0, z0, w0, x1, y1, z1, w1;
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(x0), "=r"(y0), "=r"(z0), "=r"(w0)
                 : "r"(buf + r * 64 + ((c ^ ((r >> 1) & 3)) << 4))
                 : "memory");
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(x1), "=r"(y1), "=r"(z1), "=r"(w1)
                 : "r"(buf + r * 64 + (((c + 1) ^ ((r >> 1) & 3)) << 4))
                 : "memory");
    const int grow = row0 + r;
    if (grow < M)
      asm volatile("st.global.v8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"l"(
                       g + (size_t)grow * ldc + col0 + c * 8),
                   "r"(x0), "r"(y0), "r"(z0), "r"(w0), "r"(x1), "r"(y1), "r"(z1), "r"(w1)
                   : "memory");
  }
#else
  const int c = lane & 3;
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int r = (lane >> 2) + 8 * k;
    uint32_t x, y, z, w;
    asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(x), "=r"(y), "=r"(z), "=r"(w)
                 : "r"(buf + r * 64 + ((c ^ ((r >> 1) & 3)) << 4))
                 : "memory");
    const int grow = row0 + r;
    if (grow < M) *reinterpret_cast<uint4 *>(g + (size_t)grow * ldc + col0 + c * 8) = make_uint4(x, y, z, w);
  }
#endif
}
// Store one warp's 32 rows x 32 columns (bf16, lane = row) to a row-major
// global tensor through a 2 KiB per-warp smem transpose: lanes write their
// row (4 x 16 B, 64B-swizzled -> conflict-free), then read back so that
// each pair of lanes (4 lanes with OOO_STG256=0) owns one 64-B row segment
// -> fully coalesced st.global.v8 (v4).  No async engine involved (TMA bulk stores would queue
// behind the producer's TMA loads), so nothing to wait for.
__device__ __forceinline__ void store32_rows(__nv_bfloat16 *g, int ldc, uint32_t buf, int lane,
                                             const float (&v)[32], int col0, int row0, int M) {
  __syncwarp();                            // previous read-back of buf finished
  const uint32_t rbase = buf + lane * 64;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const uint32_t a = rbase + ((c ^ ((lane >> 1) & 3)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a),
                 "r"(pack_bf2(v[8 * c + 0], v[8 * c + 1])), "r"(pack_bf2(v[8 * c + 2], v[8 * c + 3])),
                 "r"(pack_bf2(v[8 * c + 4], v[8 * c + 5])), "r"(pack_bf2(v[8 * c + 6], v[8 * c + 7]))
                 : "memory");
  }
  __syncwarp();
  readback_store32(g, ldc, buf, lane, col0, row0, M);
}
// store32_rows for values already packed to bf16 pairs (u[j] = columns 2j, 2j+1).
__device__ __forceinline__ void store32_rows_packed(__nv_bfloat16 *g, int ldc, uint32_t buf, int lane,
                                                    const uint32_t (&u)[16], int col0, int row0, int M) {
  __syncwarp();
  const uint32_t rbase = buf + lane * 64;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const uint32_t a = rbase + ((c ^ ((lane >> 1) & 3)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(u[4 * c]), "r"(u[4 * c + 1]),
                 "r"(u[4 * c + 2]), "r"(u[4 * c + 3])
                 : "memory");
  }
  __syncwarp();
  readback_store32(g, ldc, buf, lane, col0, row0, M);
}
__device__ __forceinline__ void pack32(const float (&f)[32], uint32_t (&u)[16]) {
#pragma unroll
  for (int j = 0; j < 16; ++j) u[j] = pack_bf2(f[2 * j], f[2 * j + 1]);
}
__device__ __forceinline__ void unpack32(const uint32_t (&u)[16], float (&f)[32]) {
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    f[2 * j] = __uint_as_float(u[j] << 16);
    f[2 * j + 1] = __uint_as_float(u[j] & 0xFFFF0000u);
  }
}
// Same for 32 rows x 32 columns into a 2 KiB 64B-swizzled buffer (16-B chunk
// c of 64-B row r at chunk c ^ ((r >> 1) & 3): conflict-free), box {32, 32}.
__device__ __forceinline__ void stage_store32(const CUtensorMap *map, uint32_t buf, int lane,
                                              const float (&v)[32], int col0, int row0) {
  if (lane == 0) tma_store_wait_read();
  __syncwarp();
  const uint32_t rbase = buf + lane * 64;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const uint32_t a = rbase + ((c ^ ((lane >> 1) & 3)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a),
                 "r"(pack_bf2(v[8 * c + 0], v[8 * c + 1])), "r"(pack_bf2(v[8 * c + 2], v[8 * c + 3])),
                 "r"(pack_bf2(v[8 * c + 4], v[8 * c + 5])), "r"(pack_bf2(v[8 * c + 6], v[8 * c + 7]))
                 : "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
  if (lane == 0) tma_store_2d(map, buf, col0, row0);
}

// stage_store32 for values already packed to bf16 pairs.
__device__ __forceinline__ void stage_store32_packed(const CUtensorMap *map, uint32_t buf, int lane,
                                                     const uint32_t (&u)[16], int col0, int row0) {
  if (lane == 0) tma_store_wait_read();
  __syncwarp();
  const uint32_t rbase = buf + lane * 64;
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const uint32_t a = rbase + ((c ^ ((lane >> 1) & 3)) << 4);
    asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(u[4 * c]), "r"(u[4 * c + 1]),
                 "r"(u[4 * c + 2]), "r"(u[4 * c + 3])
                 : "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();
  if (lane == 0) tma_store_2d(map, buf, col0, row0);
}

}  // namespace tc
}  // namespace ooo
