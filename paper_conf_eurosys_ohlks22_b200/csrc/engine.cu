// Persistent dataflow engine kernel (see engine.h for the design rationale).
//
// Roles per CTA (one CTA per SM, persistent):
//   warp 0 lane 0 : dispenser + TMA producer.  Takes the next task index
//                   (atomicAdd on the pass dispenser, so tiles are started in
//                   queue = priority order), publishes it to the other roles
//                   through a 4-deep smem task ring, waits until the task's
//                   input rows are complete (acquire on a completion counter,
//                   spin with timeout -> trap, never a silent hang), then
//                   streams its A / B k-blocks with TMA into the smem ring.
//   warp 1        : TMEM allocator; lane 0 issues tcgen05.mma (M=128, N=bn)
//                   into accumulator j & 1 (double-buffered, 2 x 256 cols).
//   warps 2..5    : epilogue of task j while task j+1's MMAs run: tcgen05.ld,
//                   fused bias/act (F_i), act-grad + bias-grad partials (dO_i),
//                   1/N scale + bias-grad reduction (dW_i), bf16 RNE, TMA bulk
//                   stores; then publish completion (release) to the counters.
// Deadlock freedom: tasks are dispensed in increasing index and every
// dependency of task t is a task with a smaller index, all CTAs are
// co-resident (grid <= #SMs, 1 CTA/SM), and each role processes its tasks in
// order; so the smallest unfinished task can always make progress.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "engine.h"
#include "kernels.h"
#include "tc_common.cuh"

namespace ooo {
namespace eng {

using namespace ooo::tc;

#ifdef OOO_TRACE
// Debug builds only (libooo_trace.so): per-task %globaltimer stamps
// [task][4] = dispensed, inputs ready (TMA issue starts), accumulator ready,
// completion published; plus the CTA that ran it in [task][4] high bits.
__device__ unsigned long long *g_etrace = nullptr;
__device__ __forceinline__ void etrace(int t, int slot) {
  if (g_etrace && t >= 0) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    g_etrace[(size_t)t * 4 + slot] = (v & 0xFFFFFFFFFFFFull) | ((unsigned long long)blockIdx.x << 48);
  }
}
#else
__device__ __forceinline__ void etrace(int, int) {}
#endif

constexpr int kEpiWarps = 8;
constexpr int kEpiThreads = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpiThreads;
constexpr int kMaxBN = 256;
constexpr int B_BYTES = kMaxBN * BK * 2;             // 32 KiB
constexpr int STAGE = A_BYTES + B_BYTES;             // 48 KiB
constexpr int STG_BYTES = kEpiWarps * 2048;
constexpr int STAGES = 4;
constexpr int Q = 4;                                 // task ring depth
constexpr int RING = STAGE * STAGES;
constexpr int STG_OFF = RING;
constexpr int BAR_OFF = STG_OFF + STG_BYTES;
// full[S] empty[S] tfull[2] tempty[2] taskfull[Q] taskempty[Q]
constexpr int SLOT_OFF = BAR_OFF + (2 * STAGES + 4 + 2 * Q) * 8;
constexpr int TASK_OFF = SLOT_OFF + 16;
constexpr int BIAS_OFF = (TASK_OFF + 4 * Q + 15) / 16 * 16;
constexpr int RED_OFF = BIAS_OFF + kMaxBN * 4;
constexpr int SMEM = RED_OFF + 4 * kMaxBN * 4 + 1024;
static_assert(SMEM <= kSmemBudget, "engine smem budget");
constexpr uint32_t TMEM_COLS = 512;

__device__ __forceinline__ void ebar() { asm volatile("bar.sync 1, %0;" ::"n"(kEpiThreads) : "memory"); }

__device__ __forceinline__ int ld_acquire(const int32_t *p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
// Polls use relaxed loads: an acquire at gpu scope invalidates the SM's L1
// (CCTL.IVALL) every time, which would hurt the epilogue warps' cached loads.
__device__ __forceinline__ int ld_relaxed(const int32_t *p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void red_release_add(int32_t *p, int v) {
  asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Wait until *p >= target.  A dependency that is not met within 4 s means a
// broken schedule: trap (the launch fails with an error) instead of hanging.
__device__ __forceinline__ void wait_ge(const int32_t *p, int target) {
  if (ld_relaxed(p) < target) {
    const uint64_t t0 = gtimer();
    while (ld_relaxed(p) < target) {
      __nanosleep(32);
      if (gtimer() - t0 > 4000000000ull) __trap();
    }
  }
  (void)ld_acquire(p);   // one acquire orders the producer tiles' stores before our reads
}

__device__ __forceinline__ const CUtensorMap *map_of(int idx, const CUtensorMap *maps,
                                                     const CUtensorMap *tmY, const CUtensorMap *tmDX) {
  if (idx >= 0) return maps + idx;
  return idx == MAP_Y ? tmY : tmDX;
}

// task index -> op (binary search over the ops' first task index)
__device__ __forceinline__ int op_of(const Params &p, int t) {
  int lo = 0, hi = p.nops - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (p.ops[mid].first <= t) lo = mid; else hi = mid - 1;
  }
  return lo;
}

struct TaskRt {
  int op, kind, layer, bn, nkb, m0, n0, M, N, mblk;
};
__device__ __forceinline__ TaskRt task_rt(const Params &p, int t) {
  TaskRt r;
  r.op = op_of(p, t);
  const Op &o = p.ops[r.op];
  const int rel = t - o.first;
  r.kind = o.kind;
  r.layer = o.layer;
  r.bn = o.bn;
  r.nkb = o.nkb;
  r.mblk = rel / o.nt;
  r.m0 = r.mblk * BM;
  r.n0 = (rel % o.nt) * o.bn;
  const LayerDev &L = p.layers[o.layer - 1];
  if (o.kind == EPI_FWD) { r.M = p.M; r.N = L.dout; }
  else if (o.kind == EPI_DGRAD) { r.M = p.M; r.N = L.din; }
  else { r.M = L.din; r.N = L.dout; }
  return r;
}

__global__ void __launch_bounds__(kThreads, 1)
    engine_kernel(const __grid_constant__ CUtensorMap tmY, const __grid_constant__ CUtensorMap tmDX,
                  const __grid_constant__ Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                              ~static_cast<uintptr_t>(1023));
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar_full = sbase + BAR_OFF;
  const uint32_t bar_empty = bar_full + 8 * STAGES;
  const uint32_t bar_tfull = bar_empty + 8 * STAGES;
  const uint32_t bar_tempty = bar_tfull + 16;
  const uint32_t bar_qfull = bar_tempty + 16;
  const uint32_t bar_qempty = bar_qfull + 8 * Q;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + SLOT_OFF);
  volatile int *task_slot = reinterpret_cast<volatile int *>(smem + TASK_OFF);
  float *bias_s = reinterpret_cast<float *>(smem + BIAS_OFF);
  float *red = reinterpret_cast<float *>(smem + RED_OFF);
  int32_t *ctr = p.ctr;
  const CounterLayout &cl = p.cl;
  int32_t *dispenser = ctr + (p.pass == 0 ? cl.fwd_base : cl.bwd_base);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_empty + 8 * s, 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(bar_tfull + 8 * a, 1);
      mbar_init(bar_tempty + 8 * a, kEpiWarps);   // one arrive per epilogue warp
    }
    for (int s = 0; s < Q; ++s) {
      mbar_init(bar_qfull + 8 * s, 1);
      mbar_init(bar_qempty + 8 * s, 2);   // MMA lane + epilogue leader
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();

  if (warp == 0) {
    // ============ dispenser + TMA producer ============
    if (lane == 0) {
      int it = 0;
      for (int j = 0;; ++j) {
        int t = atomicAdd(dispenser, 1);
        if (t >= p.ntasks) t = -1;
        etrace(t, 0);
        const int slot = j % Q;
        if (j >= Q) mbar_wait(bar_qempty + 8 * slot, ((j / Q) - 1) & 1);
        task_slot[slot] = t;
        mbar_arrive(bar_qfull + 8 * slot);
        if (t < 0) break;
        const TaskRt T = task_rt(p, t);
        const Op &o = p.ops[T.op];
        const LayerDev &Ld = p.layers[T.layer - 1];
        // ---- dependencies (all on tasks with smaller indices)
        if (T.kind == EPI_FWD) {
          if (T.layer > 1) {
            const LayerDev &Lp = p.layers[T.layer - 2];
            wait_ge(ctr + cl.fwd_base + 1 + (T.layer - 2) * cl.MT + T.mblk, Lp.fwd_nt);
          }
          if (p.gate_ar) wait_ge(ctr + cl.ar_done + Ld.bucket, 1);
        } else if (T.kind == EPI_DGRAD) {
          if (T.layer < cl.L) {
            const LayerDev &Ln = p.layers[T.layer];
            wait_ge(ctr + cl.dz_rows + (T.layer - 1) * cl.MT + T.mblk, Ln.dx_nt);
            if (p.in_order) wait_ge(ctr + cl.dw_done + T.layer, Ln.dw_tiles);
          }
        } else {
          if (T.layer < cl.L) {
            const LayerDev &Ln = p.layers[T.layer];
            wait_ge(ctr + cl.dz_total + (T.layer - 1), cl.MT * Ln.dx_nt);
          }
        }
        asm volatile("fence.proxy.async.global;" ::: "memory");   // TMA reads see the producers' data
        etrace(t, 1);
        const CUtensorMap *mA = map_of(o.mapA, p.maps, &tmY, &tmDX);
        const CUtensorMap *mB = map_of(o.mapB, p.maps, &tmY, &tmDX);
        const bool a_mn = T.kind == EPI_WGRAD;
        const bool b_mn = T.kind != EPI_DGRAD;
        const uint32_t bytes = A_BYTES + T.bn * BK * 2;
        for (int kb = 0; kb < T.nkb; ++kb, ++it) {
          const int s = it % STAGES;
          if (it >= STAGES) mbar_wait(bar_empty + 8 * s, ((it / STAGES) - 1) & 1);
          const uint32_t fb = bar_full + 8 * s;
          mbar_expect_tx(fb, bytes);
          const uint32_t sa = sbase + s * STAGE;
          const uint32_t sb = sa + A_BYTES;
          const int k0 = kb * BK;
          if (!a_mn) {
            tma_load_2d(sa, mA, fb, k0, T.m0);                 // box {64 K, 128 M}
          } else {
            tma_load_2d(sa, mA, fb, T.m0, k0);                 // box {64 M, 64 K}
            tma_load_2d(sa + 8192, mA, fb, T.m0 + 64, k0);
          }
          if (!b_mn) {
            tma_load_2d(sb, mB, fb, k0, T.n0);                 // box {64 K, bn N}
          } else {
            for (int c = 0; c < T.bn / 64; ++c) tma_load_2d(sb + 8192 * c, mB, fb, T.n0 + 64 * c, k0);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ============ MMA issuer ============
    if (lane == 0) {
      int it = 0;
      for (int j = 0;; ++j) {
        const int slot = j % Q;
        mbar_wait(bar_qfull + 8 * slot, (j / Q) & 1);
        const int t = task_slot[slot];
        mbar_arrive(bar_qempty + 8 * slot);
        if (t < 0) break;
        const TaskRt T = task_rt(p, t);
        const bool a_mn = T.kind == EPI_WGRAD;
        const bool b_mn = T.kind != EPI_DGRAD;
        const uint32_t ID = idesc_rt(T.bn, a_mn, b_mn);
        const int acc = j & 1;
        if (j >= 2) mbar_wait(bar_tempty + 8 * acc, ((j >> 1) - 1) & 1);
        fence_after();
        const uint32_t dtm = tmem + (uint32_t)(acc * kMaxBN);
        for (int kb = 0; kb < T.nkb; ++kb, ++it) {
          const int s = it % STAGES;
          mbar_wait(bar_full + 8 * s, (it / STAGES) & 1);
          fence_after();
          const uint32_t sa = sbase + s * STAGE;
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            const uint64_t ad = a_mn ? sdesc(sa + kk * 2048, 8192, 1024) : sdesc(sa + kk * 32, 16, 1024);
            const uint64_t bd = b_mn ? sdesc(sb + kk * 2048, 8192, 1024) : sdesc(sb + kk * 32, 16, 1024);
            umma_bf16(dtm, ad, bd, ID, (kb | kk) != 0 ? 1u : 0u);
          }
          umma_commit(bar_empty + 8 * s);
        }
        umma_commit(bar_tfull + 8 * acc);
      }
    }
    __syncwarp();
  } else {
    // ============ epilogue (warps 2..9: two per TMEM lane quarter) ============
    const int q = warp & 3;                  // lane quarter (TMEM access restriction)
    const int h = (warp - 2) >> 2;           // column half: 32-col chunks c = h, h+2, ...
    const int et = threadIdx.x - 64;         // 0..255
    const uint32_t stg = sbase + STG_OFF + (warp - 2) * 2048;
    for (int j = 0;; ++j) {
      const int slot = j % Q;
      mbar_wait(bar_qfull + 8 * slot, (j / Q) & 1);
      const int t = task_slot[slot];
      ebar();                                   // everyone read the slot; previous task done with smem
      if (et == 0) mbar_arrive(bar_qempty + 8 * slot);
      if (t < 0) break;
      const TaskRt T = task_rt(p, t);
      const Op &o = p.ops[T.op];
      const LayerDev &Ld = p.layers[T.layer - 1];
      const int acc = j & 1;
      const int row0 = T.m0 + q * 32;
      const int row = row0 + lane;
      const bool row_ok = row < T.M;
      // outputs (row-major, ldc = N): F_i -> X_{i+1} (+ Z_i), dO_i -> dZ_{i-1} (or dX), dW_i -> bucket
      __nv_bfloat16 *out;
      __nv_bfloat16 *zout = nullptr;
      if (T.kind == EPI_FWD) {
        out = reinterpret_cast<__nv_bfloat16 *>(T.layer == cl.L ? p.y_out : Ld.Xn);
        zout = reinterpret_cast<__nv_bfloat16 *>(const_cast<void *>(Ld.Z));
      } else if (T.kind == EPI_DGRAD) {
        out = reinterpret_cast<__nv_bfloat16 *>(T.layer >= 2 ? p.layers[T.layer - 2].dZ : p.dx_out);
      } else {
        out = reinterpret_cast<__nv_bfloat16 *>(Ld.gw);
      }
      const __nv_bfloat16 *zin = nullptr;
      float *dbpart = nullptr;
      if (T.kind == EPI_FWD) {
        const __nv_bfloat16 *bias = reinterpret_cast<const __nv_bfloat16 *>(Ld.bias);
        for (int c = et; c < T.bn; c += kEpiThreads) {
          const int n = T.n0 + c;
          bias_s[c] = n < T.N ? __bfloat162float(bias[n]) : 0.f;
        }
        ebar();
      } else if (T.kind == EPI_DGRAD && T.layer >= 2) {
        const LayerDev &Lp = p.layers[T.layer - 2];
        zin = reinterpret_cast<const __nv_bfloat16 *>(Lp.Z);   // null for identity act_{i-1}
        dbpart = Lp.dbpart;
      }
      const int nch = T.bn / 32;
      // param-space fields -> registers once per task (see act_chunk32)
      const int act = o.act;
      const int dbg = p.dbg;
      const float alpha = p.alpha;
      const bool need_z = (T.kind == EPI_DGRAD) && act != ACT_ID && zin != nullptr && row_ok;
      const __nv_bfloat16 *zrow = zin ? zin + (size_t)row * T.N + T.n0 : nullptr;
      uint4 zr[4];
      if (need_z && h < nch) ld_raw32(zrow + h * 32, zr);     // act' input, prefetched before the wait
      mbar_wait(bar_tfull + 8 * acc, (j >> 1) & 1);
      fence_after();
      if (et == 0) etrace(t, 2);
      for (int c = h; c < nch; c += 2) {
        const int col0 = T.n0 + c * 32;
        if (col0 >= T.N) break;
        float v[32];
        {
          uint32_t r[32];
          tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * kMaxBN + c * 32), r);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
        }
        if (T.kind == EPI_FWD) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __bfloat162float(__float2bfloat16_rn(v[i] + bias_s[c * 32 + i]));
          if (zout && !(dbg & 2)) store32_rows(zout, T.N, stg, lane, v, col0, row0, T.M);   // Z_i
          if (!(dbg & 1)) act_chunk32(act, v);
          if (!(dbg & 2)) store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);  // X_{i+1} (or Y)
        } else if (T.kind == EPI_DGRAD) {
          if (need_z && !(dbg & 1)) {
            float z[32];
            unpack_bf16x32(zr, z);
            if (c + 2 < nch && col0 + 64 < T.N) ld_raw32(zrow + (c + 2) * 32, zr);
            act_grad_mul_chunk32(act, v, z);
          }
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = row_ok ? __bfloat162float(__float2bfloat16_rn(v[i])) : 0.f;
          if (!(dbg & 2)) store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);  // dZ_{i-1} (or dX)
          if (dbpart) red[q * kMaxBN + c * 32 + lane] = warp_colsum32(v, lane);
        } else {  // EPI_WGRAD: one split, scaled bf16 straight into the gradient bucket
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] *= alpha;
          store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);
        }
      }
      // accumulator buffer free for task j+2
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(bar_tempty + 8 * acc);
      if (T.kind == EPI_DGRAD && dbpart) {
        ebar();
        for (int cc = et; cc < T.bn; cc += kEpiThreads) {
          const int col = T.n0 + cc;
          if (col < T.N) {
            const float s = ((red[cc] + red[kMaxBN + cc]) + red[2 * kMaxBN + cc]) + red[3 * kMaxBN + cc];
            dbpart[(size_t)T.mblk * T.N + col] = s;
          }
        }
      }
      if (T.kind == EPI_WGRAD && T.m0 == 0) {
        // db_i = (1/N) sum over row blocks of the bias-grad partials (fixed order)
        if (T.layer < cl.L) wait_ge(ctr + cl.dz_total + (T.layer - 1), cl.MT * p.layers[T.layer].dx_nt);
        __nv_bfloat16 *db = reinterpret_cast<__nv_bfloat16 *>(Ld.db_out);
        for (int cc = et; cc < T.bn; cc += kEpiThreads) {
          const int col = T.n0 + cc;
          if (col < T.N) {
            float s = 0.f;
            for (int r = 0; r < p.R; ++r) s += __ldcg(Ld.dbpart + (size_t)r * T.N + col);
            db[col] = __float2bfloat16_rn(s * p.alpha);
          }
        }
      }
      // ---- publish completion (release): the tile's global stores happen-before the counter
      ebar();
      if (et == 0) {
        // release reductions are cumulative: every store of the tile (all
        // epilogue warps, ordered by the barrier above) is visible before the count
        if (T.kind == EPI_FWD) {
          red_release_add(ctr + cl.fwd_base + 1 + (T.layer - 1) * cl.MT + T.mblk, 1);
        } else if (T.kind == EPI_DGRAD) {
          if (T.layer >= 2) {
            red_release_add(ctr + cl.dz_rows + (T.layer - 2) * cl.MT + T.mblk, 1);
            red_release_add(ctr + cl.dz_total + (T.layer - 2), 1);
          }
        } else {
          red_release_add(ctr + cl.dw_done + (T.layer - 1), 1);
          red_release_add(ctr + cl.bucket_done + Ld.bucket, 1);
        }
        etrace(t, 3);
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == 1) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS)
                 : "memory");
  }
}

int engine_smem_bytes() { return SMEM; }

#ifdef OOO_TRACE
cudaError_t engine_set_trace(void *p) { return cudaMemcpyToSymbol(g_etrace, &p, sizeof(p)); }
#endif

cudaError_t engine_init() {
  return cudaFuncSetAttribute(engine_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
}

cudaError_t launch_engine(const Params &p, const CUtensorMap *tmY, const CUtensorMap *tmDX, int ctas,
                          cudaStream_t stream, int priority) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(ctas, 1, 1);
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = priority;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, engine_kernel, *tmY, *tmDX, p);
}

}  // namespace eng
}  // namespace ooo
