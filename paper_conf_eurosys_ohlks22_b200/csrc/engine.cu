// Persistent dataflow engine kernel (see engine.h for the design rationale).
//
// Template CG = CTAs per tile (tcgen05 cta_group):
//   CG = 1 : one CTA per 128 x bn tile, B fully in its smem (48 KiB stages).
//   CG = 2 : a CTA pair (cluster of 2) per 256 x bn tile; CTA rank r owns rows
//            [m0 + 128 r, +128) and streams its own 128 rows of A and half of
//            B (bn/2 columns); the leader's single thread issues
//            tcgen05.mma.cta_group::2 (M = 256), reading A and B from both
//            CTAs, so each SM moves 32 KiB per k-block and 6 stages fit.
// Each CTA's TMEM holds its 128 accumulator rows (2 buffers x 256 columns).
//
// Roles per CTA (one CTA per SM, persistent):
//   warp 0 lane 0 : producer.  The leader also dispenses: atomicAdd on the
//                   launch's dispenser gives the next task (queue = priority
//                   order), written to the 4-deep smem task ring(s).
//                   X -> X_1 copy tasks (EPI_COPY) have no loads and no MMA:
//                   only the epilogue warps run them.
//                   Each producer waits until its input rows are complete
//                   (acquire on a completion counter, timeout -> trap), then
//                   issues its TMA loads, completing on the leader's barrier.
//   warp 1        : TMEM allocator; the leader's lane 0 issues the MMAs into
//                   accumulator j & 1 of its j-th GEMM task (double-buffered).
//   warps 2..9    : epilogue of task j while task j+1's MMAs run: tcgen05.ld,
//                   fused bias/act (F_i), act-grad + bias-grad partials (dO_i),
//                   1/N scale + bias-grad reduction (dW_i), bf16 RNE, coalesced
//                   stores; then publish completion (release) to the counters.
// Deadlock freedom: tasks are dispensed in increasing index and every
// dependency of task t is a task with a smaller index (or, for F_i at N > 1,
// the comm stream's all-reduce of a bucket whose dW tasks all precede t), all CTAs are
// co-resident (grid <= #SMs, 1 CTA/SM), and each role processes its tasks in
// order; so the smallest unfinished task can always make progress.  Every
// wait is bounded (globaltimer) and traps instead of hanging.
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>

#include "engine.h"
#include "kernels.h"
#include "tc_common.cuh"

namespace ooo {
namespace eng {

using namespace ooo::tc;

#ifdef OOO_TRACE
__device__ __forceinline__ uint32_t cta_rank_raw() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
// Debug builds only (libooo_trace.so): per-task stamps [task][8]:
// globaltimer at dispensed / inputs ready / accumulator ready / published
// (leader CTA; CTA index in the top 16 bits), then clock64 at the same points.
__device__ unsigned long long *g_etrace = nullptr;
__device__ __forceinline__ void etrace(int t, int slot) {
  if (g_etrace && t >= 0) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    g_etrace[(size_t)t * 8 + slot] = (v & 0xFFFFFFFFFFFFull) | ((unsigned long long)blockIdx.x << 48);
    g_etrace[(size_t)t * 8 + 4 + slot] = clock64();
  }
}
// epilogue phase clocks [task][8] (leader CTA, epilogue thread 0)
__device__ unsigned long long *g_etrace2 = nullptr;
__device__ __forceinline__ void etrace2(int t, int slot) {
  if (g_etrace2 && t >= 0) g_etrace2[(size_t)t * 8 + slot] = clock64();
}
// pipeline globaltimer stamps [task][8] (third region): 4 accumulator free
// (MMA may start), 5 last MMA issued, 6 first k-block landed, 7 last landed
__device__ unsigned long long *g_etrace3 = nullptr;
__device__ __forceinline__ void etrace_gt(int t, int slot) {
  if (g_etrace3 && t >= 0) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    g_etrace3[(size_t)t * 8 + slot] = v;
  }
}
// per-k-block clocks of task g_ktask (leader CTA; OOO_KTASK, default 0):
// [150000 + kb][slot], slot 0 producer issue, 2 MMA wait start, 3 wait passed,
// 4 MMAs + commit issued
__device__ int g_ktask = 0;
__device__ __forceinline__ void ktrace(int t, int kb, int slot) {
  if (g_etrace3 && t == g_ktask && kb < 1024 && cta_rank_raw() == 0)
    g_etrace3[(size_t)(150000 + kb) * 8 + slot] = clock64();
}
#else
__device__ __forceinline__ void etrace(int, int) {}
__device__ __forceinline__ void etrace2(int, int) {}
__device__ __forceinline__ void etrace_gt(int, int) {}
__device__ __forceinline__ void ktrace(int, int, int) {}
#endif

#ifndef OOO_ENGINE_PDL
#define OOO_ENGINE_PDL 1
#endif
#ifndef OOO_EPI_WARPS
#define OOO_EPI_WARPS 8
#endif
constexpr int kEpiWarps = OOO_EPI_WARPS;             // multiple of 4 (TMEM lane quarters)
constexpr int kEpiPerQ = kEpiWarps / 4;              // warps sharing a lane quarter (column split)
constexpr int kEpiThreads = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpiThreads;
constexpr int kMaxBN = 256;
constexpr int STG_BYTES = kEpiWarps * 2048;
constexpr int Q = 4;                                 // task ring depth
constexpr uint32_t TMEM_COLS = 512;
// Bound of every wait (ns), from Params::timeout_ns (the stack's
// wait_timeout_ms): a wait that exceeds it traps (the launch fails with an
// error) instead of hanging.  Written by thread 0 before the prologue's
// barrier; every wait follows that barrier.
__shared__ uint64_t s_timeout_ns;

#ifndef OOO_CG1_MAXBN
#define OOO_CG1_MAXBN 256   // experiment: widest B share a 1-CTA stage holds
#endif
#ifndef OOO_CG1_STAGES
#define OOO_CG1_STAGES 4
#endif
// 64-deep k-blocks per ring stage: 2 = one full-barrier wait and one MMA
// commit per 128-deep stage (the MMA issuer's per-stage overhead halves; C4
// 3.11 -> 2.92 ms, C2 neutral); 1-CTA stacks keep 1 (only 2 stages would fit:
// C5 +2.7 %)
#ifndef OOO_KPS2
#define OOO_KPS2 2
#endif
#ifndef OOO_KPS1
#define OOO_KPS1 1
#endif
template <int CG> struct Cfg {
  static constexpr int KPS = CG == 2 ? OOO_KPS2 : OOO_KPS1;
  static constexpr int B_BYTES = (CG == 1 ? OOO_CG1_MAXBN : kMaxBN / CG) * BK * 2;   // this CTA's share of B
  static constexpr int SUB = A_BYTES + B_BYTES;      // one k-block: A rows, then this CTA's B share
  static constexpr int STAGE = SUB * KPS;
  static constexpr int STAGES = (CG == 2 ? (kEpiWarps > 8 ? 5 : 6) : (kEpiWarps > 8 ? 3 : OOO_CG1_STAGES)) / KPS;
  static constexpr int RING = STAGE * STAGES;
  static constexpr int STG_OFF = RING;
  static constexpr int BAR_OFF = STG_OFF + STG_BYTES;
  // full[S] empty[S] tfull[2] tempty[2] taskfull[Q] taskempty[Q]
  static constexpr int SLOT_OFF = BAR_OFF + (2 * STAGES + 4 + 2 * Q) * 8;
  static constexpr int TASK_OFF = SLOT_OFF + 16;
  static constexpr int BIAS_OFF = (TASK_OFF + 4 * Q + 15) / 16 * 16;
  static constexpr int RED_OFF = BIAS_OFF + kMaxBN * 4;
  static constexpr int SKF_OFF = RED_OFF + 4 * kMaxBN * 4;   // split-K "last arrival" flag
  static constexpr int SMEM = SKF_OFF + 16 + 1024;
  static_assert(SMEM <= kSmemBudget, "engine smem budget");
  static_assert(STAGE % 1024 == 0, "stage alignment");
};

__device__ __forceinline__ void ebar() { asm volatile("bar.sync 1, %0;" ::"n"(kEpiThreads) : "memory"); }

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// ---- cluster (CTA pair) helpers
__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t mapa(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// Relaxed arrive (a bare SYNCS.ARRIVE): for the peer's "slot read" and
// "accumulator read" signals, which publish no memory -- the slot reads are
// performed before it (CTA barrier), the TMEM reads completed (tcgen05.wait::ld
// + fence::before_thread_sync).  OOO_RELAXED_ARRIVE=0: release arrives (A/B).
#ifndef OOO_RELAXED_ARRIVE
#define OOO_RELAXED_ARRIVE 1
#endif
__device__ __forceinline__ void mbar_arrive_cluster_signal(uint32_t cluster_addr) {
  if (OOO_RELAXED_ARRIVE)
    asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
  else
    asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// Acquire of shared::cluster data (a peer's st.shared::cluster into this CTA's
// smem, released by its arrive): no instruction on sm_100a, where
// fence.acq_rel.cluster is MEMBAR.ALL.GPU + CCTL.IVALL.
__device__ __forceinline__ void acquire_cluster_smem() {
  if (OOO_RELAXED_ARRIVE) asm volatile("fence.acquire.sync_restrict::shared::cluster.cluster;" ::: "memory");
  else asm volatile("fence.acq_rel.cluster;" ::: "memory");
}
// Bounded mbarrier wait with the default (CTA-scope) semantics.  Spinning
// with .acquire.cluster would emit an L1 invalidation (CCTL.IVALL) on every
// poll -- measured at 2/3 of all warp samples.
// The timeout clock is read only every 1024 polls: a globaltimer read on
// every poll delays the reaction to the phase flip (hot mainloop waits).
__device__ __forceinline__ void mbar_wait_b(uint32_t bar, uint32_t parity) {
  uint64_t t0 = 0;
  for (uint32_t n = 1; !mbar_try_wait(bar, parity); ++n) {
    if ((n & 1023u) == 0) {
      if (t0 == 0) t0 = gtimer();
      else if (gtimer() - t0 > s_timeout_ns) __trap();
    }
  }
}
// Idle-waiting variant for the epilogue warps: sleep between polls so that
// eight waiting warps do not take issue slots from the producer / MMA
// threads of the same SM sub-partitions.
#ifndef OOO_EPI_SLEEP_NS
#define OOO_EPI_SLEEP_NS 64
#endif
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  uint64_t t0 = 0;
  for (uint32_t n = 1; !mbar_try_wait(bar, parity); ++n) {
    if (OOO_EPI_SLEEP_NS > 0) __nanosleep(OOO_EPI_SLEEP_NS);
    if ((n & 255u) == 0) {
      if (t0 == 0) t0 = gtimer();
      else if (gtimer() - t0 > s_timeout_ns) __trap();
    }
  }
}
// For barriers that receive arrivals from the peer CTA: one acquire of the
// shared::cluster data after the wait, not one per poll.
__device__ __forceinline__ void mbar_wait_cl(uint32_t bar, uint32_t parity) {
  mbar_wait_b(bar, parity);
  acquire_cluster_smem();
}
__device__ __forceinline__ void tma_load_2d_pair(uint32_t dst, const CUtensorMap *map, uint32_t leader_bar,
                                                 int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(leader_bar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void umma_bf16_pair(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                               uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
// completion of the leader's MMAs arrives on the same barrier in both CTAs
__device__ __forceinline__ void umma_commit_pair(uint32_t bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          bar),
      "h"((unsigned short)3)
      : "memory");
}

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
__device__ __forceinline__ int atom_add_acq_rel(int32_t *p, int v) {
  int old;
  asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ void red_release_add(int32_t *p, int v) {
  asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
// Wait until *p >= target.  A dependency that is not met within the bound
// means a broken schedule or a stalled peer rank: trap (the launch fails with
// an error) instead of hanging.
__device__ __forceinline__ void wait_ge(const int32_t *p, int target) {
  if (ld_relaxed(p) < target) {
    const uint64_t t0 = gtimer();
    while (ld_relaxed(p) < target) {
      __nanosleep(32);
      if (gtimer() - t0 > s_timeout_ns) __trap();
    }
  }
  (void)ld_acquire(p);   // one acquire orders the producer tiles' stores before our reads
}

__device__ __forceinline__ const CUtensorMap *map_of(int idx, const CUtensorMap *maps,
                                                     const CUtensorMap *tmY, const CUtensorMap *tmDX,
                                                     const CUtensorMap *tmX) {
  if (idx >= 0) return maps + idx;
  return idx == MAP_Y ? tmY : (idx == MAP_DX ? tmDX : tmX);
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
  int op, kind, layer, bn, nkb, m0, n0, M, N, mblk0;   // m0 / mblk0: first row (block) of the tile
  int kb0, ks, s, tile;   // split-K: first k-block, splits, this task's split, tile index within the op
};
template <int CG>
__device__ __forceinline__ TaskRt task_rt(const Params &p, int t) {
  TaskRt r;
  r.op = op_of(p, t);
  const Op &o = p.ops[r.op];
  int rel = t - o.first;
  r.kind = o.kind;
  r.layer = o.layer;
  r.bn = o.bn;
  r.ks = o.ks > 1 ? o.ks : 1;
  r.s = rel % r.ks;               // the splits of one tile are consecutive tasks
  rel /= r.ks;
  r.tile = rel;
  const int kps = (o.nkb + r.ks - 1) / r.ks;
  r.kb0 = r.s * kps;
  r.nkb = min(o.nkb, r.kb0 + kps) - r.kb0;
  r.mblk0 = o.m_off + CG * (rel / o.nt);
  r.m0 = r.mblk0 * BM;
  r.n0 = (rel % o.nt) * o.bn;
  const LayerDev &L = p.layers[o.layer - 1];
  if (o.kind == EPI_FWD) { r.M = p.M; r.N = L.dout; }
  else if (o.kind == EPI_DGRAD || o.kind == EPI_COPY) { r.M = p.M; r.N = L.din; }
  else { r.M = L.din; r.N = L.dout; }
  return r;
}

// Dependencies of task T for row block mblk: all on tasks earlier in the
// queue (the host planner emits ops in a topological order), or on the comm
// stream's all-reduce of a bucket whose dW tasks all precede T.  kWait: block
// until met (bounded); else: report whether met now.
template <bool kWait>
__device__ __forceinline__ bool dep_ge(const int32_t *c, int target) {
  if (kWait) { wait_ge(c, target); return true; }
  return ld_relaxed(c) >= target;
}
template <bool kWait>
__device__ __forceinline__ bool deps(const Params &p, const TaskRt &T, int mblk) {
  const CounterLayout &cl = p.cl;
  const int32_t *ctr = p.ctr;
  const LayerDev &Ld = p.layers[T.layer - 1];
  bool ok = true;
  if (T.kind == EPI_FWD) {
    // (F_1 reads the caller's X directly; the X -> X_1 copy for the next
    // backward's dW_1 is off the chain)
    if (mblk < cl.MT && T.layer > 1)
      ok = dep_ge<kWait>(ctr + cl.fwd_rows + (T.layer - 2) * cl.MT + mblk, p.layers[T.layer - 2].fwd_nt);
    if (ok && p.fwd_gate == 1) ok = dep_ge<kWait>(ctr + cl.dw_done + (T.layer - 1), Ld.dw_tiles);   // P:84, N = 1
    else if (ok && p.fwd_gate == 2) ok = dep_ge<kWait>(ctr + cl.ar_done + Ld.bucket, 1);          // P:84, S[dW_i]
    if (ok && p.fwd_gate && T.layer < cl.L)      // WAR: dW_{i+1} reads X_{i+1}
      ok = dep_ge<kWait>(ctr + cl.dw_done + T.layer, p.layers[T.layer].dw_tiles);
  } else if (T.kind == EPI_DGRAD) {
    if (T.layer < cl.L) {
      const LayerDev &Ln = p.layers[T.layer];
      if (mblk < cl.MT) ok = dep_ge<kWait>(ctr + cl.dz_rows + (T.layer - 1) * cl.MT + mblk, Ln.dx_nt);
      if (ok && p.in_order) ok = dep_ge<kWait>(ctr + cl.dw_done + T.layer, Ln.dw_tiles);
    }
  } else if (T.kind == EPI_WGRAD) {
    if (T.layer < cl.L) ok = dep_ge<kWait>(ctr + cl.dz_total + (T.layer - 1), cl.MT * p.layers[T.layer].dx_nt);
  } else {   // EPI_COPY: dW_1 of the pending backward still reads X_1
    if (p.fwd_gate) ok = dep_ge<kWait>(ctr + cl.dw_done, p.layers[0].dw_tiles);
  }
  return ok;
}

// F_i's gate on the weights: S[dW_i] done (N = 1: dW_i's tiles, N > 1:
// the bucket's all-reduce flag), blocking.
__device__ __forceinline__ void wgate(const Params &p, const TaskRt &T) {
  const LayerDev &Ld = p.layers[T.layer - 1];
  if (p.fwd_gate == 1) wait_ge(p.ctr + p.cl.dw_done + (T.layer - 1), Ld.dw_tiles);
  else if (p.fwd_gate == 2) wait_ge(p.ctr + p.cl.ar_done + Ld.bucket, 1);
}

// TMA loads of one k-block stage: this CTA's A rows / its share of B,
// completing on the leader's full barrier.
template <int CG, bool A_MN>
__device__ __forceinline__ void load_a(const CUtensorMap *mA, uint32_t sa, uint32_t lb, int am, int k0) {
  if (CG == 2) {
    if (!A_MN) {
      tma_load_2d_pair(sa, mA, lb, k0, am);                       // box {64 K, 128 M}
    } else {
      tma_load_2d_pair(sa, mA, lb, am, k0);                       // box {64 M, 64 K}
      tma_load_2d_pair(sa + 8192, mA, lb, am + 64, k0);
    }
  } else {
    if (!A_MN) {
      tma_load_2d(sa, mA, lb, k0, am);
    } else {
      tma_load_2d(sa, mA, lb, am, k0);
      tma_load_2d(sa + 8192, mA, lb, am + 64, k0);
    }
  }
}
template <int CG, bool B_MN>
__device__ __forceinline__ void load_b(const CUtensorMap *mB, uint32_t sb, uint32_t lb, int bn0, int bh, int k0) {
  if (CG == 2) {
    if (!B_MN) {
      tma_load_2d_pair(sb, mB, lb, k0, bn0);                      // box {64 K, bn/2 N}
    } else {
      tma_load_2d_pair(sb, mB, lb, bn0, k0);                      // boxes {64 N, 64 K}
      if (bh > 64) tma_load_2d_pair(sb + 8192, mB, lb, bn0 + 64, k0);
    }
  } else {
    if (!B_MN) {
      tma_load_2d(sb, mB, lb, k0, bn0);                           // box {64 K, bn N}
    } else {
      for (int c = 0; c < bh / 64; ++c) tma_load_2d(sb + 8192 * c, mB, lb, bn0 + 64 * c, k0);
    }
  }
}

// Weight prefetch: the B operand of F_i / dO_i is W_i, which does not depend
// on the row-local chain, so the first npre stages are claimed and their W
// tiles requested before the producer waits for the activation rows (the
// HBM latency of the weights overlaps the chain hand-off).  The full
// barrier's expect_tx (leader) already counts the A bytes issued later.
template <int CG, bool B_MN>
__device__ __forceinline__ void prefetch_b(const CUtensorMap *mB, uint32_t sbase, uint32_t bar_empty,
                                           uint32_t bar_full, uint32_t L_full, bool leader, uint32_t bytes, int bn0,
                                           int bh, int it, int npre, int nkb, int kb0) {
  using C = Cfg<CG>;
  int s = it % C::STAGES;
  uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;
  for (int st = 0; st < npre; ++st) {
    const int kc = min(C::KPS, nkb - st * C::KPS);        // k-blocks in this stage
    if (it + st >= C::STAGES) mbar_wait_b(bar_empty + 8 * s, ph ^ 1u);
    if (leader) mbar_expect_tx(bar_full + 8 * s, bytes * kc);
    for (int sub = 0; sub < kc; ++sub)
      load_b<CG, B_MN>(mB, sbase + s * C::STAGE + sub * C::SUB + A_BYTES, L_full + 8 * s, bn0, bh,
                       (kb0 + st * C::KPS + sub) * BK);
    if (++s == C::STAGES) {
      s = 0;
      ph ^= 1u;
    }
  }
}

// L2 prefetch of the B operand (= W_j) slice a chain tile of layer j would
// load: this CTA's columns [bn0, bn0 + bh) over all nkb k-blocks.
template <int CG, bool B_MN>
__device__ __forceinline__ void prefetch_b_l2(const CUtensorMap *mB, int bn0, int bh, int nkb) {
  for (int kb = 0; kb < nkb; ++kb) {
    if (B_MN) {
      for (int c = 0; c < (bh + 63) / 64; ++c) tma_prefetch_l2_2d(mB, bn0 + 64 * c, kb * BK);
    } else {
      tma_prefetch_l2_2d(mB, kb * BK, bn0);
    }
  }
}

// Producer k-loop of one task, specialised per operand layout (no per-k-block
// branches; stage / phase advanced incrementally): waits for a free ring
// stage, then TMA-loads this CTA's A rows and its share of B, completing on
// the leader's full barrier.  The first npre stages were claimed by
// prefetch_b: only their A loads remain.
template <int CG, bool A_MN, bool B_MN>
__device__ __forceinline__ void produce(const TaskRt &T, const CUtensorMap *mA, const CUtensorMap *mB, uint32_t sbase,
                                        uint32_t bar_empty, uint32_t bar_full, uint32_t L_full, bool leader,
                                        uint32_t bytes, int am, int bn0, int bh, int &it, int t, int npre) {
  using C = Cfg<CG>;
  const int nst = (T.nkb + C::KPS - 1) / C::KPS;         // ring stages of this task
  int s = it % C::STAGES;
  uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;   // phase of the stage's next fill
  for (int st = 0; st < npre; ++st) {
    const int kc = min(C::KPS, T.nkb - st * C::KPS);
    for (int sub = 0; sub < kc; ++sub) {
      ktrace(t, st * C::KPS + sub, 0);
      load_a<CG, A_MN>(mA, sbase + s * C::STAGE + sub * C::SUB, L_full + 8 * s, am, (T.kb0 + st * C::KPS + sub) * BK);
    }
    if (++s == C::STAGES) {
      s = 0;
      ph ^= 1u;
    }
  }
  for (int st = npre; st < nst; ++st) {
    const int kc = min(C::KPS, T.nkb - st * C::KPS);
    if (it + st >= C::STAGES) mbar_wait_b(bar_empty + 8 * s, ph ^ 1u);
    if (leader) mbar_expect_tx(bar_full + 8 * s, bytes * kc);
    const uint32_t lb = L_full + 8 * s;
    for (int sub = 0; sub < kc; ++sub) {
      const int kb = st * C::KPS + sub;
      ktrace(t, kb, 0);
      const uint32_t sa = sbase + s * C::STAGE + sub * C::SUB;
      load_a<CG, A_MN>(mA, sa, lb, am, (T.kb0 + kb) * BK);
      load_b<CG, B_MN>(mB, sa + A_BYTES, lb, bn0, bh, (T.kb0 + kb) * BK);
    }
    if (++s == C::STAGES) {
      s = 0;
      ph ^= 1u;
    }
  }
  it += nst;
}

// X -> X_1 copy of one tile (epilogue threads), 8 vector loads in flight per
// thread (a dependent load -> store loop waits one memory latency per
// vector).  Not inlined: its registers stay out of the GEMM epilogue's
// allocation (168-register cap, no spills).
__device__ __noinline__ void copy_rows(const uint4 *__restrict__ src, uint4 *__restrict__ dst, size_t ld, int row0,
                                       int c0, int vpr, int nv, int et) {
  for (int v0 = et; v0 < nv; v0 += 8 * kEpiThreads) {
    uint4 r[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int v = v0 + u * kEpiThreads;
      if (v < nv) r[u] = __ldg(src + (size_t)(row0 + v / vpr) * ld + c0 + v % vpr);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int v = v0 + u * kEpiThreads;
      if (v < nv) dst[(size_t)(row0 + v / vpr) * ld + c0 + v % vpr] = r[u];
    }
  }
}

// SK: the kernel contains the split-K epilogue path (launched only when the
// queue has split ops -- skinny stacks), so the common path (C2, C3) carries
// none of its registers.
template <int CG, bool SK>
__global__ void __launch_bounds__(kThreads, 1)
    engine_kernel(const __grid_constant__ CUtensorMap tmY, const __grid_constant__ CUtensorMap tmDX,
                  const __grid_constant__ CUtensorMap tmX,
                  const __grid_constant__ Params p) {
  using C = Cfg<CG>;
  extern __shared__ uint8_t smem_raw[];
  // 1 KiB alignment by pointer arithmetic on the __shared__ array, so that the
  // compiler keeps the shared address space (LDS/STS, not generic LD/ST)
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar_full = sbase + C::BAR_OFF;
  const uint32_t bar_empty = bar_full + 8 * C::STAGES;
  const uint32_t bar_tfull = bar_empty + 8 * C::STAGES;
  const uint32_t bar_tempty = bar_tfull + 16;
  const uint32_t bar_qfull = bar_tempty + 16;
  const uint32_t bar_qempty = bar_qfull + 8 * Q;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + C::SLOT_OFF);
  volatile int *task_slot = reinterpret_cast<volatile int *>(smem + C::TASK_OFF);
  float *bias_s = reinterpret_cast<float *>(smem + C::BIAS_OFF);
  float *red = reinterpret_cast<float *>(smem + C::RED_OFF);
  volatile int *sk_flag = reinterpret_cast<volatile int *>(smem + C::SKF_OFF);
  int32_t *ctr = p.ctr;
  const CounterLayout &cl = p.cl;

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = CG == 2 ? cta_rank() : 0;   // 0 = leader (issues the MMAs)
  const bool leader = rank == 0;

  if (warp == 0 && lane == 0) {
    s_timeout_ns = p.timeout_ns;
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);           // leader's expect_tx arrival (+ the CTAs' bytes)
      mbar_init(bar_empty + 8 * s, 1);          // leader's MMA commit
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(bar_tfull + 8 * a, 1);          // leader's MMA commit
      mbar_init(bar_tempty + 8 * a, CG * kEpiWarps);   // epilogue warps of all CTAs (leader's copy)
    }
    for (int s = 0; s < Q; ++s) {
      mbar_init(bar_qfull + 8 * s, 1);          // leader: its producer; peer: its own arm (+ the leader's st.async bytes)
      mbar_init(bar_qempty + 8 * s, 2 * CG);    // MMA + epi (+ peer producer + peer epi)
      if (CG == 2 && rank != 0) mbar_expect_tx(bar_qfull + 8 * s, 4);   // phase 0 armed
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 1) {
    if (CG == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                       smem_u32(tmem_slot)),
                   "r"(TMEM_COLS)
                   : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                       smem_u32(tmem_slot)),
                   "r"(TMEM_COLS)
                   : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
  }
  fence_before();
  if (CG == 2) cluster_sync(); else __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();
  // the leader's barriers as seen from this CTA (== local ones for CG = 1)
  const uint32_t L_full = CG == 2 ? mapa(bar_full, 0) : bar_full;
  const uint32_t L_tempty = CG == 2 ? mapa(bar_tempty, 0) : bar_tempty;
  const uint32_t L_qempty = CG == 2 ? mapa(bar_qempty, 0) : bar_qempty;

  if (warp == 0) {
    // ============ dispenser (leader) + TMA producer ============
    if (lane == 0) {
      const uint32_t P_qfull = CG == 2 ? mapa(bar_qfull, 1) : 0;
      const uint32_t P_slot = CG == 2 ? mapa(smem_u32(const_cast<int *>(task_slot)), 1) : 0;
      int it = 0;
      for (int j = 0;; ++j) {
        const int slot = j % Q;
        int t;
        if (leader) {
          t = atomicAdd(ctr, 1);
          if (t >= p.ntasks) t = -1;
          etrace(t, 0);
          if (j >= Q) {
            if (CG == 2) mbar_wait_cl(bar_qempty + 8 * slot, ((j / Q) - 1) & 1);
            else mbar_wait_b(bar_qempty + 8 * slot, ((j / Q) - 1) & 1);
          }
          task_slot[slot] = t;
          mbar_arrive(bar_qfull + 8 * slot);
          if (CG == 2) {
            // the peer's copy of the slot: a remote store that completes 4
            // transaction bytes on the peer's full barrier (armed by the peer)
            // -- no release fence (MEMBAR.ALL.GPU) on the dispenser's path
            asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(
                             P_slot + 4 * slot),
                         "r"(t), "r"(P_qfull + 8 * slot)
                         : "memory");
          }
        } else {
          mbar_wait_cl(bar_qfull + 8 * slot, (j / Q) & 1);
          t = task_slot[slot];
          if (t >= 0) mbar_expect_tx(bar_qfull + 8 * slot, 4);   // arm the slot's next phase
          mbar_arrive_cluster_signal(L_qempty + 8 * slot);
        }
        if (t < 0) break;
        const TaskRt T = task_rt<CG>(p, t);
        if (T.kind == EPI_COPY) continue;        // epilogue warps only
        const Op &o = p.ops[T.op];
        const LayerDev &Ld = p.layers[T.layer - 1];
        const CUtensorMap *mA = map_of(o.mapA, p.maps, &tmY, &tmDX, &tmX);
        const CUtensorMap *mB = map_of(o.mapB, p.maps, &tmY, &tmDX, &tmX);
        tma_prefetch(mA);      // descriptors live in global memory: warm the TMA descriptor cache
        tma_prefetch(mB);
        const bool a_mn = T.kind == EPI_WGRAD;
        const bool b_mn = T.kind != EPI_DGRAD;
        const int bh = T.bn / CG;                                 // this CTA's B columns
        // MN-major B arrives in whole 64-column boxes (a 96-column share of a
        // 192-wide pair tile fetches 128 columns; the MMA reads the first 96)
        const int bh_ld = b_mn ? (bh + 63) / 64 * 64 : bh;
        const uint32_t a_bytes = T.kind == EPI_WGRAD ? (uint32_t)A_BYTES : (uint32_t)p.a_rows * (BK * 2);
        const uint32_t bytes = CG * (a_bytes + bh_ld * BK * 2);   // all CTAs, on the leader's barrier
        const int am = T.m0 + BM * (int)rank;
        const int bn0 = T.n0 + bh * (int)rank;
        int npre = 0;
        if (T.kind != EPI_WGRAD && !(p.dbg & 16)) {
          // B = W_i: only F_i's gate on S[dW_i] guards the weights
          if (T.kind == EPI_FWD && p.fwd_gate) {
            wgate(p, T);
            asm volatile("fence.proxy.async.global;" ::: "memory");
          }
          npre = min((T.nkb + C::KPS - 1) / C::KPS, C::STAGES);   // ring stages claimed for W
          if (b_mn) prefetch_b<CG, true>(mB, sbase, bar_empty, bar_full, L_full, leader, bytes, bn0, bh, it, npre, T.nkb, T.kb0);
          else prefetch_b<CG, false>(mB, sbase, bar_empty, bar_full, L_full, leader, bytes, bn0, bh, it, npre, T.nkb, T.kb0);
        }
        if (T.kind == EPI_DGRAD && o.mapZ >= 0 && am < T.M && !(p.dbg & 32)) {
          // the epilogue multiplies by act'(Z_{i-1}) read from the Z_{i-1}
          // store (written by the forward, long evicted from L2): request this
          // CTA's rows of it now, a mainloop ahead of the epilogue's loads
          const CUtensorMap *mZ = p.maps + o.mapZ;
          const int ncol = min(T.bn, T.N - T.n0);
          for (int c = 0; c < ncol; c += 64) tma_prefetch_l2_2d(mZ, T.n0 + c, am);
        }
        deps<true>(p, T, T.mblk0 + (int)rank);    // this CTA's row block (no-op after a ready claim)
        asm volatile("fence.proxy.async.global;" ::: "memory");   // TMA reads see the producers' data
        if (leader) etrace(t, 1);
        switch ((a_mn ? 2 : 0) + (b_mn ? 1 : 0)) {
          case 1: produce<CG, false, true>(T, mA, mB, sbase, bar_empty, bar_full, L_full, leader, bytes, am, bn0, bh, it, t, npre); break;
          case 0: produce<CG, false, false>(T, mA, mB, sbase, bar_empty, bar_full, L_full, leader, bytes, am, bn0, bh, it, t, npre); break;
          default: produce<CG, true, true>(T, mA, mB, sbase, bar_empty, bar_full, L_full, leader, bytes, am, bn0, bh, it, t, npre); break;
        }
        if (p.pf_dist > 0 && T.kind != EPI_WGRAD && T.m0 == 0 && T.s == 0) {
          // the weights pf_dist layers ahead on this chain (F: upwards, dO:
          // downwards), this tile's column slice -- issued after the tile's
          // own loads, so they never queue behind the prefetch
          const int j = T.kind == EPI_FWD ? T.layer + p.pf_dist : T.layer - p.pf_dist;
          if (j >= 1 && j <= cl.L && o.mapB >= 0) {
            const LayerDev &Lj = p.layers[j - 1];
            const CUtensorMap *mBj = p.maps + o.mapB + (j - T.layer) * p.maps_per_layer;
            const int nj = T.kind == EPI_FWD ? Lj.dout : Lj.din;        // output width of op j
            const int kj = T.kind == EPI_FWD ? Lj.din : Lj.dout;        // its reduction length
            if (bn0 < nj) {
              if (b_mn) prefetch_b_l2<CG, true>(mBj, bn0, min(bh, nj - bn0), (kj + BK - 1) / BK);
              else prefetch_b_l2<CG, false>(mBj, bn0, bh, (kj + BK - 1) / BK);
            }
          }
        }
      }
    }
  } else if (warp == 1) {
    // ============ MMA issuer (leader CTA only) ============
    if (leader && lane == 0) {
      int it = 0, ja = 0;   // k-block stages, accumulator uses (GEMM tasks only)
      for (int j = 0;; ++j) {
        const int slot = j % Q;
        mbar_wait_b(bar_qfull + 8 * slot, (j / Q) & 1);
        const int t = task_slot[slot];
        mbar_arrive(bar_qempty + 8 * slot);
        if (t < 0) break;
        const TaskRt T = task_rt<CG>(p, t);
        if (T.kind == EPI_COPY) continue;        // no accumulator
        const bool a_mn = T.kind == EPI_WGRAD;
        const bool b_mn = T.kind != EPI_DGRAD;
        // M = 128 * CG across the CTAs, N = bn
        const uint32_t ID = (1u << 4) | (1u << 7) | (1u << 10) | ((a_mn ? 1u : 0u) << 15) |
                            ((b_mn ? 1u : 0u) << 16) | ((uint32_t)(T.bn >> 3) << 17) |
                            ((uint32_t)((BM * CG) >> 4) << 24);
        const int acc = ja & 1;
        if (ja >= 2) {
          if (CG == 2) mbar_wait_cl(bar_tempty + 8 * acc, ((ja >> 1) - 1) & 1);
          else mbar_wait_b(bar_tempty + 8 * acc, ((ja >> 1) - 1) & 1);
        }
        ++ja;
        fence_after();
        etrace_gt(t, 4);                         // accumulator free: MMA may start
        const uint32_t dtm = tmem + (uint32_t)(acc * kMaxBN);
        // Stage-0 / k-step-0 descriptors, advanced by plain adds in the loop
        // (address field = bits 0-13, bytes >> 4): + STAGE >> 4 per stage,
        // + 2 per 16-deep k-step K-major (32 B), + 128 MN-major (2 KiB).  No
        // per-MMA branches or divisions: the issue loop must keep the tensor
        // pipe fed (measured: the generic loop cost ~870 cycles per k-block
        // against 512 of MMA work).
        const uint64_t a0 = a_mn ? sdesc(sbase, 8192, 1024) : sdesc(sbase, 16, 1024);
        const uint64_t b0 = b_mn ? sdesc(sbase + A_BYTES, 8192, 1024) : sdesc(sbase + A_BYTES, 16, 1024);
        const uint64_t astep = a_mn ? 128u : 2u, bstep = b_mn ? 128u : 2u;
        int s = it % C::STAGES;
        uint32_t ph = (uint32_t)(it / C::STAGES) & 1u;
        const int nst = (T.nkb + C::KPS - 1) / C::KPS;
        for (int st = 0; st < nst; ++st) {
          const int kb0 = st * C::KPS;
          const int kc = min(C::KPS, T.nkb - kb0);
          ktrace(t, kb0, 2);
          mbar_wait_b(bar_full + 8 * s, ph);
          ktrace(t, kb0, 3);
          if (st == 0) etrace_gt(t, 6);           // first k-block landed
          if (st == nst - 1) etrace_gt(t, 7);     // last k-block landed
          fence_after();
          for (int sub = 0; sub < kc; ++sub) {
            const uint64_t soff = (uint64_t)((s * C::STAGE + sub * C::SUB) >> 4);
            const uint64_t ad = a0 + soff, bd = b0 + soff;
            const uint32_t acc0 = (kb0 + sub) != 0 ? 1u : 0u;
            if (CG == 2) {
              umma_bf16_pair(dtm, ad, bd, ID, acc0);
              umma_bf16_pair(dtm, ad + astep, bd + bstep, ID, 1u);
              umma_bf16_pair(dtm, ad + 2 * astep, bd + 2 * bstep, ID, 1u);
              umma_bf16_pair(dtm, ad + 3 * astep, bd + 3 * bstep, ID, 1u);
            } else {
              umma_bf16(dtm, ad, bd, ID, acc0);
              umma_bf16(dtm, ad + astep, bd + bstep, ID, 1u);
              umma_bf16(dtm, ad + 2 * astep, bd + 2 * bstep, ID, 1u);
              umma_bf16(dtm, ad + 3 * astep, bd + 3 * bstep, ID, 1u);
            }
          }
          if (CG == 2) umma_commit_pair(bar_empty + 8 * s); else umma_commit(bar_empty + 8 * s);
          ktrace(t, kb0, 4);
          if (++s == C::STAGES) {
            s = 0;
            ph ^= 1u;
          }
        }
        it += nst;
        if (CG == 2) umma_commit_pair(bar_tfull + 8 * acc); else umma_commit(bar_tfull + 8 * acc);
        etrace_gt(t, 5);                         // last MMA issued
      }
    }
    __syncwarp();
  } else {
    // ============ epilogue (warps 2..9: two per TMEM lane quarter) ============
    const int q = warp & 3;                  // lane quarter (TMEM access restriction)
    const int h = (warp - 2) >> 2;           // column slot: 32-col chunks c = h, h + kEpiPerQ, ...
    const int et = threadIdx.x - 64;         // 0..255
    const uint32_t stg = sbase + C::STG_OFF + (warp - 2) * 2048;
    // epilogue thread 0, after a barrier that orders every epilogue store of
    // the publication: +1 on counters a, b, c (indices; -1 none).  One release
    // fence (a MEMBAR.ALL.GPU: it waits for the stores in flight) for all of
    // them, then relaxed increments -- a red.release per counter would pay
    // the MEMBAR once per counter (dW tiles publish two)
    auto publish = [&](int a, int b, int c) {
      asm volatile("fence.acq_rel.gpu;" ::: "memory");
      if (a >= 0) asm volatile("red.relaxed.gpu.global.add.s32 [%0], 1;" ::"l"(ctr + a) : "memory");
      if (b >= 0) asm volatile("red.relaxed.gpu.global.add.s32 [%0], 1;" ::"l"(ctr + b) : "memory");
      if (c >= 0) asm volatile("red.relaxed.gpu.global.add.s32 [%0], 1;" ::"l"(ctr + c) : "memory");
    };
    for (int j = 0, ja = 0;; ++j) {
      const int slot = j % Q;
      mbar_wait_sleep(bar_qfull + 8 * slot, (j / Q) & 1);
      if (!leader) acquire_cluster_smem();   // the leader's st.shared::cluster of the slot
      const int t = task_slot[slot];
      ebar();                                   // everyone read the slot; previous task done with smem
      if (et == 0) {
        if (leader) mbar_arrive(bar_qempty + 8 * slot);
        else mbar_arrive_cluster_signal(L_qempty + 8 * slot);
      }
      if (t < 0) break;
      const TaskRt T = task_rt<CG>(p, t);
      const int mblk = T.mblk0 + (int)rank;
      const int mrow0 = T.m0 + BM * (int)rank;  // this CTA's first row
      if (T.kind == EPI_COPY) {
        // caller's X rows [mrow0, +128) x [n0, +bn) -> X_1 store (dW_1 of the
        // pending backward reads X_1: WAR wait first)
        if (mrow0 < T.M) {
          if (p.fwd_gate && et == 0) wait_ge(ctr + cl.dw_done, p.layers[0].dw_tiles);
          ebar();
          const int rows = min(BM, T.M - mrow0);
          const int vpr = min(T.bn, T.N - T.n0) / 8;     // 16-byte vectors per row
          const uint4 *src = reinterpret_cast<const uint4 *>(p.x_in);
          uint4 *dst = reinterpret_cast<uint4 *>(p.layers[0].X);
          const size_t ld = (size_t)T.N / 8;
          for (int v = et; v < rows * vpr; v += kEpiThreads) {
            const size_t e = (size_t)(mrow0 + v / vpr) * ld + T.n0 / 8 + v % vpr;
            dst[e] = __ldg(src + e);
          }
          ebar();
          if (et == 0) red_release_add(ctr + cl.xcopy + mblk, 1);
        }
        if (et == 0 && leader) { etrace(t, 1); etrace(t, 2); etrace(t, 3); }
        continue;
      }
      const Op &o = p.ops[T.op];
      const LayerDev &Ld = p.layers[T.layer - 1];
      const int acc = ja & 1;
      const int jacc = ja++;
      const int row0 = mrow0 + q * 32;
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
      // dO_i after a GELU layer: the Z_{i-1} store holds gelu'(Z_{i-1}) (see F_i below)
      const int act = (T.kind == EPI_DGRAD && o.act == ACT_GELU) ? (int)ACT_DSTORED : (int)o.act;
      const int dbg = p.dbg;
      const float alpha = p.alpha;
      const bool need_z = (T.kind == EPI_DGRAD) && act != ACT_ID && zin != nullptr && row_ok;
      const __nv_bfloat16 *zrow = zin ? zin + (size_t)row * T.N + T.n0 : nullptr;
      uint4 zr[4];
      if (need_z && h < nch) ld_raw32(zrow + h * 32, zr);     // act' input, prefetched before the wait
      mbar_wait_sleep(bar_tfull + 8 * acc, (jacc >> 1) & 1);
      fence_after();
      if (et == 0 && leader) etrace(t, 2);
      const bool tr2 = et == 0 && leader;
      if (tr2) etrace2(t, 0);
      // TMEM loads run one chunk ahead of the epilogue math (tcgen05.ld is
      // asynchronous until tcgen05.wait::ld)
      const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(acc * kMaxBN);
      const int cend = min(nch, (T.N - T.n0 + 31) >> 5);   // chunks with col0 < N
      // Work the row-local successor does not need is done after the early
      // publish below, from the accumulator still in TMEM (pass 2): the Z_i
      // store of an activated F_i, and the bias-gradient column sums of an
      // identity-activation dO_i (round(acc) again; act' = 1).
      // split-K chain op (skinny stacks): every split stores its fp32 partial
      // and arrives on the tile's counter (one per CTA); the last to arrive
      // sums the partials in split order (deterministic) and runs the epilogue
      const bool sk = SK && T.ks > 1;
      const bool late_z = !sk && T.kind == EPI_FWD && zout != nullptr && act == ACT_RELU && !(dbg & 1);
      const bool late_db = !sk && T.kind == EPI_DGRAD && dbpart != nullptr && act == ACT_ID;
      // partial [s][row block][32-col chunk][8 float4 columns][128 rows] --
      // float4 j of chunk c of this thread's row; a warp's 32 rows are 512
      // contiguous bytes per float4 (coalesced stores and loads)
      float4 *skrow = sk ? reinterpret_cast<float4 *>(p.skpart) + ((size_t)mblk * p.sk_nc + (T.n0 >> 5)) * 8 * 128 +
                               (q * 32 + lane)
                         : nullptr;
      const size_t sk_split = (size_t)cl.MT * p.sk_nc * 8 * 128;   // float4 per split
      if (sk) {
        for (int c = h; c < cend; c += kEpiPerQ) {
          uint32_t r2[32];
          tmem_ld32_issue(tbase + (uint32_t)(c * 32), r2);
          tmem_ld_wait(r2);
          if (row_ok) {
            float4 *dst = skrow + T.s * sk_split + (size_t)c * 8 * 128;
#pragma unroll
            for (int j = 0; j < 8; ++j)
              __stcg(dst + j * 128, make_float4(__uint_as_float(r2[4 * j]), __uint_as_float(r2[4 * j + 1]),
                                                __uint_as_float(r2[4 * j + 2]), __uint_as_float(r2[4 * j + 3])));
          }
        }
        fence_before();                          // the accumulator is free again (TMEM no longer read)
        __syncwarp();
        if (lane == 0) {
          if (leader) mbar_arrive(bar_tempty + 8 * acc);
          else mbar_arrive_cluster_signal(L_tempty + 8 * acc);
        }
        ebar();                                  // all partial stores of this CTA precede the arrival
        if (tr2) etrace2(t, 6);
        if (et == 0) {
          const int old = atom_add_acq_rel(ctr + cl.sk + o.sk_base + T.tile * CG + (int)rank, 1);
          *sk_flag = old == T.ks - 1;
        }
        if (tr2) etrace2(t, 7);
        ebar();
        if (!*sk_flag) continue;                 // another split finishes this tile
      }
      uint32_t ra[32];
      if (!sk && h < cend) tmem_ld32_issue(tbase + (uint32_t)(h * 32), ra);
      for (int c = h; c < cend; c += kEpiPerQ) {
        const int col0 = T.n0 + c * 32;
        float v[32];
        if (sk) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
          if (row_ok) {
            // split order (deterministic whoever arrived last); all loads of a
            // split issued before its adds, splits unrolled up to 8
#pragma unroll
            for (int s2 = 0; s2 < 8; ++s2) {
              if (s2 < T.ks) {
                const float4 *src = skrow + s2 * sk_split + (size_t)c * 8 * 128;
                float4 f[8];
#pragma unroll
                for (int j = 0; j < 8; ++j) f[j] = __ldcg(src + j * 128);
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                  v[4 * j] += f[j].x;
                  v[4 * j + 1] += f[j].y;
                  v[4 * j + 2] += f[j].z;
                  v[4 * j + 3] += f[j].w;
                }
              }
            }
          }
        } else {
          tmem_ld_wait(ra);
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(ra[i]);
          if (c + kEpiPerQ < cend) tmem_ld32_issue(tbase + (uint32_t)((c + kEpiPerQ) * 32), ra);
        }
        if (tr2 && c == h) etrace2(t, 1);
        if (T.kind == EPI_FWD) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] += bias_s[c * 32 + i];
          uint32_t u[16];
          pack32(v, u);                                         // Z_i in bf16 (RNE)
          if (act == ACT_ID || (dbg & 1)) {
            if (!(dbg & 2)) store32_rows_packed(out, T.N, stg, lane, u, col0, row0, T.M);   // X_{i+1} = Z_i (or Y)
          } else if (act == ACT_GELU) {
            // X_{i+1} = gelu(Z_i) and, for the next backward, gelu'(Z_i) in
            // the Z_i store (one Phi / e^{-z^2/2} evaluation for both; the
            // backward's dO_{i+1} epilogue then only multiplies)
            unpack32(u, v);
            float d[32];
            gelu_and_grad_chunk32(v, d);
            if (!(dbg & 2)) {
              store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);    // X_{i+1} (or Y)
              store32_rows(zout, T.N, stg, lane, d, col0, row0, T.M);   // gelu'(Z_i)
            }
          } else {
            // ReLU: Z_i (needed only by the next backward) is stored in pass 2
            unpack32(u, v);
            act_chunk32(act, v);
            if (!(dbg & 2)) store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);  // X_{i+1} (or Y)
          }
        } else if (T.kind == EPI_DGRAD) {
          if (need_z && !(dbg & 1)) {
            float z[32];
            unpack_bf16x32(zr, z);
            if (c + kEpiPerQ < cend) ld_raw32(zrow + (c + kEpiPerQ) * 32, zr);
            act_grad_mul_chunk32(act, v, z);
          }
          uint32_t u[16];
          pack32(v, u);                                         // dZ_{i-1} in bf16 (RNE)
#pragma unroll
          for (int j = 0; j < 16; ++j) u[j] = row_ok ? u[j] : 0u;
          if (!(dbg & 2)) store32_rows_packed(out, T.N, stg, lane, u, col0, row0, T.M);  // dZ_{i-1} (or dX)
          if (dbpart && !late_db) {
            unpack32(u, v);
            red[q * kMaxBN + c * 32 + lane] = warp_colsum32(v, lane);
          }
        } else {  // EPI_WGRAD: one split, scaled bf16 straight into the gradient bucket
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] *= alpha;
          store32_rows(out, T.N, stg, lane, v, col0, row0, T.M);
        }
        if (tr2 && c == h) etrace2(t, 2);
      }
      if (tr2) etrace2(t, 3);
      // ---- early publish of the row-local chain output (X_{i+1} / dZ_{i-1}):
      // release reductions are cumulative, so every store of the pass above
      // (all epilogue warps, ordered by the barrier) is visible before the count
      if (T.kind != EPI_WGRAD) {
        ebar();
        if (et == 0 && mrow0 < T.M) {
          if (T.kind == EPI_FWD) publish(cl.fwd_rows + (T.layer - 1) * cl.MT + mblk, -1, -1);
          else if (T.layer >= 2) publish(cl.dz_rows + (T.layer - 2) * cl.MT + mblk, -1, -1);
          else publish(cl.dx_total, -1, -1);   // dX (the input gradient a previous stage waits for)
          if (leader) etrace(t, 3);
        }
      }
      if (late_z || late_db) {   // ---- pass 2: off-critical-path work from TMEM
        if (h < cend) tmem_ld32_issue(tbase + (uint32_t)(h * 32), ra);
        for (int c = h; c < cend; c += kEpiPerQ) {
          const int col0 = T.n0 + c * 32;
          tmem_ld_wait(ra);
          float v[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(ra[i]);
          if (c + kEpiPerQ < cend) tmem_ld32_issue(tbase + (uint32_t)((c + kEpiPerQ) * 32), ra);
          uint32_t u[16];
          if (late_z) {
#pragma unroll
            for (int i = 0; i < 32; ++i) v[i] += bias_s[c * 32 + i];
            pack32(v, u);
            if (!(dbg & 2)) store32_rows_packed(zout, T.N, stg, lane, u, col0, row0, T.M);   // Z_i
          } else {
            pack32(v, u);
#pragma unroll
            for (int j = 0; j < 16; ++j) u[j] = row_ok ? u[j] : 0u;
            unpack32(u, v);
            red[q * kMaxBN + c * 32 + lane] = warp_colsum32(v, lane);
          }
        }
      }
      // accumulator buffer free for task j+2 (the leader's barrier counts all
      // CTAs; a split-K task released it after storing its partial)
      if (!sk) {
        fence_before();
        __syncwarp();
        if (lane == 0) {
          if (leader) mbar_arrive(bar_tempty + 8 * acc);
          else mbar_arrive_cluster_signal(L_tempty + 8 * acc);
        }
      }
      if (T.kind == EPI_DGRAD && dbpart && mblk < cl.MT) {
        ebar();
        for (int cc = et; cc < T.bn; cc += kEpiThreads) {
          const int col = T.n0 + cc;
          if (col < T.N) {
            const float s = ((red[cc] + red[kMaxBN + cc]) + red[2 * kMaxBN + cc]) + red[3 * kMaxBN + cc];
            dbpart[(size_t)mblk * T.N + col] = s;
          }
        }
      }
      if (T.kind == EPI_WGRAD && mrow0 == 0) {
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
      // ---- publish completion of this CTA's rows (release)
      if (tr2) etrace2(t, 4);
      ebar();
      if (tr2) etrace2(t, 5);
      if (et == 0 && mrow0 < T.M) {
        // release reductions are cumulative: every store of the tile (all
        // epilogue warps, ordered by the barrier above) is visible before the count
        // (F_i: nothing left to publish -- its Z_i store is ordered before the
        // next backward by the launch boundary)
        if (T.kind == EPI_DGRAD) {
          if (T.layer >= 2) publish(cl.dz_total + (T.layer - 2), -1, -1);   // + the db partials
        } else if (T.kind == EPI_WGRAD) {
          publish(cl.dw_done + (T.layer - 1), cl.bucket_done + Ld.bucket, -1);
          if (leader) etrace(t, 3);
        }
      }
    }
  }
  fence_before();
  if (CG == 2) cluster_sync(); else __syncthreads();   // no CTA leaves while its peer may still signal it
  if (warp == 1) {
    fence_after();
    if (CG == 2)
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS)
                   : "memory");
    else
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS)
                   : "memory");
  }
}

int engine_smem_bytes(int cg) { return cg == 2 ? Cfg<2>::SMEM : Cfg<1>::SMEM; }

#ifdef OOO_TRACE
cudaError_t engine_set_trace(void *p) {
  const char *kt = getenv("OOO_KTASK");
  const int ktask = kt && *kt ? atoi(kt) : 0;
  cudaError_t e0 = cudaMemcpyToSymbol(g_ktask, &ktask, sizeof(ktask));
  if (e0 != cudaSuccess) return e0;
  // [task][8] phase stamps, [task][8] epilogue clocks, [task][8] pipeline stamps (same buffer)
  void *p2 = p ? static_cast<char *>(p) + (size_t)200000 * 8 * 8 : nullptr;
  void *p3 = p ? static_cast<char *>(p) + (size_t)2 * 200000 * 8 * 8 : nullptr;
  cudaError_t e = cudaMemcpyToSymbol(g_etrace, &p, sizeof(p));
  if (e == cudaSuccess) e = cudaMemcpyToSymbol(g_etrace2, &p2, sizeof(p2));
  if (e == cudaSuccess) e = cudaMemcpyToSymbol(g_etrace3, &p3, sizeof(p3));
  return e;
}
#endif

cudaError_t engine_init() {
  cudaError_t e = cudaFuncSetAttribute(engine_kernel<1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<1>::SMEM);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(engine_kernel<2, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<2>::SMEM);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(engine_kernel<1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<1>::SMEM);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(engine_kernel<2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg<2>::SMEM);
  return e;
}

cudaError_t launch_engine(int cg, const Params &p, const CUtensorMap *tmY, const CUtensorMap *tmDX,
                          const CUtensorMap *tmX, int ctas,
                          cudaStream_t stream, int priority) {
  bool sk = false;
  for (int j = 0; j < p.nops && !sk; ++j) sk = p.ops[j].ks > 1;
  cudaLaunchConfig_t cfg = {};
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.stream = stream;
  cudaLaunchAttribute attr[3];
  attr[0].id = cudaLaunchAttributePriority;
  attr[0].val.priority = priority;
  // programmatic dependent launch: the prologue (TMEM allocation, barrier
  // setup, cluster sync) overlaps the preceding kernel (the seed); every
  // read of its data follows griddepcontrol.wait (pdl_wait)
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = OOO_ENGINE_PDL;
  if (cg == 2) {
    cfg.gridDim = dim3((ctas / 2) * 2, 1, 1);   // whole CTA pairs
    cfg.dynamicSmemBytes = Cfg<2>::SMEM;
    attr[2].id = cudaLaunchAttributeClusterDimension;
    attr[2].val.clusterDim.x = 2;
    attr[2].val.clusterDim.y = 1;
    attr[2].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 3;
    return sk ? cudaLaunchKernelEx(&cfg, engine_kernel<2, true>, *tmY, *tmDX, *tmX, p)
              : cudaLaunchKernelEx(&cfg, engine_kernel<2, false>, *tmY, *tmDX, *tmX, p);
  }
  cfg.gridDim = dim3(ctas, 1, 1);
  cfg.dynamicSmemBytes = Cfg<1>::SMEM;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  return sk ? cudaLaunchKernelEx(&cfg, engine_kernel<1, true>, *tmY, *tmDX, *tmX, p)
            : cudaLaunchKernelEx(&cfg, engine_kernel<1, false>, *tmY, *tmDX, *tmX, p);
}

}  // namespace eng
}  // namespace ooo
