// Skinny-stack step kernel: see skinny.h for the design.  Same step and the
// same stores / counters as engine.cu (paper §2: F_i, dO_i, dW_i;
// §5.1: F_i(t+1) gated on S[dW_i]); only the tiling of a 16-row chain
// op (K split over an 8-CTA cluster, DSMEM reduction) and the static chain
// schedule differ.
#include <cuda_bf16.h>

#include "skinny.h"
#include "tc_common.cuh"

namespace ooo {
namespace sk {

using namespace ooo::tc;
using eng::CounterLayout;
using eng::EPI_COPY;
using eng::LayerDev;

namespace {

constexpr int kThreads = 192;    // warps 0-3: TMEM lane quarters (epilogue), 4: producer, 5: MMA
constexpr int STAGES = 7;        // chain ring: one 64-deep k-block per stage
constexpr int A_SK = 2048;       // 16 rows x 128 B (K-major, SW128)
constexpr int B_SK = 16384;      // <= 128 N x 64 K bf16
constexpr int STAGE = A_SK + B_SK;
constexpr int RING = STAGES * STAGE;
// Chain-tile reduction (reduce-scatter over the cluster): CTA o owns columns
// [o cs, o cs + cs) of the tile (cs = tn / kCl); each CTA sends the owner its
// fp32 partial of those columns (a block of kMaxM rows x RS floats, RS = cs + 4:
// the pad spreads the rows over the banks) into the owner's receive slot
// [sender], double-buffered by task parity.
constexpr int RS_MAX = 128 / kCl + 4;
constexpr int BLK_MAX = kMaxM * RS_MAX * 4;          // one sender -> owner block (bytes)
constexpr int SEND_OFF = RING;                       // [2][kCl owners][BLK_MAX]
constexpr int RECV_OFF = SEND_OFF + 2 * kCl * BLK_MAX;   // [2][kCl senders][BLK_MAX]
constexpr int STG_OFF = (RECV_OFF + 2 * kCl * BLK_MAX + 1023) / 1024 * 1024;
constexpr int BAR_OFF = STG_OFF + 4 * 2048;
constexpr int NBARS = 2 * STAGES + 6 + 8 + 8;
constexpr int SLOT_OFF = BAR_OFF + NBARS * 8;
constexpr int SMEM = SLOT_OFF + 64 + 1024;
constexpr int DW_BUF = 16384;    // dW role: A (2 panels x 2 KB) + B (<= 4 panels x 2 KB) per buffer
constexpr int Q = 4;             // dW task ring
constexpr uint32_t TMEM_COLS = 512;
static_assert(SMEM <= kSmemBudget, "skinny smem budget");
static_assert(STAGE % 1024 == 0 && RING % 1024 == 0, "alignment");
static_assert(2 * DW_BUF <= RING, "dW buffers live in the ring");

__shared__ uint64_t s_tmo;

#ifdef OOO_TRACE
// debug builds: globaltimer stamps per chain task [op j][tile t < 32][8]
__device__ unsigned long long *g_sktrace = nullptr;
__device__ __forceinline__ void sktrace(int j, int t, int slot) {
  if (g_sktrace) {
    unsigned long long v;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(v));
    g_sktrace[((size_t)j * 32 + t) * 8 + slot] = v;
  }
}
#else
__device__ __forceinline__ void sktrace(int, int, int) {}
#endif

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t cluster_id() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
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
// Relaxed arrive on a peer's barrier (a bare SYNCS.ARRIVE; the release form
// is a MEMBAR.ALL.GPU that waits for this thread's global stores in flight):
// the receive-slot "free" signal publishes no memory -- the slot's reads are
// performed before it (CTA barrier).
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
// non-blocking phase test (try_wait may suspend the thread for a while: the
// producer's loop polls two cursors and must not stall on either)
__device__ __forceinline__ bool mbar_test(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
// bounded waits (trap instead of hanging: a broken schedule or a stalled peer rank)
__device__ __forceinline__ void wait_bar(uint32_t bar, uint32_t parity, bool sleep) {
  uint64_t t0 = 0;
  for (uint32_t n = 1; !mbar_try_wait(bar, parity); ++n) {
    if (sleep) __nanosleep(32);
    if ((n & 1023u) == 0) {
      if (t0 == 0) t0 = gtimer();
      else if (gtimer() - t0 > s_tmo) __trap();
    }
  }
}
__device__ __forceinline__ int ld_relaxed(const int32_t *p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_acquire(const int32_t *p) {
  int v;
  asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void wait_ge(const int32_t *p, int target) {
  if (ld_relaxed(p) < target) {
    const uint64_t t0 = gtimer();
    while (ld_relaxed(p) < target) {
      __nanosleep(32);
      if (gtimer() - t0 > s_tmo) __trap();
    }
  }
  (void)ld_acquire(p);
}
__device__ __forceinline__ void red_add(int32_t *p, int v) {
  asm volatile("red.relaxed.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void red_release_add(int32_t *p, int v) {
  asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}


// The chain op's shape: output width N, reduction length K, tile width.
struct OpShape {
  int kind, layer, N, K, tn, ntiles, nkb;
};
__device__ __forceinline__ OpShape shape_of(const Params &p, int j) {
  OpShape s;
  s.kind = p.chain[j].kind;
  s.layer = p.chain[j].layer;
  const LayerDev &L = p.layers[s.layer - 1];
  s.N = s.kind == EPI_FWD ? L.dout : L.din;
  s.K = s.kind == EPI_FWD ? L.din : L.dout;
  s.tn = s.kind == EPI_FWD ? L.fwd_bn : L.dx_bn;
  s.ntiles = s.N / s.tn;
  s.nkb = (s.K + 63) / 64;
  return s;
}
// this CTA's k-blocks of a chain tile: [kb0, kb1)
__device__ __forceinline__ int kb_lo(int nkb, int r) { return nkb * r / kCl; }

// The chain tasks of cluster c, in chain order: (op j, tile t = c, c + nclu, ...).
struct Cur {
  int j, t;
  bool done;
};
__device__ __forceinline__ void cur_next(const Params &p, Cur &c, int clu, OpShape &sh) {
  if (c.j >= 0) c.t += p.nclu;
  if (c.j >= 0 && c.t < sh.ntiles) return;
  for (;;) {
    ++c.j;
    if (c.j >= p.nchain) {
      c.done = true;
      return;
    }
    sh = shape_of(p, c.j);
    c.t = clu;
    if (c.t < sh.ntiles) return;
  }
}

// Gates of F_i: S[dW_i] done (N = 1: its dW tiles; N > 1: its
// bucket's all-reduce flag) and dW_{i+1} done (it reads X_{i+1}, which F_i
// overwrites).  dO_i (in_order, conventional backprop): dW_{i+1} first.
// Counter c reached target: relaxed poll, then (met) one acquire load of it.
__device__ __forceinline__ bool reached(const int32_t *c, int target) {
  if (ld_relaxed(c) < target) return false;
  (void)ld_acquire(c);
  return true;
}
template <bool ACQ>
__device__ __forceinline__ bool gate_ok(const Params &p, const OpShape &sh) {
  const CounterLayout &cl = p.cl;
  const int i = sh.layer;
  if (sh.kind == EPI_FWD) {
    if (!p.fwd_gate) return true;
    const LayerDev &L = p.layers[i - 1];
    if (p.fwd_gate == 1 && !reached(p.ctr + cl.dw_done + i - 1, L.dw_tiles)) return false;
    if (p.fwd_gate == 2 && !reached(p.ctr + cl.ar_done + L.bucket, 1)) return false;
    if (i < cl.L && !reached(p.ctr + cl.dw_done + i, p.layers[i].dw_tiles)) return false;
    return true;
  }
  if (p.in_order && i < cl.L && !reached(p.ctr + cl.dw_done + i, p.layers[i].dw_tiles)) return false;
  return true;
}
// The op's A rows complete: F_i reads X_i (F_{i-1}'s tiles; F_1: the caller's
// X), dO_i reads dZ_i (dO_{i+1}'s tiles; dO_L: the seed's dZ_L).
__device__ __forceinline__ bool input_ok(const Params &p, const OpShape &sh) {
  const CounterLayout &cl = p.cl;
  const int i = sh.layer;
  if (sh.kind == EPI_FWD) {
    if (i == 1) return true;
    return reached(p.ctr + cl.fwd_rows + (i - 2) * cl.MT, p.layers[i - 2].fwd_nt * kPubPerTile);
  }
  if (i == cl.L) return true;
  return reached(p.ctr + cl.dz_rows + (i - 1) * cl.MT, p.layers[i].dx_nt * kPubPerTile);
}

// dW workers: a dynamic queue of dW_i tiles in D's order
// (Alg. 2) and the X -> X_1 copy; warps 0-3 epilogue, 4 dispenser +
// producer, 5 MMA.  dw_base: 2 x DW_BUF operand buffers; stg_base: 4 x 2 KB
// store staging; the barrier addresses are this CTA's.
__device__ __forceinline__ void dw_worker(const Params &p, int warp, int lane, uint32_t tmem, uint32_t dw_base,
                                          uint32_t stg_base, volatile int *task_slot, uint32_t d_buffull,
                                          uint32_t d_bufempty, uint32_t d_accfull, uint32_t d_accfree,
                                          uint32_t qfull, uint32_t qempty) {
  const CounterLayout &cl = p.cl;
  int32_t *ctr = p.ctr;
  // ================================================================ dW workers
  const int M = p.M;
  const int ksteps = (M + 15) / 16;   // 16-deep MMA K steps over the tokens (TMA zero-fills rows >= M)
  auto decode = [&](int t, int &op, int &rt, int &ct) {
    int lo = 0, hi = p.ndw - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (p.dw[mid].first <= t) lo = mid; else hi = mid - 1;
    }
    op = lo;
    const int rel = t - p.dw[op].first;
    if (p.dw[op].kind == EPI_COPY) {
      rt = ct = 0;
      return;
    }
    const LayerDev &L = p.layers[p.dw[op].layer - 1];
    const int nt = (L.dout + L.dw_bn - 1) / L.dw_bn;   // the last tile may be ragged
    rt = rel / nt;
    ct = rel % nt;
  };
  if (warp == 4 && lane == 0) {
    // ---- dispenser + producer
    int g = 0;
    for (int j = 0;; ++j) {
      const int slot = j % Q;
      if (j >= Q) wait_bar(qempty + 8 * slot, ((j / Q) - 1) & 1, false);
      int t = atomicAdd(ctr + 1, 1);
      if (t >= p.ntasks_dw) t = -1;
      task_slot[slot] = t;
      mbar_arrive(qfull + 8 * slot);
      if (t < 0) break;
      int op, rt, ct;
      decode(t, op, rt, ct);
      if (p.dw[op].kind == EPI_COPY) continue;
      const int i = p.dw[op].layer;
      const LayerDev &L = p.layers[i - 1];
      const int b = g & 1;
      if (g >= 2) wait_bar(d_bufempty + 8 * b, ((g >> 1) - 1) & 1, false);
      if (i < cl.L) wait_ge(ctr + cl.dz_total + (i - 1), cl.MT * p.layers[i].dx_nt * kPubPerTile);   // dZ_i complete
      asm volatile("fence.proxy.async.global;" ::: "memory");
      const uint32_t buf = dw_base + b * DW_BUF;
      const int npb = L.dw_bn / 64;
      mbar_expect_tx(d_buffull + 8 * b, 2 * 2048 + npb * 2048);
      const CUtensorMap *mX = p.maps + (size_t)(i - 1) * p.maps_per_layer + p.map_x;
      const CUtensorMap *mD = p.maps + (size_t)(i - 1) * p.maps_per_layer + p.map_dz;
      for (int c = 0; c < 2; ++c) tma_load_2d(buf + 2048 * c, mX, d_buffull + 8 * b, rt * 128 + 64 * c, 0);
      for (int c = 0; c < npb; ++c) tma_load_2d(buf + 4096 + 2048 * c, mD, d_buffull + 8 * b, ct * L.dw_bn + 64 * c, 0);
      ++g;
    }
  } else if (warp == 5 && lane == 0) {
    // ---- MMA: dW tile = X_i^T (MN-major, 128 features) x dZ_i (MN-major), K = tokens
    int g = 0;
    for (int j = 0;; ++j) {
      const int slot = j % Q;
      wait_bar(qfull + 8 * slot, (j / Q) & 1, false);
      const int t = task_slot[slot];
      mbar_arrive(qempty + 8 * slot);
      if (t < 0) break;
      int op, rt, ct;
      decode(t, op, rt, ct);
      if (p.dw[op].kind == EPI_COPY) continue;
      const LayerDev &L = p.layers[p.dw[op].layer - 1];
      const int b = g & 1;
      if (g >= 2) wait_bar(d_accfree + 8 * b, ((g >> 1) - 1) & 1, false);
      wait_bar(d_buffull + 8 * b, (g >> 1) & 1, false);
      fence_after();
      const uint32_t buf = dw_base + b * DW_BUF;
      const uint64_t ad = sdesc(buf, 2048, 1024), bd = sdesc(buf + 4096, 2048, 1024);
      const uint32_t ID = idesc_rt(L.dw_bn, true, true);
      for (int kk = 0; kk < ksteps; ++kk)
        umma_bf16(tmem + (uint32_t)(b * 256), ad + 128u * kk, bd + 128u * kk, ID, kk > 0 ? 1u : 0u);
      umma_commit(d_bufempty + 8 * b);
      umma_commit(d_accfull + 8 * b);
      ++g;
    }
  } else if (warp < 4) {
    // ---- epilogue: scaled bf16 dW_i into the gradient bucket; db_i; the X -> X_1 copy
    const int q = warp;
    const int et = threadIdx.x;   // 0..127
    const uint32_t stg = stg_base + q * 2048;
    int g = 0;
    for (int j = 0;; ++j) {
      const int slot = j % Q;
      wait_bar(qfull + 8 * slot, (j / Q) & 1, true);
      const int t = task_slot[slot];
      epi_bar();
      if (et == 0) mbar_arrive(qempty + 8 * slot);
      if (t < 0) break;
      int op, rt, ct;
      decode(t, op, rt, ct);
      if (p.dw[op].kind == EPI_COPY) {
        // caller's X -> X_1 store (the next backward's dW_1 input); the
        // pending dW_1 still reads X_1: wait for it first
        if (p.fwd_gate && et == 0) wait_ge(ctr + cl.dw_done, p.layers[0].dw_tiles);
        epi_bar();
        const int n = M * p.layers[0].din / 8;
        const uint4 *src = reinterpret_cast<const uint4 *>(p.x_in);
        uint4 *dst = reinterpret_cast<uint4 *>(p.layers[0].X);
        for (int v = et; v < n; v += 128) dst[v] = __ldg(src + v);
        continue;
      }
      const int i = p.dw[op].layer;
      const LayerDev &L = p.layers[i - 1];
      const int b = g & 1;
      wait_bar(d_accfull + 8 * b, (g >> 1) & 1, true);
      fence_after();
      const uint32_t tb = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(b * 256);
      __nv_bfloat16 *gw = reinterpret_cast<__nv_bfloat16 *>(L.gw);
      const int cend = min(L.dw_bn, L.dout - ct * L.dw_bn) / 32;   // chunks inside dW_i's columns
      for (int ch = 0; ch < cend; ++ch) {
        uint32_t r[32];
        tmem_ld32(tb + (uint32_t)(ch * 32), r);
        float v[32];
#pragma unroll
        for (int x = 0; x < 32; ++x) v[x] = __uint_as_float(r[x]) * p.alpha;
        store32_rows(gw, L.dout, stg, lane, v, ct * L.dw_bn + ch * 32, rt * 128 + q * 32, L.din);
      }
      fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(d_accfree + 8 * b);
      if (rt == 0) {
        // db_i = (1/N) x the bias-gradient partial of the only row block
        __nv_bfloat16 *db = reinterpret_cast<__nv_bfloat16 *>(L.db_out);
        for (int cc = et; cc < L.dw_bn; cc += 128) {
          const int col = ct * L.dw_bn + cc;
          if (col < L.dout) db[col] = __float2bfloat16_rn(__ldcg(L.dbpart + col) * p.alpha);
        }
      }
      epi_bar();
      if (et == 0) {
        red_release_add(ctr + cl.dw_done + (i - 1), 1);
        red_add(ctr + cl.bucket_done + L.bucket, 1);
      }
      ++g;
    }
  }
}

__global__ void __launch_bounds__(kThreads, 1)
    skinny_kernel(const __grid_constant__ CUtensorMap tmX, const __grid_constant__ Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t *smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  const uint32_t sbase = smem_u32(smem);
  const uint32_t bar_full = sbase + BAR_OFF;
  const uint32_t bar_empty = bar_full + 8 * STAGES;
  const uint32_t c_accfull = bar_empty + 8 * STAGES;
  const uint32_t c_accfree = c_accfull + 8;
  const uint32_t rfull = c_accfree + 8;     // [2] owner: every sender's block of its columns landed
  const uint32_t rfree = rfull + 16;        // [2] sender: every owner has read its block
  const uint32_t d_buffull = rfree + 16;    // [2]
  const uint32_t d_bufempty = d_buffull + 16;
  const uint32_t d_accfull = d_bufempty + 16;
  const uint32_t d_accfree = d_accfull + 16;
  const uint32_t qfull = d_accfree + 16;    // [Q]
  const uint32_t qempty = qfull + 8 * Q;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(smem + SLOT_OFF);
  volatile int *task_slot = reinterpret_cast<volatile int *>(smem + SLOT_OFF + 16);
  const CounterLayout &cl = p.cl;
  int32_t *ctr = p.ctr;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cta_rank();
  const int clu = (int)cluster_id();
  const bool chain_role = clu < p.nclu;

  if (threadIdx.x == 0) {
    s_tmo = p.timeout_ns;
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(bar_full + 8 * s, 1);
      mbar_init(bar_empty + 8 * s, 1);
    }
    mbar_init(c_accfull, 1);
    mbar_init(c_accfree, 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(rfull + 8 * b, 1);     // the owner's expect_tx; the senders' bulk copies complete_tx
      mbar_init(rfree + 8 * b, kCl);   // one arrival per owner
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(d_buffull + 8 * b, 1);
      mbar_init(d_bufempty + 8 * b, 1);
      mbar_init(d_accfull + 8 * b, 1);
      mbar_init(d_accfree + 8 * b, 4);
    }
    for (int s = 0; s < Q; ++s) {
      mbar_init(qfull + 8 * s, 1);
      mbar_init(qempty + 8 * s, 2);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  if (warp == 5) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  fence_before();
  cluster_sync();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_wait();

  if (chain_role) {
    // =================================================================== chain
    if (warp == 4 && lane == 0) {
      // ---- producer: B (weights) as soon as a ring stage is free, A (the
      // activation rows) once the producer op's tiles are all published.
      Cur b = {-1, 0, false}, a = {-1, 0, false};
      OpShape bs = {}, as = {};
      cur_next(p, b, clu, bs);
      cur_next(p, a, clu, as);
      int bkb = kb_lo(bs.nkb, rank), sB = 0;   // B cursor: next k-block, stages claimed
      bool bgate = false;
      int sA = 0;                              // A cursor: next stage to fill with activation rows
      int akb = kb_lo(as.nkb, rank);           // its next k-block
      bool aready = false;                     // its task's input rows are complete
      uint64_t t_last = gtimer();
      while (!a.done) {
        bool prog = false;
        if (!b.done) {
          const int kb1 = kb_lo(bs.nkb, rank + 1);
          if (bkb >= kb1) {
            cur_next(p, b, clu, bs);
            if (!b.done) bkb = kb_lo(bs.nkb, rank);
            bgate = false;
            prog = true;
          } else {
            const int s = sB % STAGES;
            const bool ahead = (p.dbg & 1) && (b.j != a.j || b.t != a.t);   // experiment: no prefetch
            const bool free = !ahead && (sB < STAGES || mbar_test(bar_empty + 8 * s, ((sB / STAGES) - 1) & 1));
            if (free && !bgate && gate_ok<true>(p, bs)) {
              // (acquire loads of the gates' counters inside) then the TMA
              // (async proxy) reads are ordered after them.  No fence.acq_rel:
              // it would wait for this thread's weight prefetches in flight
              asm volatile("fence.proxy.async.global;" ::: "memory");
              bgate = true;
              if (rank == 0) sktrace(b.j, b.t, 4);
            }
            if (free && bgate) {
              const uint32_t st = sbase + s * STAGE;
              mbar_expect_tx(bar_full + 8 * s, A_SK + bs.tn * 128);
              const CUtensorMap *mW = p.maps + (size_t)(bs.layer - 1) * p.maps_per_layer + p.map_w;
              const int n0 = b.t * bs.tn;
              for (int c = 0; c < bs.tn / 64; ++c) {
                if (bs.kind == EPI_FWD) tma_load_2d(st + A_SK + 8192 * c, mW, bar_full + 8 * s, n0 + 64 * c, bkb * 64);
                else tma_load_2d(st + A_SK + 8192 * c, mW, bar_full + 8 * s, bkb * 64, n0 + 64 * c);
              }
              ++sB;
              ++bkb;
              prog = true;
            }
          }
        }
        {
          // A cursor: k-block akb of task a, whose stage sA the B cursor has
          // claimed, once the op's input rows are complete (checked once)
          const int akb1 = kb_lo(as.nkb, rank + 1);
          if (akb >= akb1) {
            cur_next(p, a, clu, as);
            if (!a.done) akb = kb_lo(as.nkb, rank);
            aready = false;
            prog = true;
          } else if (sB > sA && (aready || input_ok(p, as))) {
            if (!aready) {
              asm volatile("fence.proxy.async.global;" ::: "memory");   // TMA reads see the producers' stores
              if (rank == 0) sktrace(a.j, a.t, 5);
              aready = true;
            }
            const CUtensorMap *mA =
                (as.kind == EPI_FWD && as.layer == 1)
                    ? &tmX
                    : p.maps + (size_t)(as.layer - 1) * p.maps_per_layer + (as.kind == EPI_FWD ? p.map_x : p.map_dz);
            for (; akb < akb1 && sA < sB; ++akb, ++sA) {
              const int s = sA % STAGES;
              tma_load_2d(sbase + s * STAGE, mA, bar_full + 8 * s, akb * 64, 0);
            }
            prog = true;
          }
        }
        if (prog) {
          t_last = gtimer();
        } else {
          __nanosleep(20);
          if (gtimer() - t_last > s_tmo) __trap();
        }
      }
    } else if (warp == 5 && lane == 0) {
      // ---- MMA issuer: the CTA's k-blocks of each task into the TMEM accumulator
      Cur c = {-1, 0, false};
      OpShape sh = {};
      cur_next(p, c, clu, sh);
      int sM = 0, uses = 0;
      while (!c.done) {
        const int kb0 = kb_lo(sh.nkb, rank), kb1 = kb_lo(sh.nkb, rank + 1);
        if (kb1 > kb0) {
          if (uses > 0) wait_bar(c_accfree, (uses - 1) & 1, false);
          fence_after();
          const bool b_mn = sh.kind == EPI_FWD;
          const uint32_t ID = idesc_rt(sh.tn, false, b_mn);
          for (int kb = kb0; kb < kb1; ++kb, ++sM) {
            const int s = sM % STAGES;
            wait_bar(bar_full + 8 * s, (sM / STAGES) & 1, false);
            fence_after();
            const uint32_t st = sbase + s * STAGE;
            const uint64_t ad = sdesc(st, 16, 1024);
            const uint64_t bd = b_mn ? sdesc(st + A_SK, 8192, 1024) : sdesc(st + A_SK, 16, 1024);
            const uint64_t bstep = b_mn ? 128u : 2u;
#pragma unroll
            for (int k = 0; k < 4; ++k) umma_bf16(tmem, ad + 2u * k, bd + bstep * k, ID, (kb > kb0 || k > 0) ? 1u : 0u);
            umma_commit(bar_empty + 8 * s);
          }
          umma_commit(c_accfull);
          ++uses;
        }
        cur_next(p, c, clu, sh);
      }
    } else if (warp < 4) {
      // ---- reduce-scatter of the K-split partials, then the epilogue of this
      // CTA's column slice.  Warp 0 reads the accumulator (TMEM lanes 0-15 =
      // token rows) into the send buffer, one block per owner, and bulk-copies
      // block o into owner o's receive slot [rank] over DSMEM (complete_tx on
      // the owner's rfull).  Every CTA (4 warps) then sums the kCl senders'
      // blocks of its cs columns in rank order (deterministic; the same order
      // as a single reducer) and runs the epilogue on 16 x cs outputs: 1-2 per
      // thread, so its latency is a fraction of one reducer's 16 per thread.
      Cur c = {-1, 0, false};
      OpShape sh = {};
      cur_next(p, c, clu, sh);
      int uses = 0, k = 0;
      const int M = p.M;
      const int et = threadIdx.x;                 // 0..127
      const uint32_t sendb = sbase + SEND_OFF;
      const uint32_t recvb = sbase + RECV_OFF;
      float *red_s = reinterpret_cast<float *>(smem + STG_OFF);   // [16 rows][cs] dbpart staging
      const int er = et >> 3;                     // epilogue: row, and 1-2 columns of the slice
      while (!c.done) {
        const int kb0 = kb_lo(sh.nkb, rank), kb1 = kb_lo(sh.nkb, rank + 1);
        const bool mine = kb1 > kb0;
        const int nch = sh.tn / 32;
        const int i = sh.layer;
        const LayerDev &Ld = p.layers[i - 1];
        const int n0 = c.t * sh.tn;
        const int cs = sh.tn / kCl;               // owned columns (8 or 16)
        const int RS = cs + 4;
        const int blk = kMaxM * RS * 4;
        const int ncol = cs / 8;                  // per thread
        const int ec = (et & 7) * ncol;           // within the slice
        const int gc = n0 + (int)rank * cs + ec;  // global column
        const int b = k & 1;
        // epilogue inputs that do not depend on the chain, requested first
        uint32_t pre = 0;
        if (sh.kind == EPI_FWD) {
          const __nv_bfloat16 *bp = reinterpret_cast<const __nv_bfloat16 *>(Ld.bias) + gc;
          pre = ncol == 2 ? __ldg(reinterpret_cast<const uint32_t *>(bp))
                          : (uint32_t)__bfloat16_as_ushort(bp[0]);
        } else if (i >= 2 && p.layers[i - 2].act != ACT_ID && p.layers[i - 2].Z && er < M) {
          const __nv_bfloat16 *zp = reinterpret_cast<const __nv_bfloat16 *>(p.layers[i - 2].Z) + (size_t)er * sh.N + gc;
          pre = ncol == 2 ? __ldg(reinterpret_cast<const uint32_t *>(zp)) : (uint32_t)__bfloat16_as_ushort(zp[0]);
        }
        int contrib = 0;
        for (int rr = 0; rr < kCl; ++rr) contrib += kb_lo(sh.nkb, rr + 1) > kb_lo(sh.nkb, rr);
        if (et == 0) {
          mbar_expect_tx(rfull + 8 * b, (uint32_t)(contrib * blk));
          if (rank == 0) sktrace(c.j, c.t, 0);
        }
        if (warp == 0 && mine) {
          // send slot b free: every owner has read task k-2's blocks
          if (k >= 2) wait_bar(rfree + 8 * b, ((k >> 1) - 1) & 1, true);
          wait_bar(c_accfull, uses & 1, true);
          fence_after();
          if (rank == 0 && et == 0) sktrace(c.j, c.t, 1);
          const uint32_t sb = sendb + b * kCl * BLK_MAX + lane * RS * 4;
          for (int ch = 0; ch < nch; ch += 2) {
            uint32_t r0[32], r1[32];
            tmem_ld32_issue(tmem + (uint32_t)(ch * 32), r0);
            tmem_ld32_issue(tmem + (uint32_t)((ch + 1) * 32), r1);
            tmem_ld_wait(r0);
            tmem_ld_wait(r1);
            if (lane < kMaxM) {
#pragma unroll
              for (int q = 0; q < 16; ++q) {       // 4 columns per store, one owner each (cs % 4 == 0)
                const int col = ch * 32 + 4 * q;
                const uint32_t *rr = q < 8 ? &r0[4 * q] : &r1[4 * (q - 8)];
                const int o = col / cs;
                asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(sb + o * blk + (col - o * cs) * 4),
                             "r"(rr[0]), "r"(rr[1]), "r"(rr[2]), "r"(rr[3])
                             : "memory");
              }
            }
          }
          fence_before();
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // send blocks -> bulk copies
          __syncwarp();
          if (lane == 0) mbar_arrive(c_accfree);
          if (lane < kCl) {                        // one lane per owner
            const uint32_t src = sendb + b * kCl * BLK_MAX + lane * blk;
            asm volatile(
                "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    mapa(recvb + (b * kCl + (int)rank) * BLK_MAX, lane)),
                "r"(src), "r"(blk), "r"(mapa(rfull + 8 * b, lane))
                : "memory");
          }
          ++uses;
        }
        // ---- owner: every sender's block of this CTA's columns landed
        wait_bar(rfull + 8 * b, (k >> 1) & 1, true);
        if (rank == 0 && et == 0) sktrace(c.j, c.t, 2);
        const bool act_row = er < M;
        float v[2] = {0.f, 0.f};
        {
          const uint32_t src0 = recvb + b * kCl * BLK_MAX + (er * RS + ec) * 4;
          for (int rr = 0; rr < kCl; ++rr) {
            if (kb_lo(sh.nkb, rr + 1) == kb_lo(sh.nkb, rr)) continue;   // that CTA had no k-blocks
            float x, y = 0.f;
            if (ncol == 2)
              asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(x), "=f"(y) : "r"(src0 + rr * BLK_MAX) : "memory");
            else
              asm volatile("ld.shared.f32 %0, [%1];" : "=f"(x) : "r"(src0 + rr * BLK_MAX) : "memory");
            v[0] += x;
            v[1] += y;
          }
        }
        const int off = er * sh.N + gc;
        bool publish_db = false;
        const float p0 = __uint_as_float(pre << 16), p1 = __uint_as_float(pre & 0xFFFF0000u);
        if (sh.kind == EPI_FWD) {
          // Z_i = acc + b_i in bf16 (RNE); X_{i+1} = act(Z_i)
          const uint32_t u = pack_bf2(v[0] + p0, v[1] + p1);
          const float z0 = bf_lo(u), z1 = bf_hi(u);
          __nv_bfloat16 *out = reinterpret_cast<__nv_bfloat16 *>(i == cl.L ? p.y_out : Ld.Xn);
          __nv_bfloat16 *zst = reinterpret_cast<__nv_bfloat16 *>(const_cast<void *>(Ld.Z));
          uint32_t o = u, d = 0;
          if (Ld.act == ACT_GELU) {
            // X_{i+1} = gelu(Z_i); the Z_i store keeps gelu'(Z_i) for the backward
            float g[2], gd[2];
            const float zz[2] = {z0, z1};
#pragma unroll
            for (int h = 0; h < 2; ++h) {
              float Phi, ez;
              gauss_cdf_exp(zz[h], Phi, ez);
              gd[h] = fmaf(zz[h] * 0.39894228040143268f, ez, Phi);
              g[h] = zz[h] * Phi;
            }
            o = pack_bf2(g[0], g[1]);
            d = pack_bf2(gd[0], gd[1]);
          } else if (Ld.act == ACT_RELU) {
            o = pack_bf2(fmaxf(z0, 0.f), fmaxf(z1, 0.f));
            d = u;                                  // ReLU: Z_i
          }
          if (act_row) {
            if (ncol == 2) {
              *reinterpret_cast<uint32_t *>(out + off) = o;
              if (Ld.act != ACT_ID) *reinterpret_cast<uint32_t *>(zst + off) = d;
            } else {
              out[off] = __ushort_as_bfloat16((unsigned short)(o & 0xFFFFu));
              if (Ld.act != ACT_ID) zst[off] = __ushort_as_bfloat16((unsigned short)(d & 0xFFFFu));
            }
          }
        } else {
          // dO_i: dZ_{i-1} = (dZ_i W_i^T) * act'_{i-1}(Z_{i-1}) (GELU: the stored gelu')
          __nv_bfloat16 *out = reinterpret_cast<__nv_bfloat16 *>(i >= 2 ? p.layers[i - 2].dZ : p.dx_out);
          const int pact = i >= 2 ? p.layers[i - 2].act : ACT_ID;
          if (pact != ACT_ID && p.layers[i - 2].Z) {
            if (pact == ACT_GELU) {
              v[0] *= p0;
              v[1] *= p1;
            } else {
              v[0] = p0 > 0.f ? v[0] : 0.f;
              v[1] = p1 > 0.f ? v[1] : 0.f;
            }
          }
          const uint32_t u = act_row ? pack_bf2(v[0], v[1]) : 0u;   // dZ_{i-1} (RNE)
          if (act_row && out) {
            if (ncol == 2) *reinterpret_cast<uint32_t *>(out + off) = u;
            else out[off] = __ushort_as_bfloat16((unsigned short)(u & 0xFFFFu));
          }
          if (i >= 2 && p.layers[i - 2].dbpart) {
            publish_db = true;
            red_s[er * 16 + ec] = bf_lo(u);
            if (ncol == 2) red_s[er * 16 + ec + 1] = bf_hi(u);
          }
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");   // outputs stored
        if (rank == 0 && et == 0) sktrace(c.j, c.t, 6);
        if (publish_db && et < cs) {
          // bias-gradient partial of the only row block: column sums of the
          // rounded dZ_{i-1} over the token rows, in row order
          float sum = 0.f;
          for (int r = 0; r < M; ++r) sum += red_s[r * 16 + et];
          p.layers[i - 2].dbpart[n0 + (int)rank * cs + et] = sum;
        }
        if (publish_db) asm volatile("bar.sync 1, 128;" ::: "memory");
        if (et == 0) {
          // publish this CTA's slice: cumulative over the 4 warps' stores
          // (ordered by bar.sync); a tile completes with kCl slices
          asm volatile("fence.acq_rel.gpu;" ::: "memory");
          if (rank == 0) sktrace(c.j, c.t, 7);
          if (sh.kind == EPI_FWD) {
            red_add(ctr + cl.fwd_rows + (i - 1) * cl.MT, 1);
          } else if (i >= 2) {
            red_add(ctr + cl.dz_rows + (i - 2) * cl.MT, 1);
            red_add(ctr + cl.dz_total + (i - 2), 1);
          } else {
            red_add(ctr + cl.dx_total, 1);
          }
          if (rank == 0) sktrace(c.j, c.t, 3);
        }
        // receive slot b read by every thread (the barriers above): free it
        // in every sender -- after the publish, which is what the chain waits
        // for (a cluster-scope release arrive costs ~1 us on the critical path)
        __syncwarp();
        if (warp == 0 && lane < kCl) mbar_arrive_cluster(mapa(rfree + 8 * b, lane));
        ++k;
        cur_next(p, c, clu, sh);
      }
    }
  } else {
    dw_worker(p, warp, lane, tmem, sbase, sbase + STG_OFF, task_slot, d_buffull, d_bufempty, d_accfull,
              d_accfree, qfull, qempty);
  }

  fence_before();
  __syncthreads();
  cluster_sync();   // no CTA leaves while a peer may still signal it
  if (warp == 5) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
  }
}


int g_max_clusters = 0;

}  // namespace

cudaError_t skinny_init() {
  cudaError_t e = cudaFuncSetAttribute(skinny_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(skinny_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 0);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  cfg.gridDim = dim3(kCl * 18, 1, 1);
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.dynamicSmemBytes = SMEM;
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kCl;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  e = cudaOccupancyMaxActiveClusters(&n, skinny_kernel, &cfg);
  if (e != cudaSuccess) return e;
  g_max_clusters = n;
  return cudaSuccess;
}

int skinny_max_clusters() { return g_max_clusters; }

#ifdef OOO_TRACE
cudaError_t skinny_set_trace(void *p) { return cudaMemcpyToSymbol(g_sktrace, &p, sizeof(p)); }
#endif

cudaError_t launch_skinny(const Params &p, const CUtensorMap *tmX, int clusters, cudaStream_t stream) {
  cudaLaunchConfig_t cfg = {};
  cudaLaunchAttribute attr[1];
  cfg.gridDim = dim3(kCl * clusters, 1, 1);
  cfg.blockDim = dim3(kThreads, 1, 1);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = stream;
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = kCl;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, skinny_kernel, *tmX, p);
}

}  // namespace sk
}  // namespace ooo
