// Persistent dataflow engine: one kernel per training step (backward(t) fused
// with forward(t+1)) that runs the whole step as a priority-ordered queue of
// output tiles.
//
// Why (paper §2, §4.1, §5.1): the paper schedules
// dO_i / dW_i ops of a layer stack so that the critical chain (dO, then the
// next forward) is never delayed and the deferrable dW ops fill idle
// resources, in Algorithm 2's order; the next forward F_i may start as soon
// as S[dW_i] is done.  On B200 a BERT-sized layer GEMM is only 3-20 us
// of tensor work, so per-kernel launch, first-load latency, exposed epilogue
// and wave tails cost as much as the math.  The engine removes those
// boundaries: CTAs take tiles in queue order (the schedule D expanded to
// tiles, then the next forward), a tile starts as soon as the rows it reads
// are complete (dO_i and F_i are row-local: output row block m needs only
// input row block m), dW_i tiles are slotted into the queue behind the
// critical dO tiles (reverse first-k keeps dW_1..dW_k at the end), and F_i
// starts as soon as dW_i is done -- the Fig. 4(c) overlap, inside one kernel.
// Completion counters in global memory replace stream events; they also
// drive the per-bucket all-reduce (the comm stream waits on them with
// cuStreamWaitValue32) and gate F_i on its bucket's all-reduce for N > 1.
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace ooo {
namespace eng {

constexpr int kMaxOps = 768;     // op table travels as a kernel parameter (<= 32 KiB)
constexpr int MAP_NONE = -1;
constexpr int MAP_Y = -2;    // kernel-parameter map of the caller's Y
constexpr int MAP_DX = -3;   // kernel-parameter map of the caller's dX
constexpr int MAP_XIN = -4;  // kernel-parameter map of the caller's X (F_1's A operand)
constexpr int EPI_COPY = 3;  // task kind: copy the caller's X rows into the X_1 store (no MMA)

// One op of the queue = one row group of a layer GEMM (F_i, dO_i or dW_i), or
// the X -> X_1 copy = mt x nt tiles starting at row block m_off.
struct Op {
  int16_t kind;     // EPI_FWD / EPI_DGRAD / EPI_WGRAD / EPI_COPY
  int16_t act;      // epilogue activation (act_i for F_i, act_{i-1} for dO_i)
  int16_t bn;       // tile width (64..256, % 64 == 0)
  int16_t layer;    // i (1-based)
  int32_t first;    // first task index of this op in the queue
  int16_t mt, nt;   // tiles: rows (128 * cg) x cols (bn)
  int16_t nkb;      // K / 64 (0 for EPI_COPY)
  int16_t mapA, mapB, mapX, mapZ;   // indices into the map table (or MAP_*)
  int16_t m_off;    // first row block of the group
  int16_t ks;       // > 1: split-K chain op -- every tile is ks tasks over consecutive k-block ranges
                    // whose fp32 partials the last-arriving task sums in split order (skinny stacks)
  int16_t sk_base;  // its first arrival counter (sk region: one per tile and CTA of the pair)
};
static_assert(sizeof(Op) == 32, "Op layout");

// Per-layer device info (static, uploaded at create).
struct LayerDev {
  const void *bias;        // b_i (bf16)
  const void *Z;           // Z_i (bf16) or null (identity: act' = 1)
  float *dbpart;           // bias-grad partials of layer i [R][d_i]
  void *db_out;            // bucket slot of db_i (bf16)
  void *Xn;                // X_{i+1} store (null for i = L: the caller's Y)
  void *dZ;                // dZ_i store
  void *gw;                // bucket slot of dW_i (bf16)
  void *X;                 // X_i store (layer 1: the copy of the caller's X)
  int32_t din, dout, act, bucket;
  int32_t fwd_nt;          // n-tiles of F_i over d_i
  int32_t dx_nt;           // n-tiles of dO_i over d_{i-1}
  int32_t dw_tiles;        // 128-row tiles of dW_i (completion count)
  int32_t fwd_bn, dx_bn, dw_bn;   // tile widths of F_i / dO_i / dW_i
  int32_t pad1[6];
};
static_assert(sizeof(LayerDev) == 128, "LayerDev layout");

// Counter layout (int32, one region in the workspace; indices are absolute):
//   [0] dispenser | [1] unused | fwd_rows[L][MT]: tiles done of row block m of X_{i+1} |
//   xcopy[MT]: X_1 rows copied | dz_rows[L][MT] | dz_total[L] | dw_done[L] |
//   bucket_done[nb] | ar_done[nb] | dx_total: tiles of dO_1's output (dX) published |
//   sk[nsk]: split-K arrivals (inside the forward-reset range [0, fwd_end))
// A forward-only launch resets [0, fwd_end); a backward resets [0, total).
struct CounterLayout {
  int L, MT, nb;
  int fwd_rows, xcopy, sk, fwd_end;
  int dz_rows, dz_total, dw_done, bucket_done, ar_done, dx_total, total;
};

struct Params {
  int32_t nops, ntasks, M, R;
  float alpha;
  int32_t in_order;        // dO_i also waits for dW_{i+1} (conventional backprop)
  int32_t fwd_gate;        // 0: none; 1: F_i waits dW_i (N = 1); 2: F_i waits ar_done[bucket(i)]
                           // (N > 1); both also wait dW_{i+1} (it reads X_{i+1}, which F_i overwrites)
  int32_t dbg;             // tuning experiments only (OOO_DBG): bit0 skip act math, bit1 skip stores, bit3 no X copy (stale X_1), bit4 no weight prefetch
  int32_t copy_nt;         // column tiles per row block of the X -> X_1 copy
  int32_t a_rows;          // rows of the row-major A box of F_i / dO_i tiles: 128, or M rounded
                           // up to 8 when all tokens fit one 128-row tile (1-CTA tiles): the
                           // MMA's rows beyond it read stale smem and are never stored
  uint64_t timeout_ns;     // bound of every in-kernel wait (trap beyond it)
  int32_t pf_dist;         // > 0: a chain tile of F_i (dO_i) also prefetches into L2 its slice of the
                           // weights of layer i + pf_dist (i - pf_dist) -- skinny stacks, where every
                           // chain op streams its W from HBM (W does not depend on the chain)
  int32_t maps_per_layer;  // map-table slots per layer (the map of layer j = the op's map + (j-i) x this)
  int32_t sk_nc;           // 32-column chunks per row of the split-K partial buffer (max width / 32)
  float *skpart;           // split-K partials [ks][MT][sk_nc][128 rows][32] fp32 (workspace)
  const CUtensorMap *maps;
  int32_t *ctr;            // counter array base
  const LayerDev *layers;  // index i-1
  void *y_out;             // caller's Y (F_L output)
  void *dx_out;            // caller's dX (dO_1 output, need_input_grad)
  const void *x_in;        // caller's X (source of the X_1 copy tasks)
  CounterLayout cl;
  Op ops[kMaxOps];
};

// cg = CTAs per tile: 1 (128-row tiles) or 2 (CTA pairs, 256-row tiles, cta_group::2)
int engine_smem_bytes(int cg);
cudaError_t engine_init();
#ifdef OOO_TRACE
cudaError_t engine_set_trace(void *p);   // debug builds: per-task timestamps buffer
#endif
cudaError_t launch_engine(int cg, const Params &p, const CUtensorMap *tmY, const CUtensorMap *tmDX,
                          const CUtensorMap *tmX, int ctas,
                          cudaStream_t stream, int priority);

}  // namespace eng
}  // namespace ooo
