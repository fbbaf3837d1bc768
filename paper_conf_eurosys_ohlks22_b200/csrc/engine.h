// Persistent dataflow engine: one kernel per pass (forward / backward) that
// runs the whole pass as a priority-ordered queue of 128 x BN output tiles.
//
// Why (paper §2, §4.1, §5.1): the paper schedules
// dO_i / dW_i ops of a layer stack so that the critical chain (dO, then the
// next forward) is never delayed and the deferrable dW ops fill idle
// resources, in Algorithm 2's order.  On B200 a BERT-sized layer GEMM is only
// 3-20 us of tensor work, so per-kernel launch, first-load latency, exposed
// epilogue and wave tails cost as much as the math.  The engine removes those
// boundaries: CTAs take tiles in queue order (the schedule D expanded to
// tiles), a tile starts as soon as the row block it reads is complete
// (dO_i and F_i are row-local: output row block m needs only input row
// block m), and dW_i tiles are slotted into the queue behind the critical
// dO tiles (reverse first-k keeps dW_1..dW_k at the end).  Completion
// counters in global memory replace stream events; they also drive the
// per-bucket all-reduce (the comm stream waits on them with
// cuStreamWaitValue32) and gate the next forward (F_i waits for its bucket).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace ooo {
namespace eng {

constexpr int kMaxOps = 512;
constexpr int MAP_NONE = -1;
constexpr int MAP_Y = -2;    // kernel-parameter map of the caller's Y
constexpr int MAP_DX = -3;   // kernel-parameter map of the caller's dX

// One op of the pass = one layer GEMM (F_i, dO_i or dW_i) = mt x nt tiles.
struct Op {
  int16_t kind;     // EPI_FWD / EPI_DGRAD / EPI_WGRAD
  int16_t act;      // epilogue activation (act_i for F_i, act_{i-1} for dO_i)
  int16_t bn;       // tile width (64..256, % 64 == 0)
  int16_t layer;    // i (1-based)
  int32_t first;    // first task index of this op in the queue
  int16_t mt, nt;   // tiles: rows (128) x cols (bn)
  int16_t nkb;      // K / 64
  int16_t mapA, mapB, mapX, mapZ;   // indices into the map table (or MAP_*)
  int16_t pad[3];
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
  void *pad0;
  int32_t din, dout, act, bucket;
  int32_t fwd_nt;          // n-tiles of F_i over d_i
  int32_t dx_nt;           // n-tiles of dO_i over d_{i-1}
  int32_t dw_tiles;        // tiles of dW_i
  int32_t pad1[9];
};
static_assert(sizeof(LayerDev) == 128, "LayerDev layout");

// Counter layout (int32, in the workspace):
//   fwd region : [0] dispenser, [1 + i*MT + m] rows of X_{i+1} done (i = 0..L-1)
//   bwd region : [0] dispenser, dz_rows[i][m], dz_total[i], dw_done[i],
//                bucket_done[b], ar_done[b]   (i = 1..L, index i-1)
struct CounterLayout {
  int L, MT, nb;
  int fwd_base, fwd_size;
  int bwd_base, bwd_size;
  int dz_rows, dz_total, dw_done, bucket_done, ar_done;   // absolute indices
};

struct Params {
  int32_t nops, ntasks, M, R;
  float alpha;
  int32_t in_order;        // dO_i also waits for dW_{i+1} (conventional backprop)
  int32_t gate_ar;         // F_i waits ar_done[bucket(i)] (N > 1)
  int32_t pass;            // 0 forward, 1 backward
  int32_t dbg;             // tuning experiments only (OOO_DBG): bit0 skip act math, bit1 skip stores
  const CUtensorMap *maps;
  int32_t *ctr;            // counter array base
  const LayerDev *layers;  // index i-1
  void *y_out;             // caller's Y (F_L output)
  void *dx_out;            // caller's dX (dO_1 output, need_input_grad)
  CounterLayout cl;
  Op ops[kMaxOps];
};

int engine_smem_bytes();
cudaError_t engine_init();
#ifdef OOO_TRACE
cudaError_t engine_set_trace(void *p);   // debug builds: per-task timestamps buffer
#endif
cudaError_t launch_engine(const Params &p, const CUtensorMap *tmY, const CUtensorMap *tmDX, int ctas,
                          cudaStream_t stream, int priority);

}  // namespace eng
}  // namespace ooo
