// Skinny-stack step kernel (tokens per GPU <= 16, e.g. C5 MLP96: 16 tokens).
//
// Why (paper §2, §5.1 P:182-210 -- the same step as engine.h; only
// the tiling differs): with so few token rows every F_i / dO_i is a chain
// op of 16 x N outputs with K = 1024 or so -- a few MMAs of work behind a
// long latency chain (the dO chain, then dW_1, then the F chain).  In
// the persistent engine each such op paid a dynamic dispatch, a k-block loop
// at the MMA issue rate on a few SMs, and (split-K) a partial round trip
// through L2 plus a gpu-scope atomic per tile.  Here:
//   * chain clusters (8 CTAs, one cluster per 64/128-wide output tile) walk
//     the chain ops of the step in order with a static tile assignment, so
//     every CTA knows its future tasks and streams their weight slices into
//     a shared-memory ring long before the activations arrive (W does not
//     depend on the chain);
//   * K is split over the 8 CTAs of the cluster; the 7 partial sums go to the
//     leader's shared memory over DSMEM (st.shared::cluster + a cluster-scope
//     mbarrier), reduced in fixed rank order (deterministic);
//   * the remaining clusters' CTAs are dW workers: a dynamic queue of dW_i
//     tiles in D's order (Alg. 2) and the X -> X_1 copy, each waiting on the
//     completion counter of dZ_i, publishing dW_i / bucket counters for the
//     all-reduce and F_i's gate exactly as the engine does (same counter
//     layout, same stores: ooo_tensor, the comm stream and the G1 test see
//     the same buffers).
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "engine.h"

namespace ooo {
namespace sk {

constexpr int kCl = 8;          // CTAs per cluster (the K split of one chain tile)
constexpr int kMaxM = 16;       // token rows of a skinny stack
constexpr int kMaxChain = 800;  // chain ops per launch (2L + 1)
constexpr int kMaxDw = 400;     // dW ops (+ the copy) per launch
// Every CTA of a chain cluster publishes its column slice of a tile: the
// fwd_rows / dz_rows / dz_total / dx_total counters of a skinny launch count
// kPubPerTile per tile (the engine's count 1; targets scale with it).
constexpr int kPubPerTile = kCl;

struct ChainOp {
  int16_t kind;    // eng::EPI_FWD / EPI_DGRAD
  int16_t layer;   // i (1-based)
};
struct DwOp {
  int16_t kind;    // EPI_WGRAD, or eng::EPI_COPY
  int16_t layer;
  int32_t first;   // first task index
};

struct Params {
  int32_t L, M, nchain, ndw, ntasks_dw, nclu;   // nclu: chain clusters (the rest are dW workers)
  int32_t in_order, fwd_gate;
  int32_t dbg;               // tuning experiments only (OOO_DBG): bit0 no weight prefetch beyond the current task
  float alpha;
  uint64_t timeout_ns;
  const CUtensorMap *maps;   // the stack's map table; per layer: map_x (X_i, box {64, 16}),
  int32_t maps_per_layer;    // map_dz (dZ_i, box {64, 16}), map_w (W_i, box {64, 64})
  int32_t map_x, map_dz, map_w;
  int32_t *ctr;              // engine counter layout (ctr[1]: the dW dispenser)
  const eng::LayerDev *layers;
  eng::CounterLayout cl;
  void *y_out;
  void *dx_out;
  const void *x_in;
  ChainOp chain[kMaxChain];
  DwOp dw[kMaxDw];
};

cudaError_t skinny_init();
int skinny_max_clusters();   // co-resident 8-CTA clusters of the kernel (0 before init)
#ifdef OOO_TRACE
cudaError_t skinny_set_trace(void *p);   // debug builds: [chain op][tile][8] timestamps
#endif
cudaError_t launch_skinny(const Params &p, const CUtensorMap *tmX, int clusters, cudaStream_t stream);

}  // namespace sk
}  // namespace ooo
