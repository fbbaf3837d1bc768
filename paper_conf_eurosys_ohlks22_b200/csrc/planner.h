// Host-side queue planner of the persistent engine (pure C++, no CUDA).
//
// The engine kernel dispenses tiles in one FIFO order; a tile whose inputs
// are incomplete makes its CTA wait.  The paper runs the critical chain (dO
// ops, then the next iteration's F ops) on a high-priority stream and the
// deferrable dW ops on a low-priority one (§4.1), in the orders of
// Algorithm 2.  The planner turns those two priority-ordered
// chains into one FIFO order by list scheduling against a timing model of
// the engine (P worker CTAs / CTA pairs, per-tile mainloop and epilogue
// times): the next critical row is emitted as soon as it is (predicted)
// ready; while it is not, deferred dW row groups fill the workers that would
// otherwise idle, as long as enough workers stay free for the critical op.
// Every op is emitted after all ops it depends on, so FIFO dispensing with
// blocking waits cannot deadlock (engine.cu).  A wrong prediction only costs
// idle time, never correctness.
#pragma once
#include <vector>

namespace ooo {
namespace plan {

enum Kind { FWD = 0, DGRAD = 1, WGRAD = 2, COPY = 3 };

// One schedulable unit = rows [m_off, m_off + mt) (in tile rows) x all nt
// column tiles of one op.
struct Unit {
  int kind, layer;   // layer 1-based
  int m_off, mt, nt;
  int nkb;           // k-blocks per tile (0 for COPY)
  int bn;            // tile width
  int act;           // epilogue activation (0 = identity)
  int ks = 1;        // split-K chain op: every tile is ks tasks of nkb = ceil(nkb_full / ks) k-blocks
  int nkb_full = 0;  // the op's whole reduction (split-K)
  int release = -1;  // deferred units: emitted only once critical op #release (index into
                     // Problem::crit) has started (region schedule, §4.1); -1 = no constraint,
                     // >= crit.size() = after the whole chain
};

struct Model {
  double t_kb = 0.47;      // us per 64-deep k-block of a 128*cg x 256 tile
  double t_fix = 1.0;      // us: first-load latency + dispatch per tile
  double stages = 6;       // producer runs this many k-blocks ahead
  double epi_fwd = 5.4, epi_fwd_act = 9.9;   // us per tile (bn = 256)
  double epi_dx = 6.6, epi_dx_act = 11.0;
  double epi_dw = 5.2, epi_copy = 1.5;
  double ar_latency = 25.0;                  // us: bucket all-reduce (N > 1)
  double lead = 2.0;                         // us: a critical row is dispatched this early
  double reserve = 0.5;                      // fraction of the critical op's width kept free of dW
};

struct Problem {
  int L = 0;
  int rows = 0;            // tile rows of the token dimension (ceil(M / (128 cg)))
  int workers = 148;       // concurrently resident tiles (CTAs / cg)
  bool in_order = false;   // dO_i waits for dW_{i+1}
  int fwd_gate = 0;        // 0 none, 1 F_i waits dW_i, 2 F_i waits its bucket's all-reduce
  std::vector<int> bucket; // [L] bucket of layer i (index i-1)
  std::vector<Unit> crit;  // critical chain in priority order (dO ops, copy, F ops)
  std::vector<Unit> defer; // deferred dW ops in D's order (whole ops; split by the planner)
};

// Returns the FIFO order as units (adjacent units of one op merged when
// their rows are contiguous), using at most `max_units` entries (coarser dW
// row groups if needed).  Empty on failure (dependency cycle).
// dw_done (optional): predicted completion time (us from the launch) of every
// dW_i in this launch (index i-1; 0 for dW ops not in it) -- the ready times
// of the prioritised all-reduce order (comm_order.cpp).
std::vector<Unit> schedule(const Problem &pb, const Model &m, int max_units, std::vector<double> *dw_done = nullptr);

// True iff every unit's dependencies are emitted before it (test hook).
bool topological(const Problem &pb, const std::vector<Unit> &order);

}  // namespace plan
}  // namespace ooo
