// Queue planner of the persistent engine (see planner.h).
#include "planner.h"

#include <algorithm>
#include <limits>

namespace ooo {
namespace plan {
namespace {

constexpr double kInf = std::numeric_limits<double>::infinity();

struct OpState {
  int total = 0, emitted = 0;       // tiles
  double done = 0.0;                // completion time of the emitted tiles (max)
  std::vector<int> row_cnt;         // emitted tiles per tile row
  std::vector<double> row_done;     // completion time per tile row (max)
};

class Sim {
 public:
  Sim(const Problem &pb, const Model &m, bool timing) : pb_(pb), m_(m), timing_(timing) {
    ops_.resize(4 * (pb.L + 2));
    auto init = [&](const Unit &u, int rows) {
      OpState &o = op(u.kind, u.layer);
      if (o.total == 0) {
        o.total = rows * u.nt * std::max(1, u.ks);
        o.row_cnt.assign(rows, 0);
        o.row_done.assign(rows, 0.0);
      }
    };
    for (const Unit &u : pb.crit) init(u, u.kind == WGRAD ? u.mt : pb.rows);
    for (const Unit &u : pb.defer) init(u, u.mt);
    const int W = std::max(1, pb.workers);
    disp_.assign(W, 0.0);
    mma_.assign(W, 0.0);
    epi_.assign(W, 0.0);
    epi_prev_.assign(W, 0.0);
    dw_until_.assign(W, 0.0);
  }

  OpState &op(int kind, int layer) { return ops_[kind * (pb_.L + 2) + layer]; }
  bool exists(int kind, int layer) { return layer >= 1 && layer <= pb_.L && op(kind, layer).total > 0; }

  // Completion time of a whole op (kInf if not fully emitted).  Ops that do
  // not exist in this launch (e.g. dW_i already done) count as done at 0.
  double op_done(int kind, int layer) {
    if (!exists(kind, layer)) return 0.0;
    OpState &o = op(kind, layer);
    return o.emitted == o.total ? o.done : kInf;
  }
  double row_done(int kind, int layer, int r) {
    if (!exists(kind, layer)) return 0.0;
    OpState &o = op(kind, layer);
    if (r >= (int)o.row_cnt.size()) return 0.0;
    return o.row_cnt[r] == o.total / (int)o.row_cnt.size() ? o.row_done[r] : kInf;
  }
  double bucket_done(int layer) {
    double t = 0.0;
    for (int j = 1; j <= pb_.L; ++j)
      if (pb_.bucket[j - 1] == pb_.bucket[layer - 1]) t = std::max(t, op_done(WGRAD, j));
    return t + m_.ar_latency;
  }

  // Earliest time the inputs of row r of unit u are complete (kInf if a
  // producer is not fully emitted yet).  Mirrors deps() in engine.cu.
  double ready(const Unit &u, int r) {
    const int i = u.layer;
    double t = 0.0;
    switch (u.kind) {
      case FWD:
        t = i > 1 ? row_done(FWD, i - 1, r) : 0.0;   // F_1 reads the caller's X
        if (pb_.fwd_gate == 1) t = std::max(t, op_done(WGRAD, i));
        if (pb_.fwd_gate == 2) t = std::max(t, bucket_done(i));
        if (pb_.fwd_gate && i < pb_.L) t = std::max(t, op_done(WGRAD, i + 1));
        break;
      case DGRAD:
        if (i < pb_.L) {
          t = row_done(DGRAD, i + 1, r);
          if (pb_.in_order) t = std::max(t, op_done(WGRAD, i + 1));
        }
        break;
      case WGRAD:
        if (i < pb_.L) t = op_done(DGRAD, i + 1);
        break;
      case COPY:
        if (pb_.fwd_gate) t = op_done(WGRAD, 1);
        break;
    }
    return t;
  }
  // The part of ready(u, r) that comes from dW ops (F_i's P:84 gate and the
  // WAR guard on dW_{i+1}; in_order dO_i on dW_{i+1}; the copy on dW_1).
  double dw_gate(const Unit &u) {
    const int i = u.layer;
    double t = 0.0;
    if (u.kind == FWD && pb_.fwd_gate) {
      t = pb_.fwd_gate == 1 ? op_done(WGRAD, i) : bucket_done(i);
      if (i < pb_.L) t = std::max(t, op_done(WGRAD, i + 1));
    } else if (u.kind == DGRAD && pb_.in_order && i < pb_.L) {
      t = op_done(WGRAD, i + 1);
    } else if (u.kind == COPY && pb_.fwd_gate) {
      t = op_done(WGRAD, 1);
    }
    return t;
  }
  bool emittable(const Unit &u) {
    if (u.kind == WGRAD) return ready(u, 0) < kInf;
    for (int r = u.m_off; r < u.m_off + u.mt; ++r)
      if (ready(u, r) == kInf) return false;
    return true;
  }

  // Time at which `need` workers are free for dispatch, optionally after the
  // tiles of unit d (ready at rd) were handed to the earliest free workers.
  double time_free(int need, const Unit *d, double rd) const {
    std::vector<double> f = disp_;
    if (d) {
      const double tkb = m_.t_kb * (0.5 + 0.5 * d->bn / 256.0);
      for (int j = 0; j < d->mt * d->nt * std::max(1, d->ks); ++j) {
        auto it = std::min_element(f.begin(), f.end());
        const double start = std::max(*it, rd);
        *it = std::max(start, start + m_.t_fix + d->nkb * tkb - m_.stages * tkb);
      }
    }
    need = std::max(1, std::min(need, (int)f.size()));
    std::nth_element(f.begin(), f.begin() + (need - 1), f.end());
    return f[need - 1];
  }

  int dw_busy(double t) const {
    int n = 0;
    for (double d : dw_until_) n += d > t;
    return n;
  }

  double epi_time(const Unit &u) const {
    const double s = u.bn / 256.0;
    switch (u.kind) {
      case FWD: return s * (u.act ? m_.epi_fwd_act : m_.epi_fwd);
      case DGRAD: return s * (u.act ? m_.epi_dx_act : m_.epi_dx);
      case WGRAD: return s * m_.epi_dw;
      default: return s * m_.epi_copy;
    }
  }

  void emit(const Unit &u) {
    OpState &o = op(u.kind, u.layer);
    const double tkb = m_.t_kb * (0.5 + 0.5 * u.bn / 256.0);
    const double epi = epi_time(u);
    for (int r = u.m_off; r < u.m_off + u.mt; ++r) {
      const double dep = timing_ ? ready(u, r) : 0.0;
      for (int n = 0; n < u.nt * std::max(1, u.ks); ++n) {   // split-K: ks tasks per tile
        double done = 0.0;
        if (timing_) {
          const int w = (int)(std::min_element(disp_.begin(), disp_.end()) - disp_.begin());
          const double t0 = disp_[w];
          if (u.kind == COPY) {
            const double s = std::max({t0, dep, epi_[w]});
            done = s + epi;
            epi_prev_[w] = epi_[w];
            epi_[w] = done;
          } else {
            const double start = std::max({t0, dep, mma_[w], epi_prev_[w]});
            const double main_end = start + m_.t_fix + u.nkb * tkb;
            done = std::max(main_end, epi_[w]) + epi;
            disp_[w] = std::max(start, main_end - m_.stages * tkb);
            mma_[w] = main_end;
            dw_until_[w] = u.kind == WGRAD ? main_end : 0.0;
            epi_prev_[w] = epi_[w];
            epi_[w] = done;
          }
        }
        o.row_cnt[r] += 1;
        o.row_done[r] = std::max(o.row_done[r], done);
        o.done = std::max(o.done, done);
        o.emitted += 1;
      }
    }
  }

 private:
  const Problem &pb_;
  const Model &m_;
  bool timing_;
  std::vector<OpState> ops_;
  std::vector<double> disp_, mma_, epi_, epi_prev_, dw_until_;
};

std::vector<Unit> merge(const std::vector<Unit> &v) {
  std::vector<Unit> out;
  for (const Unit &u : v) {
    if (!out.empty()) {
      Unit &b = out.back();
      if (b.kind == u.kind && b.layer == u.layer && b.nt == u.nt && b.m_off + b.mt == u.m_off) {
        b.mt += u.mt;
        continue;
      }
    }
    out.push_back(u);
  }
  return out;
}

// List scheduling in dispatch order.  The critical chain is emitted row by
// row (F_i / dO_i are row-local); at each step the next dispatch goes to the
// earliest free worker at time t:
//  * the next critical row if its inputs are (predicted) complete by t + lead;
//  * else the next dW row group if it is ready and the workers busy with dW
//    stay below P minus the critical op's width (so the chain keeps the
//    workers it needs when its rows become ready);
//  * else the critical row anyway (its worker waits), or the dW group if the
//    chain cannot proceed.
std::vector<Unit> plan_once(const Problem &pb, const Model &m, int group_rows, std::vector<double> *dw_done) {
  Sim sim(pb, m, true);
  std::vector<Unit> def;   // dW ops split into row groups
  for (const Unit &u : pb.defer)
    for (int r = 0; r < u.mt; r += group_rows) {
      Unit g = u;
      g.m_off = u.m_off + r;
      g.mt = std::min(group_rows, u.mt - r);
      def.push_back(g);
    }
  std::vector<Unit> crit;  // row-local critical ops split into rows
  std::vector<int> width;  // tiles of the whole op each critical unit belongs to
  std::vector<int> whole;  // index of that op in pb.crit
  for (size_t o = 0; o < pb.crit.size(); ++o) {
    const Unit &u = pb.crit[o];
    const bool rowwise = u.kind != WGRAD;
    for (int r = 0; r < u.mt; r += rowwise ? 1 : u.mt) {
      Unit g = u;
      g.m_off = u.m_off + r;
      g.mt = rowwise ? 1 : u.mt;
      crit.push_back(g);
      width.push_back(u.mt * u.nt);
      whole.push_back((int)o);
    }
  }
  // region release (§4.1): has critical op #rel started?
  auto released = [&](const Unit &d, size_t ci) {
    if (d.release < 0 || ci >= crit.size()) return true;
    const int started = ci == 0 ? 0 : whole[ci - 1] + 1;   // ops whose first row was emitted
    return started > d.release;
  };
  const int P = std::max(1, pb.workers);
  std::vector<Unit> out;
  size_t ci = 0, di = 0;
  while (ci < crit.size() || di < def.size()) {
    const bool c_ok = ci < crit.size() && sim.emittable(crit[ci]);
    const bool d_dep = di < def.size() && sim.emittable(def[di]);
    if (!c_ok && !d_dep) return {};   // dependency cycle: cannot happen for valid inputs
    // a release constraint never blocks the only unit that can proceed
    const bool d_ok = d_dep && (released(def[di], ci) || !c_ok);
    bool take_c = c_ok;
    if (c_ok && d_ok) {
      const double t = sim.time_free(1, nullptr, 0.0);
      const double rc = sim.ready(crit[ci], crit[ci].m_off);
      const double rd = sim.ready(def[di], 0);
      // a chain waiting for dW ops (F_i's gate) makes those dW ops critical: no cap
      const bool gated = sim.dw_gate(crit[ci]) >= rc - 1e-9;
      const int cap = gated ? P : P - std::min(P, (int)(m.reserve * width[ci] + 0.5));
      if (rc > t + m.lead && rd <= t + m.lead && sim.dw_busy(t) + def[di].mt * def[di].nt <= cap) take_c = false;
    }
    if (take_c) {
      sim.emit(crit[ci]);
      out.push_back(crit[ci++]);
    } else {
      sim.emit(def[di]);
      out.push_back(def[di++]);
    }
  }
  if (dw_done) {
    dw_done->assign(pb.L, 0.0);
    for (int i = 1; i <= pb.L; ++i) (*dw_done)[i - 1] = sim.op_done(WGRAD, i);
  }
  return merge(out);
}

}  // namespace

std::vector<Unit> schedule(const Problem &pb, const Model &m, int max_units, std::vector<double> *dw_done) {
  int maxrows = 1;
  for (const Unit &u : pb.defer) maxrows = std::max(maxrows, u.mt);
  for (int g = 1;; g *= 2) {
    std::vector<Unit> q = plan_once(pb, m, std::min(g, maxrows), dw_done);
    if (q.empty() || (int)q.size() <= max_units || g >= maxrows) return (int)q.size() <= max_units ? q : std::vector<Unit>{};
  }
}

bool topological(const Problem &pb, const std::vector<Unit> &order) {
  Sim sim(pb, Model(), false);
  for (const Unit &u : order) {
    if (!sim.emittable(u)) return false;
    sim.emit(u);
  }
  return true;
}

}  // namespace plan
}  // namespace ooo
