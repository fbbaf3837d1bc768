// Cross-layer model parallelism with gradient fast-forwarding and modulo
// layer allocation (§5.2.1), built on the
// public stack ABI.
//
// The L layers are split into G groups of group_layers consecutive layers;
// group j lives on stage (GPU) stage_of(j): contiguous = G/n consecutive
// groups per stage (the conventional allocation), modulo = j mod n
// ("modulo layer allocation"; the paper allocates transformer
// blocks).  One iteration without micro-batches:
//   forward : F of group 0, 1, ..., G-1, each after the previous group's
//             output (the activation hand-off between stages);
//   backward: group G-1 first; group j-1 starts on group j's input gradient
//             dX_j -- conventional backprop: after group j's whole backward
//             (Fig. 5(a)); gradient fast-forwarding: as soon as the
//             dO chain of group j has produced dX_j, in the middle of its
//             engine kernel (ooo_input_grad_wait), so group j's dW ops overlap
//             group j-1's backward on another stage (Fig. 5(b)/(c)).
// Each group is an ooo_stack (the same engine kernels), restricted to its
// stage's SM partition (engine_ctas = SMs / n); every stage has one stream.
// The hand-off buffers (group outputs, input gradients) are in the
// pipeline's workspace; on n GPUs they would be the NCCL send/recv buffers.
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "../../include/ooo.h"
#include "internal.h"

namespace {

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

struct GroupDesc {
  int first = 0, nl = 0;    // first layer (0-based) and layer count
  std::vector<int32_t> dims, acts;
};

ooo_status check_desc(const ooo_pipeline_desc *d) {
  if (!d || !d->dims || !d->acts) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL pipeline desc");
  if (d->num_layers < 1 || d->group_layers < 1 || d->num_layers % d->group_layers != 0)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "group_layers must divide num_layers");
  const int G = d->num_layers / d->group_layers;
  if (d->n_stages < 1 || d->n_stages > G)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "n_stages must be in [1, number of groups]");
  if (d->placement != 0 && d->placement != 1) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "placement 0 or 1");
  if (d->placement == 0 && G % d->n_stages != 0)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "contiguous placement: n_stages must divide the groups");
  return OOO_OK;
}

std::vector<GroupDesc> groups_of(const ooo_pipeline_desc *d) {
  std::vector<GroupDesc> g(d->num_layers / d->group_layers);
  for (size_t j = 0; j < g.size(); ++j) {
    g[j].first = (int)j * d->group_layers;
    g[j].nl = d->group_layers;
    g[j].dims.assign(d->dims + g[j].first, d->dims + g[j].first + g[j].nl + 1);
    g[j].acts.assign(d->acts + g[j].first, d->acts + g[j].first + g[j].nl);
  }
  return g;
}

int stage_of(const ooo_pipeline_desc *d, int j) {
  const int G = d->num_layers / d->group_layers;
  if (j < 0 || j >= G) return -1;
  return d->placement == 1 ? j % d->n_stages : j / (G / d->n_stages);
}

ooo_stack_desc stack_desc(const ooo_pipeline_desc *d, const GroupDesc &g, int j, int sms) {
  ooo_stack_desc s;
  memset(&s, 0, sizeof(s));
  s.num_layers = g.nl;
  s.dims = g.dims.data();
  s.acts = g.acts.data();
  s.tokens = d->tokens;
  s.dtype = OOO_BF16;
  s.need_input_grad = j > 0 ? 1 : 0;     // group 0's input gradient is not needed (reading Q1)
  s.bucket_layers = g.nl;
  s.world_size = 1;
  s.comm_enabled = 1;
  s.engine_ctas = std::max(2, sms / d->n_stages / 2 * 2);   // whole CTA pairs per stage partition
  if (d->W) s.W = d->W + g.first;
  if (d->b) s.b = d->b + g.first;
  return s;
}

}  // namespace

struct ooo_pipeline {
  ooo_pipeline_desc d;
  std::vector<int32_t> dims, acts;
  std::vector<GroupDesc> g;
  std::vector<ooo_stack *> stk;
  std::vector<cudaStream_t> st;              // one per stage
  std::vector<void *> out, dx;               // group j's output (j < G-1) / input gradient (j > 0)
  std::vector<cudaEvent_t> ev_f, ev_b;       // forward done / input gradient released, per group
  cudaEvent_t ev_fork = nullptr;
  std::vector<cudaEvent_t> ev_join;          // per stage
};

namespace {

// sizes: per group workspace + grads; hand-off buffers (outputs, input grads)
ooo_status plan_sizes(const ooo_pipeline_desc *d, std::vector<size_t> *ws_off, std::vector<size_t> *gr_off,
                      std::vector<size_t> *out_off, std::vector<size_t> *dx_off, size_t *ws_total,
                      size_t *gr_total) {
  ooo_status st = check_desc(d);
  if (st != OOO_OK) return st;
  std::vector<GroupDesc> g = groups_of(d);
  const int G = (int)g.size();
  size_t ws = 0, gr = 0;
  for (int j = 0; j < G; ++j) {
    ooo_stack_desc sd = stack_desc(d, g[j], j, 148);
    size_t w = 0, b = 0;
    if ((st = ooo_query_sizes(&sd, &w, &b)) != OOO_OK) return st;
    if (ws_off) ws_off->push_back(ws);
    if (gr_off) gr_off->push_back(gr);
    ws += align256(w);
    gr += align256(b);
  }
  for (int j = 0; j < G; ++j) {   // group outputs (inputs of the next group) and input gradients
    const size_t ob = (size_t)d->tokens * d->dims[g[j].first + g[j].nl] * 2;
    const size_t ib = (size_t)d->tokens * d->dims[g[j].first] * 2;
    if (out_off) out_off->push_back(j < G - 1 ? ws : SIZE_MAX);
    if (j < G - 1) ws += align256(ob);
    if (dx_off) dx_off->push_back(j > 0 ? ws : SIZE_MAX);
    if (j > 0) ws += align256(ib);
  }
  *ws_total = std::max<size_t>(ws, 256);
  *gr_total = std::max<size_t>(gr, 256);
  return OOO_OK;
}

}  // namespace

extern "C" {

ooo_status ooo_pipeline_query_sizes(const ooo_pipeline_desc *d, size_t *workspace_bytes, size_t *grads_bytes) {
  if (!workspace_bytes || !grads_bytes) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  return plan_sizes(d, nullptr, nullptr, nullptr, nullptr, workspace_bytes, grads_bytes);
}

ooo_status ooo_pipeline_grads_offset(const ooo_pipeline_desc *d, int32_t group, int64_t *offset) {
  if (!offset) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  std::vector<size_t> gr;
  size_t w = 0, b = 0;
  ooo_status st = plan_sizes(d, nullptr, &gr, nullptr, nullptr, &w, &b);
  if (st != OOO_OK) return st;
  if (group < 0 || group >= (int)gr.size()) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "group out of range");
  *offset = (int64_t)gr[group];
  return OOO_OK;
}

int32_t ooo_pipeline_stage_of(const ooo_pipeline *p, int32_t group) { return p ? stage_of(&p->d, group) : -1; }

ooo_status ooo_pipeline_destroy(ooo_pipeline *p) {
  if (!p) return OOO_OK;
  for (ooo_stack *s : p->stk)
    if (s) ooo_destroy(s);
  for (cudaStream_t s : p->st)
    if (s) cudaStreamDestroy(s);
  for (cudaEvent_t e : p->ev_f) if (e) cudaEventDestroy(e);
  for (cudaEvent_t e : p->ev_b) if (e) cudaEventDestroy(e);
  for (cudaEvent_t e : p->ev_join) if (e) cudaEventDestroy(e);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  delete p;
  return OOO_OK;
}

ooo_status ooo_pipeline_create(const ooo_pipeline_desc *d, ooo_pipeline **out) {
  if (!out) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  *out = nullptr;
  std::vector<size_t> wso, gro, oo, dxo;
  size_t wt = 0, gt = 0;
  ooo_status st = plan_sizes(d, &wso, &gro, &oo, &dxo, &wt, &gt);
  if (st != OOO_OK) return st;
  if (!d->W || !d->b || !d->workspace || !d->grads)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "W/b/workspace/grads NULL");
  if (reinterpret_cast<uintptr_t>(d->workspace) % 256 || reinterpret_cast<uintptr_t>(d->grads) % 256)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "workspace/grads must be 256-byte aligned");
  ooo_pipeline *p = new ooo_pipeline();
  p->d = *d;
  p->dims.assign(d->dims, d->dims + d->num_layers + 1);
  p->acts.assign(d->acts, d->acts + d->num_layers);
  p->d.dims = p->dims.data();
  p->d.acts = p->acts.data();
  p->g = groups_of(&p->d);
  const int G = (int)p->g.size();
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint8_t *ws = static_cast<uint8_t *>(d->workspace), *gr = static_cast<uint8_t *>(d->grads);
  auto bail = [&](ooo_status s) {
    ooo_pipeline_destroy(p);
    return s;
  };
  for (int j = 0; j < G; ++j) {
    ooo_stack_desc sd = stack_desc(&p->d, p->g[j], j, sms);
    size_t w = 0, b = 0;
    if ((st = ooo_query_sizes(&sd, &w, &b)) != OOO_OK) return bail(st);
    sd.workspace = ws + wso[j];
    sd.grads = gr + gro[j];
    ooo_stack *s = nullptr;
    if ((st = ooo_create_stack(&sd, &s)) != OOO_OK) return bail(st);
    p->stk.push_back(s);
    p->out.push_back(oo[j] == SIZE_MAX ? nullptr : ws + oo[j]);
    p->dx.push_back(dxo[j] == SIZE_MAX ? nullptr : ws + dxo[j]);
  }
  int lo = 0, hi = 0;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  p->st.assign(d->n_stages, nullptr);
  p->ev_join.assign(d->n_stages, nullptr);
  for (int k = 0; k < d->n_stages; ++k) {
    if (cudaStreamCreateWithPriority(&p->st[k], cudaStreamNonBlocking, hi) != cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_join[k], cudaEventDisableTiming) != cudaSuccess)
      return bail(ooo::set_error(OOO_ERR_CUDA, "stage stream / event create failed"));
  }
  p->ev_f.assign(G, nullptr);
  p->ev_b.assign(G, nullptr);
  for (int j = 0; j < G; ++j)
    if (cudaEventCreateWithFlags(&p->ev_f[j], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_b[j], cudaEventDisableTiming) != cudaSuccess)
      return bail(ooo::set_error(OOO_ERR_CUDA, "event create failed"));
  if (cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming) != cudaSuccess)
    return bail(ooo::set_error(OOO_ERR_CUDA, "event create failed"));
  *out = p;
  return OOO_OK;
}

// One iteration enqueued on `cap` (being captured): see the header comment.
static ooo_status enqueue_step(ooo_pipeline *p, const void *X, const void *dY, void *Y, int ff, cudaStream_t cap) {
  const int G = (int)p->g.size();
  const int n = p->d.n_stages;
  ooo_status st;
#define PL_CU(x)                                                             \
  do {                                                                       \
    if ((x) != cudaSuccess) return ooo::set_error(OOO_ERR_CUDA, #x " failed"); \
  } while (0)
#define PL_TRY(x)                  \
  do {                             \
    if ((st = (x)) != OOO_OK) return st; \
  } while (0)
  PL_CU(cudaEventRecord(p->ev_fork, cap));
  for (int k = 0; k < n; ++k) PL_CU(cudaStreamWaitEvent(p->st[k], p->ev_fork, 0));
  // forward: group j after group j-1 (its output is group j's input)
  for (int j = 0; j < G; ++j) {
    cudaStream_t s = p->st[stage_of(&p->d, j)];
    if (j > 0) PL_CU(cudaStreamWaitEvent(s, p->ev_f[j - 1], 0));
    PL_TRY(ooo_forward(p->stk[j], j == 0 ? X : p->out[j - 1], j == G - 1 ? Y : p->out[j], s));
    PL_CU(cudaEventRecord(p->ev_f[j], s));
  }
  // backward: group G-1 first; group j-1 on group j's input gradient.  A
  // stage runs one group's kernel at a time (it is one GPU: its SM
  // partition), so a group's backward also waits for the stage's previous one
  std::vector<int> last(n, -1);
  for (int j = G - 1; j >= 0; --j) {
    const int k = stage_of(&p->d, j);
    cudaStream_t s = p->st[k];
    if (j < G - 1) PL_CU(cudaStreamWaitEvent(s, p->ev_b[j + 1], 0));
    if (last[k] >= 0) PL_TRY(ooo_join(p->stk[last[k]], s));
    last[k] = j;
    ooo_schedule sch;
    sch.kind = ff ? OOO_SCHED_FIRST_K : OOO_SCHED_IN_ORDER;
    sch.k = ff ? p->g[j].nl : 0;   // fast-forwarding: every dW after the dO chain
    PL_TRY(ooo_backward(p->stk[j], j == G - 1 ? dY : p->dx[j + 1], sch, j > 0 ? p->dx[j] : nullptr, s));
    if (j > 0) {
      if (ff) PL_TRY(ooo_input_grad_wait(p->stk[j], s));   // dX released mid-kernel
      else PL_TRY(ooo_join(p->stk[j], s));                  // after the whole backward
      PL_CU(cudaEventRecord(p->ev_b[j], s));
    }
  }
  for (int j = 0; j < G; ++j) PL_TRY(ooo_join(p->stk[j], p->st[stage_of(&p->d, j)]));
  for (int k = 0; k < n; ++k) {
    PL_CU(cudaEventRecord(p->ev_join[k], p->st[k]));
    PL_CU(cudaStreamWaitEvent(cap, p->ev_join[k], 0));
  }
#undef PL_CU
#undef PL_TRY
  return OOO_OK;
}

ooo_status ooo_pipeline_graph_create(ooo_pipeline *p, const void *X, const void *dY, void *Y, int32_t fast_forward,
                                     ooo_graph **out) {
  if (!p || !X || !dY || !Y || !out) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  *out = nullptr;
  cudaStream_t cap;
  if (cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking) != cudaSuccess)
    return ooo::set_error(OOO_ERR_CUDA, "stream create failed");
  if (cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal) != cudaSuccess) {
    cudaStreamDestroy(cap);
    return ooo::set_error(OOO_ERR_CUDA, "begin capture failed");
  }
  ooo_status st = enqueue_step(p, X, dY, Y, fast_forward, cap);
  cudaGraph_t g = nullptr;
  cudaError_t e = cudaStreamEndCapture(cap, &g);
  cudaStreamDestroy(cap);
  if (st != OOO_OK) {
    if (g) cudaGraphDestroy(g);
    return st;
  }
  if (e != cudaSuccess) return ooo::set_error(OOO_ERR_CUDA, cudaGetErrorString(e));
  cudaGraphExec_t ex = nullptr;
  if ((e = cudaGraphInstantiateWithFlags(&ex, g, cudaGraphInstantiateFlagUseNodePriority)) != cudaSuccess) {
    cudaGraphDestroy(g);
    return ooo::set_error(OOO_ERR_CUDA, cudaGetErrorString(e));
  }
  *out = ooo::wrap_graph(g, ex);
  return OOO_OK;
}

}  // extern "C"
