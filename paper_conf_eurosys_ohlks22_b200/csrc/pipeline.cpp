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
// Each group is an ooo_stack (the same engine kernels).  Without a
// communicator the stages are SM partitions of one GPU (engine_ctas = SMs /
// n, one stream per stage, hand-offs through device buffers).  With one, each
// rank is a stage holding only its groups and the hand-offs are ncclSend /
// ncclRecv on a comm stream (loopback at world_size 1: self send / recv).
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "../../include/ooo.h"
#include "internal.h"
#include "nccl_dyn.h"

namespace {

size_t align256(size_t x) { return (x + 255) / 256 * 256; }

struct GroupDesc {
  int first = 0, nl = 0;    // first layer (0-based) and layer count
  std::vector<int32_t> dims, acts;
};

bool comm_mode(const ooo_pipeline_desc *d) { return d->nccl_unique_id != nullptr; }

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
  if (d->world_size < 1 || d->rank < 0 || d->rank >= d->world_size)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "world_size / rank invalid");
  if (comm_mode(d) ? d->n_stages != d->world_size : d->world_size != 1)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT,
                          "with a communicator n_stages == world_size (one stage per rank); without one world_size 1");
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
// this process computes group j
bool owned(const ooo_pipeline_desc *d, int j) { return !comm_mode(d) || stage_of(d, j) == d->rank; }
// the boundary between groups j and j + 1 is an NCCL transfer
bool xfer(const ooo_pipeline_desc *d, int j) {
  return comm_mode(d) && (d->world_size == 1 || stage_of(d, j) != stage_of(d, j + 1));
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
  // one SM partition per stage; with NCCL, all SMs but the P2P kernels' reserve
  s.engine_ctas = comm_mode(d) ? std::max(2, (sms - 16) / 2 * 2) : std::max(2, sms / d->n_stages / 2 * 2);
  if (d->W) s.W = d->W + g.first;
  if (d->b) s.b = d->b + g.first;
  return s;
}

size_t act_bytes(const ooo_pipeline_desc *d, int width) { return (size_t)d->tokens * width * 2; }

}  // namespace

struct ooo_pipeline {
  ooo_pipeline_desc d;
  std::vector<int32_t> dims, acts;
  std::vector<GroupDesc> g;
  std::vector<ooo_stack *> stk;              // null for groups another rank owns
  std::vector<cudaStream_t> st;              // one per stage (this rank's only, with a communicator)
  std::vector<void *> out, in, dxs, dyr;     // per group: output, input, dX sent, dY received
  std::vector<cudaEvent_t> ev_f, ev_b, ev_xf, ev_xb;   // forward done / dX released / recv done (fwd, bwd)
  cudaEvent_t ev_fork = nullptr, ev_cj = nullptr;
  std::vector<cudaEvent_t> ev_join;          // per stage
  cudaStream_t comm = nullptr;
  const ooo::NcclApi *api = nullptr;
  ncclComm_t nccl = nullptr;
  std::vector<char> uid;
};

namespace {

// Per owned group: stack workspace and gradients; hand-off buffers.  Without
// a communicator (or inside one rank) group j's input is group j-1's output
// and its dY is group j+1's dX; across an NCCL boundary the receiver has its
// own buffer.
struct Layout {
  std::vector<size_t> ws, gr, out, in, dxs, dyr;   // SIZE_MAX: none / aliased
  size_t ws_total = 0, gr_total = 0;
};

ooo_status plan_sizes(const ooo_pipeline_desc *d, Layout *lay) {
  ooo_status st = check_desc(d);
  if (st != OOO_OK) return st;
  std::vector<GroupDesc> g = groups_of(d);
  const int G = (int)g.size();
  size_t ws = 0, gr = 0;
  auto take = [&](size_t bytes) {
    size_t o = ws;
    ws += align256(bytes);
    return o;
  };
  lay->ws.assign(G, SIZE_MAX);
  lay->gr.assign(G, SIZE_MAX);
  lay->out.assign(G, SIZE_MAX);
  lay->in.assign(G, SIZE_MAX);
  lay->dxs.assign(G, SIZE_MAX);
  lay->dyr.assign(G, SIZE_MAX);
  for (int j = 0; j < G; ++j) {
    if (!owned(d, j)) continue;
    ooo_stack_desc sd = stack_desc(d, g[j], j, 148);
    size_t w = 0, b = 0;
    if ((st = ooo_query_sizes(&sd, &w, &b)) != OOO_OK) return st;
    lay->ws[j] = take(w);
    lay->gr[j] = gr;
    gr += align256(b);
    const int din = d->dims[g[j].first], dout = d->dims[g[j].first + g[j].nl];
    if (j < G - 1) lay->out[j] = take(act_bytes(d, dout));
    if (j > 0) lay->dxs[j] = take(act_bytes(d, din));
    if (j > 0 && xfer(d, j - 1)) lay->in[j] = take(act_bytes(d, din));
    if (j < G - 1 && xfer(d, j)) lay->dyr[j] = take(act_bytes(d, dout));
  }
  lay->ws_total = std::max<size_t>(ws, 256);
  lay->gr_total = std::max<size_t>(gr, 256);
  return OOO_OK;
}

}  // namespace

extern "C" {

ooo_status ooo_pipeline_query_sizes(const ooo_pipeline_desc *d, size_t *workspace_bytes, size_t *grads_bytes) {
  if (!workspace_bytes || !grads_bytes) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  Layout lay;
  ooo_status st = plan_sizes(d, &lay);
  if (st != OOO_OK) return st;
  *workspace_bytes = lay.ws_total;
  *grads_bytes = lay.gr_total;
  return OOO_OK;
}

ooo_status ooo_pipeline_grads_offset(const ooo_pipeline_desc *d, int32_t group, int64_t *offset) {
  if (!offset) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  Layout lay;
  ooo_status st = plan_sizes(d, &lay);
  if (st != OOO_OK) return st;
  if (group < 0 || group >= (int)lay.gr.size() || lay.gr[group] == SIZE_MAX)
    return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "group out of range or owned by another rank");
  *offset = (int64_t)lay.gr[group];
  return OOO_OK;
}

int32_t ooo_pipeline_stage_of(const ooo_pipeline *p, int32_t group) { return p ? stage_of(&p->d, group) : -1; }

ooo_status ooo_pipeline_destroy(ooo_pipeline *p) {
  if (!p) return OOO_OK;
  for (ooo_stack *s : p->stk)
    if (s) ooo_destroy(s);
  if (p->comm) cudaStreamSynchronize(p->comm);
  if (p->nccl && p->api) p->api->CommDestroy(p->nccl);
  for (cudaStream_t s : p->st)
    if (s) cudaStreamDestroy(s);
  if (p->comm) cudaStreamDestroy(p->comm);
  for (auto *v : {&p->ev_f, &p->ev_b, &p->ev_xf, &p->ev_xb, &p->ev_join})
    for (cudaEvent_t e : *v)
      if (e) cudaEventDestroy(e);
  if (p->ev_fork) cudaEventDestroy(p->ev_fork);
  if (p->ev_cj) cudaEventDestroy(p->ev_cj);
  delete p;
  return OOO_OK;
}

ooo_status ooo_pipeline_create(const ooo_pipeline_desc *d, ooo_pipeline **out) {
  if (!out) return ooo::set_error(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  *out = nullptr;
  Layout lay;
  ooo_status st = plan_sizes(d, &lay);
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
  if (d->nccl_unique_id) {                 // keep a copy: the mode (comm_mode) is read at every capture
    p->uid.assign(static_cast<const char *>(d->nccl_unique_id),
                  static_cast<const char *>(d->nccl_unique_id) + OOO_UNIQUE_ID_BYTES);
    p->d.nccl_unique_id = p->uid.data();
  }
  p->g = groups_of(&p->d);
  const bool cm = comm_mode(d);
  const int G = (int)p->g.size();
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint8_t *ws = static_cast<uint8_t *>(d->workspace), *gr = static_cast<uint8_t *>(d->grads);
  auto bail = [&](ooo_status s) {
    ooo_pipeline_destroy(p);
    return s;
  };
  auto at = [&](size_t o) { return o == SIZE_MAX ? nullptr : static_cast<void *>(ws + o); };
  p->stk.assign(G, nullptr);
  p->out.assign(G, nullptr);
  p->in.assign(G, nullptr);
  p->dxs.assign(G, nullptr);
  p->dyr.assign(G, nullptr);
  for (int j = 0; j < G; ++j) {
    if (!owned(d, j)) continue;
    ooo_stack_desc sd = stack_desc(d, p->g[j], j, sms);
    sd.workspace = ws + lay.ws[j];
    sd.grads = gr + lay.gr[j];
    if ((st = ooo_create_stack(&sd, &p->stk[j])) != OOO_OK) return bail(st);
    p->out[j] = at(lay.out[j]);
    p->in[j] = at(lay.in[j]);
    p->dxs[j] = at(lay.dxs[j]);
    p->dyr[j] = at(lay.dyr[j]);
  }
  for (int j = 0; j < G; ++j) {   // same-process boundaries: the buffers are shared
    if (!owned(d, j)) continue;
    if (j > 0 && !xfer(d, j - 1)) p->in[j] = p->out[j - 1];
    if (j < G - 1 && !xfer(d, j)) p->dyr[j] = p->dxs[j + 1];
  }
  int lo = 0, hi = 0;
  cudaDeviceGetStreamPriorityRange(&lo, &hi);
  const int nst = cm ? 1 : d->n_stages;    // with a communicator this process is one stage
  p->st.assign(nst, nullptr);
  p->ev_join.assign(nst, nullptr);
  for (int k = 0; k < nst; ++k) {
    if (cudaStreamCreateWithPriority(&p->st[k], cudaStreamNonBlocking, hi) != cudaSuccess ||
        cudaEventCreateWithFlags(&p->ev_join[k], cudaEventDisableTiming) != cudaSuccess)
      return bail(ooo::set_error(OOO_ERR_CUDA, "stage stream / event create failed"));
  }
  for (auto *v : {&p->ev_f, &p->ev_b, &p->ev_xf, &p->ev_xb}) {
    v->assign(G, nullptr);
    for (cudaEvent_t &e : *v)
      if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
        return bail(ooo::set_error(OOO_ERR_CUDA, "event create failed"));
  }
  if (cudaEventCreateWithFlags(&p->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&p->ev_cj, cudaEventDisableTiming) != cudaSuccess)
    return bail(ooo::set_error(OOO_ERR_CUDA, "event create failed"));
  if (cm) {
    const char *why = nullptr;
    p->api = ooo::nccl_api(&why);
    if (!p->api) return bail(ooo::set_error(OOO_ERR_NCCL, why ? why : "NCCL unavailable"));
    if (cudaStreamCreateWithPriority(&p->comm, cudaStreamNonBlocking, hi) != cudaSuccess)
      return bail(ooo::set_error(OOO_ERR_CUDA, "comm stream create failed"));
    ncclUniqueId id;
    memcpy(&id, d->nccl_unique_id, sizeof(id));
    ncclResult_t r;
    if (p->api->CommInitRankConfig) {
      ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
      cfg.maxCTAs = 16;                      // the SMs the engines leave free
      r = p->api->CommInitRankConfig(&p->nccl, d->world_size, id, d->rank, &cfg);
    } else {
      r = p->api->CommInitRank(&p->nccl, d->world_size, id, d->rank);
    }
    if (r != ncclSuccess) {
      p->nccl = nullptr;
      return bail(ooo::set_error(OOO_ERR_NCCL, p->api->GetErrorString(r)));
    }
  }
  *out = p;
  return OOO_OK;
}

// One iteration enqueued on `cap` (being captured): see the header comment.
static ooo_status enqueue_step(ooo_pipeline *p, const void *X, const void *dY, void *Y, int ff, cudaStream_t cap) {
  const ooo_pipeline_desc *d = &p->d;
  const int G = (int)p->g.size();
  const bool cm = p->nccl != nullptr;
  const int nst = (int)p->st.size();
  auto sidx = [&](int j) { return cm ? 0 : stage_of(d, j); };
  ooo_status st;
#define PL_CU(x)                                                             \
  do {                                                                       \
    if ((x) != cudaSuccess) return ooo::set_error(OOO_ERR_CUDA, #x " failed"); \
  } while (0)
#define PL_TRY(x)                        \
  do {                                   \
    if ((st = (x)) != OOO_OK) return st; \
  } while (0)
#define PL_NC(x)                                                                     \
  do {                                                                               \
    ncclResult_t _r = (x);                                                           \
    if (_r != ncclSuccess) return ooo::set_error(OOO_ERR_NCCL, p->api->GetErrorString(_r)); \
  } while (0)
  PL_CU(cudaEventRecord(p->ev_fork, cap));
  for (int k = 0; k < nst; ++k) PL_CU(cudaStreamWaitEvent(p->st[k], p->ev_fork, 0));
  if (cm) PL_CU(cudaStreamWaitEvent(p->comm, p->ev_fork, 0));
  // NCCL hand-off across the boundary between group a (sender) and group b
  // (receiver); every rank issues the boundaries in the same global order
  auto handoff = [&](int a, int b, const void *src, void *dst, size_t bytes, cudaEvent_t done) -> ooo_status {
    const bool snd = owned(d, a), rcv = owned(d, b);
    if (!snd && !rcv) return OOO_OK;
    const size_t n = bytes / 2;
    if (snd && rcv) PL_NC(p->api->GroupStart());
    if (snd) PL_NC(p->api->Send(src, n, ncclBfloat16, stage_of(d, b) % d->world_size, p->nccl, p->comm));
    if (rcv) PL_NC(p->api->Recv(dst, n, ncclBfloat16, stage_of(d, a) % d->world_size, p->nccl, p->comm));
    if (snd && rcv) PL_NC(p->api->GroupEnd());
    if (rcv) PL_CU(cudaEventRecord(done, p->comm));
    return OOO_OK;
  };
  // forward: group j after group j-1 (its output is group j's input)
  for (int j = 0; j < G; ++j) {
    if (owned(d, j)) {
      cudaStream_t s = p->st[sidx(j)];
      if (j > 0) PL_CU(cudaStreamWaitEvent(s, xfer(d, j - 1) ? p->ev_xf[j] : p->ev_f[j - 1], 0));
      PL_TRY(ooo_forward(p->stk[j], j == 0 ? X : p->in[j], j == G - 1 ? Y : p->out[j], s));
      PL_CU(cudaEventRecord(p->ev_f[j], s));
      if (j < G - 1 && xfer(d, j)) PL_CU(cudaStreamWaitEvent(p->comm, p->ev_f[j], 0));
    }
    if (j < G - 1 && xfer(d, j))
      PL_TRY(handoff(j, j + 1, p->out[j], p->in[j + 1], act_bytes(d, d->dims[p->g[j].first + p->g[j].nl]),
                     p->ev_xf[j + 1]));
  }
  // backward: group G-1 first; group j-1 on group j's input gradient.  A
  // stage runs one group's kernel at a time (it is one GPU: its SMs), so a
  // group's backward also waits for the stage's previous one
  std::vector<int> last(nst, -1);
  for (int j = G - 1; j >= 0; --j) {
    if (owned(d, j)) {
      const int k = sidx(j);
      cudaStream_t s = p->st[k];
      if (j < G - 1) PL_CU(cudaStreamWaitEvent(s, xfer(d, j) ? p->ev_xb[j] : p->ev_b[j + 1], 0));
      if (last[k] >= 0) PL_TRY(ooo_join(p->stk[last[k]], s));
      last[k] = j;
      ooo_schedule sch;
      sch.kind = ff ? OOO_SCHED_FIRST_K : OOO_SCHED_IN_ORDER;
      sch.k = ff ? p->g[j].nl : 0;   // fast-forwarding: every dW after the dO chain
      PL_TRY(ooo_backward(p->stk[j], j == G - 1 ? dY : p->dyr[j], sch, j > 0 ? p->dxs[j] : nullptr, s));
      if (j > 0) {
        // dX released mid-kernel or after the whole backward
        cudaStream_t w = xfer(d, j - 1) ? p->comm : s;
        if (ff) PL_TRY(ooo_input_grad_wait(p->stk[j], w));
        else PL_TRY(ooo_join(p->stk[j], w));
        if (!xfer(d, j - 1)) PL_CU(cudaEventRecord(p->ev_b[j], s));
      }
    }
    if (j > 0 && xfer(d, j - 1))
      PL_TRY(handoff(j, j - 1, p->dxs[j], p->dyr[j - 1], act_bytes(d, d->dims[p->g[j].first]), p->ev_xb[j - 1]));
  }
  for (int j = 0; j < G; ++j)
    if (owned(d, j)) PL_TRY(ooo_join(p->stk[j], p->st[sidx(j)]));
  for (int k = 0; k < nst; ++k) {
    PL_CU(cudaEventRecord(p->ev_join[k], p->st[k]));
    PL_CU(cudaStreamWaitEvent(cap, p->ev_join[k], 0));
  }
  if (cm) {
    PL_CU(cudaEventRecord(p->ev_cj, p->comm));
    PL_CU(cudaStreamWaitEvent(cap, p->ev_cj, 0));
  }
#undef PL_CU
#undef PL_TRY
#undef PL_NC
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
