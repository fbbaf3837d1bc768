// C ABI (include/ooo.h) and the dependency-driven scheduler of the
// out-of-order backprop data-parallel hot path.
//
// Paper mapping ("P:N" = line of /root/reference/PAPER.md):
//   * iteration = backward(t) + S[dW_i] + forward(t+1), F_i gated on S[dW_i]
//     (§2 problem statement, eq. at)
//   * dW_i is consumed only by the update (§3) -> it may run out of
//     order on a low-priority stream while the critical dO chain runs on a
//     high-priority stream (§4.1; the sub-stream serialises its
//     kernels); events enforce the cross-stream dependencies (§7)
//   * the dW order is Algorithm 2 "Reverse First-K" (§5.1); S[dW_i]
//     is one NCCL all-reduce per bucket issued in that order on a comm stream
//   * a step can be captured as one executable CUDA graph (§4.2)
//   * static per-stream workspaces planned at create time replace the paper's
//     separate sub-stream allocator / XLA heap simulator (§7)
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>
#include <mutex>
#include <string>
#include <vector>

#include "../../include/ooo.h"
#include "engine.h"
#include "kernels.h"
#include "nccl_dyn.h"
#include "planner.h"
#include "skinny.h"

using namespace ooo;

// ------------------------------------------------------------------ errors
namespace {
thread_local std::string t_err;

ooo_status fail(ooo_status st, const char *fmt, ...) {
  char buf[512];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  t_err = buf;
  return st;
}

#define CU_TRY(expr)                                                                   \
  do {                                                                                 \
    cudaError_t _e = (expr);                                                           \
    if (_e != cudaSuccess)                                                             \
      return fail(OOO_ERR_CUDA, "%s failed: %s (%s:%d)", #expr, cudaGetErrorString(_e), \
                  __FILE__, __LINE__);                                                 \
  } while (0)

#define OOO_TRY(expr)                  \
  do {                                 \
    ooo_status _s = (expr);            \
    if (_s != OOO_OK) return _s;       \
  } while (0)

size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// ------------------------------------------------------------------ plan
struct GemmPlan {
  int bn = 128;
  int splits = 1;
  int kb_per_split = 1;
  dim3 grid;
};

struct LayerPlan {
  int din = 0, dout = 0, act = 0;
  size_t off_X = 0;            // X_i (input of layer i)
  size_t off_Z = SIZE_MAX;     // Z_i (only for non-identity act)
  size_t off_Xn = SIZE_MAX;    // X_{i+1} (i < L)
  size_t off_dZ = 0;
  size_t off_db = 0;           // bias-grad partials [R][dout] fp32
  int64_t goff_w = 0, goff_b = 0;
  int bucket = 0;
  GemmPlan fwd, dx, dw;
  int ebn_fwd = 0, ebn_dx = 0, ebn_dw = 0;   // engine tile widths
  int ks_fwd = 1, ks_dx = 1;                 // split-K factors of the chain ops (skinny stacks)
  int sk_fwd = 0, sk_dx = 0;                 // their first split-K arrival counter (CounterLayout::sk)
};

// Map-table slots per layer (engine): operand loads and output stores.
enum MapSlot { MS_FWD_A = 0, MS_FWD_B, MS_FWD_X, MS_FWD_Z, MS_DX_A, MS_DX_B, MS_DZ_X, MS_DW_A, MS_DW_B,
               MS_GW_X, MS_Z_PF, MS_SK_X, MS_SK_DZ, MS_COUNT };

struct Plan {
  int L = 0, M = 0, dtype = 0, elt = 2, R = 0, nbuckets = 0;
  std::vector<LayerPlan> layer;  // index i-1
  std::vector<int> bucket_first, bucket_last;
  std::vector<std::vector<int64_t>> chunk_start;   // [bucket] element offsets (in grads) of its chunks, + end
  size_t off_wpart = 0, wpart_bytes = 0;
  size_t workspace_bytes = 0;
  int64_t grad_elems = 0;
  // engine (bf16): map table, layer table, completion counters
  bool engine = false;
  int cg = 2;                      // engine CTAs per tile (2 = CTA pairs, cta_group::2)
  bool skinny = false;             // <= 16 tokens: the skinny-stack kernel (skinny.h) runs every engine launch
  size_t off_maps = 0, off_layers = 0, off_ctr = 0;
  size_t off_skpart = 0;           // split-K partials (0 bytes when no op splits)
  int sk_nc = 0;                   // 32-column chunks per partial row
  ooo::eng::CounterLayout cl{};
};

constexpr int kSMs = 148;

int env_int(const char *name, int dflt) {
  const char *v = getenv(name);
  return v && *v ? atoi(v) : dflt;
}

// Engine tile width for an output of width N: the widest of 256/192/128/64
// that divides N (the dataflow pipeline hides wave quantisation, so wider
// tiles -- better MMA efficiency, less L2 traffic per FLOP -- win).
int engine_bn(int N, bool chain, int cg, int row_tiles, int workers, int K = 0) {
  int forced = env_int(chain ? "OOO_EBN_CHAIN" : "OOO_EBN_DW", 0);
  if (!forced) forced = env_int("OOO_EBN", 0);
  if (forced && N % forced == 0 && (cg == 1 || forced % 64 == 0) && (cg == 1 || forced >= 128)) return forced;
  // skinny token dimension (one CTA row): 64-wide chain tiles spread the
  // weight stream of F_i / dO_i over 4x more SMs (1-CTA tiles only)
  if (chain && cg == 1 && row_tiles * (N / 256) * 4 <= workers && N % 64 == 0) return 64;
  // few token rows (e.g. 512 tokens = 2 pair rows): 128-wide chain tiles put
  // twice the pairs on each F_i / dO_i while they still fit the workers
  // (C4: 3.62 -> 3.14 ms; on C2's 16 rows the same change costs 25 %)
  if (chain && cg == 2 && N % 128 == 0 && row_tiles * (N / 128) <= workers) return 128;
  // CTA pairs split B in halves of >= 64 columns: bn in {128, 256}
  return N % 256 == 0 ? 256 : 128;
}

GemmPlan plan_simt(int M, int N, int K, bool weight_grad) {
  GemmPlan p;
  p.bn = 64;
  const int nkb = (K + 15) / 16;
  const int tiles = ((M + 63) / 64) * ((N + 63) / 64);
  int S = 1;
  if (weight_grad && tiles < kSMs) S = std::max(1, std::min(kSMs / tiles, nkb / 8));
  p.kb_per_split = (nkb + S - 1) / S;
  p.splits = (nkb + p.kb_per_split - 1) / p.kb_per_split;
  p.grid = dim3((M + 63) / 64, (N + 63) / 64, p.splits);
  return p;
}

ooo_status validate_desc(const ooo_stack_desc *d, bool need_pointers) {
  if (!d) return fail(OOO_ERR_INVALID_ARGUMENT, "desc is NULL");
  if (d->num_layers < 1) return fail(OOO_ERR_INVALID_ARGUMENT, "num_layers must be >= 1");
  if (!d->dims || !d->acts) return fail(OOO_ERR_INVALID_ARGUMENT, "dims/acts NULL");
  for (int i = 0; i <= d->num_layers; ++i) {
    if (d->dims[i] < 64 || d->dims[i] % 64 != 0)
      return fail(OOO_ERR_UNSUPPORTED, "dims[%d] = %d: widths must be >= 64 and multiples of 64", i,
                  d->dims[i]);
  }
  for (int i = 0; i < d->num_layers; ++i)
    if (d->acts[i] < 0 || d->acts[i] > 2)
      return fail(OOO_ERR_INVALID_ARGUMENT, "acts[%d] = %d invalid", i, d->acts[i]);
  if (d->tokens < 1 || d->tokens % 8 != 0)
    return fail(OOO_ERR_UNSUPPORTED, "tokens = %d: must be >= 1 and a multiple of 8", d->tokens);
  if (d->dtype != OOO_BF16 && d->dtype != OOO_FP32)
    return fail(OOO_ERR_INVALID_ARGUMENT, "dtype %d invalid", d->dtype);
  if (d->bucket_layers < 1) return fail(OOO_ERR_INVALID_ARGUMENT, "bucket_layers must be >= 1");
  if (d->dtype == OOO_BF16 && 2 * d->num_layers > ooo::eng::kMaxOps)
    return fail(OOO_ERR_UNSUPPORTED, "bf16 stacks: num_layers = %d > %d (engine op table)", d->num_layers,
                ooo::eng::kMaxOps / 2);
  if (d->world_size < 1 || d->rank < 0 || d->rank >= d->world_size)
    return fail(OOO_ERR_INVALID_ARGUMENT, "world_size %d / rank %d invalid", d->world_size, d->rank);
  if (need_pointers) {
    if (!d->W || !d->b) return fail(OOO_ERR_INVALID_ARGUMENT, "W/b arrays NULL");
    for (int i = 0; i < d->num_layers; ++i)
      if (!d->W[i] || !d->b[i]) return fail(OOO_ERR_INVALID_ARGUMENT, "W[%d]/b[%d] NULL", i, i);
    if (!d->grads || !d->workspace) return fail(OOO_ERR_INVALID_ARGUMENT, "grads/workspace NULL");
    if (reinterpret_cast<uintptr_t>(d->workspace) % 256 != 0 ||
        reinterpret_cast<uintptr_t>(d->grads) % 256 != 0)
      return fail(OOO_ERR_INVALID_ARGUMENT, "grads/workspace must be 256-byte aligned");
    if (d->world_size > 1 && !d->nccl_unique_id)
      return fail(OOO_ERR_INVALID_ARGUMENT, "world_size > 1 needs nccl_unique_id");
  }
  return OOO_OK;
}

Plan make_plan(const ooo_stack_desc *d) {
  Plan p;
  p.L = d->num_layers;
  p.M = d->tokens;
  p.dtype = d->dtype;
  p.elt = d->dtype == OOO_BF16 ? 2 : 4;
  const int bm = d->dtype == OOO_BF16 ? kTcBM : kSimtBM;
  p.R = (p.M + bm - 1) / bm;
  p.layer.resize(p.L);
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 256);
    return o;
  };
  const size_t M = p.M;
  // X_1, then per layer Z_i (non-identity) and X_{i+1}
  size_t xoff = take(M * d->dims[0] * p.elt);
  int64_t goff = 0;
  size_t wpart = 0;
  for (int i = 1; i <= p.L; ++i) {
    LayerPlan &lp = p.layer[i - 1];
    lp.din = d->dims[i - 1];
    lp.dout = d->dims[i];
    lp.act = d->acts[i - 1];
    lp.off_X = xoff;
    if (lp.act != OOO_ACT_IDENTITY) lp.off_Z = take(M * lp.dout * p.elt);
    if (i < p.L) {
      lp.off_Xn = take(M * lp.dout * p.elt);
      xoff = lp.off_Xn;
    }
    lp.goff_w = goff;
    lp.goff_b = goff + (int64_t)lp.din * lp.dout;
    goff = lp.goff_b + lp.dout;
    lp.bucket = (i - 1) / d->bucket_layers;
    if (p.dtype == OOO_FP32) {   // per-layer SIMT GEMMs on the hi / lo streams
      lp.fwd = plan_simt(p.M, lp.dout, lp.din, false);
      lp.dx = plan_simt(p.M, lp.din, lp.dout, false);
      lp.dw = plan_simt(lp.din, lp.dout, p.M, true);
    }
    if (lp.dw.splits > 1) wpart = std::max(wpart, (size_t)lp.dw.splits * lp.din * lp.dout * 4);
  }
  for (int i = 1; i <= p.L; ++i) p.layer[i - 1].off_dZ = take(M * p.layer[i - 1].dout * p.elt);
  for (int i = 1; i <= p.L; ++i) p.layer[i - 1].off_db = take((size_t)p.R * p.layer[i - 1].dout * 4);
  p.wpart_bytes = wpart;
  p.off_wpart = wpart ? take(wpart) : 0;
  p.nbuckets = (p.L + d->bucket_layers - 1) / d->bucket_layers;
  // persistent dataflow engine (bf16): map table, layer table, counters
  p.engine = p.dtype == OOO_BF16;   // bf16: the persistent dataflow engine (validate_desc bounds L)
  if (p.engine) {
    // CTA pairs (256-row tiles) unless the token dimension fits one 128-row tile
    const int cg_env = env_int("OOO_CG", 0);
    p.cg = cg_env == 1 ? 1 : (cg_env == 2 ? 2 : (p.M <= 128 ? 1 : 2));
    const int workers = kSMs / p.cg;
    const int MT = (p.M + 127) / 128;
    const int PT = (MT + p.cg - 1) / p.cg;                      // tile rows of F_i / dO_i
    for (int i = 1; i <= p.L; ++i) {
      LayerPlan &lp = p.layer[i - 1];
      lp.ebn_fwd = engine_bn(lp.dout, true, p.cg, PT, workers, lp.din);
      lp.ebn_dx = engine_bn(lp.din, true, p.cg, PT, workers, lp.dout);
      lp.ebn_dw = engine_bn(lp.dout, false, p.cg, PT, workers);
    }
    // <= 16 tokens: chain ops as 8-CTA clusters with a DSMEM K-split
    // reduction (skinny.h; OOO_SKINNY=0 keeps the engine): 128-wide chain
    // tiles where the width allows (the kernel's tile widths)
    p.skinny = p.cg == 1 && p.M <= ooo::sk::kMaxM && env_int("OOO_SKINNY", 1) != 0;
    if (p.skinny)
      for (int i = 1; i <= p.L; ++i) {
        LayerPlan &lp = p.layer[i - 1];
        lp.ebn_fwd = lp.dout % 128 == 0 ? 128 : 64;
        lp.ebn_dx = lp.din % 128 == 0 ? 128 : 64;
      }
    // split-K chain ops when all tokens fit one 128-row tile (C5 through the
    // engine, OOO_SKINNY=0 / > 16 tokens):
    // a chain op's latency is its k-blocks at the MMA issue rate, whatever its
    // width (profiles/r02_mainloop_issue.md), so its K is spread over up to 8
    // workers while the split tiles still fit them (>= 4 k-blocks each: C5
    // 1.434 -> 1.363 ms with 4 splits, 1.614 with 8 splits of 2); the
    // fp32 partials of so few rows cost little.  With more rows the partial
    // traffic outweighs the k-blocks saved (C4, 512 tokens: 2.90 -> 3.70 ms
    // with 4 splits, profiles/r02_splitk.md).  Not for ReLU F_i (their Z_i
    // store is a pass over the TMEM accumulator, which a split task no longer
    // holds).  OOO_SPLITK=0: off; OOO_SPLITK_MAX / OOO_SPLITK_MINKB: tuning.
    int nsk = 0, maxw = 0;
    for (int i = 0; i <= p.L; ++i) maxw = std::max(maxw, d->dims[i]);
    // with more rows, only the long-K chain ops split (>= longk k-blocks: C4's
    // K = 4096 ops, 8 tiles x 64 k-blocks = 28 us each on the chain): C4
    // 2.82 -> 2.72 ms; the split epilogue (~10 us: its fp32 partial round
    // trips through L2) loses on shorter K.  OOO_SPLITK_LONGK=0: off
    const int longk = env_int("OOO_SPLITK_LONGK", 64);
    auto ksplit = [&](int N, int bn, int K, bool allowed) {
      if (!allowed || p.skinny || env_int("OOO_SPLITK", 1) == 0) return 1;
      if (p.M > 128 && (longk <= 0 || (K + 63) / 64 < longk)) return 1;
      const int tiles = PT * ((N + bn - 1) / bn);
      const int minkb = std::max(1, env_int("OOO_SPLITK_MINKB", 4));
      const int ks = std::min({std::min(8, env_int("OOO_SPLITK_MAX", 8)), ((K + 63) / 64) / minkb, workers / tiles});
      return ks >= 2 ? ks : 1;
    };
    int ksmax = 1;
    for (int i = 1; i <= p.L; ++i) {
      LayerPlan &lp = p.layer[i - 1];
      lp.ks_fwd = ksplit(lp.dout, lp.ebn_fwd, lp.din, lp.act != OOO_ACT_RELU);
      lp.ks_dx = ksplit(lp.din, lp.ebn_dx, lp.dout, true);
      ksmax = std::max({ksmax, lp.ks_fwd, lp.ks_dx});
      lp.sk_fwd = nsk;
      if (lp.ks_fwd > 1) nsk += PT * ((lp.dout + lp.ebn_fwd - 1) / lp.ebn_fwd) * p.cg;
      lp.sk_dx = nsk;
      if (lp.ks_dx > 1) nsk += PT * ((lp.din + lp.ebn_dx - 1) / lp.ebn_dx) * p.cg;
    }
    p.sk_nc = maxw / 32;
    p.off_maps = take((size_t)p.L * MS_COUNT * sizeof(CUtensorMap));
    p.off_layers = take((size_t)p.L * sizeof(ooo::eng::LayerDev));
    ooo::eng::CounterLayout &cl = p.cl;
    cl.L = p.L;
    cl.MT = (p.M + 127) / 128;
    cl.nb = p.nbuckets;
    cl.fwd_rows = 2;
    cl.xcopy = cl.fwd_rows + p.L * cl.MT;
    cl.sk = cl.xcopy + cl.MT;
    cl.fwd_end = cl.sk + nsk;
    cl.dz_rows = (int)align_up(cl.fwd_end, 32);
    cl.dz_total = cl.dz_rows + p.L * cl.MT;
    cl.dw_done = cl.dz_total + p.L;
    cl.bucket_done = cl.dw_done + p.L;
    cl.ar_done = cl.bucket_done + p.nbuckets;
    cl.dx_total = cl.ar_done + p.nbuckets;
    cl.total = cl.dx_total + 1;
    p.off_ctr = take((size_t)cl.total * 4);
    if (nsk > 0) p.off_skpart = take((size_t)ksmax * cl.MT * p.sk_nc * 128 * 32 * 4);   // [split][row block][chunk]
  }
  p.workspace_bytes = std::max<size_t>(off, 256);
  p.grad_elems = goff;
  p.bucket_first.resize(p.nbuckets);
  p.bucket_last.resize(p.nbuckets);
  p.chunk_start.resize(p.nbuckets);
  for (int b = 0; b < p.nbuckets; ++b) {
    p.bucket_first[b] = b * d->bucket_layers + 1;
    p.bucket_last[b] = std::min(p.L, (b + 1) * d->bucket_layers);
    // fixed chunk boundaries (schedule independent): NEXT-4 partitioning
    const int64_t e0 = p.layer[p.bucket_first[b] - 1].goff_w;
    const int64_t e1 = p.layer[p.bucket_last[b] - 1].goff_b + p.layer[p.bucket_last[b] - 1].dout;
    int64_t ce = d->comm_chunk_bytes > 0 ? d->comm_chunk_bytes / p.elt / 256 * 256 : 0;
    if (ce <= 0) ce = e1 - e0;
    for (int64_t e = e0; e < e1; e += ce) p.chunk_start[b].push_back(e);
    p.chunk_start[b].push_back(e1);
  }
  return p;
}

// Alg. 2 lines 3-6.  Reading Q1: dO_1 only if need_input_grad.
// in_order (k = 0, dO_i first within a layer, reading Q2).
void schedule_ops(int L, int kind, int k, bool need_dx, std::vector<int> &D) {
  D.clear();
  if (kind == OOO_SCHED_IN_ORDER) {
    for (int i = L; i >= 1; --i) {
      if (i > 1 || need_dx) D.push_back(+i);
      D.push_back(-i);
    }
    return;
  }
  k = std::min(std::max(k, 0), L);
  for (int i = L; i >= 1; --i) {           // l.3
    if (i > k) D.push_back(-i);            // l.4
    if (i > 1 || need_dx) D.push_back(+i); // l.5
  }
  for (int i = 1; i <= k; ++i) D.push_back(-i);   // l.6
}

// ------------------------------------------------------------ tensor maps
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                  const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void *p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  return fn;
}

// 2-D bf16 row-major tensor [outer][inner], 128-B swizzled box {box_inner, box_outer}.
ooo_status make_map(CUtensorMap *m, const void *ptr, uint64_t inner, uint64_t outer,
                    uint32_t box_inner, uint32_t box_outer, int swizzle_bytes = 128) {
  EncodeTiledFn enc = get_encode();
  if (!enc) return fail(OOO_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {inner * 2};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = enc(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void *>(ptr), dims, strides, box,
                   es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   swizzle_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_128B,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(OOO_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return OOO_OK;
}

}  // namespace

// ------------------------------------------------------------------ stack
struct LayerRt {
  void *W = nullptr, *b = nullptr;
  void *X = nullptr, *Z = nullptr, *Xn = nullptr, *dZ = nullptr;
  float *db = nullptr;
  void *gw = nullptr, *gb = nullptr;
};

struct TimedRec {
  ooo_launch_record info;
  cudaEvent_t a = nullptr, b = nullptr;
};

struct ooo_stack {
  ooo_stack_desc d;
  std::vector<int> dims, acts;
  Plan p;
  std::vector<LayerRt> lr;
  uint8_t *ws = nullptr;
  uint8_t *grads = nullptr;
  cudaStream_t hi = nullptr, lo = nullptr, comm = nullptr;
  int prio_hi = 0, prio_lo = 0;
  std::vector<cudaEvent_t> ev_dz, ev_pack, ev_ar;   // ev_dz[i], ev_pack[i] (1-based), ev_ar[b]
  cudaEvent_t ev_fork = nullptr, ev_j_hi = nullptr, ev_j_lo = nullptr, ev_j_comm = nullptr;
  cudaEvent_t ev_reset = nullptr;             // engine: counters reset (the comm stream's value-waits start after it)
  bool have_fwd = false;
  bool bwd_pending = false;
  ncclComm_t nccl = nullptr;
  const NcclApi *api = nullptr;
  bool timing = false;
  bool pdl = true;
  std::vector<TimedRec> recs;
  size_t rec_cursor = 0;
  std::vector<int> D;
  // persistent dataflow engine (bf16)
  int32_t *ctr = nullptr;                     // completion counters (workspace)
  const CUtensorMap *dmaps = nullptr;         // map table (workspace)
  const ooo::eng::LayerDev *dlayers = nullptr;
  int engine_ctas = 148;
  bool comm_stack = false;                    // a NCCL communicator (N > 1, or the one-rank mode)
  int timeout_ms = 4000;                      // engine wait bound (desc.wait_timeout_ms)
  bool test_comm_gate = false;                // OOO_TEST_COMM_GATE=1 (N = 1 only): see comm_active
  int test_drop_flag = -1;                    // OOO_TEST_DROP_AR_FLAG=b: bucket b's flag is never written
                                              // (tests that the engine's wait bound traps instead of hanging)
  // emulated all-reduce (N = 1 only; OOO_EMULATE_AR_N = n >= 2): each bucket's
  // S[dW] holds the comm stream for the ring time 2(n-1)/n x bytes / BW + lat
  int emu_n = 0;
  double emu_gbps = 900.0, emu_lat_us = 8.0;
  bool eng_pending = false;                   // ooo_backward enqueued, its kernel deferred
  std::vector<ooo::plan::Unit> eng_crit, eng_defer;   // the deferred backward's chains
  double eng_flops = 0;
  void *eng_dX = nullptr;
  bool eng_in_order = false;
  bool eng_comm = false;                      // the deferred backward's per-bucket S[dW] still to enqueue
  std::vector<double> pred_dw;                // planner: predicted dW_i completion (us) of the last launch
  std::vector<int> comm_b, comm_c;            // the last step's all-reduce chunk issue order (introspection)
  // region plan (OOO_SCHED_REGIONS, §4.1; ooo_plan_regions)
  bool has_regions = false;
  std::vector<int> reg_D;          // backward order D of the plan
  std::vector<int> reg_release;    // [L] release of dW_i: >= 0 index into the backward chain,
                                   // <= -2: F_m of the next forward (m = -tag - 1)
  std::vector<int> reg_region_of;  // [L] main-stream region of dW_i
  std::vector<double> reg_tmain;   // profiled region times (ms)
  int reg_kpre = 0;
#ifdef OOO_TRACE
  std::vector<ooo::eng::Op> last_queue;       // debug: the most recent engine launch's ops
#endif
};

struct ooo_graph {
  ooo_stack *s = nullptr;
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  // per-launch timing (ooo_graph_set_timing_slots): the timing brackets
  // captured into the graph (record info in capture order), their event-record
  // nodes, and `slots` sets of events the nodes are re-pointed to, one set per
  // launch, so every launch of a timed region keeps its own measurement
  struct TNode { cudaGraphNode_t node; int rec, which; };
  std::vector<ooo_launch_record> tinfo;
  std::vector<TNode> tnodes;
  std::vector<cudaEvent_t> sev;    // [slot][rec][2]
  int slots = 0;
  long launches = 0;
  // host-buffer steps (ooo_graph_upload / ooo_graph_launch_host): the
  // device buffers baked into the graph and the events ordering the copies
  void *dX = nullptr, *dY = nullptr, *dYout = nullptr;
  size_t x_bytes = 0, dy_bytes = 0, y_bytes = 0;
  cudaEvent_t ev_in = nullptr, ev_done = nullptr;
  bool launched = false;
};

namespace {

// Timing events become event-record nodes when the stream is being captured
// (cudaEventRecordExternal); outside capture they are plain records.
cudaError_t record_timing_event(cudaEvent_t ev, cudaStream_t st) {
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  cudaError_t e = cudaStreamIsCapturing(st, &cs);
  if (e != cudaSuccess) return e;
  if (cs == cudaStreamCaptureStatusActive) return cudaEventRecordWithFlags(ev, st, cudaEventRecordExternal);
  return cudaEventRecord(ev, st);
}

ooo_status begin_rec(ooo_stack *s, cudaStream_t st, int kind, int layer, int sid, TimedRec **out) {
  *out = nullptr;
  if (!s->timing) return OOO_OK;
  if (s->rec_cursor >= s->recs.size()) {
    TimedRec r;
    CU_TRY(cudaEventCreate(&r.a));
    CU_TRY(cudaEventCreate(&r.b));
    s->recs.push_back(r);
  }
  TimedRec *r = &s->recs[s->rec_cursor++];
  memset(&r->info, 0, sizeof(r->info));
  r->info.kind = kind;
  r->info.layer = layer;
  r->info.stream = sid;
  CU_TRY(record_timing_event(r->a, st));
  *out = r;
  return OOO_OK;
}
ooo_status end_rec(TimedRec *r, cudaStream_t st, int grid, double flops, double bytes) {
  if (!r) return OOO_OK;
  r->info.grid = grid;
  r->info.flops = flops;
  r->info.bytes = bytes;
  CU_TRY(record_timing_event(r->b, st));
  return OOO_OK;
}

// Pack/scale factor of the gradients (reading Q9: 1/N before the sum all-reduce).
float grad_alpha(const ooo_stack *s) {
  return 1.0f / (float)(s->d.average_over > 0 ? s->d.average_over : s->d.world_size);
}

// ---- op launchers ------------------------------------------------------
ooo_status launch_fwd(ooo_stack *s, int i, void *Y, cudaStream_t st, int prio) {
  const LayerPlan &lp = s->p.layer[i - 1];
  LayerRt &r = s->lr[i - 1];
  EpiArgs a = {};
  a.M = s->p.M; a.N = lp.dout; a.K = lp.din;
  a.kb_per_split = lp.fwd.kb_per_split; a.splits = 1;
  a.act = lp.act; a.ldc = lp.dout; a.alpha = 1.f;
  a.bias = r.b; a.z_out = r.Z; a.x_out = (i == s->p.L) ? Y : r.Xn;
  TimedRec *tr;
  OOO_TRY(begin_rec(s, st, 0, i, 0, &tr));
  LaunchCtx ctx{st, prio, s->pdl};
  int grid = 0;
  SimtOperands o{static_cast<const float *>(r.X), lp.din, 1, static_cast<const float *>(r.W), lp.dout, 1};
  CU_TRY(launch_gemm_simt(EPI_FWD, o, a, ctx, &grid));
  return end_rec(tr, st, grid, 2.0 * s->p.M * lp.din * lp.dout, 0);
}

// dO_i: i >= 2 -> dZ_{i-1} (+ db_{i-1} partials); i == 1 -> dX (no epilogue)
ooo_status launch_dx(ooo_stack *s, int i, void *dX, cudaStream_t st, int prio) {
  const LayerPlan &lp = s->p.layer[i - 1];
  LayerRt &r = s->lr[i - 1];
  EpiArgs a = {};
  a.M = s->p.M; a.N = lp.din; a.K = lp.dout;
  a.kb_per_split = lp.dx.kb_per_split; a.splits = 1;
  a.ldc = lp.din; a.alpha = 1.f;
  if (i >= 2) {
    const LayerPlan &pp = s->p.layer[i - 2];
    LayerRt &pr = s->lr[i - 2];
    a.act = pp.act;
    a.zin = pr.Z;            // null for identity (act' = 1, not read)
    a.x_out = pr.dZ;
    a.dbpart = pr.db;
  } else {
    a.act = OOO_ACT_IDENTITY;
    a.x_out = dX;
    a.dbpart = nullptr;
  }
  TimedRec *tr;
  OOO_TRY(begin_rec(s, st, 1, i, st == s->hi ? 0 : 1, &tr));
  LaunchCtx ctx{st, prio, s->pdl};
  int grid = 0;
  SimtOperands o{static_cast<const float *>(r.dZ), lp.dout, 1, static_cast<const float *>(r.W), 1, lp.dout};
  CU_TRY(launch_gemm_simt(EPI_DGRAD, o, a, ctx, &grid));
  return end_rec(tr, st, grid, 2.0 * s->p.M * lp.din * lp.dout, 0);
}

// dW_i (+ pack: split-K reduction, db reduction, 1/N scale -> bucket)
ooo_status launch_dw_pack(ooo_stack *s, int i, cudaStream_t st, int prio, int sid) {
  const LayerPlan &lp = s->p.layer[i - 1];
  LayerRt &r = s->lr[i - 1];
  const float alpha = grad_alpha(s);
  EpiArgs a = {};
  a.M = lp.din; a.N = lp.dout; a.K = s->p.M;
  a.kb_per_split = lp.dw.kb_per_split; a.splits = lp.dw.splits;
  a.ldc = lp.dout; a.alpha = alpha;
  a.x_out = r.gw;
  a.fpart = reinterpret_cast<float *>(s->ws + s->p.off_wpart);
  TimedRec *tr;
  OOO_TRY(begin_rec(s, st, 2, i, sid, &tr));
  LaunchCtx ctx{st, prio, s->pdl};
  int grid = 0;
  SimtOperands o{static_cast<const float *>(r.X), 1, lp.din, static_cast<const float *>(r.dZ), lp.dout, 1};
  CU_TRY(launch_gemm_simt(EPI_WGRAD, o, a, ctx, &grid));
  OOO_TRY(end_rec(tr, st, grid, 2.0 * s->p.M * lp.din * lp.dout, 0));
  // pack (plain launch: it does not use griddepcontrol)
  ctx.pdl = false;
  OOO_TRY(begin_rec(s, st, 4, i, sid, &tr));
  const bool split = lp.dw.splits > 1;
  const long long wcount = (long long)lp.din * lp.dout;
  int pgrid = 0;
  CU_TRY(launch_pack(s->p.dtype == OOO_BF16, split ? a.fpart : nullptr, lp.dw.splits, wcount, r.gw, r.db,
                     s->p.R, lp.dout, r.gb, alpha, ctx, &pgrid));
  const double pbytes = (split ? (double)wcount * (4.0 * lp.dw.splits + s->p.elt) : 0.0) +
                        (double)lp.dout * (4.0 * s->p.R + s->p.elt);
  return end_rec(tr, st, pgrid, 0, pbytes);
}

ooo_status launch_seed_op(ooo_stack *s, const void *dY, cudaStream_t st, int prio) {
  const int L = s->p.L;
  const LayerPlan &lp = s->p.layer[L - 1];
  LayerRt &r = s->lr[L - 1];
  TimedRec *tr;
  OOO_TRY(begin_rec(s, st, 3, L, 0, &tr));
  int grid = 0;
  LaunchCtx ctx{st, prio};
  const int bm = s->p.dtype == OOO_BF16 ? kTcBM : kSimtBM;
  // the engine's F_L stores gelu'(Z_L) in place of Z_L (engine.cu)
  const int act = s->p.engine && lp.act == OOO_ACT_GELU_ERF ? (int)ACT_DSTORED : (int)lp.act;
  CU_TRY(launch_seed(s->p.dtype == OOO_BF16, dY, r.Z, act, r.dZ, r.db, s->p.M, lp.dout, bm, ctx, &grid));
  const double bytes = (double)s->p.M * lp.dout * s->p.elt * (lp.act != OOO_ACT_IDENTITY ? 3.0 : 2.0) +
                       (double)s->p.R * lp.dout * 4.0;
  return end_rec(tr, st, grid, 0, bytes);
}

// S[dW] of chunk c of bucket b (the whole bucket when it is not partitioned).
ooo_status launch_allreduce(ooo_stack *s, int b, int c) {
  const int64_t e0 = s->p.chunk_start[b][c], e1 = s->p.chunk_start[b][c + 1];
  if (s->emu_n > 1) {
    TimedRec *tr;
    OOO_TRY(begin_rec(s, s->comm, 5, b, 2, &tr));
    const double n = s->emu_n;
    const double ring = 2.0 * (n - 1) / n * (double)(e1 - e0) * s->p.elt;
    const double ns = ring / (s->emu_gbps * 1e9) * 1e9 + s->emu_lat_us * 1e3;
    CU_TRY(launch_delay((unsigned long long)ns, s->comm));
    OOO_TRY(end_rec(tr, s->comm, 1, 0, ring));
    return OOO_OK;
  }
  if (s->nccl && s->d.comm_enabled) {
    TimedRec *tr;
    OOO_TRY(begin_rec(s, s->comm, 5, b, 2, &tr));
    void *buf = s->grads + e0 * s->p.elt;
    ncclResult_t rr = s->api->AllReduce(buf, buf, (size_t)(e1 - e0),
                                        s->p.dtype == OOO_BF16 ? ncclBfloat16 : ncclFloat32, ncclSum,
                                        s->nccl, s->comm);
    if (rr != ncclSuccess)
      return fail(OOO_ERR_NCCL, "ncclAllReduce: %s", s->api->GetErrorString(rr));
    const double n = s->d.world_size;
    OOO_TRY(end_rec(tr, s->comm, 0, 0, 2.0 * (n - 1) / n * (double)(e1 - e0) * s->p.elt));
  }
  return OOO_OK;
}
ooo_status launch_allreduce(ooo_stack *s, int b) {
  for (int c = 0; c + 1 < (int)s->p.chunk_start[b].size(); ++c) OOO_TRY(launch_allreduce(s, b, c));
  return OOO_OK;
}

ooo_status fork_from(ooo_stack *s, cudaStream_t st) {
  CU_TRY(cudaEventRecord(s->ev_fork, st));
  CU_TRY(cudaStreamWaitEvent(s->hi, s->ev_fork, 0));
  CU_TRY(cudaStreamWaitEvent(s->lo, s->ev_fork, 0));
  CU_TRY(cudaStreamWaitEvent(s->comm, s->ev_fork, 0));
  return OOO_OK;
}

ooo_status join_into(ooo_stack *s, cudaStream_t st) {
  CU_TRY(cudaEventRecord(s->ev_j_hi, s->hi));
  CU_TRY(cudaEventRecord(s->ev_j_lo, s->lo));
  CU_TRY(cudaEventRecord(s->ev_j_comm, s->comm));
  CU_TRY(cudaStreamWaitEvent(st, s->ev_j_hi, 0));
  CU_TRY(cudaStreamWaitEvent(st, s->ev_j_lo, 0));
  CU_TRY(cudaStreamWaitEvent(st, s->ev_j_comm, 0));
  return OOO_OK;
}

// Caller activation buffers: the bf16 engine's epilogue stores rows with
// 32-byte vector stores (st.global.v8.b32) and its X -> X_1 copy reads 16-byte
// vectors, so X / Y / dY / dX must be 32-byte aligned (TMA descriptors alone
// would accept 16); fp32 stacks need 16 bytes.
ooo_status check_align(const ooo_stack *s, const void *p, const char *name) {
  const uintptr_t a = s->p.dtype == OOO_BF16 ? 32 : 16;
  if (reinterpret_cast<uintptr_t>(p) % a != 0)
    return fail(OOO_ERR_INVALID_ARGUMENT, "%s must be %d-byte aligned", name, (int)a);
  return OOO_OK;
}

ooo_status check_async(ooo_stack *s) {
  if (s->nccl) {
    ncclResult_t ar = ncclSuccess;
    ncclResult_t rr = s->api->CommGetAsyncError(s->nccl, &ar);
    if (rr != ncclSuccess || ar != ncclSuccess)
      return fail(OOO_ERR_NCCL, "NCCL async error: %s",
                  s->api->GetErrorString(rr != ncclSuccess ? rr : ar));
  }
  cudaError_t e = cudaPeekAtLastError();
  if (e != cudaSuccess) return fail(OOO_ERR_CUDA, "pending CUDA error: %s", cudaGetErrorString(e));
  return OOO_OK;
}

// ---- persistent dataflow engine (bf16) ---------------------------------
typedef CUresult (*StreamValueFn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

StreamValueFn stream_value_fn(const char *name) {
  void *p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess)
    return nullptr;
  return reinterpret_cast<StreamValueFn>(p);
}

int map_index(int layer, int slot) { return (layer - 1) * MS_COUNT + slot; }

// The comm stream takes part in the step (bucket all-reduces + ar_done flags
// gating F_i).  test_comm_gate: world_size 1 with the same wait-value /
// write-value chain but no all-reduce, so single-GPU tests exercise the N > 1
// gating of the fused step.
bool comm_active(const ooo_stack *s) {
  return (s->nccl != nullptr && s->d.comm_enabled) || s->test_comm_gate || s->emu_n > 1;
}

namespace pl = ooo::plan;
static_assert(pl::FWD == EPI_FWD && pl::DGRAD == EPI_DGRAD && pl::WGRAD == EPI_WGRAD &&
                  pl::COPY == ooo::eng::EPI_COPY, "planner kinds = engine task kinds");

// Planner timing model (tuning knobs for experiments: OOO_PLAN_LEAD, OOO_PLAN_RESERVE).
pl::Model plan_model() {
  pl::Model m;
  if (const char *v = getenv("OOO_PLAN_LEAD")) m.lead = atof(v);
  if (const char *v = getenv("OOO_PLAN_RESERVE")) m.reserve = atof(v);
  return m;
}

// Rows of the A box of row-local (F_i / dO_i) tiles: all tokens fit one
// 1-CTA tile -> only the M valid rows are fetched (no 128-row OOB fill).
int a_box_rows(const Plan &p) {
  if (p.cg == 1 && p.M < 128 && env_int("OOO_SMALL_ABOX", 1)) return (p.M + 7) / 8 * 8;
  return 128;
}

int copy_bn(int d0) { return d0 % 256 == 0 ? 256 : (d0 % 128 == 0 ? 128 : 64); }

// Whole-op planner units.  Row-local ops (F_i, dO_i, copy) span the PT =
// ceil(MT / cg) token tile rows; dW_i spans the ceil(d_{i-1} / (128 cg)) rows
// of its weight-gradient tile grid.
pl::Unit unit_of(const ooo_stack *s, int kind, int i) {
  const Plan &p = s->p;
  const int PT = (p.cl.MT + p.cg - 1) / p.cg;
  pl::Unit u = {};
  u.kind = kind;
  u.layer = i;
  u.m_off = 0;
  if (kind == pl::COPY) {
    u.layer = 1;
    u.bn = copy_bn(s->dims[0]);
    u.mt = PT;
    u.nt = (s->dims[0] + u.bn - 1) / u.bn;
    u.nkb = 0;
    return u;
  }
  const LayerPlan &lp = p.layer[i - 1];
  if (kind == pl::FWD) {
    u.act = lp.act;
    u.bn = lp.ebn_fwd;
    u.mt = PT;
    u.nt = (lp.dout + u.bn - 1) / u.bn;
    u.nkb = (lp.din + 63) / 64;
    u.ks = lp.ks_fwd;
  } else if (kind == pl::DGRAD) {
    u.act = i >= 2 ? p.layer[i - 2].act : OOO_ACT_IDENTITY;
    u.bn = lp.ebn_dx;
    u.mt = PT;
    u.nt = (lp.din + u.bn - 1) / u.bn;
    u.nkb = (lp.dout + 63) / 64;
    u.ks = lp.ks_dx;
  } else {
    u.act = OOO_ACT_IDENTITY;
    u.bn = lp.ebn_dw;
    u.mt = ((lp.din + 127) / 128 + p.cg - 1) / p.cg;
    u.nt = (lp.dout + u.bn - 1) / u.bn;
    u.nkb = (p.M + 63) / 64;
  }
  u.nkb_full = u.nkb;
  if (u.ks > 1) u.nkb = (u.nkb + u.ks - 1) / u.ks;   // the planner's per-task k-blocks
  return u;
}

ooo::eng::Op op_of_unit(const ooo_stack *s, const pl::Unit &u) {
  const Plan &p = s->p;
  const int i = u.layer;
  ooo::eng::Op o = {};
  o.kind = (int16_t)u.kind;
  o.layer = (int16_t)i;
  o.act = (int16_t)u.act;
  o.bn = (int16_t)u.bn;
  o.m_off = (int16_t)(p.cg * u.m_off);   // 128-row blocks
  o.mt = (int16_t)u.mt;
  o.nt = (int16_t)u.nt;
  o.nkb = (int16_t)u.nkb_full;
  o.ks = (int16_t)std::max(1, u.ks);
  if (u.ks > 1) {   // arrival counters of this unit's tiles: after the op's earlier rows
    const LayerPlan &lp = p.layer[i - 1];
    o.sk_base = (int16_t)((u.kind == pl::FWD ? lp.sk_fwd : lp.sk_dx) + u.m_off * u.nt * p.cg);
  }
  o.mapA = o.mapB = o.mapX = o.mapZ = ooo::eng::MAP_NONE;
  if (u.kind == pl::FWD) {
    o.mapA = (int16_t)(i == 1 ? ooo::eng::MAP_XIN : map_index(i, MS_FWD_A));   // F_1 reads the caller's X
    o.mapB = (int16_t)map_index(i, MS_FWD_B);
    o.mapX = (int16_t)(i == p.L ? ooo::eng::MAP_Y : map_index(i, MS_FWD_X));
    o.mapZ = (int16_t)(s->lr[i - 1].Z ? map_index(i, MS_FWD_Z) : ooo::eng::MAP_NONE);
  } else if (u.kind == pl::DGRAD) {
    o.mapA = (int16_t)map_index(i, MS_DX_A);
    o.mapB = (int16_t)map_index(i, MS_DX_B);
    o.mapX = (int16_t)(i >= 2 ? map_index(i - 1, MS_DZ_X) : ooo::eng::MAP_DX);
    // the epilogue's act'(Z_{i-1}) input, L2-prefetched at dispatch
    o.mapZ = (int16_t)(i >= 2 && s->lr[i - 2].Z ? map_index(i - 1, MS_Z_PF) : ooo::eng::MAP_NONE);
  } else if (u.kind == pl::WGRAD) {
    o.mapA = (int16_t)map_index(i, MS_DW_A);
    o.mapB = (int16_t)map_index(i, MS_DW_B);
    o.mapX = (int16_t)map_index(i, MS_GW_X);
  }
  return o;
}

// Backward chains.  ooo schedules: critical = the dO chain in D's order,
// deferred = the dW ops in D's order (Alg. 2: dW_L..dW_{k+1}, then the
// reversed first-k dW_1..dW_k); the planner interleaves them (two priority
// streams).  in_order (conventional backprop): one chain =
// D, and the kernel adds the dW_{i+1} -> dO_i dependency.
void engine_bwd_units(const ooo_stack *s, bool in_order, bool regions, std::vector<pl::Unit> &crit,
                      std::vector<pl::Unit> &defer, double &flops) {
  const Plan &p = s->p;
  for (int op : s->D) {
    const int i = op > 0 ? op : -op;
    pl::Unit u = unit_of(s, op > 0 ? pl::DGRAD : pl::WGRAD, i);
    if (regions && op < 0) u.release = s->reg_release[i - 1];   // Algorithm 1's region (§4.1)
    (op < 0 && !in_order ? defer : crit).push_back(u);
    flops += 2.0 * p.M * p.layer[i - 1].din * p.layer[i - 1].dout;
  }
}

// Skinny stacks (skinny.h): the chain ops (F_i, dO_i) in chain order for the
// chain clusters, the dW ops in D's order (Alg. 2) and the X -> X_1 copy for
// the dW workers; same counters, gates and stores as the engine.
ooo_status skinny_launch(ooo_stack *s, const std::vector<pl::Unit> &crit, const std::vector<pl::Unit> &defer,
                         void *Y, void *dX, const void *X, bool in_order, int fwd_gate, int rec_kind, double flops) {
  const Plan &p = s->p;
  static ooo::sk::Params P;   // ~7 KB: not on the stack (launches are serialised by the caller)
  memset(&P, 0, sizeof(P));
  P.L = p.L;
  P.M = p.M;
  P.in_order = in_order ? 1 : 0;
  P.fwd_gate = fwd_gate;
  P.dbg = env_int("OOO_DBG", 0);
  P.alpha = grad_alpha(s);
  P.timeout_ns = (uint64_t)s->timeout_ms * 1000000ull;
  P.maps = s->dmaps;
  P.maps_per_layer = MS_COUNT;
  P.map_x = MS_SK_X;
  P.map_dz = MS_SK_DZ;
  P.map_w = MS_FWD_B;
  P.ctr = s->ctr;
  P.layers = s->dlayers;
  P.cl = p.cl;
  P.y_out = Y;
  P.dx_out = dX;
  P.x_in = X;
  int max_tiles = 0, ntask = 0;
  auto add_chain = [&](const pl::Unit &u) {
    if (P.nchain >= ooo::sk::kMaxChain) return false;
    P.chain[P.nchain].kind = (int16_t)u.kind;
    P.chain[P.nchain].layer = (int16_t)u.layer;
    ++P.nchain;
    const LayerPlan &lp = p.layer[u.layer - 1];
    max_tiles = std::max(max_tiles, u.kind == pl::FWD ? lp.dout / lp.ebn_fwd : lp.din / lp.ebn_dx);
    return true;
  };
  auto add_dw = [&](const pl::Unit &u) {
    if (P.ndw >= ooo::sk::kMaxDw) return false;
    ooo::sk::DwOp &o = P.dw[P.ndw++];
    o.kind = (int16_t)u.kind;
    o.layer = (int16_t)u.layer;
    o.first = ntask;
    const LayerPlan &lp = p.layer[u.layer - 1];
    ntask += u.kind == pl::COPY ? 1 : ((lp.din + 127) / 128) * ((lp.dout + lp.ebn_dw - 1) / lp.ebn_dw);
    return true;
  };
  for (const std::vector<pl::Unit> *v : {&crit, &defer})
    for (const pl::Unit &u : *v)
      if ((u.kind == pl::FWD || u.kind == pl::DGRAD) && !add_chain(u))
        return fail(OOO_ERR_UNSUPPORTED, "skinny: too many chain ops");
  for (const std::vector<pl::Unit> *v : {&crit, &defer})
    for (const pl::Unit &u : *v)
      if (u.kind == pl::WGRAD && !add_dw(u)) return fail(OOO_ERR_UNSUPPORTED, "skinny: too many dW ops");
  for (const std::vector<pl::Unit> *v : {&crit, &defer})
    for (const pl::Unit &u : *v)
      if (u.kind == pl::COPY && !add_dw(u)) return fail(OOO_ERR_UNSUPPORTED, "skinny: too many dW ops");
  P.ntasks_dw = ntask;
  // clusters: as many chain clusters as the widest chain op has tiles, at
  // least one dW-worker cluster when there are dW tasks
  const int total = std::min(s->engine_ctas / ooo::sk::kCl, ooo::sk::skinny_max_clusters());
  if (total < (P.nchain > 0) + (P.ndw > 0)) return fail(OOO_ERR_UNSUPPORTED, "skinny: %d clusters fit", total);
  P.nclu = P.nchain > 0 ? std::max(1, std::min(max_tiles, total - (P.ndw > 0 ? 1 : 0))) : 0;
  const int clusters = P.ndw > 0 ? total : P.nclu;
  if (env_int("OOO_SKINNY_VERBOSE", 0))
    fprintf(stderr, "[skinny] max_clusters %d total %d chain clusters %d (widest op %d tiles) launch %d; "
            "chain ops %d, dW ops %d (%d tasks)\n", ooo::sk::skinny_max_clusters(), total, P.nclu, max_tiles,
            clusters, P.nchain, P.ndw, P.ntasks_dw);
  CUtensorMap tmX;
  OOO_TRY(make_map(&tmX, X ? X : s->lr[0].X, s->dims[0], p.M, 64, 16));
  TimedRec *tr;
  OOO_TRY(begin_rec(s, s->hi, rec_kind, 0, 0, &tr));
  CU_TRY(ooo::sk::launch_skinny(P, &tmX, clusters, s->hi));
  return end_rec(tr, s->hi, clusters * ooo::sk::kCl, flops, 0);
}

// Plans the FIFO order (planner.h) and launches the engine on it.
ooo_status engine_launch(ooo_stack *s, const std::vector<pl::Unit> &crit, const std::vector<pl::Unit> &defer,
                         void *Y, void *dX, const void *X, bool in_order, int fwd_gate, int rec_kind, double flops) {
  const Plan &p = s->p;
  if (p.skinny) return skinny_launch(s, crit, defer, Y, dX, X, in_order, fwd_gate, rec_kind, flops);
  pl::Problem pb;
  pb.L = p.L;
  pb.rows = (p.cl.MT + p.cg - 1) / p.cg;
  pb.workers = std::max(1, s->engine_ctas / p.cg);
  pb.in_order = in_order;
  pb.fwd_gate = fwd_gate;
  pb.bucket.resize(p.L);
  for (int i = 1; i <= p.L; ++i) pb.bucket[i - 1] = p.layer[i - 1].bucket;
  pb.crit = crit;
  pb.defer = defer;
  const std::vector<pl::Unit> order = pl::schedule(pb, plan_model(), ooo::eng::kMaxOps, &s->pred_dw);
  if (order.empty()) return fail(OOO_ERR_UNSUPPORTED, "engine queue does not fit the op table (%d ops)", ooo::eng::kMaxOps);
  ooo::eng::Params P = {};
  P.M = p.M;
  P.R = p.R;
  P.alpha = grad_alpha(s);
  P.in_order = in_order ? 1 : 0;
  P.fwd_gate = fwd_gate;
  P.dbg = env_int("OOO_DBG", 0);
  P.copy_nt = (s->dims[0] + copy_bn(s->dims[0]) - 1) / copy_bn(s->dims[0]);
  P.a_rows = a_box_rows(p);
  P.timeout_ns = (uint64_t)s->timeout_ms * 1000000ull;
  // skinny stacks (the tokens fill at most two tile rows: C4, C5): every chain
  // op streams its W_i from HBM; prefetch the weights a few layers ahead into
  // L2 (OOO_PF_DIST overrides; 0 = off)
  P.pf_dist = env_int("OOO_PF_DIST", pb.rows <= 2 ? 4 : 0);
  P.maps_per_layer = MS_COUNT;
  P.sk_nc = p.sk_nc;
  P.skpart = p.off_skpart ? reinterpret_cast<float *>(s->ws + p.off_skpart) : nullptr;
  P.maps = s->dmaps;
  P.ctr = s->ctr;
  P.layers = s->dlayers;
  P.y_out = Y;
  P.dx_out = dX;
  P.x_in = X;
  P.cl = p.cl;
  int first = 0;
  for (size_t j = 0; j < order.size(); ++j) {
    P.ops[j] = op_of_unit(s, order[j]);
    P.ops[j].first = first;
    first += order[j].mt * order[j].nt * std::max(1, order[j].ks);
  }
  P.nops = (int)order.size();
  P.ntasks = first;
#ifdef OOO_TRACE
  s->last_queue.assign(P.ops, P.ops + P.nops);
#endif
  CUtensorMap tmY, tmDX, tmX;
  // F_1's A operand: the caller's X (no X -> X_1 copy on the chain); a
  // launch without X (region profiling) reads the X_1 store instead
  OOO_TRY(make_map(&tmX, X ? X : s->lr[0].X, s->dims[0], p.M, 64, a_box_rows(p)));
  if (Y) OOO_TRY(make_map(&tmY, Y, p.layer[p.L - 1].dout, p.M, 32, 32, 64));
  else memset(&tmY, 0, sizeof(tmY));    // unused placeholder
  if (dX) OOO_TRY(make_map(&tmDX, dX, s->dims[0], p.M, 32, 32, 64));
  else memset(&tmDX, 0, sizeof(tmDX));
  TimedRec *tr;
  OOO_TRY(begin_rec(s, s->hi, rec_kind, 0, 0, &tr));
  CU_TRY(ooo::eng::launch_engine(p.cg, P, &tmY, &tmDX, &tmX, s->engine_ctas, s->hi, s->prio_hi));
  return end_rec(tr, s->hi, s->engine_ctas, flops, 0);
}

// The deferred backward's S[dW] per bucket on the comm stream, enqueued
// right AFTER the engine kernel whose counters it waits on: an eager
// cuStreamWaitValue32 followed by a kernel on the comm stream, submitted
// before the engine kernel that satisfies the wait, hangs the device (the
// stream-ordered graph capture has no such hazard, but one order serves both).
ooo_status engine_comm(ooo_stack *s) {
  if (!s->eng_comm) return OOO_OK;
  s->eng_comm = false;
  const Plan &p = s->p;
  const int L = p.L;
  CU_TRY(cudaStreamWaitEvent(s->comm, s->ev_reset, 0));   // value-waits observe the reset counters
  // S[dW] per bucket in D's dW order: the comm stream waits for the bucket's
  // dW tiles (engine counter), all-reduces, and publishes ar_done for F_i.
  static StreamValueFn wait_fn = stream_value_fn("cuStreamWaitValue32");
  static StreamValueFn write_fn = stream_value_fn("cuStreamWriteValue32");
  if (!wait_fn || !write_fn) return fail(OOO_ERR_CUDA, "stream memory operations unavailable");
  const int nb = p.nbuckets;
  std::vector<int> left(nb), tiles(nb, 0), rank(nb, 0), nch(nb);
  for (int b = 0; b < nb; ++b) {
    left[b] = p.bucket_last[b] - p.bucket_first[b] + 1;
    nch[b] = (int)p.chunk_start[b].size() - 1;
  }
  for (int i = 1; i <= L; ++i) {
    const LayerPlan &lp = p.layer[i - 1];
    tiles[lp.bucket] += ((lp.din + 127) / 128) * ((lp.dout + lp.ebn_dw - 1) / lp.ebn_dw);
  }
  int pos = 0;   // FIFO = the order in which D completes each bucket's dW ops
  for (int op : s->D)
    if (op < 0 && --left[p.layer[-op - 1].bucket] == 0) rank[p.layer[-op - 1].bucket] = pos++;
  // chunk issue order (§5.1, ooo_comm_schedule): FIFO, or prioritised
  // from the planner's predicted bucket ready times and a ring-time model
  std::vector<double> ready(nb, 0.0), dur;
  std::vector<int32_t> prio(nb);
  const bool emu = s->emu_n > 1;
  const double n = emu ? s->emu_n : s->d.world_size;
  const double gbps = emu ? s->emu_gbps : (s->d.comm_model_gbps > 0 ? s->d.comm_model_gbps : 700.0);
  const double lat = emu ? s->emu_lat_us : 8.0;
  for (int b = 0; b < nb; ++b) {
    prio[b] = p.bucket_first[b];
    for (int i = p.bucket_first[b]; i <= p.bucket_last[b]; ++i)
      if (i - 1 < (int)s->pred_dw.size()) ready[b] = std::max(ready[b], s->pred_dw[i - 1]);
    for (int c = 0; c < nch[b]; ++c) {
      const double bytes = (double)(p.chunk_start[b][c + 1] - p.chunk_start[b][c]) * p.elt;
      dur.push_back(lat + 2.0 * (n - 1) / n * bytes / (gbps * 1e3));   // us
    }
  }
  const int total = (int)dur.size();
  std::vector<int32_t> ob(total), oc(total);
  OOO_TRY(ooo_comm_schedule(nb, ready.data(), nch.data(), dur.data(), prio.data(), rank.data(),
                            s->d.comm_priority ? 1 : 0, ob.data(), oc.data(), nullptr));
  // per chunk: the bucket's dW counter (before its first chunk), the
  // all-reduce, and after its last chunk the flag F_i waits on
  std::vector<int> todo = nch;
  std::vector<char> waited(nb, 0);
  for (int j = 0; j < total; ++j) {
    const int b = ob[j];
    if (!waited[b]) {
      CUresult r = wait_fn(s->comm, reinterpret_cast<CUdeviceptr>(s->ctr + p.cl.bucket_done + b),
                           (cuuint32_t)tiles[b], CU_STREAM_WAIT_VALUE_GEQ);
      if (r != CUDA_SUCCESS) return fail(OOO_ERR_CUDA, "cuStreamWaitValue32 failed (%d)", (int)r);
      waited[b] = 1;
    }
    OOO_TRY(launch_allreduce(s, b, oc[j]));
    if (--todo[b] == 0 && b != s->test_drop_flag) {
      CUresult r = write_fn(s->comm, reinterpret_cast<CUdeviceptr>(s->ctr + p.cl.ar_done + b), 1, 0);
      if (r != CUDA_SUCCESS) return fail(OOO_ERR_CUDA, "cuStreamWriteValue32 failed (%d)", (int)r);
    }
  }
  s->comm_b.assign(ob.begin(), ob.end());
  s->comm_c.assign(oc.begin(), oc.end());
  return OOO_OK;
}

// A backward whose kernel is still deferred (engine): run it alone.
ooo_status engine_flush(ooo_stack *s) {
  if (!s->eng_pending) return OOO_OK;
  s->eng_pending = false;
  std::vector<pl::Unit> defer = s->eng_defer;
  for (pl::Unit &u : defer)
    if (u.release <= -2) u.release = (int)s->eng_crit.size();   // its forward region: after the chain
  OOO_TRY(engine_launch(s, s->eng_crit, defer, nullptr, s->eng_dX, nullptr, s->eng_in_order, 0, 8,
                        s->eng_flops));
  return engine_comm(s);
}

ooo_status engine_forward(ooo_stack *s, const void *X, void *Y, cudaStream_t st) {
  const Plan &p = s->p;
  const int L = p.L;
  OOO_TRY(fork_from(s, st));
  double flops = 0;
  for (int i = 1; i <= L; ++i) flops += 2.0 * p.M * p.layer[i - 1].din * p.layer[i - 1].dout;
  // the next forward: F_1..F_L (critical chain; F_1 reads the caller's X),
  // then the copy X -> X_1 that the next backward's dW_1 reads (off the
  // chain: it only waits for the pending dW_1, which still reads X_1)
  std::vector<pl::Unit> fwd;
  for (int i = 1; i <= L; ++i) fwd.push_back(unit_of(s, pl::FWD, i));
  if (!(env_int("OOO_DBG", 0) & 8)) fwd.push_back(unit_of(s, pl::COPY, 1));   // bit 3: timing experiments only
  if (s->eng_pending && env_int("OOO_FUSE", 1) == 0) OOO_TRY(engine_flush(s));   // experiments: unfused
  if (s->eng_pending) {
    if (s->emu_n > 1 || (s->nccl && s->d.comm_enabled)) {
      cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
      CU_TRY(cudaStreamIsCapturing(st, &cs));
      if (cs != cudaStreamCaptureStatusActive)
        return fail(OOO_ERR_UNSUPPORTED, "communicating stack: run the fused step (ooo_backward; ooo_forward) "
                                         "through ooo_graph_create, or ooo_join before ooo_forward (an eager "
                                         "fused step with kernels on the comm stream stalls, see ooo.h)");
    }
    // backward(t) + forward(t+1) in one launch (Fig. 4(c)); counters were
    // reset by ooo_backward.  F_i is gated on dW_i (N = 1) or on its bucket's
    // all-reduce (N > 1) and on dW_{i+1} (it reads X_{i+1}).
    s->eng_pending = false;
    const bool ar = comm_active(s);
    std::vector<pl::Unit> crit = s->eng_crit;
    crit.insert(crit.end(), fwd.begin(), fwd.end());
    std::vector<pl::Unit> defer = s->eng_defer;
    const int f1 = (int)(s->eng_crit.size());   // index of F_1 in the chain
    for (pl::Unit &u : defer)
      if (u.release <= -2) u.release = f1 + (-u.release - 1) - 1;   // region starting at F_m
    OOO_TRY(engine_launch(s, crit, defer, Y, s->eng_dX, X, s->eng_in_order, ar ? 2 : 1, 9,
                          s->eng_flops + flops));
    OOO_TRY(engine_comm(s));
  } else {
    CU_TRY(cudaMemsetAsync(s->ctr, 0, (size_t)p.cl.fwd_end * 4, s->hi));
    OOO_TRY(engine_launch(s, fwd, {}, Y, nullptr, X, false, 0, 7, flops));
  }
  s->bwd_pending = false;
  s->have_fwd = true;
  return join_into(s, st);
}

// Enqueues the counter reset, the seed and the comm stream's all-reduces; the
// engine kernel itself is deferred to the next ooo_forward (fused step) or
// ooo_join (backward alone).
ooo_status engine_backward(ooo_stack *s, const void *dY, bool in_order, bool regions, void *dX,
                           cudaStream_t st) {
  const Plan &p = s->p;
  const int L = p.L;
  OOO_TRY(fork_from(s, st));
  CU_TRY(cudaMemsetAsync(s->ctr, 0, (size_t)p.cl.total * 4, s->hi));
  const bool comm = comm_active(s);
  if (comm) CU_TRY(cudaEventRecord(s->ev_reset, s->hi));   // the comm stream's value-waits start after it
  OOO_TRY(launch_seed_op(s, dY, s->hi, s->prio_hi));
  s->eng_crit.clear();
  s->eng_defer.clear();
  s->eng_flops = 0;
  engine_bwd_units(s, in_order, regions, s->eng_crit, s->eng_defer, s->eng_flops);
  s->eng_dX = dX;
  s->eng_in_order = in_order;
  s->eng_pending = true;
  s->eng_comm = comm;   // enqueued right after the engine launch (engine_comm)
  s->have_fwd = false;
  s->bwd_pending = true;
  return OOO_OK;
}

ooo_status enqueue_forward(ooo_stack *s, const void *X, void *Y, cudaStream_t st) {
  if (s->p.engine) return engine_forward(s, X, Y, st);
  const int L = s->p.L;
  OOO_TRY(fork_from(s, st));
  const bool pend = s->bwd_pending;
  if (pend) CU_TRY(cudaStreamWaitEvent(s->hi, s->ev_pack[1], 0));   // dW_1(t) still reads X_1
  {
    TimedRec *tr;
    OOO_TRY(begin_rec(s, s->hi, 6, 1, 0, &tr));
    const size_t bytes = (size_t)s->p.M * s->dims[0] * s->p.elt;
    CU_TRY(cudaMemcpyAsync(s->lr[0].X, X, bytes, cudaMemcpyDeviceToDevice, s->hi));
    OOO_TRY(end_rec(tr, s->hi, 0, 0, 2.0 * bytes));
  }
  for (int i = 1; i <= L; ++i) {
    if (pend) {
      // T(F_i) >= T(S[dW_i]) + S[dW_i]
      CU_TRY(cudaStreamWaitEvent(s->hi, s->ev_ar[s->p.layer[i - 1].bucket], 0));
      // WAR guard of the static buffers: dW_{i+1}(t) reads X_{i+1}, which F_i overwrites
      if (i < L) CU_TRY(cudaStreamWaitEvent(s->hi, s->ev_pack[i + 1], 0));
    }
    OOO_TRY(launch_fwd(s, i, Y, s->hi, s->prio_hi));
  }
  s->bwd_pending = false;
  s->have_fwd = true;
  return join_into(s, st);
}

ooo_status enqueue_backward(ooo_stack *s, const void *dY, ooo_schedule sch, void *dX, cudaStream_t st) {
  const int L = s->p.L;
  int k = sch.k;
  if (sch.kind == OOO_SCHED_FIRST_K) {
    int mk = ooo_max_k(L, 0, nullptr, nullptr, 0);
    if (s->d.max_temp_bytes > 0) {
      std::vector<int64_t> mdo(L), mdw(L);
      int64_t mf = (int64_t)s->p.M * s->dims[0] * s->p.elt;
      for (int i = 1; i <= L; ++i) {
        const LayerPlan &lp = s->p.layer[i - 1];
        const int64_t act_bytes = (int64_t)s->p.M * lp.din * s->p.elt +
                                  (lp.act != OOO_ACT_IDENTITY ? (int64_t)s->p.M * lp.dout * s->p.elt : 0);
        mdo[i - 1] = act_bytes;
        mdw[i - 1] = (int64_t)s->p.M * lp.dout * s->p.elt;
        mf += (lp.act != OOO_ACT_IDENTITY ? (int64_t)s->p.M * lp.dout * s->p.elt : 0) +
              (i < L ? (int64_t)s->p.M * lp.dout * s->p.elt : 0);
      }
      mk = ooo_max_k(L, mf, mdo.data(), mdw.data(), s->d.max_temp_bytes);
    }
    k = std::min(k, mk);
  }
  if (sch.kind == OOO_SCHED_REGIONS) {
    if (!s->has_regions) return fail(OOO_ERR_STATE, "OOO_SCHED_REGIONS needs ooo_plan_regions first");
    s->D = s->reg_D;
  } else {
    schedule_ops(L, sch.kind, k, s->d.need_input_grad != 0, s->D);
  }
  if (s->timing) s->rec_cursor = 0;
  if (s->p.engine)
    return engine_backward(s, dY, sch.kind == OOO_SCHED_IN_ORDER, sch.kind == OOO_SCHED_REGIONS, dX, st);
  OOO_TRY(fork_from(s, st));
  const bool single = sch.kind == OOO_SCHED_IN_ORDER;
  cudaStream_t wst = single ? s->hi : s->lo;
  const int wprio = single ? s->prio_hi : s->prio_lo;
  const int wsid = single ? 0 : 1;
  // seed dO_{L+1} at time 0
  OOO_TRY(launch_seed_op(s, dY, s->hi, s->prio_hi));
  CU_TRY(cudaEventRecord(s->ev_dz[L], s->hi));
  std::vector<int> left(s->p.nbuckets);
  for (int b = 0; b < s->p.nbuckets; ++b) left[b] = s->p.bucket_last[b] - s->p.bucket_first[b] + 1;
  for (int op : s->D) {
    if (op > 0) {
      const int i = op;
      OOO_TRY(launch_dx(s, i, dX, s->hi, s->prio_hi));
      if (i >= 2) CU_TRY(cudaEventRecord(s->ev_dz[i - 1], s->hi));
    } else {
      const int i = -op;
      if (!single) CU_TRY(cudaStreamWaitEvent(s->lo, s->ev_dz[i], 0));
      OOO_TRY(launch_dw_pack(s, i, wst, wprio, wsid));
      CU_TRY(cudaEventRecord(s->ev_pack[i], wst));
      const int b = s->p.layer[i - 1].bucket;
      if (--left[b] == 0) {
        // S[dW] for the bucket, issued in D's dW order on every rank (FIFO comm stream)
        CU_TRY(cudaStreamWaitEvent(s->comm, s->ev_pack[i], 0));
        OOO_TRY(launch_allreduce(s, b));
        CU_TRY(cudaEventRecord(s->ev_ar[b], s->comm));
      }
    }
  }
  s->have_fwd = false;
  s->bwd_pending = true;
  return OOO_OK;
}


// ---- region planning (OOO_SCHED_REGIONS, §4.1) ---------------
int fwd_nt_of(const Plan &p, int i) { return (p.layer[i - 1].dout + p.layer[i - 1].ebn_fwd - 1) / p.layer[i - 1].ebn_fwd; }
int dx_nt_of(const Plan &p, int i) { return (p.layer[i - 1].din + p.layer[i - 1].ebn_dx - 1) / p.layer[i - 1].ebn_dx; }
int dw_tiles_of(const Plan &p, int i) {
  const LayerPlan &lp = p.layer[i - 1];
  return ((lp.din + 127) / 128) * ((lp.dout + lp.ebn_dw - 1) / lp.ebn_dw);
}

// One profiling launch of the engine on the given ops alone: the completion
// counters of every op NOT in the launch are preset to "complete", so the
// launched ops wait only for each other (step 1 of §4.1).  Minimum
// device time over `reps` timed launches after one warm-up (ms).
ooo_status profile_launch(ooo_stack *s, const std::vector<pl::Unit> &crit, const std::vector<pl::Unit> &defer,
                          int reps, double *ms) {
  const Plan &p = s->p;
  const ooo::eng::CounterLayout &cl = p.cl;
  auto in = [&](int kind, int i) {
    for (const pl::Unit &u : crit)
      if (u.kind == kind && u.layer == i) return true;
    for (const pl::Unit &u : defer)
      if (u.kind == kind && u.layer == i) return true;
    return false;
  };
  std::vector<int32_t> img(cl.total, 0);
  const int pub = p.skinny ? ooo::sk::kPubPerTile : 1;   // publications per chain tile
  for (int i = 1; i <= p.L; ++i) {
    if (!in(pl::FWD, i))
      for (int m = 0; m < cl.MT; ++m) img[cl.fwd_rows + (i - 1) * cl.MT + m] = fwd_nt_of(p, i) * pub;
    if (i >= 2 && !in(pl::DGRAD, i)) {
      for (int m = 0; m < cl.MT; ++m) img[cl.dz_rows + (i - 2) * cl.MT + m] = dx_nt_of(p, i) * pub;
      img[cl.dz_total + i - 2] = cl.MT * dx_nt_of(p, i) * pub;
    }
    if (!in(pl::WGRAD, i)) img[cl.dw_done + i - 1] = dw_tiles_of(p, i);
  }
  const int copy_nt = (s->dims[0] + copy_bn(s->dims[0]) - 1) / copy_bn(s->dims[0]);
  for (int m = 0; m < cl.MT; ++m) img[cl.xcopy + m] = copy_nt;
  void *Y = s->lr[p.L - 1].dZ;                                  // scratch M x d_L target for F_L
  void *dX = s->d.need_input_grad ? s->lr[0].X : nullptr;      // scratch M x d_0 target for dO_1
  cudaEvent_t e0, e1;
  CU_TRY(cudaEventCreate(&e0));
  CU_TRY(cudaEventCreate(&e1));
  double best = 1e30;
  ooo_status st = OOO_OK;
  for (int r = 0; r <= reps && st == OOO_OK; ++r) {
    cudaError_t ce = cudaMemcpyAsync(s->ctr, img.data(), img.size() * 4, cudaMemcpyHostToDevice, s->hi);
    if (ce == cudaSuccess) ce = cudaEventRecord(e0, s->hi);
    if (ce != cudaSuccess) {
      st = fail(OOO_ERR_CUDA, "profile launch: %s", cudaGetErrorString(ce));
      break;
    }
    st = engine_launch(s, crit, defer, Y, dX, nullptr, false, 0, 10, 0.0);
    if (st != OOO_OK) break;
    ce = cudaEventRecord(e1, s->hi);
    if (ce == cudaSuccess) ce = cudaEventSynchronize(e1);
    float t = 0.f;
    if (ce == cudaSuccess) ce = cudaEventElapsedTime(&t, e0, e1);
    if (ce != cudaSuccess) st = fail(OOO_ERR_CUDA, "profile launch: %s", cudaGetErrorString(ce));
    else if (r > 0) best = std::min(best, (double)t);
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  *ms = best;
  return st;
}

ooo_status plan_regions(ooo_stack *s, int rl, int reps) {
  const Plan &p = s->p;
  const int L = p.L;
  const bool need_dx = s->d.need_input_grad != 0;
  // step 2: main-stream regions (backward dO blocks from the top, then forward F blocks)
  struct Region { std::vector<pl::Unit> ops; std::vector<double> flops; std::vector<int> layers; bool fwd; };
  std::vector<Region> R;
  for (int hi = L; hi >= 1; hi -= rl) {
    Region g;
    g.fwd = false;
    for (int i = hi; i > std::max(0, hi - rl); --i) {
      if (i == 1 && !need_dx) continue;
      g.ops.push_back(unit_of(s, pl::DGRAD, i));
      g.flops.push_back(2.0 * p.M * p.layer[i - 1].din * p.layer[i - 1].dout);
      g.layers.push_back(i);
    }
    if (!g.ops.empty()) R.push_back(g);
  }
  const int nb = (int)R.size();
  std::vector<int> fwd_region(L + 1, 0);
  for (int lo = 1; lo <= L; lo += rl) {
    Region g;
    g.fwd = true;
    for (int i = lo; i <= std::min(L, lo + rl - 1); ++i) {
      g.ops.push_back(unit_of(s, pl::FWD, i));
      g.flops.push_back(2.0 * p.M * p.layer[i - 1].din * p.layer[i - 1].dout);
      g.layers.push_back(i);
      fwd_region[i] = (int)R.size();
    }
    R.push_back(g);
  }
  const int N = (int)R.size();
  // step 1: profile -- regions alone, candidates alone, co-runs
  std::vector<double> t_main(N), start(N);
  for (int r = 0; r < N; ++r) OOO_TRY(profile_launch(s, R[r].ops, {}, reps, &t_main[r]));
  double acc = 0;
  for (int r = 0; r < N; ++r) {
    start[r] = acc;
    acc += t_main[r];
  }
  // candidates dW_2..dW_L (c = L - i: the paper's U in descending layer order)
  const int K = L - 1;
  std::vector<double> ready(K), t_alone(K), t_sub((size_t)K * N), sp((size_t)K * N, 0.0);
  std::vector<int32_t> last(K);
  std::vector<int64_t> nbytes(K);
  for (int c = 0; c < K; ++c) {
    const int i = L - c;
    // runnable once dO_{i+1} is done: its completion inside its region, by FLOPs
    ready[c] = 0.0;
    if (i < L) {
      for (int r = 0; r < nb; ++r) {
        double f = 0, tot = 0;
        bool here = false;
        for (size_t j = 0; j < R[r].layers.size(); ++j) {
          tot += R[r].flops[j];
          if (!here) f += R[r].flops[j];
          if (R[r].layers[j] == i + 1) here = true;
        }
        if (here) ready[c] = start[r] + t_main[r] * (tot > 0 ? f / tot : 1.0);
      }
    }
    last[c] = std::max(0, fwd_region[i - 1] - 1);   // before F_{i-1} (WAR on X_i) and F_i
    nbytes[c] = (int64_t)p.M * p.layer[i - 1].dout * p.elt;   // dZ_i kept alive (§3)
    OOO_TRY(profile_launch(s, {}, {unit_of(s, pl::WGRAD, i)}, reps, &t_alone[c]));
  }
  for (int c = 0; c < K; ++c) {
    const int i = L - c;
    for (int r = 0; r < N; ++r) {
      t_sub[(size_t)c * N + r] = t_alone[c];   // reading A6: T_sub(k, R) = k's profiled time
      if (start[r] + t_main[r] <= ready[c] || r > last[c]) continue;   // never runnable there
      double tc = 0;
      OOO_TRY(profile_launch(s, R[r].ops, {unit_of(s, pl::WGRAD, i)}, reps, &tc));
      sp[(size_t)c * N + r] = (t_main[r] + t_alone[c]) / tc;
    }
  }
  // steps 3-5: Algorithm 1 (+ P:162 memory bound)
  std::vector<int32_t> region_of(std::max(K, 1)), order(std::max(K, 1));
  int32_t kpre = 0;
  OOO_TRY(ooo_region_schedule(N, t_main.data(), K, t_sub.data(), sp.data(), ready.data(), last.data(),
                              nbytes.data(), s->d.max_temp_bytes, region_of.data(), order.data(), &kpre));
  // the plan: D = per backward region its dO ops then its dW ops, then dW_1
  // and the forward regions' dW ops; release tags for the engine queue
  std::vector<std::vector<int>> S(N);
  for (int j = 0; j < K; ++j) S[region_of[order[j]]].push_back(L - order[j]);
  s->reg_D.clear();
  s->reg_release.assign(L, -1);
  s->reg_region_of.assign(L, nb);
  int ci = 0;   // backward chain index
  for (int r = 0; r < nb; ++r) {
    const int first = ci;
    for (int i : R[r].layers) {
      s->reg_D.push_back(+i);
      ++ci;
    }
    for (int i : S[r]) {
      s->reg_D.push_back(-i);
      s->reg_release[i - 1] = first;
      s->reg_region_of[i - 1] = r;
    }
  }
  s->reg_D.push_back(-1);                    // dW_1 gates F_1: as soon as ready (reading A4)
  s->reg_release[0] = ci;                    // after the last dO (the chain end if no forward follows)
  for (int r = nb; r < N; ++r)
    for (int i : S[r]) {
      s->reg_D.push_back(-i);
      s->reg_release[i - 1] = -(1 + R[r].layers[0]);   // region starting at F_m
      s->reg_region_of[i - 1] = r;
    }
  s->reg_tmain = t_main;
  s->reg_kpre = kpre;
  s->has_regions = true;
  return OOO_OK;
}

}  // namespace

// ======================================================================
extern "C" {

int32_t ooo_abi_version(void) { return OOO_ABI_VERSION; }

const char *ooo_last_error(void) { return t_err.c_str(); }

const char *ooo_status_string(int32_t st) {
  switch (st) {
    case OOO_OK: return "OOO_OK";
    case OOO_ERR_INVALID_ARGUMENT: return "OOO_ERR_INVALID_ARGUMENT";
    case OOO_ERR_UNSUPPORTED: return "OOO_ERR_UNSUPPORTED";
    case OOO_ERR_CUDA: return "OOO_ERR_CUDA";
    case OOO_ERR_NCCL: return "OOO_ERR_NCCL";
    case OOO_ERR_STATE: return "OOO_ERR_STATE";
  }
  return "unknown";
}

ooo_status ooo_query_sizes(const ooo_stack_desc *d, size_t *workspace_bytes, size_t *grads_bytes) {
  OOO_TRY(validate_desc(d, false));
  if (!workspace_bytes || !grads_bytes) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  Plan p = make_plan(d);
  *workspace_bytes = p.workspace_bytes;
  *grads_bytes = align_up((size_t)p.grad_elems * p.elt, 256);
  return OOO_OK;
}

ooo_status ooo_grad_offsets(const ooo_stack_desc *d, int64_t *offsets) {
  OOO_TRY(validate_desc(d, false));
  if (!offsets) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  Plan p = make_plan(d);
  for (int i = 0; i < p.L; ++i) {
    offsets[2 * i] = p.layer[i].goff_w;
    offsets[2 * i + 1] = p.layer[i].goff_b;
  }
  return OOO_OK;
}

ooo_status ooo_schedule_order(int32_t L, ooo_schedule sch, int32_t need_input_grad, int32_t *ops,
                              int32_t *n) {
  if (L < 1) return fail(OOO_ERR_INVALID_ARGUMENT, "L must be >= 1");
  if (sch.kind != OOO_SCHED_IN_ORDER && sch.kind != OOO_SCHED_FIRST_K)
    return fail(OOO_ERR_INVALID_ARGUMENT, "schedule kind %d invalid", sch.kind);
  if (sch.k < 0) return fail(OOO_ERR_INVALID_ARGUMENT, "k must be >= 0");
  if (!ops || !n) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  std::vector<int> D;
  schedule_ops(L, sch.kind, sch.k, need_input_grad != 0, D);
  for (size_t j = 0; j < D.size(); ++j) ops[j] = D[j];
  *n = (int32_t)D.size();
  return OOO_OK;
}

int32_t ooo_max_k(int32_t L, int64_t m_fwd, const int64_t *m_dO, const int64_t *m_dW, int64_t mxm) {
  if (mxm <= 0 || !m_dO || !m_dW) return L;
  // f(j) = m_fwd - sum_{i=j+1..L} m_dO[i] + sum_{i=1..j} m_dW[i]   (Alg. 2 l.1, reading Q3)
  int best = 0;
  for (int j = 0; j <= L; ++j) {
    int64_t f = m_fwd;
    for (int i = j + 1; i <= L; ++i) f -= m_dO[i - 1];
    for (int i = 1; i <= j; ++i) f += m_dW[i - 1];
    if (f < mxm) best = j;
  }
  return best;
}

int64_t ooo_deferral_bytes(const ooo_stack_desc *d, int32_t k) {
  if (validate_desc(d, false) != OOO_OK) return -1;
  int64_t s = 0;
  const int elt = d->dtype == OOO_BF16 ? 2 : 4;
  for (int i = 2; i <= std::min<int>(k, d->num_layers); ++i) s += (int64_t)d->tokens * d->dims[i] * elt;
  return s;
}

ooo_status ooo_engine_plan(const ooo_stack_desc *d, ooo_schedule sch, int32_t fused, int32_t workers,
                           int32_t *out, int32_t cap, int32_t *n, int32_t *topological) {
  OOO_TRY(validate_desc(d, false));
  if (!n || !topological || (cap > 0 && !out)) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  if (sch.kind != OOO_SCHED_IN_ORDER && sch.kind != OOO_SCHED_FIRST_K)
    return fail(OOO_ERR_INVALID_ARGUMENT, "schedule kind %d invalid", sch.kind);
  if (sch.k < 0) return fail(OOO_ERR_INVALID_ARGUMENT, "k must be >= 0");
  ooo_stack tmp;
  tmp.d = *d;
  tmp.dims.assign(d->dims, d->dims + d->num_layers + 1);
  tmp.p = make_plan(d);
  if (!tmp.p.engine) return fail(OOO_ERR_UNSUPPORTED, "no engine for this stack (fp32 or OOO_ENGINE=0)");
  const bool in_order = sch.kind == OOO_SCHED_IN_ORDER;
  schedule_ops(tmp.p.L, sch.kind, sch.k, d->need_input_grad != 0, tmp.D);
  std::vector<pl::Unit> crit, defer;
  double flops = 0;
  engine_bwd_units(&tmp, in_order, false, crit, defer, flops);
  if (fused) {
    for (int i = 1; i <= tmp.p.L; ++i) crit.push_back(unit_of(&tmp, pl::FWD, i));
    crit.push_back(unit_of(&tmp, pl::COPY, 1));
  }
  pl::Problem pb;
  pb.L = tmp.p.L;
  pb.rows = (tmp.p.cl.MT + tmp.p.cg - 1) / tmp.p.cg;
  pb.workers = workers > 0 ? workers : std::max(1, kSMs / tmp.p.cg);
  pb.in_order = in_order;
  pb.fwd_gate = fused ? ((d->world_size > 1 || d->nccl_unique_id) && d->comm_enabled ? 2 : 1) : 0;
  pb.bucket.resize(pb.L);
  for (int i = 1; i <= pb.L; ++i) pb.bucket[i - 1] = tmp.p.layer[i - 1].bucket;
  pb.crit = crit;
  pb.defer = defer;
  const std::vector<pl::Unit> order = pl::schedule(pb, plan_model(), ooo::eng::kMaxOps);
  if (order.empty()) return fail(OOO_ERR_UNSUPPORTED, "queue does not fit the op table");
  for (size_t j = 0; j < order.size() && (int32_t)j < cap; ++j) {
    const pl::Unit &u = order[j];
    int32_t *o = out + 5 * j;
    o[0] = u.kind; o[1] = u.layer; o[2] = u.m_off; o[3] = u.mt; o[4] = u.nt;
  }
  *n = (int32_t)order.size();
  *topological = pl::topological(pb, order) ? 1 : 0;
  return OOO_OK;
}

ooo_status ooo_get_unique_id(void *out) {
  if (!out) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  const char *why = nullptr;
  const NcclApi *api = nccl_api(&why);
  if (!api) return fail(OOO_ERR_NCCL, "NCCL unavailable: %s", why);
  ncclUniqueId id;
  ncclResult_t r = api->GetUniqueId(&id);
  if (r != ncclSuccess) return fail(OOO_ERR_NCCL, "ncclGetUniqueId: %s", api->GetErrorString(r));
  memcpy(out, &id, sizeof(id) < OOO_UNIQUE_ID_BYTES ? sizeof(id) : OOO_UNIQUE_ID_BYTES);
  return OOO_OK;
}

ooo_status ooo_create_stack(const ooo_stack_desc *d, ooo_stack **out) {
  if (!out) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL output");
  *out = nullptr;
  OOO_TRY(validate_desc(d, true));
  ooo_stack *s = new ooo_stack();
  s->d = *d;
  s->dims.assign(d->dims, d->dims + d->num_layers + 1);
  s->acts.assign(d->acts, d->acts + d->num_layers);
  s->d.dims = s->dims.data();
  s->d.acts = s->acts.data();
  s->p = make_plan(d);
  s->pdl = env_int("OOO_PDL", 1) != 0;
  s->comm_stack = d->world_size > 1 || d->nccl_unique_id != nullptr;
  s->timeout_ms = d->wait_timeout_ms > 0 ? d->wait_timeout_ms : (s->comm_stack ? 120000 : 4000);
  s->test_comm_gate = d->world_size == 1 && s->p.engine && env_int("OOO_TEST_COMM_GATE", 0) != 0;
  if (s->test_comm_gate) s->test_drop_flag = env_int("OOO_TEST_DROP_AR_FLAG", -1);
  s->ws = static_cast<uint8_t *>(d->workspace);
  s->grads = static_cast<uint8_t *>(d->grads);
  const Plan &p = s->p;
  auto cleanup_fail = [&](ooo_status st) {
    std::string msg = t_err;
    ooo_destroy(s);
    t_err = msg;
    return st;
  };
  s->lr.resize(p.L);
  for (int i = 1; i <= p.L; ++i) {
    const LayerPlan &lp = p.layer[i - 1];
    LayerRt &r = s->lr[i - 1];
    r.W = const_cast<void *>(d->W[i - 1]);
    r.b = const_cast<void *>(d->b[i - 1]);
    r.X = s->ws + lp.off_X;
    r.Z = lp.off_Z != SIZE_MAX ? s->ws + lp.off_Z : nullptr;
    r.Xn = lp.off_Xn != SIZE_MAX ? s->ws + lp.off_Xn : nullptr;
    r.dZ = s->ws + lp.off_dZ;
    r.db = reinterpret_cast<float *>(s->ws + lp.off_db);
    r.gw = s->grads + lp.goff_w * p.elt;
    r.gb = s->grads + lp.goff_b * p.elt;
  }
  if (p.engine) {
    static std::once_flag eng_once;
    static cudaError_t eng_err = cudaSuccess;
    std::call_once(eng_once, [] {
      eng_err = ooo::eng::engine_init();
      if (eng_err == cudaSuccess) eng_err = ooo::sk::skinny_init();
    });
    if (eng_err != cudaSuccess)
      return cleanup_fail(fail(OOO_ERR_CUDA, "engine init: %s", cudaGetErrorString(eng_err)));
    std::vector<CUtensorMap> maps((size_t)p.L * MS_COUNT);
    std::vector<ooo::eng::LayerDev> ldev(p.L);
    for (int i = 1; i <= p.L; ++i) {
      const LayerPlan &lp = p.layer[i - 1];
      LayerRt &r = s->lr[i - 1];
      CUtensorMap *m = &maps[(size_t)(i - 1) * MS_COUNT];
      memset(m, 0, sizeof(CUtensorMap) * MS_COUNT);
      ooo_status st;
      if ((st = make_map(&m[MS_FWD_A], r.X, lp.din, p.M, 64, a_box_rows(p))) != OOO_OK ||
          (st = make_map(&m[MS_FWD_B], r.W, lp.dout, lp.din, 64, 64)) != OOO_OK ||
          (r.Xn && (st = make_map(&m[MS_FWD_X], r.Xn, lp.dout, p.M, 32, 32, 64)) != OOO_OK) ||
          (r.Z && (st = make_map(&m[MS_FWD_Z], r.Z, lp.dout, p.M, 32, 32, 64)) != OOO_OK) ||
          (st = make_map(&m[MS_DX_A], r.dZ, lp.dout, p.M, 64, a_box_rows(p))) != OOO_OK ||
          (st = make_map(&m[MS_DX_B], r.W, lp.dout, lp.din, 64, lp.ebn_dx / p.cg)) != OOO_OK ||
          (st = make_map(&m[MS_DZ_X], r.dZ, lp.dout, p.M, 32, 32, 64)) != OOO_OK ||
          (st = make_map(&m[MS_DW_A], r.X, lp.din, p.M, 64, 64)) != OOO_OK ||
          (st = make_map(&m[MS_DW_B], r.dZ, lp.dout, p.M, 64, 64)) != OOO_OK ||
          (st = make_map(&m[MS_GW_X], r.gw, lp.dout, lp.din, 32, 32, 64)) != OOO_OK ||
          (r.Z && (st = make_map(&m[MS_Z_PF], r.Z, lp.dout, p.M, 64, 128)) != OOO_OK) ||
          (p.skinny && (st = make_map(&m[MS_SK_X], r.X, lp.din, p.M, 64, 16)) != OOO_OK) ||
          (p.skinny && (st = make_map(&m[MS_SK_DZ], r.dZ, lp.dout, p.M, 64, 16)) != OOO_OK))
        return cleanup_fail(st);
      ooo::eng::LayerDev &L = ldev[i - 1];
      memset(&L, 0, sizeof(L));
      L.bias = r.b;
      L.Z = r.Z;
      L.dbpart = r.db;
      L.db_out = r.gb;
      L.X = r.X;
      L.Xn = r.Xn;
      L.dZ = r.dZ;
      L.gw = r.gw;
      L.din = lp.din;
      L.dout = lp.dout;
      L.act = lp.act;
      L.bucket = lp.bucket;
      L.fwd_nt = (lp.dout + lp.ebn_fwd - 1) / lp.ebn_fwd;
      L.dx_nt = (lp.din + lp.ebn_dx - 1) / lp.ebn_dx;
      L.dw_tiles = ((lp.din + 127) / 128) * ((lp.dout + lp.ebn_dw - 1) / lp.ebn_dw);
      L.fwd_bn = lp.ebn_fwd;
      L.dx_bn = lp.ebn_dx;
      L.dw_bn = lp.ebn_dw;
    }
    cudaError_t ce = cudaMemcpy(s->ws + p.off_maps, maps.data(), maps.size() * sizeof(CUtensorMap),
                                cudaMemcpyHostToDevice);
    if (ce == cudaSuccess)
      ce = cudaMemcpy(s->ws + p.off_layers, ldev.data(), ldev.size() * sizeof(ooo::eng::LayerDev),
                      cudaMemcpyHostToDevice);
    if (ce == cudaSuccess)
      ce = cudaMemset(s->ws + p.off_ctr, 0, (size_t)p.cl.total * 4);
    if (ce != cudaSuccess)
      return cleanup_fail(fail(OOO_ERR_CUDA, "engine tables upload: %s", cudaGetErrorString(ce)));
    s->dmaps = reinterpret_cast<const CUtensorMap *>(s->ws + p.off_maps);
    s->dlayers = reinterpret_cast<const ooo::eng::LayerDev *>(s->ws + p.off_layers);
    s->ctr = reinterpret_cast<int32_t *>(s->ws + p.off_ctr);
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    // emulated all-reduce (measurement aid, N = 1): see ooo_stack::emu_n
    if (!s->comm_stack && env_int("OOO_EMULATE_AR_N", 0) > 1) {
      s->emu_n = env_int("OOO_EMULATE_AR_N", 0);
      if (const char *v = getenv("OOO_EMULATE_AR_GBPS")) s->emu_gbps = atof(v);
      if (const char *v = getenv("OOO_EMULATE_AR_LAT_US")) s->emu_lat_us = atof(v);
    }
    // N > 1 (or its emulation): leave SMs for the NCCL kernels the engine's counters wait on
    const int reserve = s->comm_stack || s->emu_n > 1 ? (d->nccl_max_ctas > 0 ? d->nccl_max_ctas : 16) : 0;
    s->engine_ctas = std::max(1, sms - reserve);
    s->engine_ctas = std::min(s->engine_ctas, env_int("OOO_ENGINE_CTAS", s->engine_ctas));
    if (d->engine_ctas > 0) s->engine_ctas = std::min(s->engine_ctas, d->engine_ctas);
  }
  int least = 0, greatest = 0;
  cudaError_t e = cudaDeviceGetStreamPriorityRange(&least, &greatest);
  if (e != cudaSuccess) return cleanup_fail(fail(OOO_ERR_CUDA, "priority range: %s", cudaGetErrorString(e)));
  s->prio_hi = greatest;
  s->prio_lo = least;
  if ((e = cudaStreamCreateWithPriority(&s->hi, cudaStreamNonBlocking, greatest)) != cudaSuccess ||
      (e = cudaStreamCreateWithPriority(&s->lo, cudaStreamNonBlocking, least)) != cudaSuccess ||
      (e = cudaStreamCreateWithPriority(&s->comm, cudaStreamNonBlocking, greatest)) != cudaSuccess)
    return cleanup_fail(fail(OOO_ERR_CUDA, "stream create: %s", cudaGetErrorString(e)));
  auto mk = [&](cudaEvent_t *ev) { return cudaEventCreateWithFlags(ev, cudaEventDisableTiming); };
  s->ev_dz.assign(p.L + 1, nullptr);
  s->ev_pack.assign(p.L + 2, nullptr);
  s->ev_ar.assign(p.nbuckets, nullptr);
  for (int i = 1; i <= p.L; ++i) {
    if ((e = mk(&s->ev_dz[i])) != cudaSuccess || (e = mk(&s->ev_pack[i])) != cudaSuccess)
      return cleanup_fail(fail(OOO_ERR_CUDA, "event create: %s", cudaGetErrorString(e)));
  }
  for (int b = 0; b < p.nbuckets; ++b)
    if ((e = mk(&s->ev_ar[b])) != cudaSuccess)
      return cleanup_fail(fail(OOO_ERR_CUDA, "event create: %s", cudaGetErrorString(e)));
  if ((e = mk(&s->ev_fork)) != cudaSuccess || (e = mk(&s->ev_j_hi)) != cudaSuccess ||
      (e = mk(&s->ev_j_lo)) != cudaSuccess || (e = mk(&s->ev_j_comm)) != cudaSuccess ||
      (e = mk(&s->ev_reset)) != cudaSuccess)
    return cleanup_fail(fail(OOO_ERR_CUDA, "event create: %s", cudaGetErrorString(e)));
  if (s->comm_stack) {
    const char *why = nullptr;
    s->api = nccl_api(&why);
    if (!s->api) return cleanup_fail(fail(OOO_ERR_NCCL, "NCCL unavailable: %s", why));
    ncclUniqueId id;
    memcpy(&id, d->nccl_unique_id, sizeof(id));
    ncclResult_t r;
    // engine: NCCL must fit in the SMs the persistent kernels leave free
    const int max_ctas = d->nccl_max_ctas > 0 ? d->nccl_max_ctas : (p.engine ? 16 : 0);
    if (s->api->CommInitRankConfig && max_ctas > 0) {
      ncclConfig_t cfg = NCCL_CONFIG_INITIALIZER;
      cfg.maxCTAs = max_ctas;
      r = s->api->CommInitRankConfig(&s->nccl, d->world_size, id, d->rank, &cfg);
    } else {
      r = s->api->CommInitRank(&s->nccl, d->world_size, id, d->rank);
    }
    if (r != ncclSuccess) {
      s->nccl = nullptr;
      return cleanup_fail(fail(OOO_ERR_NCCL, "ncclCommInitRank: %s", s->api->GetErrorString(r)));
    }
    // warm-up: every bucket's all-reduce once (lazy channel connection, NVLS
    // setup) so that no training step pays it under the engine's wait bound
    ooo_status st = OOO_OK;
    cudaError_t ce = cudaMemsetAsync(s->grads, 0, (size_t)p.grad_elems * p.elt, s->comm);
    if (ce != cudaSuccess) st = fail(OOO_ERR_CUDA, "warm-up memset: %s", cudaGetErrorString(ce));
    for (int b = p.nbuckets - 1; b >= 0 && st == OOO_OK && d->comm_enabled; --b) st = launch_allreduce(s, b);
    if (st == OOO_OK && (ce = cudaStreamSynchronize(s->comm)) != cudaSuccess)
      st = fail(OOO_ERR_CUDA, "warm-up all-reduce: %s", cudaGetErrorString(ce));
    if (st == OOO_OK) st = check_async(s);
    if (st != OOO_OK) return cleanup_fail(st);
  }
  *out = s;
  return OOO_OK;
}

ooo_status ooo_forward(ooo_stack *s, const void *X, void *Y, void *stream) {
  if (!s || !X || !Y) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  OOO_TRY(check_align(s, X, "X"));
  OOO_TRY(check_align(s, Y, "Y"));
  OOO_TRY(check_async(s));
  return enqueue_forward(s, X, Y, static_cast<cudaStream_t>(stream));
}

ooo_status ooo_backward(ooo_stack *s, const void *dY, ooo_schedule sch, void *dX, void *stream) {
  if (!s || !dY) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  if (sch.kind != OOO_SCHED_IN_ORDER && sch.kind != OOO_SCHED_FIRST_K && sch.kind != OOO_SCHED_REGIONS)
    return fail(OOO_ERR_INVALID_ARGUMENT, "schedule kind %d invalid", sch.kind);
  if (sch.k < 0) return fail(OOO_ERR_INVALID_ARGUMENT, "k must be >= 0");
  if (s->d.need_input_grad && !dX) return fail(OOO_ERR_INVALID_ARGUMENT, "need_input_grad set but dX NULL");
  if (!s->d.need_input_grad && dX) return fail(OOO_ERR_INVALID_ARGUMENT, "dX given but need_input_grad = 0");
  if (!s->have_fwd) return fail(OOO_ERR_STATE, "ooo_backward without a preceding ooo_forward");
  OOO_TRY(check_align(s, dY, "dY"));
  if (dX) OOO_TRY(check_align(s, dX, "dX"));
  OOO_TRY(check_async(s));
  return enqueue_backward(s, dY, sch, dX, static_cast<cudaStream_t>(stream));
}

ooo_status ooo_join(ooo_stack *s, void *stream) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  OOO_TRY(engine_flush(s));
  OOO_TRY(join_into(s, static_cast<cudaStream_t>(stream)));
  return check_async(s);
}

ooo_status ooo_input_grad_wait(ooo_stack *s, void *stream) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  if (!s->p.engine || !s->d.need_input_grad)
    return fail(OOO_ERR_UNSUPPORTED, "input-gradient wait needs a bf16 engine stack with need_input_grad");
  if (!s->bwd_pending) return fail(OOO_ERR_STATE, "no backward to wait for");
  OOO_TRY(engine_flush(s));   // the deferred backward kernel runs now (on hi)
  static StreamValueFn wait_fn = stream_value_fn("cuStreamWaitValue32");
  if (!wait_fn) return fail(OOO_ERR_CUDA, "stream memory operations unavailable");
  // every 128-row block of dO_1's output, once per column tile (engine.cu: dx_total)
  const uint32_t target = (uint32_t)(s->p.cl.MT * ((s->dims[0] + s->p.layer[0].ebn_dx - 1) / s->p.layer[0].ebn_dx) *
                                     (s->p.skinny ? ooo::sk::kPubPerTile : 1));
  CUresult r = wait_fn(static_cast<cudaStream_t>(stream), reinterpret_cast<CUdeviceptr>(s->ctr + s->p.cl.dx_total),
                       target, CU_STREAM_WAIT_VALUE_GEQ);
  if (r != CUDA_SUCCESS) return fail(OOO_ERR_CUDA, "cuStreamWaitValue32 failed (%d)", (int)r);
  return OOO_OK;
}


ooo_status ooo_comm_issue_order(const ooo_stack *s, int32_t *bucket, int32_t *chunk, int32_t cap, int32_t *n) {
  if (!s || !n) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  const int m = (int)s->comm_b.size();
  for (int j = 0; j < m && j < cap; ++j) {
    if (bucket) bucket[j] = s->comm_b[j];
    if (chunk) chunk[j] = s->comm_c[j];
  }
  *n = m;
  return OOO_OK;
}

ooo_status ooo_allreduce_buckets(ooo_stack *s, void *stream) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  if (!s->nccl) return fail(OOO_ERR_STATE, "stack has no communicator");
  OOO_TRY(check_async(s));
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  OOO_TRY(engine_flush(s));
  OOO_TRY(fork_from(s, st));
  if (s->timing) s->rec_cursor = 0;
  for (int b = s->p.nbuckets - 1; b >= 0; --b) {
    if (s->d.comm_enabled) OOO_TRY(launch_allreduce(s, b));
  }
  return join_into(s, st);
}

ooo_status ooo_graph_create(ooo_stack *s, const void *X, void *Y, const void *dY, ooo_schedule sch,
                            void *dX, ooo_graph **out) {
  if (!s || !X || !Y || !dY || !out) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  *out = nullptr;
  if (!s->have_fwd) return fail(OOO_ERR_STATE, "ooo_graph_create needs a preceding ooo_forward");
  if (sch.kind != OOO_SCHED_IN_ORDER && sch.kind != OOO_SCHED_FIRST_K && sch.kind != OOO_SCHED_REGIONS)
    return fail(OOO_ERR_INVALID_ARGUMENT, "schedule kind %d invalid", sch.kind);
  if (sch.k < 0) return fail(OOO_ERR_INVALID_ARGUMENT, "k must be >= 0");
  if (s->d.need_input_grad && !dX) return fail(OOO_ERR_INVALID_ARGUMENT, "need_input_grad set but dX NULL");
  if (!s->d.need_input_grad && dX) return fail(OOO_ERR_INVALID_ARGUMENT, "dX given but need_input_grad = 0");
  OOO_TRY(check_align(s, X, "X"));
  OOO_TRY(check_align(s, Y, "Y"));
  OOO_TRY(check_align(s, dY, "dY"));
  if (dX) OOO_TRY(check_align(s, dX, "dX"));
  cudaStream_t cap;
  CU_TRY(cudaStreamCreateWithFlags(&cap, cudaStreamNonBlocking));
  cudaError_t e = cudaStreamBeginCapture(cap, cudaStreamCaptureModeThreadLocal);
  if (e != cudaSuccess) {
    cudaStreamDestroy(cap);
    return fail(OOO_ERR_CUDA, "begin capture: %s", cudaGetErrorString(e));
  }
  ooo_status st = enqueue_backward(s, dY, sch, dX, cap);
  if (st == OOO_OK) st = enqueue_forward(s, X, Y, cap);
  cudaGraph_t g = nullptr;
  e = cudaStreamEndCapture(cap, &g);
  cudaStreamDestroy(cap);
  if (st != OOO_OK) {
    if (g) cudaGraphDestroy(g);
    return st;
  }
  if (e != cudaSuccess) return fail(OOO_ERR_CUDA, "end capture: %s", cudaGetErrorString(e));
  cudaGraphExec_t ex = nullptr;
  e = cudaGraphInstantiateWithFlags(&ex, g, cudaGraphInstantiateFlagUseNodePriority);
  if (e != cudaSuccess) {
    cudaGraphDestroy(g);
    return fail(OOO_ERR_CUDA, "graph instantiate: %s", cudaGetErrorString(e));
  }
  ooo_graph *gr = new ooo_graph();
  gr->s = s;
  gr->graph = g;
  gr->exec = ex;
  gr->dX = const_cast<void *>(X);
  gr->dY = const_cast<void *>(dY);
  gr->dYout = Y;
  gr->x_bytes = (size_t)s->p.M * s->dims[0] * s->p.elt;
  gr->dy_bytes = gr->y_bytes = (size_t)s->p.M * s->dims[s->p.L] * s->p.elt;
  if (s->timing && s->rec_cursor > 0) {
    for (size_t j = 0; j < s->rec_cursor; ++j) gr->tinfo.push_back(s->recs[j].info);
    size_t nn = 0;
    if (cudaGraphGetNodes(g, nullptr, &nn) == cudaSuccess && nn > 0) {
      std::vector<cudaGraphNode_t> nodes(nn);
      if (cudaGraphGetNodes(g, nodes.data(), &nn) == cudaSuccess) {
        for (cudaGraphNode_t n : nodes) {
          cudaGraphNodeType ty;
          cudaEvent_t ev = nullptr;
          if (cudaGraphNodeGetType(n, &ty) != cudaSuccess || ty != cudaGraphNodeTypeEventRecord) continue;
          if (cudaGraphEventRecordNodeGetEvent(n, &ev) != cudaSuccess) continue;
          for (size_t j = 0; j < s->rec_cursor; ++j) {
            if (s->recs[j].a == ev) gr->tnodes.push_back({n, (int)j, 0});
            else if (s->recs[j].b == ev) gr->tnodes.push_back({n, (int)j, 1});
          }
        }
      }
    }
    (void)cudaGetLastError();
  }
  *out = gr;
  return OOO_OK;
}

ooo_status ooo_graph_set_timing_slots(ooo_graph *g, int32_t slots) {
  if (!g) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL graph");
  if (slots < 1) return fail(OOO_ERR_INVALID_ARGUMENT, "slots must be >= 1");
  if (g->tnodes.empty()) return fail(OOO_ERR_STATE, "graph was captured without timing (ooo_set_timing before ooo_graph_create)");
  for (cudaEvent_t e : g->sev) cudaEventDestroy(e);
  g->sev.assign((size_t)slots * g->tinfo.size() * 2, nullptr);
  for (cudaEvent_t &e : g->sev) CU_TRY(cudaEventCreate(&e));
  g->slots = slots;
  g->launches = 0;
  return OOO_OK;
}

ooo_status ooo_graph_timing_read(ooo_graph *g, ooo_launch_record *out, int32_t cap, int32_t *n, int32_t *per_launch) {
  if (!g || !n) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  const int nrec = (int)g->tinfo.size();
  const long used = std::min<long>(g->launches, g->slots);
  if (per_launch) *per_launch = nrec;
  int32_t cnt = 0;
  for (long l = 0; l < used; ++l) {
    for (int j = 0; j < nrec; ++j, ++cnt) {
      if (!out || cnt >= cap) continue;
      cudaEvent_t a = g->sev[((size_t)l * nrec + j) * 2], b = g->sev[((size_t)l * nrec + j) * 2 + 1];
      out[cnt] = g->tinfo[j];
      float ms = 0.f, st = 0.f;
      cudaError_t e = cudaEventElapsedTime(&ms, a, b);
      out[cnt].ms = e == cudaSuccess ? ms : -1.f;
      if (e != cudaSuccess) (void)cudaGetLastError();
      e = cudaEventElapsedTime(&st, g->sev[0], a);
      out[cnt].start_ms = e == cudaSuccess ? st : -1.f;
      if (e != cudaSuccess) (void)cudaGetLastError();
    }
  }
  *n = cnt;
  return OOO_OK;
}

ooo_status ooo_graph_launch(ooo_graph *g, void *stream) {
  if (!g) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL graph");
  if (g->slots > 0 && g->launches <= g->slots) {
    // re-point the timing nodes: launch l records into slot l's events; after
    // the last slot, back to the stack's own events (slots keep their values)
    const int nrec = (int)g->tinfo.size();
    for (const ooo_graph::TNode &t : g->tnodes) {
      cudaEvent_t ev = g->launches < g->slots ? g->sev[((size_t)g->launches * nrec + t.rec) * 2 + t.which]
                                              : (t.which ? g->s->recs[t.rec].b : g->s->recs[t.rec].a);
      CU_TRY(cudaGraphExecEventRecordNodeSetEvent(g->exec, t.node, ev));
    }
  }
  CU_TRY(cudaGraphLaunch(g->exec, static_cast<cudaStream_t>(stream)));
  if (g->slots > 0) ++g->launches;
  return OOO_OK;
}

ooo_status ooo_graph_upload(ooo_graph *g, const void *X_host, const void *dY_host, void *copy_stream) {
  if (!g || !X_host || !dY_host) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  if (!g->dX) return fail(OOO_ERR_UNSUPPORTED, "not a stack step graph");
  cudaStream_t cs = static_cast<cudaStream_t>(copy_stream);
  if (!g->ev_in) {
    CU_TRY(cudaEventCreateWithFlags(&g->ev_in, cudaEventDisableTiming));
    CU_TRY(cudaEventCreateWithFlags(&g->ev_done, cudaEventDisableTiming));
  }
  if (g->launched) CU_TRY(cudaStreamWaitEvent(cs, g->ev_done, 0));   // the last launch has read X / dY
  CU_TRY(cudaMemcpyAsync(g->dX, X_host, g->x_bytes, cudaMemcpyHostToDevice, cs));
  CU_TRY(cudaMemcpyAsync(g->dY, dY_host, g->dy_bytes, cudaMemcpyHostToDevice, cs));
  CU_TRY(cudaEventRecord(g->ev_in, cs));
  return OOO_OK;
}

ooo_status ooo_graph_launch_host(ooo_graph *g, void *Y_host, void *stream, void *copy_stream) {
  if (!g || !Y_host) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  if (!g->ev_in) return fail(OOO_ERR_STATE, "ooo_graph_upload must precede ooo_graph_launch_host");
  cudaStream_t st = static_cast<cudaStream_t>(stream), cs = static_cast<cudaStream_t>(copy_stream);
  CU_TRY(cudaStreamWaitEvent(st, g->ev_in, 0));
  OOO_TRY(ooo_graph_launch(g, stream));
  CU_TRY(cudaEventRecord(g->ev_done, st));
  g->launched = true;
  CU_TRY(cudaStreamWaitEvent(cs, g->ev_done, 0));
  CU_TRY(cudaMemcpyAsync(Y_host, g->dYout, g->y_bytes, cudaMemcpyDeviceToHost, cs));
  return OOO_OK;
}

ooo_status ooo_graph_destroy(ooo_graph *g) {
  if (!g) return OOO_OK;
  if (g->ev_in) cudaEventDestroy(g->ev_in);
  if (g->ev_done) cudaEventDestroy(g->ev_done);
  for (cudaEvent_t e : g->sev) cudaEventDestroy(e);
  if (g->exec) cudaGraphExecDestroy(g->exec);
  if (g->graph) cudaGraphDestroy(g->graph);
  delete g;
  return OOO_OK;
}

ooo_status ooo_destroy(ooo_stack *s) {
  if (!s) return OOO_OK;
  if (s->eng_pending) (void)engine_flush(s);   // the comm stream may be waiting on its counters
  if (s->hi) cudaStreamSynchronize(s->hi);
  if (s->lo) cudaStreamSynchronize(s->lo);
  if (s->comm) cudaStreamSynchronize(s->comm);
  if (s->nccl && s->api) s->api->CommDestroy(s->nccl);
  for (auto e : s->ev_dz) if (e) cudaEventDestroy(e);
  for (auto e : s->ev_pack) if (e) cudaEventDestroy(e);
  for (auto e : s->ev_ar) if (e) cudaEventDestroy(e);
  for (cudaEvent_t e : {s->ev_fork, s->ev_j_hi, s->ev_j_lo, s->ev_j_comm, s->ev_reset}) if (e) cudaEventDestroy(e);
  for (auto &r : s->recs) {
    if (r.a) cudaEventDestroy(r.a);
    if (r.b) cudaEventDestroy(r.b);
  }
  if (s->hi) cudaStreamDestroy(s->hi);
  if (s->lo) cudaStreamDestroy(s->lo);
  if (s->comm) cudaStreamDestroy(s->comm);
  delete s;
  return OOO_OK;
}

ooo_status ooo_tensor(ooo_stack *s, int32_t kind, int32_t layer, void **ptr, int64_t *rows) {
  if (!s || !ptr) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  if (layer < 1 || layer > s->p.L) return fail(OOO_ERR_INVALID_ARGUMENT, "layer %d out of range", layer);
  LayerRt &r = s->lr[layer - 1];
  int64_t nrows = s->p.M;
  switch (kind) {
    case 0: *ptr = r.X; break;
    case 1: *ptr = r.Z; break;
    case 2: *ptr = r.dZ; break;
    case 3: *ptr = r.db; nrows = s->p.R; break;
    default: return fail(OOO_ERR_INVALID_ARGUMENT, "kind %d invalid", kind);
  }
  if (rows) *rows = nrows;
  return OOO_OK;
}

ooo_status ooo_set_timing(ooo_stack *s, int32_t enable) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  s->timing = enable != 0;
  s->rec_cursor = 0;
  return OOO_OK;
}

ooo_status ooo_timing_read(ooo_stack *s, ooo_launch_record *out, int32_t cap, int32_t *n) {
  if (!s || !n) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL argument");
  int32_t cnt = 0;
  for (size_t j = 0; j < s->rec_cursor && j < s->recs.size(); ++j) {
    if (out && cnt < cap) {
      TimedRec &r = s->recs[j];
      out[cnt] = r.info;
      float ms = 0.f, st = 0.f;
      cudaError_t e = cudaEventElapsedTime(&ms, r.a, r.b);
      out[cnt].ms = e == cudaSuccess ? ms : -1.f;
      if (e != cudaSuccess) (void)cudaGetLastError();
      e = cudaEventElapsedTime(&st, s->recs[0].a, r.a);
      out[cnt].start_ms = e == cudaSuccess ? st : -1.f;
      if (e != cudaSuccess) (void)cudaGetLastError();
    }
    ++cnt;
  }
  *n = cnt;
  return OOO_OK;
}


ooo_status ooo_plan_regions(ooo_stack *s, int32_t region_layers, int32_t reps, void *stream) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  if (region_layers < 1 || reps < 1) return fail(OOO_ERR_INVALID_ARGUMENT, "region_layers and reps must be >= 1");
  if (!s->p.engine) return fail(OOO_ERR_UNSUPPORTED, "region planning profiles the bf16 engine (fp32 stack)");
  if (s->p.L < 2) return fail(OOO_ERR_UNSUPPORTED, "region planning needs L >= 2");
  // single-GPU method (§4): a plan profiled per rank could differ between
  // ranks, and the all-reduce issue order (D's dW order) must be identical
  if (s->d.world_size > 1) return fail(OOO_ERR_UNSUPPORTED, "region scheduling is single-GPU (world_size 1)");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  OOO_TRY(engine_flush(s));
  OOO_TRY(join_into(s, st));
  CU_TRY(cudaStreamSynchronize(st));
  CU_TRY(cudaStreamSynchronize(s->hi));
  const bool timing = s->timing;
  s->timing = false;
  ooo_status r = plan_regions(s, region_layers, reps);
  s->timing = timing;
  s->have_fwd = false;       // activations / gradients were overwritten by the profiling launches
  s->bwd_pending = false;
  OOO_TRY(r);
  CU_TRY(cudaStreamSynchronize(s->hi));
  return check_async(s);
}

ooo_status ooo_region_plan(const ooo_stack *s, int32_t *n_regions, int32_t *k_pre, int32_t *region_of,
                           int32_t *ops, int32_t *n_ops, double *t_main, int32_t t_main_cap) {
  if (!s) return fail(OOO_ERR_INVALID_ARGUMENT, "NULL stack");
  if (!s->has_regions) return fail(OOO_ERR_STATE, "no region plan (ooo_plan_regions)");
  if (n_regions) *n_regions = (int32_t)s->reg_tmain.size();
  if (k_pre) *k_pre = s->reg_kpre;
  if (region_of)
    for (int i = 0; i < s->p.L; ++i) region_of[i] = s->reg_region_of[i];
  if (ops)
    for (size_t j = 0; j < s->reg_D.size(); ++j) ops[j] = s->reg_D[j];
  if (n_ops) *n_ops = (int32_t)s->reg_D.size();
  if (t_main)
    for (int i = 0; i < std::min<int>(t_main_cap, (int)s->reg_tmain.size()); ++i) t_main[i] = s->reg_tmain[i];
  return OOO_OK;
}

}  // extern "C"

// ---- internal (pipeline.cpp): error message and graph wrapping
namespace ooo {
ooo_status set_error(ooo_status st, const char *msg) { return fail(st, "%s", msg); }
ooo_graph *wrap_graph(cudaGraph_t g, cudaGraphExec_t e) {
  ooo_graph *gr = new ooo_graph();
  gr->graph = g;
  gr->exec = e;
  return gr;
}
}  // namespace ooo

#ifdef OOO_TRACE
// Debug builds only (libooo_trace.so): device buffer of [task][4] u64 stamps
// filled by the engine kernels (tools/engine_trace.py).
extern "C" ooo_status ooo_debug_set_trace(void *dev_ptr) {
  CU_TRY(ooo::eng::engine_set_trace(dev_ptr));
#ifdef OOO_TRACE
  // skinny stacks: after the engine's three 200000 x 8 stamp arrays
  CU_TRY(ooo::sk::skinny_set_trace(dev_ptr ? static_cast<char *>(dev_ptr) + (size_t)3 * 200000 * 8 * 8 : nullptr));
#endif
  return OOO_OK;
}

// the most recent engine launch's queue as (kind, layer, m_off in 128-row
// blocks, tile rows, column tiles) per op; returns the number of ops.
extern "C" int32_t ooo_debug_last_queue(ooo_stack *s, int32_t *out, int32_t cap) {
  int32_t n = 0;
  for (const auto &o : s->last_queue) {
    if (n < cap) {
      out[5 * n] = o.kind;
      out[5 * n + 1] = o.layer;
      out[5 * n + 2] = o.m_off;
      out[5 * n + 3] = o.mt;
      out[5 * n + 4] = o.nt * (o.ks > 1 ? o.ks : 1);   // tasks per tile row (split-K: ks per tile)
    }
    ++n;
  }
  return n;
}
#endif
