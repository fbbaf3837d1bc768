/*
 * ooo.h -- C ABI of the B200-native out-of-order backprop (ooo backprop)
 *          data-parallel hot path.
 *
 * Paper: H. Oh, J. Lee, H. Kim, J. Seo, "Out-Of-Order BackProp: An Effective
 * Scheduling Technique for Deep Learning", EuroSys'22.  "P:N" = line N of the
 * paper text, followed by the section it is in.
 *
 * What one iteration is (§2, problem statement P:81-95): starting from the
 * loss gradient dO_{L+1} at time 0, the backward ops of every layer -- the
 * output-gradient op dO_i and the weight-gradient op dW_i -- then the
 * gradient synchronisation S[dW_i] of every layer (data parallelism, §5.1
 * P:176-180), and finally the next iteration's forward F_1..F_L, where
 * F_i may start only after S[dW_i] (T(F_i) >= T(S[dW_i]) + S[dW_i]).
 * dW_i feeds no other gradient (§3), so it may run out of layer order;
 * ooo_backward(schedule = OOO_SCHED_FIRST_K, k) issues the dW ops in the
 * order of Algorithm 2 "Reverse First-K Scheduling".
 *
 * Model: a stack of L dense (Linear) layers, layer i = 1..L:
 *     Z_i = X_i W_i + 1 b_i^T,      X_{i+1} = act_i(Z_i)
 *     W_i: d_{i-1} x d_i, row-major (d_i contiguous);  b_i: d_i
 *     X_i, Z_i, dZ_i: M x d, row-major (d contiguous), M = tokens per rank.
 *   Backward (dY = dLoss/dX_{L+1}, given by the caller; reading Q8):
 *     dZ_L     = dY (.) act_L'(Z_L)                               (seed)
 *     dO_i:  dZ_{i-1} = (dZ_i W_i^T) (.) act_{i-1}'(Z_{i-1})      (i >= 2)
 *            dX       =  dZ_1 W_1^T       (i == 1, only if need_input_grad)
 *     dW_i:  dW_i = X_i^T dZ_i,  db_i = 1^T dZ_i
 *   Data parallel (§5.1): every rank holds the same W, b and its own M-token
 *   shard; the library returns the rank average (1/N) sum_r dW_i^(r)
 *   (reading Q9: pre-scaled by 1/N, then an in-place NCCL sum all-reduce per
 *   bucket, issued in the order the dW ops complete).
 *
 * Precision (reading Q10): OOO_BF16 = bf16 storage of X, Z, dZ, W, b and
 * gradients, fp32 accumulation (tcgen05 tensor cores), bf16 RNE rounding at
 * every store; OOO_FP32 = fp32 everywhere (exact fp32 FFMA, no TF32).
 *
 * Memory ownership: every device buffer is allocated by the caller (e.g. a
 * torch tensor); the library never allocates device memory.  The stack owns
 * host objects only: CUDA streams and events, TMA descriptors, the NCCL
 * communicator and captured graphs.
 *
 * Stream semantics: every call is stream-ordered after prior work on the
 * caller's stream `st`.  ooo_backward returns with work still in flight on
 * the library's internal streams (hi priority: dO ops; lo priority: dW ops;
 * comm: all-reduces) -- or, on the bf16 engine path, with its kernel
 * deferred: the next ooo_forward then runs backward(t) and forward(t+1) as
 * ONE persistent kernel whose F_i tiles start as soon as S[dW_i] and
 * dW_{i+1} are done (Fig. 4(c)).  ooo_forward finally joins everything into
 * `st`; ooo_join runs/joins an outstanding backward explicitly.  Gradients in
 * `grads` and dX are valid only after one of those.  No call synchronises the host or allocates, so the
 * sequence ooo_backward; ooo_forward is CUDA-graph capturable on `st`.
 *
 * Errors: argument/shape errors are detected before anything is enqueued;
 * the call returns a non-zero ooo_status and ooo_last_error() describes it.
 * Asynchronous CUDA / NCCL failures surface as OOO_ERR_CUDA / OOO_ERR_NCCL
 * from a later call (ooo_join polls ncclCommGetAsyncError).  No C++
 * exception crosses this ABI.  Threading: one stack is used by one host
 * thread at a time; ooo_last_error is thread-local.  GPU sharing: a bf16
 * step is one persistent kernel holding one CTA per SM (N > 1: all but the
 * SMs reserved for NCCL); steps of two stacks must not run concurrently on
 * one GPU (a second persistent grid pending for SMs can starve the comm
 * stream's all-reduce kernels the first one waits on).
 *
 * Collective rule: with world_size > 1 every rank must call ooo_backward with
 * the same schedule (D and the NCCL issue order depend only on (L, k));
 * a mismatch is undefined behaviour (NCCL hang).
 */
#ifndef OOO_H_
#define OOO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define OOO_ABI_VERSION 2
#define OOO_UNIQUE_ID_BYTES 128

typedef struct ooo_stack ooo_stack;   /* opaque */
typedef struct ooo_graph ooo_graph;   /* opaque, a captured [backward; forward] step */

typedef enum {
  OOO_OK = 0,
  OOO_ERR_INVALID_ARGUMENT = 1,
  OOO_ERR_UNSUPPORTED = 2,
  OOO_ERR_CUDA = 3,
  OOO_ERR_NCCL = 4,
  OOO_ERR_STATE = 5
} ooo_status;

typedef enum { OOO_BF16 = 0, OOO_FP32 = 1 } ooo_dtype;

/* act_i of layer i (applied to Z_i).  ReLU: relu'(0) = 0.  GELU: exact erf
 * form gelu(z) = z Phi(z), gelu'(z) = Phi(z) + z phi(z). */
typedef enum { OOO_ACT_IDENTITY = 0, OOO_ACT_RELU = 1, OOO_ACT_GELU_ERF = 2 } ooo_act;

/* OOO_SCHED_IN_ORDER: conventional backprop with per-layer
 *   overlapped sync (wait-free backprop): one compute stream runs, for
 *   i = L..1, dO_i then dW_i (+ its bucket pack); each bucket's all-reduce is
 *   issued as soon as it is packed.
 * OOO_SCHED_FIRST_K: Algorithm 2 with k <- min(max_k, k)
 *   (l.1-2): dO ops on the high-priority stream, dW ops on the low-priority
 *   stream in D's order (critical ops high priority, sub-stream
 *   kernels serialise), all-reduces on the comm stream in D's dW order.
 *   k = 0 is dual-stream without reordering (the P:312 ablation). */
/* OOO_SCHED_REGIONS: single-GPU multi-stream ooo computation (§4.1,
 *   P:117-162): the critical ops (dO, then the next forward) form the
 *   main-stream, split into regions; every dW_i (i >= 2) runs in the region
 *   Algorithm 1 assigned it (multi-region joint scheduling, with
 *   the memory-bounded pre-scheduling of P:162), dW_1 as soon as it is ready
 *   (it gates F_1).  Needs a plan from ooo_plan_regions on the same stack
 *   (OOO_ERR_STATE otherwise); k is ignored.  The backward order D is the
 *   plan's (ooo_region_plan); the all-reduces follow D's dW order. */
typedef enum { OOO_SCHED_IN_ORDER = 0, OOO_SCHED_FIRST_K = 1, OOO_SCHED_REGIONS = 2 } ooo_sched_kind;

typedef struct {
  int32_t kind;   /* ooo_sched_kind */
  int32_t k;      /* >= 0; clamped to [0, min(L, max_k)] (Alg. 2 l.2); k < 0 -> INVALID_ARGUMENT */
} ooo_schedule;

typedef struct {
  int32_t num_layers;          /* L >= 1 */
  const int32_t *dims;         /* L+1 host ints d_0..d_L; each >= 64 and % 64 == 0, else UNSUPPORTED */
  const int32_t *acts;         /* L host ints (ooo_act) */
  int32_t tokens;              /* M rows per rank per call; >= 1 and % 8 == 0 (TMA row alignment) */
  int32_t dtype;               /* ooo_dtype */
  int32_t need_input_grad;     /* 1: emit dO_1 and write dX (reading Q1); 0: omit dO_1 */
  int32_t bucket_layers;       /* >= 1 consecutive layers per all-reduce bucket; schedule independent */
  int64_t max_temp_bytes;      /* MXM of Alg. 2 l.1 (bytes); <= 0 = unlimited */
  const void *const *W;        /* L device pointers, W_i [d_{i-1}][d_i] row-major, dtype */
  const void *const *b;        /* L device pointers, b_i [d_i], dtype */
  void *grads;                 /* device, grads_bytes (ooo_query_sizes), dtype: layer i at
                                  ooo_grad_offsets: dW_i [d_{i-1}][d_i] row-major then db_i [d_i];
                                  layers contiguous in increasing i, so a bucket of consecutive
                                  layers is one contiguous all-reduce buffer.  Output. */
  void *workspace;             /* device, workspace_bytes (ooo_query_sizes), 256-B aligned:
                                  X_i / Z_i / dZ_i stores, split-K and bias-grad partials */
  int32_t world_size;          /* N >= 1 */
  int32_t rank;                /* 0 <= rank < N */
  const void *nccl_unique_id;  /* OOO_UNIQUE_ID_BYTES from ooo_get_unique_id on rank 0, shared by
                                  the caller (e.g. torch.distributed broadcast).  Required for N > 1.
                                  N == 1: NULL = no communicator; non-NULL = a ONE-rank NCCL
                                  communicator, so a single GPU runs the whole N > 1 data plane
                                  (per-bucket ncclAllReduce on the comm stream, F_i gated on the
                                  all-reduce flags, the SM reserve) -- the all-reduce of one rank is
                                  the identity, so results equal the non-communicating stack's. */
  int32_t comm_enabled;        /* 1: all-reduce each bucket.  0: comm-off control -- same streams,
                                  events and kernels, the all-reduce is skipped (exposed-comm
                                  measurement); gradients are then the local shard's. */
  int32_t nccl_max_ctas;       /* > 0: ncclConfig_t.maxCTAs (bounds SMs taken from the GEMMs); 0 = NCCL default */
  int32_t wait_timeout_ms;     /* bound of every wait inside the bf16 engine kernel (dependency
                                  counters; F_i's wait for its bucket's all-reduce, which peer ranks
                                  drive): beyond it the kernel traps and the CUDA context reports an
                                  error instead of hanging.  <= 0 = default: 4000 ms for a stack
                                  without a communicator, 120000 ms with one. */
  int32_t comm_priority;       /* issue order of the all-reduce chunks on the comm stream (§5.1 P:180,
                                  Fig. 4; ooo_comm_schedule): 0 = FIFO in D's dW order (Fig. 4(a)/(c));
                                  1 = prioritised: the ready chunk of the lowest-layer bucket first
                                  (Fig. 4(b)), planned per step from the engine planner's predicted dW
                                  completion times (bf16 engine; the fp32 path stays FIFO) */
  int32_t comm_model_gbps;     /* chunk-duration model of the prioritised order: ring bytes
                                  2(N-1)/N x chunk bytes at this many GB/s + 8 us per call;
                                  <= 0 = 700 (the emulated all-reduce uses its own parameters) */
  int64_t comm_chunk_bytes;    /* > 0: every bucket's all-reduce is partitioned into chunks of at most
                                  this many bytes (rounded down to 256 elements), with boundaries
                                  fixed per stack -- so every schedule reduces the same element ranges
                                  and stays bit-exact -- and the channel can switch buckets between
                                  chunks (the partitioning of [28, 38] behind P:180); <= 0 = one
                                  all-reduce per bucket */
  int32_t average_over;        /* > 0: the gradients are scaled by 1 / average_over before the sum
                                  all-reduce (pack/scale step, reading Q9) instead of 1 / world_size --
                                  e.g. to average over a global batch of several local steps; 0 =
                                  world_size (the data-parallel mean) */
  int32_t engine_ctas;         /* > 0: at most this many CTAs (SMs) for the bf16 engine kernels of this
                                  stack (one SM partition per pipeline stage, ooo_pipeline_*); <= 0 = all
                                  SMs (minus the NCCL reserve of a communicating stack) */
} ooo_stack_desc;

/* ---------------------------------------------------------------- info */
int32_t ooo_abi_version(void);
const char *ooo_last_error(void);                  /* thread-local message of the last non-OK status */
const char *ooo_status_string(int32_t status);

/* ------------------------------------------------------ host-only helpers */
/* Sizes of the caller-allocated device buffers.  No device access. */
ooo_status ooo_query_sizes(const ooo_stack_desc *d, size_t *workspace_bytes, size_t *grads_bytes);

/* offsets[2*(i-1)] = element offset of dW_i, offsets[2*(i-1)+1] = of db_i, inside `grads`. */
ooo_status ooo_grad_offsets(const ooo_stack_desc *d, int64_t *offsets /* 2L */);

/* The backward order D as the library issues it (Alg. 2 lines 3-6, P:195-201;
 * within a layer the paper's order dW_i before dO_i; IN_ORDER = dO_i first).
 * ops[j] = +i for dO_i, -i for dW_i.  `ops` has room for 2L entries; *n
 * receives the count.  `k` is clamped to [0, L] only (memory clamp: ooo_max_k). */
ooo_status ooo_schedule_order(int32_t L, ooo_schedule sch, int32_t need_input_grad,
                              int32_t *ops, int32_t *n);

/* Alg. 2 line 1 (garbled in the text; reading Q3, parity unpinned):
 * max_k = largest j in [0, L] with f(j) = m_fwd - sum_{i>j} m_dO[i-1] + sum_{i<=j} m_dW[i-1] < mxm;
 * mxm <= 0 -> L.  Byte counts are host arrays of length L. */
int32_t ooo_max_k(int32_t L, int64_t m_fwd, const int64_t *m_dO, const int64_t *m_dW, int64_t mxm);

/* Algorithm 1 "Multi-Region Joint Scheduling" (§4.1) and the
 * memory-bounded pre-scheduling of P:162.  Pure host function.
 *   n_regions N >= 1 main-stream regions R[0..N-1] in execution order,
 *   t_main[N] = T_main(R[i]) (regions run back to back: start[i] = sum_{j<i}).
 *   n_cands K >= 0 sub-stream kernels; row-major [K][N] tables t_sub =
 *   T_sub(k, R[i]) and speedup = co-run speedup p of kernel k in R[i];
 *   ready[K] = main-stream time at which kernel k's input is complete;
 *   last_region[K] = last region k may run in (NULL: N-1);
 *   nbytes[K] = bytes kernel k keeps alive while deferred (NULL: 0);
 *   mxm = memory bound on the bytes held at region ends (<= 0: unlimited).
 * Readings: runnable in R[i] = ready[k] <= start[i] + now[i] and
 * i <= last_region[k]; ties -> first kernel / smallest region; when no open
 * region has a runnable kernel the rest run as soon as ready (in the region
 * in which they become ready); while the peak held bytes exceed mxm, one
 * more leading region is pre-scheduled as soon as ready and Algorithm 1
 * re-runs on the rest.
 * Outputs (caller-owned host arrays): region_of[K]; order[K] = kernels in
 * schedule order (region 0's list, then region 1's, ...); *k_pre = regions
 * pre-scheduled.  OOO_ERR_INVALID_ARGUMENT on bad sizes / pointers / regions. */
ooo_status ooo_region_schedule(int32_t n_regions, const double *t_main, int32_t n_cands, const double *t_sub,
                               const double *speedup, const double *ready, const int32_t *last_region,
                               const int64_t *nbytes, int64_t mxm, int32_t *region_of, int32_t *order,
                               int32_t *k_pre);

/* Heuristic search for reverse first-k's k (§5.1; readings in
 * DESIGN.md Q4, parity unpinned beyond the prose): dk0 = max(1, round(L/10)),
 * scan k = 0, dk, ... < L, then the open range (best - dk, best + dk) with dk
 * halved, until a pass with dk == 1; ties -> smaller k; each k measured once
 * through `throughput(k, ctx)` (higher is better; the caller times the step).
 * visited (room for L + 1 entries, may be NULL) receives the measured ks in
 * order, *n_visited their count.  Returns the best k, or -1 if L < 1 or
 * throughput is NULL.  Pure host function. */
int32_t ooo_k_search(int32_t L, double (*throughput)(int32_t k, void *ctx), void *ctx, int32_t *visited,
                     int32_t *n_visited);

/* Issue order of partitioned all-reduces on one FIFO channel (§5.1 P:180,
 * Fig. 4(b); readings C1-C3 in DESIGN.md).  Pure host function.
 *   n_buckets B; ready[B] = time bucket b's dW ops are complete; n_chunks[B]
 *   >= 1; dur = chunk durations, bucket after bucket (sum n_chunks entries);
 *   prio[B] = priority key (lower = more urgent: the bucket's first layer);
 *   fifo_rank[B] = position in the FIFO order (NULL = bucket index).
 *   policy 0 = FIFO: buckets by fifo_rank, chunks in order, each chunk
 *   starting at max(channel free, ready); 1 = PRIORITY: whenever the channel
 *   is free the next chunk of the ready bucket with the lowest prio (ties:
 *   lower index) goes, an idle channel waits for the earliest ready bucket.
 * Outputs (caller-owned): order_b / order_c = the (bucket, chunk) issue
 * order (sum n_chunks entries); done[B] (may be NULL) = completion time of
 * each bucket's last chunk.  OOO_ERR_INVALID_ARGUMENT on bad sizes. */
ooo_status ooo_comm_schedule(int32_t n_buckets, const double *ready, const int32_t *n_chunks, const double *dur,
                             const int32_t *prio, const int32_t *fifo_rank, int32_t policy, int32_t *order_b,
                             int32_t *order_c, double *done);

/* Extra bytes kept alive by deferring dW_1..dW_k (the memory cost of
 * deferral, §3; E8 at P:352-354): sum_{i=2..k} |dZ_i|. */
int64_t ooo_deferral_bytes(const ooo_stack_desc *d, int32_t k);

/* Host only (no GPU): the tile queue the bf16 engine dispenses for one step,
 * as planned from the two priority chains (critical: dO ops in D's order,
 * then -- if `fused` -- the X -> X_1 copy and F_1..F_L of the next forward;
 * deferred: dW ops in D's order; §4.1, Alg. 2) for
 * `workers` concurrently resident tiles (<= 0: 148 / CTAs per tile).
 * Writes up to `cap` ops as 5 int32 each: kind (0 F, 1 dO, 2 dW, 3 copy),
 * layer i, first tile row, tile rows, column tiles; *n receives the count.
 * *topological = 1 iff every op follows all ops it depends on (the engine's
 * deadlock-freedom condition).  OOO_ERR_UNSUPPORTED for fp32 stacks. */
ooo_status ooo_engine_plan(const ooo_stack_desc *d, ooo_schedule sch, int32_t fused, int32_t workers,
                           int32_t *out, int32_t cap, int32_t *n, int32_t *topological);

/* NCCL bootstrap id (rank 0 calls, caller broadcasts).  Needs libnccl.so.2. */
ooo_status ooo_get_unique_id(void *out /* OOO_UNIQUE_ID_BYTES */);

/* ------------------------------------------------------------- the path */
/* Validates, plans the workspace, encodes TMA descriptors, creates the
 * priority streams / events and (nccl_unique_id given) the NCCL communicator
 * -- collective over ranks.  With a communicator it then warms NCCL up: it
 * zeroes `grads` and all-reduces every bucket once (NCCL connects its
 * channels lazily on first use; a cold first call inside a training step
 * could take longer than the engine's wait bound) and waits for it.  Uses
 * the current CUDA device. */
ooo_status ooo_create_stack(const ooo_stack_desc *d, ooo_stack **out);

/* F_1..F_L: X [M][d_0] (device, dtype) -> Y [M][d_L] (device, dtype).
 * X and Y (and dY, dX of ooo_backward / ooo_graph_create) must be 32-byte
 * aligned for bf16 stacks (the engine stores 32-byte row vectors), 16-byte for
 * fp32; OOO_ERR_INVALID_ARGUMENT otherwise.
 * X is copied into the stack's X_1 store; Y is written by F_L.  If a backward
 * is pending, F_i first waits for layer i's synchronised gradient (and for
 * dW_{i+1}, which still reads X_{i+1}).  A communicating bf16 stack (a NCCL
 * communicator, or the emulated all-reduce OOO_EMULATE_AR_N) runs its fused
 * training steps only through ooo_graph_create / ooo_graph_launch: an eager
 * ooo_forward after ooo_backward returns OOO_ERR_UNSUPPORTED (an EAGER fused
 * step whose comm stream holds kernels behind the per-bucket value-waits was
 * observed to stall on B200; the graph-launched step is unaffected).  Eager
 * ooo_backward + ooo_join (no forward in the same launch) is allowed. */
ooo_status ooo_forward(ooo_stack *s, const void *X, void *Y, void *stream /* cudaStream_t */);

/* Backward of the last forward: dY [M][d_L] (device, dtype).  dX [M][d_0]
 * (device) is written iff need_input_grad, else must be NULL.
 * OOO_ERR_STATE if no forward preceded it. */
ooo_status ooo_backward(ooo_stack *s, const void *dY, ooo_schedule sch, void *dX, void *stream);

/* `stream` waits for all outstanding backward work, all-reduces included. */
ooo_status ooo_join(ooo_stack *s, void *stream);

/* Gradient fast-forwarding across pipeline stages (§5.2.1): make
 * `stream` wait until the input gradient dX of this stack's last
 * ooo_backward is complete -- in the middle of the engine kernel, as soon as
 * the dO chain has produced dX and before the deferrable dW ops finish -- so
 * the previous stage can start on it.  Launches the deferred backward kernel
 * if it has not run yet (as ooo_join would, without joining it).  bf16
 * engine stacks with need_input_grad only (OOO_ERR_UNSUPPORTED otherwise);
 * OOO_ERR_STATE without a backward.  Like every mid-kernel wait on another
 * stream, run it inside a captured graph (see ooo_forward). */
ooo_status ooo_input_grad_wait(ooo_stack *s, void *stream);

/* S[dW] of every bucket back to back on the stack's comm stream and
 * communicator, no compute (collective: every rank calls it): the
 * stand-alone all-reduce time the hidden fraction is measured against
 * (SURVEY §8d AR_ms), with exactly the buckets, sizes, dtype and
 * communicator a training step uses.  `grads` is summed in place again
 * (its values change; run a backward afterwards for valid gradients).
 * Buckets are issued from the last (layer L) to the first.  `stream` waits
 * for the all-reduces.  OOO_ERR_STATE for a stack without communicator. */
ooo_status ooo_allreduce_buckets(ooo_stack *s, void *stream);

/* The (bucket, chunk) order in which the most recently enqueued step issued
 * its all-reduces on the comm stream (engine path; ooo_comm_schedule with
 * desc.comm_priority).  *n = count (only the first `cap` are written).  An
 * empty list for a stack that does not communicate. */
ooo_status ooo_comm_issue_order(const ooo_stack *s, int32_t *bucket, int32_t *chunk, int32_t cap, int32_t *n);

/* Plans OOO_SCHED_REGIONS (single-GPU multi-stream ooo, §4.1) for
 * this stack, by the paper's steps 1-5:
 *   1. profile on the GPU, for every region pair, the main-stream region
 *      alone, each candidate dW_i alone and the two co-run (one engine
 *      launch each, `reps` timed repetitions, the minimum kept); speedup =
 *      (T_main + T_sub) / T_co-run;
 *   2. main-stream = dO_L..dO_2 (dO_1 iff need_input_grad), then F_1..F_L of
 *      the next iteration, in regions of `region_layers` consecutive layers;
 *   3. candidates dW_2..dW_L (dW_1 gates F_1 and runs as soon as ready),
 *      runnable once dO_{i+1} is done (interpolated by FLOPs inside its
 *      region) and up to the region before F_{i-1} (which overwrites X_i);
 *   4-5. Algorithm 1 with the memory bound desc.max_temp_bytes on the
 *      deferred dZ_i bytes (ooo_region_schedule).
 * Synchronous (host waits for the profiling launches; not capturable) and
 * destructive: activations and gradients are overwritten, so an ooo_forward
 * must run before the next ooo_backward (OOO_ERR_STATE otherwise).  bf16
 * stacks with world_size 1 only (OOO_ERR_UNSUPPORTED otherwise: the paper's
 * single-GPU method, and per-rank profiles could order the all-reduces
 * differently on different ranks); region_layers >= 1, reps >= 1. */
ooo_status ooo_plan_regions(ooo_stack *s, int32_t region_layers, int32_t reps, void *stream);

/* The current region plan: *n_regions, *k_pre (pre-scheduled regions),
 * region_of[L] (main-stream region of dW_i; that of dW_1 = the first
 * forward region), ops[2L] / *n_ops = the backward order D it issues (+i dO_i,
 * -i dW_i), t_main[n_regions] (profiled region times, ms; may be NULL).
 * OOO_ERR_STATE without a plan. */
ooo_status ooo_region_plan(const ooo_stack *s, int32_t *n_regions, int32_t *k_pre, int32_t *region_of,
                           int32_t *ops, int32_t *n_ops, double *t_main, int32_t t_main_cap);

/* Pre-compiled issue (§4.2): capture one training step
 * [ooo_backward(dY, sch, dX); ooo_forward(X, Y)] into an executable CUDA graph
 * instantiated with per-node priorities.  A plain ooo_forward(X, Y) must have
 * run before.  Pointers are baked into the graph. */
ooo_status ooo_graph_create(ooo_stack *s, const void *X, void *Y, const void *dY, ooo_schedule sch,
                            void *dX, ooo_graph **out);
ooo_status ooo_graph_launch(ooo_graph *g, void *stream);
ooo_status ooo_graph_destroy(ooo_graph *g);

/* A training step with HOST buffers (the end-to-end path): ooo_graph_upload
 * copies the step's inputs X [M][d_0] and dY [M][d_L] from host memory into
 * the device buffers baked into the graph, on `copy_stream`, after the
 * graph's previous launch has finished reading them; ooo_graph_launch_host
 * launches the step on `stream` once that upload is complete and then copies
 * Y [M][d_L] back to host memory on `copy_stream` (Y_host is written when
 * copy_stream reaches that point).  Pinned host memory makes the copies
 * asynchronous.  Two graphs over two buffer sets, used alternately
 * (upload(t+1); launch_host(t)), overlap the copies with the compute.  Stack
 * step graphs only (not pipeline graphs: OOO_ERR_UNSUPPORTED). */
ooo_status ooo_graph_upload(ooo_graph *g, const void *X_host, const void *dY_host, void *copy_stream);
ooo_status ooo_graph_launch_host(ooo_graph *g, void *Y_host, void *stream, void *copy_stream);

ooo_status ooo_destroy(ooo_stack *s);             /* joins, then frees host/NCCL resources */

/* --------------------------------------- cross-layer model parallelism (§5.2) */
/* A stack of L layers split into groups of group_layers consecutive layers
 * (the unit of allocation; the paper allocates transformer blocks),
 * groups allocated to n_stages pipeline stages (GPUs): placement 0 =
 * contiguous (G/n consecutive groups per stage, the conventional allocation,
 * P:234), 1 = modulo (group j on stage j mod n, "modulo layer allocation",
 * P:234-238).  One training iteration (no micro-batches, §5.2.1) = the
 * forward of every group in layer order, then the backward from the last
 * group: with fast_forward = 0 conventional backprop (each group in order, a
 * stage starts after the next group's whole backward, P:101 / Fig. 5(a));
 * with fast_forward = 1 gradient fast-forwarding (each group's dO chain first
 * and its dX released mid-kernel to the previous group, whose backward
 * overlaps this group's dW ops, Fig. 5(b)/(c)).
 * Two modes.  Without a communicator (nccl_unique_id NULL, world_size 1) the
 * stages are SM partitions of the current GPU (148 / n SMs each, one stream
 * per stage, hand-offs through device buffers): the data plane of n GPUs on
 * one device.  With a communicator every rank is one stage (n_stages ==
 * world_size), holds only its groups (ooo_pipeline_query_sizes then sizes
 * that rank's buffers), uses all SMs but an NCCL reserve of 16, and hands
 * activations and input gradients to the neighbouring stages with
 * ncclSend / ncclRecv on a comm stream -- after the group's forward, and
 * after its dX (fast-forwarding: ooo_input_grad_wait on the comm stream,
 * mid-kernel) or its whole backward (conventional).  Every rank walks the
 * groups in the same global order, so each pair of ranks posts matching
 * send / recv sequences.  world_size 1 with a communicator = loopback: every
 * group boundary is a send / recv to itself (the P2P data plane on one GPU).
 * Gradients of group j (owned groups only) are in its own gradient buffer
 * (ooo_pipeline_grads_offset). */
typedef struct ooo_pipeline ooo_pipeline;
typedef struct {
  int32_t num_layers;          /* L */
  const int32_t *dims;         /* L+1 widths (as ooo_stack_desc) */
  const int32_t *acts;         /* L activations */
  int32_t tokens;              /* M */
  int32_t group_layers;        /* >= 1, divides L */
  int32_t n_stages;            /* >= 1; n_stages <= number of groups */
  int32_t placement;           /* 0 contiguous, 1 modulo */
  const void *const *W, *const *b;   /* L device pointers (bf16) */
  void *workspace;             /* device, ooo_pipeline_query_sizes, 256-B aligned */
  void *grads;                 /* device, ooo_pipeline_query_sizes: groups' gradient buffers back to back */
  int32_t world_size;          /* 1, or the number of ranks (= n_stages) with a communicator */
  int32_t rank;
  const void *nccl_unique_id;  /* NULL: SM-partition stages on one GPU; else OOO_UNIQUE_ID_BYTES (rank 0's) */
} ooo_pipeline_desc;
ooo_status ooo_pipeline_query_sizes(const ooo_pipeline_desc *d, size_t *workspace_bytes, size_t *grads_bytes);
/* byte offset of group j's gradient buffer (layout of ooo_grad_offsets for the group's layers);
 * OOO_ERR_INVALID_ARGUMENT for a group another rank owns */
ooo_status ooo_pipeline_grads_offset(const ooo_pipeline_desc *d, int32_t group, int64_t *offset);
ooo_status ooo_pipeline_create(const ooo_pipeline_desc *d, ooo_pipeline **out);
/* Captures one iteration [forward(X) -> Y; backward(dY)] into a graph
 * (launch / destroy with ooo_graph_launch / ooo_graph_destroy).  X [M][d_0],
 * dY [M][d_L], Y [M][d_L]: caller device buffers, baked into the graph. */
ooo_status ooo_pipeline_graph_create(ooo_pipeline *p, const void *X, const void *dY, void *Y, int32_t fast_forward,
                                     ooo_graph **out);
/* Stage of group j under the pipeline's placement; -1 if out of range. */
int32_t ooo_pipeline_stage_of(const ooo_pipeline *p, int32_t group);
ooo_status ooo_pipeline_destroy(ooo_pipeline *p);

/* ------------------------------------------------- introspection / timing */
/* Device pointer of an internal store (teacher-forced parity tests):
 * kind 0 = X_i (i = 1..L), 1 = Z_i (NULL for identity layers: Z_i aliases
 * X_{i+1}; for GELU layers of a bf16 engine stack it holds gelu'(Z_i), the
 * factor the backward needs), 2 = dZ_i, 3 = bias-grad partials of layer i ([rows][d_i] fp32). */
ooo_status ooo_tensor(ooo_stack *s, int32_t kind, int32_t layer, void **ptr, int64_t *rows);

/* Per-launch timing.  ooo_set_timing(s, 1) makes subsequently enqueued or
 * captured calls bracket every kernel launch with CUDA events on the stream
 * it is launched on.  After the work completed (e.g. after the last graph
 * replay of a timed region), ooo_timing_read fills up to `cap` records
 * describing the most recent execution of each bracketed launch. */
typedef struct {
  int32_t kind;       /* 0 fwd GEMM, 1 dX GEMM, 2 dW GEMM, 3 seed act-grad, 4 pack, 5 all-reduce, 6 copy,
                         7 engine forward, 8 engine backward, 9 engine step (backward + next forward) */
  int32_t layer;
  int32_t stream;     /* 0 hi, 1 lo, 2 comm */
  int32_t grid;       /* CTAs launched */
  double flops;       /* algorithmic FLOPs of the launch (GEMMs) */
  double bytes;       /* algorithmic HBM bytes of the launch (pack / seed / copy / all-reduce payload) */
  float ms;           /* event-measured duration */
  float start_ms;     /* start relative to the first record's start (timeline) */
} ooo_launch_record;
ooo_status ooo_set_timing(ooo_stack *s, int32_t enable);
ooo_status ooo_timing_read(ooo_stack *s, ooo_launch_record *out, int32_t cap, int32_t *n);

/* Per-launch timing of a captured step over a whole timed region.  For a
 * graph captured while the stack's timing was on: the next `slots` calls of
 * ooo_graph_launch each record into their own set of CUDA events (the graph's
 * event-record nodes are re-pointed before each launch, host side; the
 * launches stay back to back on the caller's stream), later launches use the
 * stack's events again.  OOO_ERR_STATE if the graph has no timing brackets. */
ooo_status ooo_graph_set_timing_slots(ooo_graph *g, int32_t slots);
/* After those launches completed: the records of every timed launch, launch
 * after launch (*per_launch records each, in capture order), `ms` measured in
 * that launch; start_ms relative to the first launch's first record.
 * *n = total records (only the first `cap` are written). */
ooo_status ooo_graph_timing_read(ooo_graph *g, ooo_launch_record *out, int32_t cap, int32_t *n,
                                 int32_t *per_launch);

#ifdef __cplusplus
}
#endif
#endif /* OOO_H_ */
