"""Thin Python binding of the C ABI (include/ooo.h).

Argument marshalling only: every step of the path runs in libooo.so's CUDA
kernels.  torch supplies device memory (workspace / gradient buffers are torch
tensors), the caller's CUDA stream and, for N > 1, the process group used to
broadcast the NCCL bootstrap id.  Function and argument names follow the ABI
(ooo_create_stack / ooo_forward / ooo_backward / ooo_join / ooo_destroy).
"""
from __future__ import annotations

import ctypes
from ctypes import c_int32, c_int64, c_size_t, c_void_p

from . import _lib
from ._lib import check, load

TORCH_DTYPE_NAMES = {"bf16": "bfloat16", "fp32": "float32"}


def _i32arr(vals):
    return (c_int32 * len(vals))(*[int(v) for v in vals])


def _desc(dims, acts, tokens, dtype, need_input_grad=False, bucket_layers=1, max_temp_bytes=0,
          world_size=1, rank=0, comm_enabled=True, nccl_max_ctas=0, wait_timeout_ms=0, comm_priority=0,
          comm_chunk_bytes=0, comm_model_gbps=0, engine_ctas=0, average_over=0):
    keep = {}
    d = _lib.StackDesc()
    d.num_layers = len(acts)
    keep["dims"] = _i32arr(dims)
    keep["acts"] = _i32arr([_lib.ACTS[a] if isinstance(a, str) else a for a in acts])
    d.dims = ctypes.cast(keep["dims"], ctypes.POINTER(c_int32))
    d.acts = ctypes.cast(keep["acts"], ctypes.POINTER(c_int32))
    d.tokens = int(tokens)
    d.dtype = _lib.DTYPES[dtype]
    d.need_input_grad = int(bool(need_input_grad))
    d.bucket_layers = int(bucket_layers)
    d.max_temp_bytes = int(max_temp_bytes)
    d.world_size = int(world_size)
    d.rank = int(rank)
    d.comm_enabled = int(bool(comm_enabled))
    d.nccl_max_ctas = int(nccl_max_ctas)
    d.wait_timeout_ms = int(wait_timeout_ms)
    d.comm_priority = int(comm_priority)
    d.comm_chunk_bytes = int(comm_chunk_bytes)
    d.comm_model_gbps = int(comm_model_gbps)
    d.engine_ctas = int(engine_ctas)
    d.average_over = int(average_over)
    return d, keep


def query_sizes(dims, acts, tokens, dtype="bf16", bucket_layers=1):
    d, _keep = _desc(dims, acts, tokens, dtype, bucket_layers=bucket_layers)
    ws, gb = c_size_t(), c_size_t()
    check(load().ooo_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)))
    return ws.value, gb.value


def grad_offsets(dims, acts, tokens, dtype="bf16"):
    d, _keep = _desc(dims, acts, tokens, dtype)
    L = len(acts)
    out = (c_int64 * (2 * L))()
    check(load().ooo_grad_offsets(ctypes.byref(d), out))
    return [(out[2 * i], out[2 * i + 1]) for i in range(L)]


def schedule_order(L: int, kind: str = "first_k", k: int = 0, need_input_grad: bool = False) -> list:
    ops = (c_int32 * (2 * L))()
    n = c_int32()
    check(load().ooo_schedule_order(int(L), _lib.schedule(kind, k), int(bool(need_input_grad)), ops,
                                    ctypes.byref(n)))
    return list(ops[: n.value])


def max_k(m_fwd: int, m_dO: list, m_dW: list, mxm: int) -> int:
    L = len(m_dO)
    a = (c_int64 * L)(*m_dO)
    b = (c_int64 * L)(*m_dW)
    return int(load().ooo_max_k(L, int(m_fwd), a, b, int(mxm)))


def deferral_bytes(dims, acts, tokens, dtype, k) -> int:
    d, _keep = _desc(dims, acts, tokens, dtype)
    return int(load().ooo_deferral_bytes(ctypes.byref(d), int(k)))


def engine_plan(dims, acts, tokens, kind="first_k", k=0, fused=True, workers=0, need_input_grad=False,
                bucket_layers=1, world_size=1):
    """The engine's planned tile queue for one step (host only): list of
    (kind, layer, first_row, rows, col_tiles) with kind 'F'/'dO'/'dW'/'copy',
    and whether it is a topological order of the step's dependencies."""
    d, _keep = _desc(dims, acts, tokens, "bf16", need_input_grad=need_input_grad,
                     bucket_layers=bucket_layers, world_size=world_size)
    cap = 4096
    out = (c_int32 * (5 * cap))()
    n, topo = c_int32(), c_int32()
    check(load().ooo_engine_plan(ctypes.byref(d), _lib.schedule(kind, k), int(bool(fused)), int(workers), out, cap,
                                 ctypes.byref(n), ctypes.byref(topo)))
    names = {0: "F", 1: "dO", 2: "dW", 3: "copy"}
    ops = [(names[out[5 * j]], out[5 * j + 1], out[5 * j + 2], out[5 * j + 3], out[5 * j + 4])
           for j in range(min(n.value, cap))]
    return ops, bool(topo.value)


def region_schedule(t_main, t_sub, speedup, ready, last_region=None, nbytes=None, mxm=0):
    """Algorithm 1 (§4.1) + the P:162 memory bound, computed by the
    library (``ooo_region_schedule``).  t_sub / speedup are [K][N] nested
    lists.  Returns (S, k_pre): S[i] = candidate indices of region i in
    schedule order."""
    N, K = len(t_main), len(ready)
    dbl = lambda v: (ctypes.c_double * max(1, len(v)))(*v)  # noqa: E731
    flat = lambda m: [float(x) for row in m for x in row]  # noqa: E731
    reg = (c_int32 * max(1, K))()
    order = (c_int32 * max(1, K))()
    kp = c_int32()
    last = _i32arr(last_region) if last_region is not None else None
    nb = (ctypes.c_int64 * max(1, K))(*nbytes) if nbytes is not None else None
    check(load().ooo_region_schedule(int(N), dbl(t_main), int(K), dbl(flat(t_sub)), dbl(flat(speedup)),
                                     dbl(ready), last, nb, int(mxm), reg, order, ctypes.byref(kp)))
    S = [[] for _ in range(N)]
    for j in range(K):
        S[reg[order[j]]].append(order[j])
    return S, kp.value


def comm_schedule(ready, dur, prio, policy="priority", fifo_rank=None):
    """The library's all-reduce chunk issue order (``ooo_comm_schedule``,
    §5.1).  dur[b] = list of bucket b's chunk durations.  Returns
    (order as [(b, c), ...], done[b])."""
    B = len(ready)
    nch = [len(d) for d in dur]
    tot = sum(nch)
    flat = [float(x) for d in dur for x in d]
    ob, oc = (c_int32 * max(1, tot))(), (c_int32 * max(1, tot))()
    done = (ctypes.c_double * max(1, B))()
    fr = _i32arr(fifo_rank) if fifo_rank is not None else None
    check(load().ooo_comm_schedule(int(B), (ctypes.c_double * max(1, B))(*ready), _i32arr(nch),
                                   (ctypes.c_double * max(1, tot))(*flat), _i32arr(prio), fr,
                                   {"fifo": 0, "priority": 1}[policy], ob, oc, done))
    return [(ob[j], oc[j]) for j in range(tot)], list(done[:B])


def get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(_lib.UNIQUE_ID_BYTES)
    check(load().ooo_get_unique_id(buf))
    return buf.raw


def broadcast_unique_id(group=None) -> bytes:
    """Rank 0 creates the NCCL bootstrap id; torch.distributed broadcasts it."""
    import torch.distributed as dist
    obj = [get_unique_id() if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=0, group=group)
    return obj[0]


def _record(r) -> dict:
    return {"kind": _lib.KIND_NAMES.get(r.kind, r.kind), "layer": r.layer, "stream": r.stream, "grid": r.grid,
            "flops": r.flops, "bytes": r.bytes, "ms": r.ms, "start_ms": r.start_ms}


def _stream_handle(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


class StepGraph:
    """A captured [ooo_backward; ooo_forward] step (pre-compiled issue, §4.2)."""

    def __init__(self, stack, handle, keep):
        self._stack = stack
        self._h = handle
        self._keep = keep

    def launch(self, stream=None):
        check(load().ooo_graph_launch(self._h, _stream_handle(stream)))

    def upload(self, X_host, dY_host, copy_stream):
        """Host -> device copy of the step's inputs (pinned CPU tensors) into
        the graph's buffers, on copy_stream (ooo_graph_upload)."""
        check(load().ooo_graph_upload(self._h, c_void_p(X_host.data_ptr()), c_void_p(dY_host.data_ptr()),
                                      _stream_handle(copy_stream)))

    def launch_host(self, Y_host, stream=None, copy_stream=None):
        """Launch after the upload, then copy Y back into the pinned CPU
        tensor Y_host on copy_stream (ooo_graph_launch_host)."""
        check(load().ooo_graph_launch_host(self._h, c_void_p(Y_host.data_ptr()), _stream_handle(stream),
                                           _stream_handle(copy_stream)))

    def set_timing_slots(self, slots: int):
        """The next `slots` launches each record their own per-kernel CUDA
        events (graph captured with the stack's timing on)."""
        check(load().ooo_graph_set_timing_slots(self._h, int(slots)))

    def timing(self) -> list:
        """Per-launch records of the timed launches: a list (one entry per
        launch) of lists of record dicts (see OooStack.timing)."""
        n, per = c_int32(), c_int32()
        check(load().ooo_graph_timing_read(self._h, None, 0, ctypes.byref(n), ctypes.byref(per)))
        recs = (_lib.LaunchRecord * max(1, n.value))()
        check(load().ooo_graph_timing_read(self._h, recs, n.value, ctypes.byref(n), ctypes.byref(per)))
        flat = [_record(r) for r in recs[: n.value]]
        p = max(1, per.value)
        return [flat[i: i + p] for i in range(0, len(flat), p)]

    def close(self):
        if self._h:
            load().ooo_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class OooStack:
    """One rank's stack: ooo_create_stack over caller-owned torch tensors."""

    def __init__(self, dims, acts, tokens, W, b, dtype="bf16", need_input_grad=False, bucket_layers=1,
                 max_temp_bytes=0, world_size=1, rank=0, unique_id: bytes | None = None,
                 comm_enabled=True, nccl_max_ctas=0, wait_timeout_ms=0, comm_priority=0, comm_chunk_bytes=0,
                 comm_model_gbps=0, engine_ctas=0, average_over=0):
        """unique_id: the NCCL bootstrap id (broadcast_unique_id); required
        for world_size > 1; with world_size == 1 it makes a one-rank
        communicator that runs the N > 1 data plane on one GPU."""
        import torch
        lib = load()
        self.dims = [int(x) for x in dims]
        self.acts = list(acts)
        self.L = len(self.acts)
        self.tokens = int(tokens)
        self.dtype = dtype
        self.tdtype = getattr(torch, TORCH_DTYPE_NAMES[dtype])
        self.need_input_grad = bool(need_input_grad)
        self.world_size = int(world_size)
        self.rank = int(rank)
        if len(W) != self.L or len(b) != self.L:
            raise ValueError("need L weights and biases")
        for i, (w, bb) in enumerate(zip(W, b)):
            if w.dtype != self.tdtype or bb.dtype != self.tdtype:
                raise ValueError(f"layer {i + 1}: W/b dtype must be {self.tdtype}")
            if tuple(w.shape) != (self.dims[i], self.dims[i + 1]) or tuple(bb.shape) != (self.dims[i + 1],):
                raise ValueError(f"layer {i + 1}: bad W/b shape")
            if not (w.is_cuda and w.is_contiguous() and bb.is_cuda and bb.is_contiguous()):
                raise ValueError(f"layer {i + 1}: W/b must be contiguous CUDA tensors")
        self.W, self.b = list(W), list(b)
        self.device = W[0].device
        d, keep = _desc(self.dims, self.acts, self.tokens, dtype, need_input_grad, bucket_layers,
                        max_temp_bytes, world_size, rank, comm_enabled, nccl_max_ctas, wait_timeout_ms,
                        comm_priority, comm_chunk_bytes, comm_model_gbps, engine_ctas, average_over)
        ws, gb = c_size_t(), c_size_t()
        check(lib.ooo_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)))
        self.workspace = torch.empty(ws.value, dtype=torch.uint8, device=self.device)
        self.grads_buf = torch.zeros(gb.value, dtype=torch.uint8, device=self.device)
        keep["W"] = (c_void_p * self.L)(*[w.data_ptr() for w in self.W])
        keep["b"] = (c_void_p * self.L)(*[x.data_ptr() for x in self.b])
        d.W = ctypes.cast(keep["W"], ctypes.POINTER(c_void_p))
        d.b = ctypes.cast(keep["b"], ctypes.POINTER(c_void_p))
        d.grads = self.grads_buf.data_ptr()
        d.workspace = self.workspace.data_ptr()
        if self.world_size > 1 and unique_id is None:
            raise ValueError("world_size > 1 needs the 128-byte NCCL unique id (broadcast_unique_id)")
        if unique_id is not None:
            if len(unique_id) != _lib.UNIQUE_ID_BYTES:
                raise ValueError("the NCCL unique id has 128 bytes")
            keep["uid"] = ctypes.create_string_buffer(unique_id, _lib.UNIQUE_ID_BYTES)
            d.nccl_unique_id = ctypes.cast(keep["uid"], c_void_p)
        self._keep = keep
        self._desc = d
        h = c_void_p()
        check(lib.ooo_create_stack(ctypes.byref(d), ctypes.byref(h)))
        self._h = h
        offs = (c_int64 * (2 * self.L))()
        check(lib.ooo_grad_offsets(ctypes.byref(d), offs))
        g = self.grads_buf.view(self.tdtype)
        self.dW, self.db = [], []
        for i in range(self.L):
            ow, ob = offs[2 * i], offs[2 * i + 1]
            din, dout = self.dims[i], self.dims[i + 1]
            self.dW.append(g[ow: ow + din * dout].view(din, dout))
            self.db.append(g[ob: ob + dout])

    # ---- the path ---------------------------------------------------------
    def _check_act(self, t, rows, cols, name):
        if t.dtype != self.tdtype or tuple(t.shape) != (rows, cols) or not t.is_contiguous() or not t.is_cuda:
            raise ValueError(f"{name}: expected contiguous CUDA {self.tdtype} [{rows}, {cols}]")

    def forward(self, X, Y=None, stream=None):
        import torch
        self._check_act(X, self.tokens, self.dims[0], "X")
        if Y is None:
            Y = torch.empty(self.tokens, self.dims[-1], dtype=self.tdtype, device=self.device)
        self._check_act(Y, self.tokens, self.dims[-1], "Y")
        check(load().ooo_forward(self._h, c_void_p(X.data_ptr()), c_void_p(Y.data_ptr()),
                                 _stream_handle(stream)))
        return Y

    def backward(self, dY, kind="first_k", k=0, dX=None, stream=None):
        self._check_act(dY, self.tokens, self.dims[-1], "dY")
        if dX is not None:
            self._check_act(dX, self.tokens, self.dims[0], "dX")
        check(load().ooo_backward(self._h, c_void_p(dY.data_ptr()), _lib.schedule(kind, k),
                                  c_void_p(dX.data_ptr() if dX is not None else None),
                                  _stream_handle(stream)))

    def join(self, stream=None):
        check(load().ooo_join(self._h, _stream_handle(stream)))

    def comm_issue_order(self) -> list:
        """(bucket, chunk) issue order of the last enqueued step's all-reduces."""
        n = c_int32()
        check(load().ooo_comm_issue_order(self._h, None, None, 0, ctypes.byref(n)))
        b, c = (c_int32 * max(1, n.value))(), (c_int32 * max(1, n.value))()
        check(load().ooo_comm_issue_order(self._h, b, c, n.value, ctypes.byref(n)))
        return [(b[j], c[j]) for j in range(n.value)]

    def allreduce_buckets(self, stream=None):
        """Every bucket's all-reduce back to back on the stack's own
        communicator (stand-alone S[dW] time; sums `grads` in place again)."""
        check(load().ooo_allreduce_buckets(self._h, _stream_handle(stream)))

    def graph(self, X, Y, dY, kind="first_k", k=0, dX=None) -> StepGraph:
        self._check_act(X, self.tokens, self.dims[0], "X")
        self._check_act(Y, self.tokens, self.dims[-1], "Y")
        self._check_act(dY, self.tokens, self.dims[-1], "dY")
        h = c_void_p()
        check(load().ooo_graph_create(self._h, c_void_p(X.data_ptr()), c_void_p(Y.data_ptr()),
                                      c_void_p(dY.data_ptr()), _lib.schedule(kind, k),
                                      c_void_p(dX.data_ptr() if dX is not None else None), ctypes.byref(h)))
        return StepGraph(self, h, (X, Y, dY, dX))

    def plan_regions(self, region_layers: int = 6, reps: int = 1, stream=None) -> dict:
        """Profile co-run speedups and plan OOO_SCHED_REGIONS (single-GPU
        multi-stream ooo, §4.1, Algorithm 1).  Overwrites activations and
        gradients: run forward() again before the next backward."""
        check(load().ooo_plan_regions(self._h, int(region_layers), int(reps), _stream_handle(stream)))
        return self.region_plan()

    def region_plan(self) -> dict:
        L = len(self.acts)
        n, kp, nops = c_int32(), c_int32(), c_int32()
        reg = (c_int32 * L)()
        ops = (c_int32 * (2 * L))()
        check(load().ooo_region_plan(self._h, ctypes.byref(n), ctypes.byref(kp), reg, ops, ctypes.byref(nops),
                                     None, 0))
        tm = (ctypes.c_double * max(1, n.value))()
        check(load().ooo_region_plan(self._h, None, None, None, None, None, tm, n.value))
        return {"n_regions": n.value, "k_pre": kp.value, "region_of": list(reg), "D": list(ops[: nops.value]),
                "t_main_ms": list(tm[: n.value])}

    # ---- introspection -----------------------------------------------------
    def tensor(self, kind: str, layer: int):
        """Views of internal stores: 'X' (X_i), 'Z' (Z_i; None for identity
        layers), 'dZ', 'dbpart' (fp32 [rows][d_i])."""
        import torch
        code = {"X": 0, "Z": 1, "dZ": 2, "dbpart": 3}[kind]
        p = c_void_p()
        rows = c_int64()
        check(load().ooo_tensor(self._h, code, int(layer), ctypes.byref(p), ctypes.byref(rows)))
        if not p.value:
            return None
        off = p.value - self.workspace.data_ptr()
        cols = self.dims[layer - 1] if kind == "X" else self.dims[layer]
        if kind == "dbpart":
            n = rows.value * cols * 4
            return self.workspace[off: off + n].view(torch.float32).view(rows.value, cols)
        esz = 2 if self.dtype == "bf16" else 4
        n = rows.value * cols * esz
        return self.workspace[off: off + n].view(self.tdtype).view(rows.value, cols)

    def set_timing(self, enable: bool = True):
        check(load().ooo_set_timing(self._h, int(bool(enable))))

    def timing(self) -> list:
        n = c_int32()
        check(load().ooo_timing_read(self._h, None, 0, ctypes.byref(n)))
        recs = (_lib.LaunchRecord * max(1, n.value))()
        check(load().ooo_timing_read(self._h, recs, n.value, ctypes.byref(n)))
        return [_record(r) for r in recs[: n.value]]

    def close(self):
        if getattr(self, "_h", None):
            load().ooo_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Pipeline:
    """Cross-layer model parallelism (§5.2.1): ooo_pipeline_create over
    caller-owned torch buffers.  placement 'contiguous' | 'modulo'.  Without
    unique_id the stages are SM partitions of the current GPU; with it every
    rank is one stage (n_stages = world_size) and the hand-offs are NCCL
    send / recv (world_size 1: loopback) -- include/ooo.h.  dW[i] / db[i] are
    None for layers another rank owns."""

    def __init__(self, dims, acts, tokens, W, b, group_layers, n_stages, placement="modulo", world_size=1,
                 rank=0, unique_id: bytes | None = None):
        import torch
        lib = load()
        self.dims, self.acts, self.tokens = [int(x) for x in dims], list(acts), int(tokens)
        self.L = len(self.acts)
        self.group_layers, self.n_stages = int(group_layers), int(n_stages)
        self.G = self.L // self.group_layers
        keep = {"dims": _i32arr(self.dims), "acts": _i32arr([_lib.ACTS[a] if isinstance(a, str) else a
                                                             for a in self.acts])}
        d = _lib.PipelineDesc()
        d.num_layers = self.L
        d.dims = ctypes.cast(keep["dims"], ctypes.POINTER(c_int32))
        d.acts = ctypes.cast(keep["acts"], ctypes.POINTER(c_int32))
        d.tokens = self.tokens
        d.group_layers = self.group_layers
        d.n_stages = self.n_stages
        d.placement = {"contiguous": 0, "modulo": 1}[placement]
        d.world_size, d.rank = int(world_size), int(rank)
        if unique_id is not None:
            keep["uid"] = ctypes.create_string_buffer(unique_id, _lib.UNIQUE_ID_BYTES)
            d.nccl_unique_id = ctypes.cast(keep["uid"], c_void_p)
        ws, gb = c_size_t(), c_size_t()
        check(lib.ooo_pipeline_query_sizes(ctypes.byref(d), ctypes.byref(ws), ctypes.byref(gb)))
        dev = W[0].device
        self.workspace = torch.empty(ws.value, dtype=torch.uint8, device=dev)
        self.grads_buf = torch.zeros(gb.value, dtype=torch.uint8, device=dev)
        self.W, self.b = list(W), list(b)
        keep["W"] = (c_void_p * self.L)(*[w.data_ptr() for w in self.W])
        keep["b"] = (c_void_p * self.L)(*[x.data_ptr() for x in self.b])
        d.W = ctypes.cast(keep["W"], ctypes.POINTER(c_void_p))
        d.b = ctypes.cast(keep["b"], ctypes.POINTER(c_void_p))
        d.workspace = self.workspace.data_ptr()
        d.grads = self.grads_buf.data_ptr()
        self._keep, self._desc = keep, d
        h = c_void_p()
        check(lib.ooo_pipeline_create(ctypes.byref(d), ctypes.byref(h)))
        self._h = h
        # gradient views: group j's buffer, laid out as ooo_grad_offsets of its layers
        g = self.grads_buf.view(torch.bfloat16)
        self.dW, self.db = [], []
        for j in range(self.G):
            off = c_int64()
            if lib.ooo_pipeline_grads_offset(ctypes.byref(d), j, ctypes.byref(off)) != 0:
                self.dW += [None] * self.group_layers      # another rank's group
                self.db += [None] * self.group_layers
                continue
            lo = j * self.group_layers
            offs = grad_offsets(self.dims[lo: lo + self.group_layers + 1], self.acts[lo: lo + self.group_layers],
                                self.tokens)
            base = off.value // 2
            for i, (ow, ob) in enumerate(offs):
                din, dout = self.dims[lo + i], self.dims[lo + i + 1]
                self.dW.append(g[base + ow: base + ow + din * dout].view(din, dout))
                self.db.append(g[base + ob: base + ob + dout])

    def stage_of(self, group: int) -> int:
        return int(load().ooo_pipeline_stage_of(self._h, int(group)))

    def graph(self, X, dY, Y, fast_forward=True) -> StepGraph:
        h = c_void_p()
        check(load().ooo_pipeline_graph_create(self._h, c_void_p(X.data_ptr()), c_void_p(dY.data_ptr()),
                                               c_void_p(Y.data_ptr()), int(bool(fast_forward)), ctypes.byref(h)))
        return StepGraph(self, h, (X, dY, Y))

    def close(self):
        if getattr(self, "_h", None):
            load().ooo_pipeline_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
