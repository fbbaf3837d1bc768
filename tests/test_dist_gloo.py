"""world_size-2 data-parallel host logic on CPU (gloo), ``-m "not gpu"``.

* S[dW_i] semantics (§5.1, reading Q9): each rank pre-scales its
  gradient by 1/N and rounds it to the bucket dtype; the sum all-reduce of
  those buckets equals the oracle's N-rank average, which equals the
  full-batch gradient / N.
* The collective rule of the ABI: the schedule D (and so the NCCL issue order)
  depends only on (L, k) -- every rank computes the same list.
* The NCCL bootstrap id is broadcast over torch.distributed (a failure is
  a test failure: ncclGetUniqueId needs no GPU).
* The rest of the N > 1 host plan is identical on every rank: the engine's
  tile queue for a communicating stack (fwd_gate 2: F_i on its bucket's
  all-reduce) and its topological order, the prioritised all-reduce chunk
  order (NEXT-4), and the model-parallel pipeline's per-rank ownership
  (NEXT-3: every group owned by exactly one rank).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle import layers as O
from oracle import schedule as S
from paper_conf_eurosys_ohlks22_b200 import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


DIMS = (64, 128, 64, 128)
ACTS = ("gelu", "id", "gelu")   # ReLU sign flips make bf16-vs-fp64 errors O(1)
M = 24


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        W, b = synth.weights(DIMS, ACTS, "bf16")
        X = synth.x_shard(M, DIMS[0], rank, "bf16")
        dY = synth.dy_shard(M, DIMS[-1], rank, "bf16")
        L = len(ACTS)
        D = S.reverse_first_k(L, 2)
        st = O.forward(X, W, b, list(ACTS), "bf16")
        bs = O.run_backward(D, st, dY, W, list(ACTS), "bf16")
        out = []
        for i in range(1, L + 1):
            # bucket contents on this rank: st(dW_i / N), st(db_i / N)
            bucket = np.concatenate([O.round_bf16(bs.dW[i] / world).ravel(), O.round_bf16(bs.db[i] / world)])
            t = torch.from_numpy(bucket)
            dist.all_reduce(t)                       # fp64 sum, one rounding at the end
            out.append(O.round_bf16(t.numpy()))
        # collective rule: identical D on every rank
        from paper_conf_eurosys_ohlks22_b200 import _lib, stack
        if os.path.exists(_lib.LIB_PATH):
            Ds = [None] * world
            dist.all_gather_object(Ds, stack.schedule_order(L, "first_k", 2))
            assert all(d == Ds[0] for d in Ds)
            uid = stack.broadcast_unique_id()
            ids = [None] * world
            dist.all_gather_object(ids, uid)
            assert len(uid) == 128 and all(x == ids[0] for x in ids)
            # the engine queue of a communicating BERT-block stack: identical, topological
            dims = [256, 256, 256, 256, 256, 1024, 256] * 1
            acts = ["id", "id", "id", "id", "gelu", "id"]
            q_ = stack.engine_plan(dims, acts, 512, "first_k", 2, fused=True, bucket_layers=2, world_size=world)
            qs = [None] * world
            dist.all_gather_object(qs, q_)
            assert q_[1] and all(x == qs[0] for x in qs)
            # the prioritised chunk order from identical predicted ready times
            co = stack.comm_schedule([30.0, 10.0, 0.0], [[4.0, 4.0], [2.0], [3.0, 3.0, 1.0]], [1, 3, 5], "priority")
            cos = [None] * world
            dist.all_gather_object(cos, co)
            assert all(x == cos[0] for x in cos)
            # pipeline ownership: every group on exactly one rank (modulo placement)
            import ctypes
            d = _lib.PipelineDesc()
            pd, pa = stack._i32arr([128] * 9), stack._i32arr([0] * 8)
            d.num_layers, d.tokens, d.group_layers, d.n_stages, d.placement = 8, 64, 2, world, 1
            d.dims = ctypes.cast(pd, ctypes.POINTER(ctypes.c_int32))
            d.acts = ctypes.cast(pa, ctypes.POINTER(ctypes.c_int32))
            d.world_size, d.rank = world, rank
            idbuf = ctypes.create_string_buffer(uid, 128)
            d.nccl_unique_id = ctypes.cast(idbuf, ctypes.c_void_p)
            mine = []
            for j in range(4):
                o = ctypes.c_int64()
                if _lib.load().ooo_pipeline_grads_offset(ctypes.byref(d), j, ctypes.byref(o)) == 0:
                    mine.append(j)
            owners = [None] * world
            dist.all_gather_object(owners, mine)
            assert sorted(j for m in owners for j in m) == [0, 1, 2, 3]
            assert owners[rank] == [j for j in range(4) if j % world == rank]
        q.put((rank, out))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))


def test_two_rank_gradient_sync_matches_oracle_average():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
    W, b = synth.weights(DIMS, ACTS, "bf16")
    Xs = [synth.x_shard(M, DIMS[0], r, "bf16") for r in range(world)]
    dYs = [synth.dy_shard(M, DIMS[-1], r, "bf16") for r in range(world)]
    ref = O.dp_step(Xs, dYs, W, b, list(ACTS), S.reverse_first_k(3, 2), "bf16")
    for i in range(3):
        want = np.concatenate([ref.gW[i].ravel(), ref.gb[i]])
        for r in range(world):
            assert np.array_equal(res[r][i], want)
    # and the average is the full-batch gradient / N up to bf16 rounding
    full = O.dp_step([np.concatenate(Xs)], [np.concatenate(dYs)], W, b, list(ACTS),
                     S.reverse_first_k(3, 2), "fp64")
    for i in range(3):
        assert O.rel_fro(ref.gW[i], full.gW[i] / world) < 2e-2
