"""Cross-layer model parallelism on SM-partition stages (§5.2.1, Fig. 5):
iteration time of conventional backprop vs gradient fast-forwarding, with
contiguous vs modulo allocation of transformer blocks (groups of 6 layers),
against the unpartitioned stack on the whole GPU.  All graphs timed in
interleaved runs.
    python tools/pipeline_bench.py [C2] [n ...]            # n SM-partition stages on one GPU
    python tools/pipeline_bench.py C2 loopback             # one-rank NCCL: every hand-off a self send/recv
    torchrun --nproc-per-node N --master-addr 127.0.0.1 tools/pipeline_bench.py C2   # one stage per GPU, NCCL
"""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack, Pipeline  # noqa: E402


def interleaved(graphs, stream, steps=20, reps=3):
    for g in graphs:
        for _ in range(3):
            g.launch(stream)
    ev = [[] for _ in graphs]
    torch.cuda.synchronize()
    for _ in range(reps):
        for j, g in enumerate(graphs):
            a, b = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record(stream)
            for _ in range(steps):
                g.launch(stream)
            b.record(stream)
            ev[j].append((a, b))
    torch.cuda.synchronize()
    return [sum(a.elapsed_time(b) for a, b in e) / (steps * len(e)) for e in ev]


def multi_rank(cfg, world, rank, loopback=False):
    """One stage per rank, hand-offs over NCCL (world 1: loopback)."""
    import torch.distributed as dist
    from paper_conf_eurosys_ohlks22_b200.stack import broadcast_unique_id, get_unique_id
    dev = torch.device("cuda", int(os.environ.get("LOCAL_RANK", "0")))
    torch.cuda.set_device(dev)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    stream = torch.cuda.current_stream()
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    Y = torch.empty(cfg.tokens, cfg.dims[-1], dtype=X.dtype, device=dev)
    keys, graphs, pipes = [], [], []
    for pl in ("contiguous", "modulo"):
        uid = broadcast_unique_id() if world > 1 else get_unique_id()
        p = Pipeline(cfg.dims, cfg.acts, cfg.tokens, W, b, group_layers=6, n_stages=world, placement=pl,
                     world_size=world, rank=rank, unique_id=uid)
        pipes.append(p)
        for ff in (False, True):
            keys.append((pl, ff))
            graphs.append(p.graph(X, dY, Y, fast_forward=ff))
    if world > 1:
        dist.barrier()
    t = interleaved(graphs, stream)
    if world > 1:
        tt = torch.tensor(t, dtype=torch.float64, device=dev)
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t = tt.tolist()
    res = {"config": cfg.name, "ranks": world, "mode": "nccl loopback" if loopback else "nccl",
           "group_layers": 6}
    for (pl, ff), ms in zip(keys, t):
        res[f"{pl}_{'fast_forward' if ff else 'conventional'}_ms"] = round(ms, 4)
    if rank == 0:
        print(json.dumps(res), flush=True)
    for g in graphs:
        g.close()
    for p in pipes:
        p.close()
    if world > 1:
        dist.destroy_process_group()


def main():
    args = [a for a in sys.argv[1:]]
    cfg = configs.get(args[0] if args else "C2")
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world > 1 or "loopback" in args:
        return multi_rank(cfg, world, int(os.environ.get("RANK", "0")), loopback=world == 1)
    ns = [int(a) for a in args[1:]] or [2, 4]
    dev = torch.device("cuda")
    stream = torch.cuda.current_stream()
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    Y = torch.empty(cfg.tokens, cfg.dims[-1], dtype=X.dtype, device=dev)
    stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b)
    stk.forward(X, Y)
    whole = stk.graph(X, Y, dY, "first_k", 0)
    for n in ns:
        keys, graphs, pipes = [], [], []
        for pl in ("contiguous", "modulo"):
            p = Pipeline(cfg.dims, cfg.acts, cfg.tokens, W, b, group_layers=6, n_stages=n, placement=pl)
            pipes.append(p)
            for ff in (False, True):
                keys.append((pl, ff))
                graphs.append(p.graph(X, dY, Y, fast_forward=ff))
        t = interleaved([whole] + graphs, stream)
        res = {"config": cfg.name, "stages": n, "group_layers": 6, "sms_per_stage": 148 // n // 2 * 2,
               "unpartitioned_whole_gpu_ms": round(t[0], 4)}
        for (pl, ff), ms in zip(keys, t[1:]):
            res[f"{pl}_{'fast_forward' if ff else 'conventional'}_ms"] = round(ms, 4)
        base = res["contiguous_conventional_ms"]
        for k in list(res):
            if k.endswith("_ms") and k.startswith(("contiguous", "modulo")):
                res[k.replace("_ms", "_speedup")] = round(base / res[k], 3)
        print(json.dumps(res), flush=True)
        for g in graphs:
            g.close()
        for p in pipes:
            p.close()


if __name__ == "__main__":
    main()
