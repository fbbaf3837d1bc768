#!/usr/bin/env python
"""Benchmark of the ooo-backprop data-parallel hot path (one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--k auto|INT]
    torchrun --nproc-per-node N bench.py --gpus N ...     (N > 1, NCCL)
    python bench.py --impl reference ...                   (the CPU oracle arm)

A step = one training iteration of the paper's problem statement (§2,
P:81-95): backward(t) of the whole dense stack (dO chain on the high-priority
stream, dW ops in Algorithm 2 "reverse first-k" order on the low-priority
stream, one NCCL all-reduce per gradient bucket) followed by forward(t+1),
each F_i gated on its layer's synchronised gradient -- captured once as a
CUDA graph (pre-compiled issue, §4.2) and replayed.  Inputs are synthetic
(seeded, shaped like BASELINE.json's configs; reading Q13) and resident in
HBM for `value`; `e2e` adds the per-step host->device copy of X, dY and the
device->host read of Y through the same public API.

The oracle (oracle/) is imported only by the cpu_baseline leg and by
--impl reference.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "train iters/sec at 1/2/4/8 B200; exposed allreduce ms/iter; ooo vs in-order"
UNIT = "iters/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C2", help="C1..C5 or a config name (default: configs[1] = BERT-base stack)")
    ap.add_argument("--k", default="auto", help="reverse first-k parameter, or 'auto' (paper's search, P:212-214)")
    ap.add_argument("--regions", type=int, default=6,
                    help="N = 1: also plan the single-GPU multi-stream schedule (Algorithm 1, §4.1) with regions of "
                         "this many layers and time the better of it and reverse first-k; 0 = off")
    ap.add_argument("--emulate-n", type=int, default=8,
                    help="N = 1: also measure exposed communication with an EMULATED ring all-reduce of this many "
                         "ranks (comm stream held for 2(n-1)/n x bucket bytes / 900 GB/s + 8 us per bucket, "
                         "16-SM NCCL reserve); 0 = off")
    ap.add_argument("--bucket-layers", type=int, default=6,
                    help="consecutive layers per all-reduce bucket (6 = one transformer block: per-call latency; "
                         "measured with the emulated all-reduce, DESIGN.md §5c)")
    ap.add_argument("--nccl-max-ctas", type=int, default=0)
    ap.add_argument("--comm-priority", type=int, default=0,
                    help="1: prioritised, partitioned all-reduce issue (Fig. 4(b), P:180) for the timed stack")
    ap.add_argument("--comm-chunk-mb", type=float, default=4.0,
                    help="all-reduce partition size (MB) of the prioritised communication")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample-tokens", type=int, default=0)
    ap.add_argument("--runs", type=int, default=10,
                    help="the K timed steps run as this many back-to-back runs (mean +- s.e. over runs), "
                         "interleaved with as many in_order runs")
    return ap.parse_args()


# --------------------------------------------------------------- helpers
def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": d["hbm_gbs"], "bf16_tflops": d["bf16_tflops"],
                "bf16_tflops_sustained": d.get("bf16_tflops_sustained", d["bf16_tflops"]), "source": "measured"}
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "source": "fallback"}


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                                       "-lms", "100", "-i", str(self.gpu)],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        self.lines = []
        if self.p is not None:
            time.sleep(0.15)
            self.p.terminate()
            try:
                out, _ = self.p.communicate(timeout=5)
            except Exception:
                self.p.kill()
                out = ""
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in self.lines:
            f = [x.strip() for x in l.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx = float(f[2])
            except ValueError:
                continue
            for n, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(n)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        loaded = [x for x in sm if x > 0.5 * max(sm)] or sm
        return {"sm_mhz": statistics.median(loaded), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


def dist_setup(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            raise SystemExit("--gpus N > 1 must be launched with torchrun --nproc-per-node N")
    return world, rank, local


def time_cpu_oracle(cfg, sample_tokens: int):
    """The fp64 oracle (bf16 storage mode) as it stands, one forward+backward
    of `sample_tokens` rows of this config; returns (seconds, threads)."""
    import numpy as np
    from oracle import layers as O
    from oracle import schedule as S
    from paper_conf_eurosys_ohlks22_b200 import synth
    try:
        from threadpoolctl import threadpool_info
        threads = max((i.get("num_threads", 1) for i in threadpool_info()), default=1)
    except Exception:
        threads = len(os.sched_getaffinity(0))
    rng = np.random.default_rng(1)
    dt = "bf16" if cfg.dtype == "bf16" else "fp32"
    W = [synth.to_storage(rng.standard_normal((cfg.dims[i], cfg.dims[i + 1])) / math.sqrt(cfg.dims[i]), dt)
         for i in range(cfg.L)]
    b = [synth.to_storage(0.1 * rng.standard_normal(cfg.dims[i + 1]), dt) for i in range(cfg.L)]
    X = synth.x_shard(sample_tokens, cfg.dims[0], 0, dt)
    dY = synth.dy_shard(sample_tokens, cfg.dims[-1], 0, dt)
    D = S.reverse_first_k(cfg.L, cfg.L)
    t0 = time.perf_counter()
    O.dp_step([X], [dY], W, b, list(cfg.acts), D, "bf16" if cfg.dtype == "bf16" else "fp64")
    return time.perf_counter() - t0, threads


def cpu_sample_tokens(cfg, requested):
    if requested:
        return requested
    # aim at ~10-30 s of fp64 work on the host cores: ~8e11 FLOP (≈ 10 s measured on the B200 hosts)
    per_token = cfg.gemm_flops() / cfg.tokens
    t = int(8e11 / per_token) // 8 * 8
    return max(8, min(cfg.tokens, t))


# ---------------------------------------------------------- reference arm
def run_reference(args):
    world, rank, _ = dist_setup(args)
    if rank != 0:
        return
    from paper_conf_eurosys_ohlks22_b200 import configs
    cfg = configs.get(args.config)
    tok = cpu_sample_tokens(cfg, args.cpu_sample_tokens)
    steps = max(1, min(args.steps, 3))
    for _ in range(min(args.warmup, 1)):
        time_cpu_oracle(cfg, min(tok, 64))
    times = []
    threads = 1
    for _ in range(steps):
        t, threads = time_cpu_oracle(cfg, tok)
        times.append(t)
    sec = statistics.mean(times)
    value = (tok / cfg.tokens) / sec        # full-config iterations per second (scaled)
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": steps, "warmup": min(args.warmup, 1), "ms_per_step": 1e3 / value, "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{cfg.name} ({cfg.note})", "tokens_per_gpu": cfg.tokens, "layers": cfg.L,
                   "parallelism": f"dp{args.gpus}"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": f"one fp64 forward+backward of {tok} of {cfg.tokens} tokens/GPU, "
                                   f"scaled by {tok}/{cfg.tokens}; {steps} step(s), mean"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ ours
def split_runs(steps: int, runs: int) -> list:
    """K timed steps as R back-to-back runs (mean +- s.e. over runs)."""
    runs = max(1, min(runs, steps))
    base, extra = divmod(steps, runs)
    return [base + (1 if r < extra else 0) for r in range(runs)]


def dp_selfcheck(world, rank, dev, stream, dist, bucket_layers=2):
    """N > 1: the library's data plane checks itself before anything is timed.
    A small stack with the bit-exact NCCL setting SURVEY §8e pins
    (NCCL_ALGO=Ring NCCL_PROTO=Simple), per-rank seeded shards (synth), shared
    W: (1) in_order and ooo_first_k(2) give bit-identical gradients on every
    rank (fixed all-reduce order); (2) every rank holds the same bytes
    (gathered sha256); (3) the all-reduced gradient equals the sum over ranks
    of each rank's local 1/N-scaled gradient (comm-off stack of the same
    library, summed in fp32 by torch.distributed) within the bf16 gate --
    i.e. every bucket was really reduced across ranks before F_i read it.
    Runs through captured steps (eager fused steps are refused at N > 1).
    At N = 1 the same check runs on a one-rank communicator (the N > 1 data
    plane on one GPU), so its code is exercised by every single-GPU bench."""
    import hashlib

    import torch
    from paper_conf_eurosys_ohlks22_b200 import synth
    from paper_conf_eurosys_ohlks22_b200.stack import OooStack, broadcast_unique_id, get_unique_id
    uid = broadcast_unique_id if world > 1 else get_unique_id
    dims, acts, M = [256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"], 264
    Wn, bn = synth.weights(dims, acts, "bf16")
    tb = lambda a: torch.from_numpy(a).to(torch.bfloat16).to(dev).contiguous()  # noqa: E731
    W, b = [tb(w) for w in Wn], [tb(x) for x in bn]
    X = tb(synth.x_shard(M, dims[0], rank, "bf16"))
    dY = tb(synth.dy_shard(M, dims[-1], rank, "bf16"))
    Y = torch.empty(M, dims[-1], dtype=torch.bfloat16, device=dev)
    saved = {k: os.environ.get(k) for k in ("NCCL_ALGO", "NCCL_PROTO")}
    os.environ.update({"NCCL_ALGO": "Ring", "NCCL_PROTO": "Simple"})
    try:
        on = OooStack(dims, acts, M, W, b, bucket_layers=bucket_layers, world_size=world, rank=rank,
                      unique_id=uid())
        off = OooStack(dims, acts, M, W, b, bucket_layers=bucket_layers, world_size=world, rank=rank,
                       unique_id=uid(), comm_enabled=False)
    finally:
        for k, v in saved.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
    out = {}
    for name, stk in (("on", on), ("off", off)):
        for sch in (("in_order", 0), ("first_k", 2)):
            stk.forward(X, Y)
            g = stk.graph(X, Y, dY, *sch)
            g.launch(stream)
            torch.cuda.synchronize()
            out[(name, sch[0])] = stk.grads_buf.clone()
            g.close()
    bit_exact = bool(torch.equal(out[("on", "in_order")], out[("on", "first_k")]) and
                     torch.equal(out[("off", "in_order")], out[("off", "first_k")]))
    h = hashlib.sha256(out[("on", "first_k")].cpu().numpy().tobytes()).hexdigest()
    hs = [h] * world
    local = out[("off", "first_k")].view(torch.bfloat16).float()
    if world > 1:
        dist.all_gather_object(hs, h)
        dist.all_reduce(local)                          # fp32 sum of the ranks' 1/N-scaled local gradients
    got = out[("on", "first_k")].view(torch.bfloat16).float()
    errs = []
    offs_w = [(w.data_ptr() - on.grads_buf.data_ptr()) // 2 for w in on.dW]
    offs_b = [(x.data_ptr() - on.grads_buf.data_ptr()) // 2 for x in on.db]
    for i in range(len(acts)):
        for o, n in ((offs_w[i], on.dW[i].numel()), (offs_b[i], on.db[i].numel())):
            r = local[o: o + n]
            errs.append(float((got[o: o + n] - r).norm() / r.norm().clamp_min(1e-30)))
    on.close()
    off.close()
    res = {"stack": f"{len(acts)} layers {dims}, {M} tokens/rank, bucket_layers {bucket_layers}",
           "nccl_env": "NCCL_ALGO=Ring NCCL_PROTO=Simple", "in_order_eq_first_k_bit_exact": bit_exact,
           "ranks_identical": len(set(hs)) == 1, "max_rel_err_vs_sum_of_local_grads": max(errs)}
    res["ok"] = bool(bit_exact and res["ranks_identical"] and res["max_rel_err_vs_sum_of_local_grads"] <= 1e-2)
    return res


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)
    import torch
    import torch.distributed as dist
    from paper_conf_eurosys_ohlks22_b200 import configs, synth
    from paper_conf_eurosys_ohlks22_b200.stack import OooStack, broadcast_unique_id, deferral_bytes

    world, rank, local = dist_setup(args)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    cfg = configs.get(args.config)
    dt = cfg.dtype
    M = cfg.tokens
    L = cfg.L
    peaks = load_peaks()
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(xs):
        """Elementwise max over ranks of a list of floats (device-timed values)."""
        if world == 1:
            return list(xs)
        t = torch.tensor(list(xs), dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return t.tolist()

    try:
        selfcheck = dp_selfcheck(world, rank, dev, stream, dist)
    except Exception as e:  # noqa: BLE001 -- reported in the line (and fatal at N > 1 below)
        selfcheck = {"ok": False, "error": str(e)[:300]}
    if not selfcheck.get("ok"):
        print(f"WARNING: data-parallel self-check failed: {selfcheck}", file=sys.stderr, flush=True)

    W, b = synth.weights_torch(cfg.dims, cfg.acts, dt, dev)
    uid = broadcast_unique_id() if world > 1 else None
    chunk = int(args.comm_chunk_mb * 2 ** 20)
    comm_kw = {"comm_priority": args.comm_priority, "comm_chunk_bytes": chunk if args.comm_priority else 0}
    stk = OooStack(cfg.dims, cfg.acts, M, W, b, dtype=dt, bucket_layers=args.bucket_layers,
                   world_size=world, rank=rank, unique_id=uid, nccl_max_ctas=args.nccl_max_ctas, **comm_kw)
    X = synth.activations_torch(M, cfg.dims[0], dt, dev, synth.SEED, rank, 0)
    dY = synth.activations_torch(M, cfg.dims[-1], dt, dev, synth.SEED, rank, 1)
    Y = torch.empty(M, cfg.dims[-1], dtype=X.dtype, device=dev)

    def interleaved(graphs, steps, runs, sampler=None):
        """Time `steps` launches of every graph in `graphs` as `runs`
        back-to-back runs per graph, interleaved A B A B ... (no host sync or
        idle inside the region), bracketed by barrier + synchronize; CUDA
        events on the launching stream; per-run times max over ranks.
        Returns per graph the list of per-run ms per step."""
        sizes = split_runs(steps, runs)
        ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in sizes]
              for _ in graphs]
        barrier()
        torch.cuda.synchronize()
        if sampler:
            sampler.__enter__()
        for r, n in enumerate(sizes):
            for gi, g in enumerate(graphs):
                ev[gi][r][0].record(stream)
                for _ in range(n):
                    g.launch(stream)
                ev[gi][r][1].record(stream)
        torch.cuda.synchronize()
        if sampler:
            sampler.__exit__(None, None, None)
        barrier()
        flat = [ev[gi][r][0].elapsed_time(ev[gi][r][1]) for gi in range(len(graphs)) for r in range(len(sizes))]
        flat = max_over_ranks(flat)
        return [[flat[gi * len(sizes) + r] / sizes[r] for r in range(len(sizes))] for gi in range(len(graphs))]

    def summary(per_run, steps, runs):
        sizes = split_runs(steps, runs)
        total = sum(ms * n for ms, n in zip(per_run, sizes))
        mean = total / sum(sizes)
        sem = statistics.stdev(per_run) / math.sqrt(len(per_run)) if len(per_run) > 1 else None
        return {"ms_per_step": mean, "value": 1e3 / mean, "runs": len(per_run), "run_steps": sizes,
                "run_ms_per_step": per_run, "sem_ms": sem}

    stk.forward(X, Y)
    torch.cuda.synchronize()
    graphs = {}

    def graph_for(kind, k, s=stk):
        key = (id(s), kind, k)
        if key not in graphs:
            graphs[key] = s.graph(X, Y, dY, kind, k)
        return graphs[key]

    # ---- choose k: the paper's heuristic search (§5.1) on measured throughput
    if args.k == "auto":
        from paper_conf_eurosys_ohlks22_b200.ksearch import search_k
        probe = max(5, min(20, args.steps // 2))

        g_ref = graph_for("first_k", 0)

        def tput(k):
            # throughput relative to first_k(0), the two timed interleaved
            # (ABAB): clock / power drift over the search cancels in the ratio
            # (timing each candidate alone favoured whichever ran first)
            g = graph_for("first_k", k)
            for _ in range(2):
                g.launch(stream)
            if k == 0:
                return 1.0
            a, r = interleaved([g, g_ref], probe, 2)
            return (sum(r) / len(r)) / (sum(a) / len(a))
        k_best, visited = search_k(L, tput)
    else:
        k_best, visited = int(args.k), []
    g_fk = graph_for("first_k", k_best)
    sched = ("first_k", k_best)
    # ---- N = 1: the paper's single-GPU method -- multi-stream ooo with
    # Algorithm 1 regions (§4.1), planned from profiled co-run
    # speedups; the better of it and reverse first-k (ABAB probe) is timed
    regions = None
    plan = None
    if world == 1 and args.regions > 0 and dt == "bf16":    # profiles the bf16 engine
        t0 = time.time()
        try:
            plan = stk.plan_regions(region_layers=args.regions, reps=3)   # min of 3: a steadier plan
        except Exception as e:  # noqa: BLE001 -- the bench line must still be printed
            regions = {"error": str(e)[:200]}
        t_plan = time.time() - t0
        stk.forward(X, Y)
        torch.cuda.synchronize()
    if plan is not None:
        g_reg = graph_for("regions", 0)
        for _ in range(3):
            g_reg.launch(stream)
            g_fk.launch(stream)
        pr = interleaved([g_reg, g_fk], max(20, min(60, args.steps)), 4)
        ms_r, ms_f = statistics.mean(pr[0]), statistics.mean(pr[1])
        regions = {"region_layers": args.regions, "n_regions": plan["n_regions"], "k_pre": plan["k_pre"],
                   "D": plan["D"], "plan_seconds": t_plan, "probe_ms_per_step": ms_r,
                   "first_k_probe_ms_per_step": ms_f}
        if ms_r < ms_f:
            sched = ("regions", 0)
    g_ooo = graph_for(*sched)
    g_in = graph_for("in_order", 0)
    for _ in range(max(3, args.warmup)):
        g_ooo.launch(stream)
        g_in.launch(stream)
    torch.cuda.synchronize()

    # ---- the timed region: K steps of the ooo schedule and K of in_order,
    # as R runs each, interleaved ABAB (drift hits both alike)
    sampler = ClockSampler(local)
    per = interleaved([g_ooo, g_in], args.steps, args.runs, sampler)
    clocks = sampler.summary()
    main_s, in_s = summary(per[0], args.steps, args.runs), summary(per[1], args.steps, args.runs)
    ms_ooo, ms_in = main_s["ms_per_step"], in_s["ms_per_step"]
    # secondary comparisons (own ABAB regions): the other ooo schedule and the
    # dual-stream control ooo_first_k(0) (no reordering)
    half = max(10, args.steps // 2)
    g_k0 = graph_for("first_k", 0)
    others = [("first_k", k_best)] if sched[0] == "regions" else ([("regions", 0)] if plan is not None else [])
    og = [g_k0] + [graph_for(*o) for o in others]
    for g in og:
        for _ in range(3):
            g.launch(stream)
    po = interleaved([g_ooo] + og, half, max(2, args.runs // 2))
    ms_k0 = statistics.mean(po[1])
    ms_other = {f"{o[0]}": statistics.mean(po[2 + j]) for j, o in enumerate(others)}
    ms_fk = ms_ooo if sched[0] == "first_k" else ms_other.get("first_k")
    if regions is not None and plan is not None:
        regions["ms_per_step"] = ms_ooo if sched[0] == "regions" else ms_other.get("regions")

    # ---- N > 1: exposed communication = same graphs with the all-reduce
    # skipped (comm-off stack, ABAB with the comm-on graphs), and the
    # stand-alone all-reduce of the library's own buckets on its own communicator
    exposed = None
    ar_ms = None
    if world > 1:
        stk_off = OooStack(cfg.dims, cfg.acts, M, W, b, dtype=dt, bucket_layers=args.bucket_layers,
                           world_size=world, rank=rank, unique_id=broadcast_unique_id(), comm_enabled=False,
                           nccl_max_ctas=args.nccl_max_ctas, **comm_kw)
        stk_off.forward(X, Y)
        g_off = stk_off.graph(X, Y, dY, *sched)
        g_off_in = stk_off.graph(X, Y, dY, "in_order", 0)
        for g in (g_off, g_off_in):
            for _ in range(3):
                g.launch(stream)
        pe = interleaved([g_ooo, g_off, g_in, g_off_in], half, max(2, args.runs // 2))
        m = [statistics.mean(x) for x in pe]
        exposed = {"ooo": m[0] - m[1], "in_order": m[2] - m[3], "ooo_comm_on_ms": m[0], "ooo_comm_off_ms": m[1],
                   "in_order_comm_on_ms": m[2], "in_order_comm_off_ms": m[3]}
        g_off.close()
        g_off_in.close()
        stk_off.close()
        reps = 10
        stk.allreduce_buckets(stream)                   # warm
        torch.cuda.synchronize()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            stk.allreduce_buckets(stream)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        ar_ms = max_over_ranks([e0.elapsed_time(e1) / reps])[0]
        stk.forward(X, Y)                               # grads were summed again: fresh step state
        torch.cuda.synchronize()

    # ---- N = 1: exposed communication against an EMULATED n-rank ring all-reduce
    # (no NCCL, no data moved: the comm stream is held for each bucket's ring
    # time; F_i waits for its bucket's flag exactly as at N = n)
    emulated = None
    if world == 1 and args.emulate_n > 1 and dt == "bf16":
        try:
            n, gbps, lat = args.emulate_n, 900.0, 8.0
            elt = 2
            nbk = (L + args.bucket_layers - 1) // args.bucket_layers
            ar_total = sum(2.0 * (n - 1) / n * (cfg.dims[i] * cfg.dims[i + 1] + cfg.dims[i + 1]) * elt / (gbps * 1e9) * 1e3
                           for i in range(L)) + nbk * lat * 1e-3
            ks = sorted({0, max(1, L // 24), L // 6, L // 2, L})
            gs = {}
            stacks = []
            # "prio": the same emulated link with the prioritised, partitioned
            # issue order (NEXT-4, Fig. 4(b)); the zero-time control is shared
            for label, bw, la, pr in (("on", gbps, lat, 0), ("prio", gbps, lat, 1), ("off", 1e9, 0.0, 0)):
                os.environ.update({"OOO_EMULATE_AR_N": str(n), "OOO_EMULATE_AR_GBPS": str(bw),
                                   "OOO_EMULATE_AR_LAT_US": str(la)})
                se = OooStack(cfg.dims, cfg.acts, M, W, b, dtype=dt, bucket_layers=args.bucket_layers,
                              comm_priority=pr, comm_chunk_bytes=chunk if pr else 0)
                stacks.append(se)
                se.forward(X, Y)
                for kind, k in [("in_order", 0)] + [("first_k", k) for k in ks]:
                    g = se.graph(X, Y, dY, kind, k)
                    for _ in range(3):
                        g.launch(stream)
                    gs[(label, kind, k)] = g
            for key in ("OOO_EMULATE_AR_N", "OOO_EMULATE_AR_GBPS", "OOO_EMULATE_AR_LAT_US"):
                os.environ.pop(key, None)
            keys = list(gs)
            pe = interleaved([gs[k] for k in keys], max(10, args.steps // 4), 2)
            times = {k: statistics.mean(v) for k, v in zip(keys, pe)}
            for g in gs.values():
                g.close()
            for se in stacks:
                se.close()
            sweep = {}
            for kind, k in [("in_order", 0)] + [("first_k", k) for k in ks]:
                off = times[("off", kind, k)]
                for label, tag in (("on", ""), ("prio", "+prio")):
                    on = times[(label, kind, k)]
                    sweep[f"{kind}({k}){tag}"] = {"ms": on, "exposed_ms": max(0.0, on - off),
                                                  "hidden_fraction": 1.0 - max(0.0, on - off) / ar_total}
            best = min((v["ms"], key) for key, v in sweep.items() if key.startswith("first_k") and "+prio" not in key)[1]
            best_p = min((v["ms"], key) for key, v in sweep.items() if "+prio" in key)[1]
            emulated = {"n": n, "link_GBps_per_direction": gbps, "latency_us_per_bucket": lat,
                        "bucket_layers": args.bucket_layers,
                        "note": "EMULATED all-reduce on one GPU (comm stream held for the ring time; no NCCL, no "
                                "data moved); the engine keeps the 16-SM NCCL reserve; all graphs timed "
                                "interleaved (2 runs each)",
                        "allreduce_total_ms": ar_total, "in_order_ms": sweep["in_order(0)"]["ms"], "best": best,
                        "best_ms": sweep[best]["ms"], "best_exposed_ms": sweep[best]["exposed_ms"],
                        "best_hidden_fraction": sweep[best]["hidden_fraction"],
                        "ooo_speedup_vs_in_order": sweep["in_order(0)"]["ms"] / sweep[best]["ms"],
                        "prioritised": {"chunk_mb": args.comm_chunk_mb, "best": best_p, "best_ms": sweep[best_p]["ms"],
                                        "best_hidden_fraction": sweep[best_p]["hidden_fraction"],
                                        "speedup_vs_fifo_best": sweep[best]["ms"] / sweep[best_p]["ms"]},
                        "k_sweep": sweep}
        except Exception as e:  # noqa: BLE001 -- the bench line must still be printed
            emulated = {"error": str(e)[:200]}
        finally:
            for key in ("OOO_EMULATE_AR_N", "OOO_EMULATE_AR_GBPS", "OOO_EMULATE_AR_LAT_US"):
                os.environ.pop(key, None)

    # ---- per-kernel durations: the same step captured with per-launch CUDA
    # events (stream-ordered on the stream each kernel runs on), every launch of
    # a K-step back-to-back region keeping its own events (timing slots)
    stk.set_timing(True)
    stk.forward(X, Y)
    g_t = stk.graph(X, Y, dY, *sched)
    stk.set_timing(False)
    for _ in range(3):
        g_t.launch(stream)
    n_t = args.steps
    g_t.set_timing_slots(n_t)
    ms_timed = statistics.mean(interleaved([g_t], n_t, 1)[0])
    per_launch = g_t.timing()
    g_t.close()
    by_kind = {}
    for recs in per_launch:
        for r in recs:
            d = by_kind.setdefault(r["kind"], {"ms": [], "flops": r["flops"], "bytes": r["bytes"], "per_launch": 0})
            d["ms"].append(max(r["ms"], 0.0))
    for recs in per_launch[:1]:
        for r in recs:
            by_kind[r["kind"]]["per_launch"] += 1
    ours = {k: v for k, v in by_kind.items() if k not in ("allreduce", "copy")}
    dom = max(ours, key=lambda k: sum(ours[k]["ms"]))
    dd = ours[dom]
    n_launch = len(per_launch)
    launches_per_step = sum(v["per_launch"] for v in ours.values())
    dom_ms = statistics.mean(dd["ms"])                      # mean over every timed launch
    dom_step_ms = sum(dd["ms"]) / max(1, n_launch)          # per step (if several launches per step)
    if dd["flops"] > 0:
        achieved = dd["flops"] / (dom_ms * 1e-3) / 1e12
        peak = peaks["bf16_tflops_sustained"] if dt == "bf16" else 75.0
        roof = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak}
    else:
        achieved = dd["bytes"] / (dom_ms * 1e-3) / 1e9
        peak = peaks["hbm_gbs"]
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak}
    roof["kernel"] = dom
    roof["algorithmic_work_per_launch"] = dd["flops"] if dd["flops"] > 0 else dd["bytes"]
    roof["timed_launches"] = len(dd["ms"])
    roof["avg_launch_us"] = dom_ms * 1e3
    roof["launch_us_sem"] = (statistics.stdev(dd["ms"]) / math.sqrt(len(dd["ms"])) * 1e3) if len(dd["ms"]) > 1 else None
    roof["share_of_step"] = dom_step_ms / ms_timed
    roof["share_ok"] = roof["share_of_step"] <= 1.0 + 1e-3
    roof["instrumented_ms_per_step"] = ms_timed
    roof["peak_source"] = f"{peaks['source']} ({'bf16_tflops_sustained' if dd['flops'] > 0 else 'hbm_gbs'})"
    traffic = None
    tp = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(tp):
        try:
            tr = json.load(open(tp))
            traffic = tr.get(cfg.name, {}).get(dom)
        except Exception:
            traffic = None
    roof["traffic"] = traffic

    # ---- north-star roofline of the whole step: max(GEMM FLOP at peak, ring AR bytes at 900 GB/s)
    flops = cfg.gemm_flops()
    t_tensor = flops / (peaks["bf16_tflops_sustained"] * 1e12) * 1e3 if dt == "bf16" else None
    grad_bytes = cfg.params() * (2 if dt == "bf16" else 4)
    link = 900e9
    t_ar = 2 * (world - 1) / world * grad_bytes / link * 1e3 if world > 1 else 0.0
    step_roof_ms = max(t_tensor or 0.0, t_ar)
    hbm_bytes = cfg.hbm_min_bytes()
    t_hbm = hbm_bytes / (peaks["hbm_gbs"] * 1e9) * 1e3

    # ---- e2e through the C ABI with HOST buffers (ooo_graph_upload /
    # ooo_graph_launch_host): every step uploads its inputs (X, dY) from
    # pinned host memory and reads its result Y back; two graphs over two
    # buffer sets, used alternately, let step t+1's upload and step t's
    # read-back overlap step t's compute on the copy stream (each step still
    # moves its own bytes inside the timed region).
    e2e = None
    if not args.no_e2e:
        cs = torch.cuda.Stream(device=dev)
        sets = []
        for p in range(2):
            if p == 0:
                g = g_ooo
            else:
                Xp, dYp, Yp = torch.empty_like(X), torch.empty_like(dY), torch.empty_like(Y)
                stk.forward(Xp, Yp)
                torch.cuda.synchronize()
                g = stk.graph(Xp, Yp, dYp, *sched)
            hX = torch.empty(X.shape, dtype=X.dtype, pin_memory=True)
            hdY = torch.empty(dY.shape, dtype=dY.dtype, pin_memory=True)
            hY = torch.empty(Y.shape, dtype=Y.dtype, pin_memory=True)
            hX.copy_(X.cpu())
            hdY.copy_(dY.cpu())
            sets.append({"g": g, "hX": hX, "hdY": hdY, "hY": hY})

        def run_steps(n, e0=None, e1=None):
            if e0 is not None:
                e0.record(cs)
            sets[0]["g"].upload(sets[0]["hX"], sets[0]["hdY"], cs)
            for t in range(n):
                b_ = sets[t % 2]
                if t + 1 < n:
                    nb = sets[(t + 1) % 2]
                    nb["g"].upload(nb["hX"], nb["hdY"], cs)     # overlaps step t
                b_["g"].launch_host(b_["hY"], stream, cs)
            if e1 is not None:
                e1.record(cs)

        run_steps(4)
        barrier()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        run_steps(args.steps, e0, e1)
        torch.cuda.synchronize()
        barrier()
        ms_e2e = max_over_ranks([e0.elapsed_time(e1) / args.steps])[0]
        ebytes = X.element_size()
        e2e = {"value": 1e3 / ms_e2e, "unit": UNIT,
               "h2d_bytes_per_step": (X.numel() + dY.numel()) * ebytes, "d2h_bytes_per_step": Y.numel() * ebytes,
               "api": "ooo_graph_upload + ooo_graph_launch_host (C ABI, pinned host buffers)",
               "overlap": "double-buffered: step t+1 upload and step t read-back overlap step t (copy stream)"}
        sets[1]["g"].close()

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        tok = cpu_sample_tokens(cfg, args.cpu_sample_tokens)
        sec, threads = time_cpu_oracle(cfg, tok)
        cpu = {"value": (tok / M) / sec, "unit": UNIT, "cores": threads, "kind": "oracle",
               "sample": f"one fp64 (bf16-storage) forward+backward of {tok} of {M} tokens of {cfg.name}, "
                         f"{sec:.1f} s, scaled by {tok}/{M}"}

    nccl = None
    if world > 1:
        try:
            ver = torch.cuda.nccl.version()
        except Exception:  # noqa: BLE001
            ver = None
        nccl = {"version": ".".join(map(str, ver)) if isinstance(ver, tuple) else ver,
                "env": {k: v for k, v in sorted(os.environ.items()) if k.startswith("NCCL_")},
                "library_communicator_max_ctas": args.nccl_max_ctas or 16}
    value = 1e3 / ms_ooo
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_ooo, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": dt, "data": "synthetic",
        "config": {"workload": f"{cfg.name} ({cfg.note})", "layers": L, "tokens_per_gpu": M,
                   "global_batch_tokens": M * world, "dims": f"{cfg.dims[0]}/{max(cfg.dims)}",
                   "schedule": (f"regions(Algorithm 1, {args.regions} layers per region)" if sched[0] == "regions"
                                else "ooo_first_k"),
                   "k": k_best, "k_search_visited": visited,
                   "bucket_layers": args.bucket_layers, "parallelism": f"dp{world}",
                   "comm": (f"prioritised, {args.comm_chunk_mb} MB chunks (Fig. 4(b))" if args.comm_priority
                            else "FIFO in D's dW order"),
                   "timing": f"{args.steps} steps as {len(main_s['run_steps'])} back-to-back runs, interleaved "
                             f"with as many in_order runs (ABAB); value = steps / summed run time",
                   "l2": "working set (weights+activations+grads) >> 126 MB L2; no flush"},
        "tokens_per_s": value * M * world,
        "runs": {"n": main_s["runs"], "mean_ms": ms_ooo, "sem_ms": main_s["sem_ms"],
                 "run_ms_per_step": main_s["run_ms_per_step"]},
        "in_order": {"value": in_s["value"], "ms_per_step": ms_in, "sem_ms": in_s["sem_ms"]},
        "ooo_speedup_vs_in_order": ms_in / ms_ooo,
        "exposed_allreduce_ms": exposed,
        "allreduce_standalone_ms": ar_ms,
        "allreduce_standalone_note": ("the library's own buckets on its own communicator (ooo_allreduce_buckets), "
                                      "back to back, no compute" if world > 1 else None),
        "hidden_fraction": (None if not exposed or not ar_ms else 1.0 - max(0.0, exposed["ooo"]) / ar_ms),
        "dp_selfcheck": selfcheck,
        "nccl": nccl,
        "ooo_first_k0": {"value": 1e3 / ms_k0, "ms_per_step": ms_k0},
        "ooo_first_k": {"k": k_best, "value": 1e3 / ms_fk if ms_fk else None, "ms_per_step": ms_fk,
                        "deferral_bytes": deferral_bytes(cfg.dims, cfg.acts, M, dt, k_best),
                        "deferral_note": "extra live bytes of deferring dW_1..dW_k (sum_{i=2..k} |dZ_i|, §3 P:111, "
                                         "E8); the engine keeps every dZ_i resident, so this is reported, not allocated"},
        "regions": regions,
        "emulated_dp": emulated,
        "step_roofline": {"ms": step_roof_ms, "frac": step_roof_ms / ms_ooo if step_roof_ms else None,
                          "tensor_ms": t_tensor, "allreduce_ms_at_900GBps": t_ar, "gemm_flops": flops,
                          "hbm_min_bytes": hbm_bytes, "hbm_ms": t_hbm,
                          "hbm_inclusive_ms": max(step_roof_ms, t_hbm)},
        "roofline": roof,
        "kernels": {k: {"mean_ms_per_launch": statistics.mean(v["ms"]), "launches_per_step": v["per_launch"]}
                    for k, v in by_kind.items()},
        "gpu_launches": launches_per_step * args.steps,
        "clocks": clocks,
        "e2e": e2e,
        "cpu_baseline": cpu,
    }
    for g in graphs.values():
        g.close()
    stk.close()
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
