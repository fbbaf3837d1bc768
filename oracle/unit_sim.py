"""Oracle: unit-time list-scheduling simulator for the paper's worked examples.

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).

The paper states its scheduling problem as a job-shop variant (§2, eq. at
P:84): start times T for {F_i, dO_i, dW_i, S[dO_i], S[dW_i]} under
    T(dO_{L+1}) = 0,
    {T(dW_i), T(dO_i)} >= T(S[dO_{i+1}]) + S[dO_{i+1}],
    T(S[dW_i]) >= T(dW_i) + dW_i,
    T(F_i) >= T(S[dW_i]) + S[dW_i],  T(F_{i+1}) >= T(F_i) + F_i,
minimising the makespan T(F_L) + F_L.  This module simulates a given
schedule in integer time steps so the tests can check the schedules of
Fig. 4 (data parallel, P:164/P:180/P:206) and Fig. 5 (cross-layer model
parallel, P:226/P:232/P:236) against the unit counts the paper prints.

Readings: unit cost for F/dO/dW; the loss gradient dO_{L+1} is
free; dO_1 is not computed (Q1); one compute stream per GPU; one
communication channel per worker; FIFO channel for conventional execution and
pre-emptive lowest-layer-first for prioritised communication ([28, 36,
38, 44, 56]); zero inter-GPU latency for the model-parallel example.
Fig. 4's per-layer sync costs are not printed (the image is missing); the
instance c = (4, 1, 1, 2, 4) is a reconstruction that reproduces every number
the text gives (-1 unit, -3 units, k = 3 and k = 4 both optimal).
"""
from __future__ import annotations

from dataclasses import dataclass, field


@dataclass
class Op:
    name: str
    resource: str
    duration: int
    deps: tuple = ()
    key: tuple = ()          # smaller = higher priority


@dataclass
class Resource:
    name: str
    policy: str              # "order" | "priority" | "fifo" | "preemptive"
    order: list = field(default_factory=list)   # op names, for policy "order"


def simulate(ops: list, resources: list, horizon: int = 10_000) -> dict:
    """Integer time-stepped simulation.  Returns {op name: finish time}."""
    by_name = {o.name: o for o in ops}
    res = {r.name: r for r in resources}
    remaining = {o.name: o.duration for o in ops}
    finish = {}
    ready_at = {}
    running = {r: None for r in res}            # non-preemptive op in progress
    idx = {o.name: n for n, o in enumerate(ops)}
    for o in ops:
        if o.resource not in res:
            raise ValueError(f"unknown resource {o.resource}")
        if o.duration == 0:
            pass
    t = 0
    while len(finish) < len(ops):
        if t > horizon:
            raise RuntimeError("simulation did not finish (cyclic deps?)")
        # zero-duration ops complete as soon as their deps are done
        progressed = True
        while progressed:
            progressed = False
            for o in ops:
                if o.name not in finish and o.duration == 0 and all(d in finish and finish[d] <= t for d in o.deps):
                    finish[o.name] = t
                    progressed = True
        for o in ops:
            if o.name not in finish and o.name not in ready_at and all(d in finish and finish[d] <= t for d in o.deps):
                ready_at[o.name] = t
        chosen = {}
        for rname, r in res.items():
            cur = running[rname]
            if cur is not None and r.policy != "preemptive":
                chosen[rname] = cur
                continue
            cands = [o for o in ops if o.resource == rname and o.name not in finish
                     and o.name in ready_at and o.duration > 0]
            pick = None
            if r.policy == "order":
                for name in r.order:
                    if name not in finish:
                        if name in ready_at:
                            pick = by_name[name]
                        break
            elif r.policy == "priority" or r.policy == "preemptive":
                if cands:
                    pick = min(cands, key=lambda o: (o.key, idx[o.name]))
            elif r.policy == "fifo":
                if cands:
                    pick = min(cands, key=lambda o: (ready_at[o.name], idx[o.name]))
            else:
                raise ValueError(r.policy)
            if pick is not None:
                chosen[rname] = pick.name
                if r.policy != "preemptive":
                    running[rname] = pick.name
        for rname, name in chosen.items():
            remaining[name] -= 1
            if remaining[name] == 0:
                finish[name] = t + 1
                running[rname] = None
        t += 1
    return finish


# --------------------------------------------------------------- Fig. 4 (DP)
def dp_iteration(L: int, D: list, sync_cost: list, comm_policy: str) -> int:
    """Makespan of one data-parallel iteration (§5.1, Fig. 4):
    backward ops executed on one GPU stream in the order D, each S[dW_i] on one
    channel (``comm_policy`` "fifo" or "preemptive" lowest-layer-first), then
    the next forward F_1..F_L gated on S[dW_i].  S[dO_*] is a no-op in
    data parallelism."""
    ops = []
    gpu_order = []
    for op in D:
        i = abs(op)
        dep = () if i == L else (f"dO{i + 1}",)
        name = f"dO{i}" if op > 0 else f"dW{i}"
        ops.append(Op(name, "gpu", 1, dep))
        gpu_order.append(name)
    for i in range(1, L + 1):
        ops.append(Op(f"S{i}", "net", sync_cost[i - 1], (f"dW{i}",), key=(i,)))
    for i in range(1, L + 1):
        deps = (f"S{i}",) + ((f"F{i - 1}",) if i > 1 else ())
        ops.append(Op(f"F{i}", "gpu", 1, deps))
        gpu_order.append(f"F{i}")
    fin = simulate(ops, [Resource("gpu", "order", gpu_order), Resource("net", comm_policy)])
    return fin[f"F{L}"]


# -------------------------------------------------- Fig. 5 (cross-layer MP)
def mp_iteration(L: int, n_gpu: int, placement: str, fast_forward: bool) -> int:
    """Makespan of one cross-layer model-parallel iteration (§5.2.1,
    P:222-236, Fig. 5): forward F_1..F_L then backward, unit costs, zero
    transfer latency, dO_1 omitted.

    placement "contiguous": layers split into n_gpu consecutive groups;
              "modulo"    : layer l on GPU (l mod n_gpu).
    fast_forward False: conventional backprop -- both gradients of layer l
                        finish before layer l-1's start;
                 True : each GPU prefers dO over dW (gradient fast-forwarding,
                        P:222/P:232), higher layer first.
    """
    def gpu_of(l):
        if placement == "contiguous":
            per = L // n_gpu
            return (l - 1) // per
        if placement == "modulo":
            return l % n_gpu
        raise ValueError(placement)

    ops = []
    for l in range(1, L + 1):
        ops.append(Op(f"F{l}", f"g{gpu_of(l)}", 1, (f"F{l - 1}",) if l > 1 else (), key=(0, l)))
    for l in range(L, 0, -1):
        g = f"g{gpu_of(l)}"
        base = (f"F{L}",) if l == L else (f"dO{l + 1}",)
        conv = () if (fast_forward or l == L) else (f"dW{l + 1}",)
        if l > 1:
            ops.append(Op(f"dO{l}", g, 1, base + conv, key=(1, -l)))
        ops.append(Op(f"dW{l}", g, 1, base + conv, key=(2 if fast_forward else 1, -l)))
    resources = [Resource(f"g{n}", "priority") for n in range(n_gpu)]
    fin = simulate(ops, resources)
    return max(fin.values())
