"""Pins of the Algorithm 1 oracle (oracle/regions.py; §4.1).

Algorithm 1 is a heuristic list scheduler, so it is pinned by a hand-expanded
trace of its pseudocode (tests/golden/alg1_trace.json), by special cases that
reduce it to a textbook operation (one unbounded region with every kernel
ready = sort by descending speedup) and by the invariants its lines imply.
"""
import json
import os
import random

import pytest

from oracle import regions as R

GOLD = os.path.join(os.path.dirname(__file__), "golden", "alg1_trace.json")


def _gold():
    with open(GOLD) as f:
        return json.load(f)


def test_hand_trace_algorithm1():
    g = _gold()
    I = g["instance"]
    S = R.algorithm1(I["t_main"], I["t_sub"], I["speedup"], I["ready"], I["last_region"])
    assert S == g["algorithm1"]
    assert R.held_bytes(S, I["t_main"], I["ready"], I["nbytes"]) == g["held_bytes_algorithm1"]


@pytest.mark.parametrize("mxm", [0, 300, 250])
def test_hand_trace_memory_bounded_preschedule(mxm):
    g = _gold()
    I = g["instance"]
    S, k = R.region_schedule(I["t_main"], I["t_sub"], I["speedup"], I["ready"], I["last_region"],
                             I["nbytes"], mxm)
    exp = g["region_schedule"][f"mxm={mxm}"]
    assert S == exp["S"] and k == exp["k"]


def test_one_unbounded_region_is_a_sort_by_speedup():
    """Lines 4-9 with one region that never closes and every kernel ready at
    time 0: each step takes the remaining kernel with the highest speedup
    (first in candidate order on ties) -> a stable sort by descending p."""
    rng = random.Random(7)
    for _ in range(50):
        K = rng.randint(1, 12)
        p = [[round(rng.uniform(0.8, 2.0), 1)] for _ in range(K)]
        S = R.algorithm1([1e9], [[1.0]] * K, p, [0.0] * K)
        assert S == [sorted(range(K), key=lambda k: -p[k][0])]


def _random_instance(rng):
    N = rng.randint(1, 6)
    K = rng.randint(1, 10)
    t_main = [float(rng.randint(1, 20)) for _ in range(N)]
    total = sum(t_main)
    ready = sorted(float(rng.randint(0, int(total))) for _ in range(K))
    last = [rng.randint(R.ready_region(t_main, ready[k]), N - 1) for k in range(K)]
    p = [[round(rng.uniform(0.8, 2.0), 2) for _ in range(N)] for _ in range(K)]
    ts = [[float(rng.randint(1, 8)) for _ in range(N)] for _ in range(K)]
    nb = [rng.randint(1, 100) for _ in range(K)]
    return t_main, ts, p, ready, last, nb


def test_invariants_random_instances():
    rng = random.Random(20220405)
    for _ in range(300):
        t_main, ts, p, ready, last, nb = _random_instance(rng)
        N, K = len(t_main), len(ready)
        S = R.algorithm1(t_main, ts, p, ready, last)
        flat = [k for lst in S for k in lst]
        assert sorted(flat) == list(range(K))               # l.9: every kernel once
        start = R.region_starts(t_main)
        for i, lst in enumerate(S):
            now = 0.0
            for k in lst:
                assert i <= last[k]                         # reading A1 (last allowed region)
                runnable = ready[k] <= start[i] + now and now < t_main[i]
                asap = i == min(R.ready_region(t_main, ready[k]), last[k])
                assert runnable or asap                     # l.5 / l.11, else reading A3
                now += ts[k][i]                             # l.10


def test_full_preschedule_is_as_soon_as_ready():
    """P:162 with every region pre-scheduled: each kernel runs in the region
    in which it becomes ready, and no deferred bytes are held."""
    rng = random.Random(3)
    for _ in range(100):
        t_main, ts, p, ready, last, nb = _random_instance(rng)
        S, k = R.region_schedule(t_main, ts, p, ready, last, nb, mxm=1e-9)
        N = len(t_main)
        assert k <= N
        assert max(R.held_bytes(S, t_main, ready, nb)) == 0
        if k == N:
            for i, lst in enumerate(S):
                exp = sorted([c for c in range(len(ready)) if min(R.ready_region(t_main, ready[c]), last[c]) == i],
                             key=lambda c: (ready[c], c))
                assert lst == exp


def test_memory_bound_respected_when_reachable():
    rng = random.Random(11)
    for _ in range(100):
        t_main, ts, p, ready, last, nb = _random_instance(rng)
        S0 = R.algorithm1(t_main, ts, p, ready, last)
        peak0 = max(R.held_bytes(S0, t_main, ready, nb))
        mxm = max(1, peak0 // 2)
        S, k = R.region_schedule(t_main, ts, p, ready, last, nb, mxm)
        assert max(R.held_bytes(S, t_main, ready, nb)) <= mxm or k == len(t_main)
        if peak0 <= mxm:
            assert k == 0 and S == S0
