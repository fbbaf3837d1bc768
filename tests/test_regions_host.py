"""The library's Algorithm 1 (``ooo_region_schedule``, regions.cpp) against
the oracle (oracle/regions.py) -- host only, no GPU.  Integer / index output:
bit-exact (same region lists in the same order, same pre-scheduled count)."""
import json
import os
import random

import pytest

from oracle import regions as R
from paper_conf_eurosys_ohlks22_b200 import stack as ST
from paper_conf_eurosys_ohlks22_b200._lib import OooError
from tests.test_oracle_regions import _random_instance

GOLD = os.path.join(os.path.dirname(__file__), "golden", "alg1_trace.json")


def test_golden_trace():
    g = json.load(open(GOLD))
    I = g["instance"]
    for m, exp in (("0", g["algorithm1"]), ("250", g["region_schedule"]["mxm=250"]["S"])):
        S, k = ST.region_schedule(I["t_main"], I["t_sub"], I["speedup"], I["ready"], I["last_region"],
                                  I["nbytes"], int(m))
        assert S == exp


@pytest.mark.parametrize("seed", range(4))
def test_library_equals_oracle_random(seed):
    rng = random.Random(1000 + seed)
    for _ in range(100):
        t_main, ts, p, ready, last, nb = _random_instance(rng)
        mxm = rng.choice([0, 1, 50, 200])
        exp, kexp = R.region_schedule(t_main, ts, p, ready, last, nb, mxm)
        got, kgot = ST.region_schedule(t_main, ts, p, ready, last, nb, mxm)
        assert got == exp and kgot == kexp


def test_invalid_arguments():
    with pytest.raises(OooError):
        ST.region_schedule([], [], [], [])
    with pytest.raises(OooError):
        ST.region_schedule([1.0], [[1.0]], [[1.0]], [0.0], last_region=[3])
