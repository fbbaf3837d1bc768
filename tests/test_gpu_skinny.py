"""Skinny stacks (<= 16 tokens per GPU, e.g. C5 MLP96): every engine launch
runs the skinny-stack kernel (csrc/skinny.cu: chain ops as 8-CTA clusters
with the K split reduced over DSMEM, dW workers on the other clusters).  Same
gates as the engine tests: the oracle within the bf16 gate, every schedule
bit-exact with every other, graph == eager; and the engine's result
(OOO_SKINNY=0) within the same gate of the oracle and of the skinny result.
The fused-step, comm-gated, emulated all-reduce, regions and one-rank NCCL
tests of test_gpu_parity.py also carry 16- / 8-token cases."""
import numpy as np
import pytest
import torch

from oracle.layers import rel_fro
from tests.gpu_helpers import Case, max_err, to_dev

pytestmark = pytest.mark.gpu

BF16_TOL = 1e-2


def _check(errs, tol):
    for k, v in errs.items():
        assert v <= tol, (k, v, errs)


@pytest.mark.parametrize("tokens", [16, 8])
def test_skinny_schedules_bit_exact_graph_equals_eager(tokens):
    case = Case([256, 512, 256, 1024, 256, 256], ["id", "gelu", "gelu", "id", "id"], tokens, "bf16")
    stk = case.stack(bucket_layers=2)
    base = case.run(stk, "in_order", 0)
    for k in range(case.L + 2):
        out = case.run(stk, "first_k", k)
        assert torch.equal(out["raw"], base["raw"]), k
        assert np.array_equal(out["Y"], base["Y"])
    for kind, k in [("in_order", 0), ("first_k", 3)]:
        out = case.run(stk, kind, k, graph=True, launches=3)
        assert torch.equal(out["raw"], base["raw"]), (kind, k)
    _check(max_err(base, case.oracle()), BF16_TOL)
    stk.close()


@pytest.mark.parametrize("tokens", [16, 8])
def test_skinny_relu_gelu_and_input_grad(tokens):
    """ReLU (its Z_i store, the mask in dO_{i+1}), GELU (gelu' store) and dX
    (dO_1), with widths that are not multiples of 128 (64-wide chain tiles)."""
    case = Case([192, 256, 320, 128, 64], ["relu", "gelu", "relu", "gelu"], tokens, "bf16", need_dx=True)
    stk = case.stack()
    out = case.run(stk, "first_k", 2)
    _check(max_err(out, case.oracle(2)), BF16_TOL)
    g = case.run(stk, "first_k", 2, graph=True, launches=2)
    assert torch.equal(g["raw"], out["raw"])
    assert np.array_equal(g["dX"], out["dX"])
    stk.close()


def test_skinny_matches_engine(monkeypatch):
    """The persistent engine (OOO_SKINNY=0) and the skinny kernel on the same
    16-token stack: both within the gate of the oracle, and of each other
    (their fp32 summation orders differ, so not bit-exact)."""
    case = Case([1024, 1024, 1024, 1024, 1024], ["gelu", "id", "gelu", "id"], 16, "bf16")
    sk = case.stack(bucket_layers=2)
    a = case.run(sk, "first_k", 1, graph=True, launches=2)
    sk.close()
    monkeypatch.setenv("OOO_SKINNY", "0")
    eng = case.stack(bucket_layers=2)
    b = case.run(eng, "first_k", 1, graph=True, launches=2)
    eng.close()
    ref = case.oracle(1)
    _check(max_err(a, ref), BF16_TOL)
    _check(max_err(b, ref), BF16_TOL)
    assert rel_fro(a["Y"], b["Y"]) <= BF16_TOL
    assert max(rel_fro(x, y) for x, y in zip(a["dW"], b["dW"])) <= BF16_TOL


def test_skinny_wide_layers_more_tiles_than_clusters():
    """A 4096-wide layer has 32 chain tiles: more than the chain clusters, so a
    cluster walks several tiles of one op."""
    case = Case([512, 4096, 512], ["gelu", "id"], 16, "bf16")
    stk = case.stack()
    out = case.run(stk, "first_k", 1, graph=True, launches=2)
    _check(max_err(out, case.oracle(1)), BF16_TOL)
    stk.close()


def test_skinny_timing_records():
    """The skinny kernel is the stack's engine launch for the timing API
    (bench.py's per-launch accounting)."""
    case = Case([256, 256, 256], ["gelu", "id"], 16, "bf16")
    stk = case.stack()
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    Y = stk.forward(X)
    stk.set_timing(True)
    stk.backward(dY, "first_k", 0)
    stk.forward(X, Y)
    stk.join()
    torch.cuda.synchronize()
    recs = stk.timing()
    stk.set_timing(False)
    assert any(r["ms"] > 0 for r in recs), recs
    stk.close()
