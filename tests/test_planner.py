"""Host-only checks of the engine's tile-queue planner (ooo_engine_plan).

The persistent engine dispenses tiles in one FIFO order and a tile waits for
its inputs, so the order must be topological (every op after the ops it
depends on) or the kernel could deadlock; it must also cover every tile of
every op exactly once, keep the dO chain in D's order and the dW ops in
Algorithm 2's order (the planner only interleaves the two chains,
§4.1).  No GPU needed.
"""
import pytest

from oracle import schedule as S
from paper_conf_eurosys_ohlks22_b200 import configs
from paper_conf_eurosys_ohlks22_b200.stack import engine_plan

def _cg(tokens):
    """Engine CTAs per tile: pairs (256-row tiles) unless the tokens fit one 128-row tile."""
    return 1 if tokens <= 128 else 2


def _rows(n, per):
    return (n + per - 1) // per


def _check_plan(dims, acts, tokens, kind, k, fused, workers, need_dx=False, bucket_layers=1):
    L = len(acts)
    ops, topo = engine_plan(dims, acts, tokens, kind, k, fused=fused, workers=workers,
                            need_input_grad=need_dx, bucket_layers=bucket_layers)
    assert topo, "planned queue is not a topological order"
    D = S.reverse_first_k(L, k, need_dx) if kind == "first_k" else S.in_order(L, need_dx)
    # coverage: every (op, tile row) exactly once, column tiles constant per op
    seen = {}
    for name, layer, r0, nr, nt in ops:
        for r in range(r0, r0 + nr):
            key = (name, layer, r)
            assert key not in seen, key
            seen[key] = nt
    want = {}
    CG = _cg(tokens)
    T = _rows(_rows(tokens, 128), CG)
    for op in D:
        i = abs(op)
        if op > 0:
            for r in range(T):
                want[("dO", i, r)] = True
        else:
            for r in range(_rows(_rows(dims[i - 1], 128), CG)):
                want[("dW", i, r)] = True
    if fused:
        for r in range(T):
            want[("copy", 1, r)] = True
        for i in range(1, L + 1):
            for r in range(T):
                want[("F", i, r)] = True
    assert set(seen) == set(want)
    # chain orders: dO ops in D's order, dW ops (first appearance) in D's order
    first = {}
    for j, (name, layer, *_rest) in enumerate(ops):
        first.setdefault((name, layer), j)
    do_order = sorted((first[("dO", i)], i) for i in {o for o in D if o > 0})
    assert [i for _, i in do_order] == [o for o in D if o > 0]
    dw_order = sorted((first[("dW", -o)], -o) for o in D if o < 0)
    assert [i for _, i in dw_order] == [-o for o in D if o < 0]
    if fused:
        f_order = sorted((first[("F", i)], i) for i in range(1, L + 1))
        assert [i for _, i in f_order] == list(range(1, L + 1))
    return ops


@pytest.mark.parametrize("cfg", [configs.C2, configs.C3, configs.C4, configs.C5], ids=lambda c: c.name)
@pytest.mark.parametrize("kind,kfrac", [("first_k", 0.0), ("first_k", 1 / 3), ("first_k", 1.0), ("in_order", 0.0)])
def test_plan_configs(cfg, kind, kfrac):
    k = int(round(kfrac * cfg.L))
    for fused in (True, False):
        _check_plan(cfg.dims, cfg.acts, cfg.tokens, kind, k, fused, workers=74)


@pytest.mark.parametrize("workers", [1, 3, 74])
@pytest.mark.parametrize("need_dx", [False, True])
def test_plan_small_ragged(workers, need_dx):
    dims, acts = [192, 320, 256, 448, 256, 192], ["gelu", "id", "gelu", "gelu", "id"]
    for k in range(len(acts) + 1):
        _check_plan(dims, acts, 400, "first_k", k, True, workers, need_dx=need_dx, bucket_layers=2)
    _check_plan(dims, acts, 8, "in_order", 0, True, workers, need_dx=need_dx)


def test_plan_in_order_is_d_then_forward():
    """Conventional backprop: the queue is exactly D, then F_1..F_L (F_1 reads
    the caller's X), then the X -> X_1 copy the next backward's dW_1 reads."""
    dims, acts = [256] * 7, ["id", "gelu"] * 3
    ops = _check_plan(dims, acts, 512, "in_order", 0, True, workers=74)
    names = [(n, l) for n, l, *_ in ops]
    D = S.in_order(6, False)
    want = [("dO", o) if o > 0 else ("dW", -o) for o in D] + [("F", i) for i in range(1, 7)] + [("copy", 1)]
    assert names == want
