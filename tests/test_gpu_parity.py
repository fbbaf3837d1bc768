"""Parity of the CUDA path (through the C ABI) against the fp64 oracle.

All inputs are seeded (paper_conf_eurosys_ohlks22_b200.synth); the oracle
computes every expected value itself from those inputs (no teacher forcing).
Gates (north star, reading in DESIGN.md): max relative Frobenius error over
Y, every dW_i, db_i (and dX) <= 1e-2 in bf16 and <= 1e-4 in fp32; in-order
and every ooo_first_k(k) schedule bit-exact with each other.
"""
import numpy as np
import pytest
import torch

from paper_conf_eurosys_ohlks22_b200 import configs
from oracle.layers import rel_fro
from tests.gpu_helpers import TDT, Case, bf16_floor, max_err, record_parity, to_dev, to_np

pytestmark = pytest.mark.gpu

BF16_TOL = 1e-2
FP32_TOL = 1e-4


def _check(errs, tol):
    for k, v in errs.items():
        assert v <= tol, (k, v, errs)


# ------------------------------------------------------------------ fp32
def test_fp32_config0_end_to_end_all_schedules():
    c = configs.C1
    case = Case(c.dims, c.acts, c.tokens, "fp32")
    ref = case.oracle()
    stk = case.stack()
    base = None
    for kind, k in [("in_order", 0)] + [("first_k", k) for k in range(c.L + 1)]:
        out = case.run(stk, kind, k)
        _check(max_err(out, ref), FP32_TOL)
        if base is None:
            base = out["raw"]
        assert torch.equal(out["raw"], base), (kind, k)
    stk.close()


def test_fp32_ragged_with_input_grad():
    case = Case([192, 320, 128, 64], ["gelu", "relu", "id"], 200, "fp32", need_dx=True)
    ref = case.oracle(2)
    stk = case.stack()
    out = case.run(stk, "first_k", 2)
    _check(max_err(out, ref), FP32_TOL)


# ------------------------------------------------------------------ bf16
@pytest.mark.parametrize("tokens", [400, 128, 16, 8])
def test_bf16_ragged_tiles_end_to_end(tokens):
    """Several tiles in every dimension plus ragged tails (M % 128 != 0,
    widths not multiples of the N tile)."""
    case = Case([192, 320, 256, 448, 192], ["gelu", "id", "gelu", "id"], tokens, "bf16")
    ref = case.oracle(2)
    stk = case.stack()
    out = case.run(stk, "first_k", 2)
    _check(max_err(out, ref), BF16_TOL)


def test_bf16_relu_and_input_grad():
    case = Case([128, 256, 128, 128], ["relu", "gelu", "relu"], 264, "bf16", need_dx=True)
    ref = case.oracle(3)
    stk = case.stack()
    out = case.run(stk, "first_k", 3)
    _check(max_err(out, ref), BF16_TOL)


def test_bf16_schedules_bit_exact_and_graph_equals_eager():
    case = Case([256, 512, 256, 1024, 256, 256], ["id", "gelu", "gelu", "id", "id"], 384, "bf16")
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


def test_bf16_deterministic_repeat():
    case = Case([768, 768, 3072, 768], ["id", "gelu", "id"], 1024, "bf16")
    stk = case.stack()
    a = case.run(stk, "first_k", 3)
    b = case.run(stk, "first_k", 3)
    assert torch.equal(a["raw"], b["raw"])


# ---------------------------------------- full-size shapes of the configs
def _block_slice(cfg, blocks):
    """The first `blocks` transformer blocks of a config at its full width and
    full tokens per GPU: every GEMM launch configuration of the config (tile
    plan depends only on (M, d_in, d_out)) is exercised."""
    n = 6 * blocks
    return list(cfg.dims[: n + 1]), list(cfg.acts[:n]), cfg.tokens


@pytest.mark.parametrize("cfg", [configs.C2, configs.C3, configs.C4], ids=["bert_base", "bert_large", "gpt2_medium"])
def test_bf16_full_size_block_slice(cfg):
    dims, acts, M = _block_slice(cfg, 2)
    case = Case(dims, acts, M, "bf16")
    ref = case.oracle(len(acts))
    stk = case.stack()
    out = case.run(stk, "first_k", len(acts))
    _check(max_err(out, ref), BF16_TOL)
    base = case.run(stk, "in_order", 0)
    assert torch.equal(out["raw"], base["raw"])


def test_bf16_long_k_split_many_rows():
    """Long-K chain ops split over K with more than one 128-row block
    (OOO_SPLITK_LONGK, default 64 k-blocks: F_2 and dO_1 have K = 4096),
    ragged rows (264 tokens): within the oracle's gate, every schedule
    bit-exact, graph == eager."""
    case = Case([256, 4096, 256], ["gelu", "id"], 264, "bf16", need_dx=True)
    stk = case.stack()
    base = case.run(stk, "in_order", 0)
    _check(max_err(base, case.oracle(0)), BF16_TOL)
    for k in (1, 2, 3):
        out = case.run(stk, "first_k", k)
        assert torch.equal(out["raw"], base["raw"]), k
        assert np.array_equal(out["dX"], base["dX"])
    g = case.run(stk, "first_k", 2, graph=True, launches=2)
    assert torch.equal(g["raw"], base["raw"])
    stk.close()


def test_bf16_mlp96_full_config():
    """Config 4 at full size (96 layers, M = 16).  End-to-end bf16 error of a
    96-layer stack is bounded by the rounding random walk:
    gate at max(1e-2, 2 x floor), floor = sqrt(2L) 2^-9 / sqrt(3)."""
    c = configs.C5
    case = Case(c.dims, c.acts, c.tokens, "bf16")
    ref = case.oracle(48)
    stk = case.stack()
    out = case.run(stk, "first_k", 48, graph=True)
    errs = max_err(out, ref)
    record_parity("g3_MLP96", {"config": c.name, "layers": c.L, "errors": errs, "floor": bf16_floor(c.L),
                               "gate": max(BF16_TOL, 2 * bf16_floor(c.L))})
    _check(errs, max(BF16_TOL, 2 * bf16_floor(c.L)))
    base = case.run(stk, "in_order", 0)
    assert torch.equal(out["raw"], base["raw"])


@pytest.mark.slow
def test_bf16_bert_base_full_config_end_to_end():
    """Config 1 (the bench workload) end to end at full size: 72 layers,
    M = 4096, graph-captured ooo_first_k as bench.py times it."""
    c = configs.C2
    case = Case(c.dims, c.acts, c.tokens, "bf16")
    ref = case.oracle(24)
    stk = case.stack()
    out = case.run(stk, "first_k", 24, graph=True)
    errs = max_err(out, ref)
    print("bert_base full-size errors", errs, "floor", bf16_floor(c.L))
    record_parity("g3_BERT-base", {"config": c.name, "layers": c.L, "errors": errs, "floor": bf16_floor(c.L),
                                   "gate": max(BF16_TOL, 2 * bf16_floor(c.L))})
    _check(errs, max(BF16_TOL, 2 * bf16_floor(c.L)))
    # bench.py's N = 1 schedule: Algorithm 1 regions of one block (§4.1), graph-captured
    stk.forward(to_dev(case.X, "bf16"))
    stk.plan_regions(region_layers=6)
    reg = case.run(stk, "regions", 0, graph=True, launches=2)
    assert torch.equal(reg["raw"], out["raw"])


# ------------------------------- fused step: backward(t) + forward(t+1)
@pytest.mark.parametrize("kind,k,tokens,need_dx", [("first_k", 2, 400, False), ("first_k", 5, 264, True),
                                                   ("in_order", 0, 512, False), ("first_k", 0, 136, False),
                                                   ("first_k", 2, 16, True), ("in_order", 0, 8, False)])
def test_bf16_fused_step_across_iterations(kind, k, tokens, need_dx):
    """ooo_backward(t); ooo_forward(X_{t+1}) runs as one engine launch whose
    F_i tiles overlap the deferred dW tiles (Fig. 4(c)).  Over three
    iterations with fresh inputs per step, check against the oracle the
    gradients of step t and Y of step t+1 (which must see the new X and no
    partially overwritten activations), and bit-exactness against the
    unfused sequence (backward; join; forward) on a second stack."""
    dims, acts = [192, 320, 256, 448, 256, 192], ["gelu", "id", "gelu", "gelu", "id"]
    cases = [Case(dims, acts, tokens, "bf16", need_dx=need_dx, step=t) for t in range(3)]
    fused = cases[0].stack(bucket_layers=2)
    plain = cases[0].stack(bucket_layers=2)
    Xs = [to_dev(c.X, "bf16") for c in cases]
    dYs = [to_dev(c.dY, "bf16") for c in cases]
    dXa = torch.empty(tokens, dims[0], dtype=TDT["bf16"], device="cuda") if need_dx else None
    dXb = torch.empty_like(dXa) if need_dx else None
    Ya = fused.forward(Xs[0])
    Yb = plain.forward(Xs[0])
    for t in range(3):
        ref = cases[t].oracle(k if kind == "first_k" else 0)
        torch.cuda.synchronize()
        assert rel_fro(to_np(Ya), ref.Y[0]) <= BF16_TOL, t
        assert torch.equal(Ya, Yb), t
        fused.backward(dYs[t], kind, k, dXa)
        plain.backward(dYs[t], kind, k, dXb)
        plain.join()
        if t < 2:
            Ya = fused.forward(Xs[t + 1])       # fused launch
            Yb = plain.forward(Xs[t + 1])
        else:
            fused.join()
        torch.cuda.synchronize()
        assert torch.equal(fused.grads_buf, plain.grads_buf), t
        if need_dx:
            assert torch.equal(dXa, dXb), t
        out = {"Y": ref.Y[0], "dW": [to_np(w) for w in fused.dW], "db": [to_np(v) for v in fused.db],
               "dX": to_np(dXa) if need_dx else None}
        _check(max_err(out, ref), BF16_TOL)
    fused.close()
    plain.close()


@pytest.mark.parametrize("tokens", [520, 16])
def test_bf16_fused_step_comm_gated(monkeypatch, tokens):
    """The N > 1 gating of the fused step (F_i waits for its bucket's
    all-reduce flag, written by the comm stream after cuStreamWaitValue32 on
    the bucket's dW counter) on one GPU: OOO_TEST_COMM_GATE runs that
    wait/write chain without the all-reduce.  Results must be bit-identical
    to the ungated stack (the all-reduce of one rank is the identity)."""
    dims, acts = [256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"]
    cases = [Case(dims, acts, tokens, "bf16", step=t) for t in range(3)]
    plain = cases[0].stack(bucket_layers=2)
    monkeypatch.setenv("OOO_TEST_COMM_GATE", "1")
    gated = cases[0].stack(bucket_layers=2)
    monkeypatch.delenv("OOO_TEST_COMM_GATE")
    Xs = [to_dev(c.X, "bf16") for c in cases]
    dYs = [to_dev(c.dY, "bf16") for c in cases]
    Ya, Yb = gated.forward(Xs[0]), plain.forward(Xs[0])
    for t in range(3):
        gated.backward(dYs[t], "first_k", 2)
        plain.backward(dYs[t], "first_k", 2)
        if t < 2:
            Ya, Yb = gated.forward(Xs[t + 1]), plain.forward(Xs[t + 1])
        else:
            gated.join()
            plain.join()
        torch.cuda.synchronize()
        assert torch.equal(Ya, Yb), t
        assert torch.equal(gated.grads_buf, plain.grads_buf), t
    _check(max_err({"Y": cases[2].oracle(2).Y[0], "dW": [to_np(w) for w in gated.dW],
                    "db": [to_np(v) for v in gated.db], "dX": None}, cases[2].oracle(2)), BF16_TOL)
    gated.close()
    plain.close()


@pytest.mark.parametrize("kind,k,tokens", [("first_k", 2, 520), ("first_k", 0, 520), ("in_order", 0, 520),
                                          ("first_k", 2, 16)])
def test_bf16_emulated_allreduce_graph(monkeypatch, kind, k, tokens):
    """The emulated N = 8 all-reduce (OOO_EMULATE_AR_N: the comm stream held
    for each bucket's ring time, 16-SM NCCL reserve; bench.py's emulated_dp)
    through the captured step as bench.py times it: bit-identical to the
    plain stack, within the gate of the oracle."""
    case = Case([256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"], tokens, "bf16")
    plain = case.stack(bucket_layers=2)
    base = case.run(plain, kind, k, graph=True, launches=2)
    plain.close()
    monkeypatch.setenv("OOO_EMULATE_AR_N", "8")
    monkeypatch.setenv("OOO_EMULATE_AR_GBPS", "50")
    emu = case.stack(bucket_layers=2)
    monkeypatch.delenv("OOO_EMULATE_AR_N")
    monkeypatch.delenv("OOO_EMULATE_AR_GBPS")
    out = case.run(emu, kind, k, graph=True, launches=2)
    assert torch.equal(out["raw"], base["raw"])
    _check(max_err(out, case.oracle(k)), BF16_TOL)
    emu.close()


# ------------------- single-GPU multi-stream ooo: Algorithm 1 regions (§4.1)
def _region_plan_valid(stk, L, need_dx=False):
    from oracle import schedule as S
    plan = stk.region_plan()
    D = plan["D"]
    assert S.is_valid_order(D, L, need_dx), D          # a topological order of the backward
    assert sorted(-op for op in D if op < 0) == list(range(1, L + 1))
    return plan


@pytest.mark.parametrize("tokens,rl,need_dx", [(384, 2, False), (264, 1, True), (136, 3, False), (16, 2, True)])
def test_bf16_regions_schedule_bit_exact(tokens, rl, need_dx):
    """OOO_SCHED_REGIONS (dW kernels placed by Algorithm 1 from profiled
    co-run speedups) gives the gradients of in_order bit for bit and the
    oracle's within the bf16 gate; eager and graph-captured alike."""
    case = Case([256, 512, 256, 1024, 256, 256, 512], ["id", "gelu", "gelu", "id", "gelu", "id"], tokens, "bf16",
                need_dx=need_dx)
    stk = case.stack(bucket_layers=2)
    stk.forward(to_dev(case.X, "bf16"))
    plan = stk.plan_regions(region_layers=rl, reps=1)
    _region_plan_valid(stk, case.L, need_dx)
    assert plan["n_regions"] >= 2 and all(t > 0 for t in plan["t_main_ms"])
    base = case.run(stk, "in_order", 0)
    out = case.run(stk, "regions", 0)
    assert torch.equal(out["raw"], base["raw"])
    if need_dx:
        assert np.array_equal(out["dX"], base["dX"])
    g = case.run(stk, "regions", 0, graph=True, launches=2)
    assert torch.equal(g["raw"], base["raw"])
    _check(max_err(out, case.oracle()), BF16_TOL)
    stk.close()


def test_bf16_regions_fused_step_and_memory_bound():
    """Regions across fused steps (backward(t) + forward(t+1) in one launch,
    deferred dW in forward regions) and the P:162 memory bound (max_temp_bytes
    below any deferral: the plan pre-schedules until nothing is held)."""
    dims, acts = [256, 512, 256, 256, 512, 256, 256], ["gelu", "id", "id", "gelu", "id", "id"]
    cases = [Case(dims, acts, 400, "bf16", step=t) for t in range(3)]
    a = cases[0].stack()
    b = cases[0].stack()
    Xs = [to_dev(c.X, "bf16") for c in cases]
    dYs = [to_dev(c.dY, "bf16") for c in cases]
    a.forward(Xs[0])
    a.plan_regions(region_layers=2)
    Ya, Yb = a.forward(Xs[0]), b.forward(Xs[0])
    for t in range(3):
        a.backward(dYs[t], "regions")
        b.backward(dYs[t], "in_order")
        if t < 2:
            Ya, Yb = a.forward(Xs[t + 1]), b.forward(Xs[t + 1])
        else:
            a.join()
            b.join()
        torch.cuda.synchronize()
        assert torch.equal(Ya, Yb), t
        assert torch.equal(a.grads_buf, b.grads_buf), t
    a.close()
    b.close()
    tight = cases[0].stack(max_temp_bytes=1)
    tight.forward(Xs[0])
    plan = tight.plan_regions(region_layers=1)
    assert 0 <= plan["k_pre"] <= plan["n_regions"]
    _region_plan_valid(tight, len(acts))
    out = cases[0].run(tight, "regions", 0)
    _check(max_err(out, cases[0].oracle()), BF16_TOL)
    tight.close()


def test_bf16_regions_full_size_block_slice():
    """Two BERT-base blocks at full width and 4096 tokens, one region per
    block (the paper's per-block regions)."""
    dims, acts, M = _block_slice(configs.C2, 2)
    case = Case(dims, acts, M, "bf16")
    stk = case.stack()
    stk.forward(to_dev(case.X, "bf16"))
    stk.plan_regions(region_layers=6)
    _region_plan_valid(stk, case.L)
    out = case.run(stk, "regions", 0, graph=True)
    base = case.run(stk, "in_order", 0)
    assert torch.equal(out["raw"], base["raw"])
    _check(max_err(out, case.oracle()), BF16_TOL)
    stk.close()


@pytest.mark.slow
@pytest.mark.parametrize("cfg", [configs.C3, configs.C4], ids=["bert_large", "gpt2_medium"])
def test_bf16_144_layer_full_configs_end_to_end(cfg):
    """Configs 2 and 3 end to end at full size (144 layers; 4096 / 512 tokens),
    graph-captured reverse first-k and the Algorithm 1 region schedule (bench
    launch configurations), gated at max(1e-2, 2 x the bf16 random-walk floor)
    (SURVEY §8c G3), and bit-exact with in_order."""
    case = Case(cfg.dims, cfg.acts, cfg.tokens, "bf16")
    ref = case.oracle(cfg.L // 6)
    stk = case.stack()
    out = case.run(stk, "first_k", cfg.L // 6, graph=True)
    errs = max_err(out, ref)
    print(cfg.name, "full-size errors", errs, "floor", bf16_floor(cfg.L))
    record_parity(f"g3_{cfg.name}", {"config": cfg.name, "layers": cfg.L, "errors": errs,
                                      "floor": bf16_floor(cfg.L), "gate": max(BF16_TOL, 2 * bf16_floor(cfg.L))})
    _check(errs, max(BF16_TOL, 2 * bf16_floor(cfg.L)))
    stk.forward(to_dev(case.X, "bf16"))
    stk.plan_regions(region_layers=6)
    reg = case.run(stk, "regions", 0, graph=True)
    assert torch.equal(reg["raw"], out["raw"])
    base = case.run(stk, "in_order", 0)
    assert torch.equal(base["raw"], out["raw"])
    stk.close()


def test_regions_error_paths():
    """OOO_SCHED_REGIONS without a plan -> OOO_ERR_STATE; planning an fp32
    stack -> OOO_ERR_UNSUPPORTED; a plan is discarded by nothing but a new
    plan, and planning leaves the stack needing a forward (OOO_ERR_STATE)."""
    from paper_conf_eurosys_ohlks22_b200._lib import OooError
    case = Case([256, 256, 256, 256], ["gelu", "id", "id"], 256, "bf16")
    stk = case.stack()
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    stk.forward(X)
    with pytest.raises(OooError, match="STATE"):
        stk.backward(dY, "regions")
    stk.forward(X)
    stk.plan_regions(region_layers=1)
    with pytest.raises(OooError, match="STATE"):
        stk.backward(dY, "regions")          # the profiling launches overwrote the activations
    stk.forward(X)
    stk.backward(dY, "regions")
    stk.join()
    stk.close()
    c32 = Case([256, 256, 256], ["relu", "id"], 32, "fp32")
    s32 = c32.stack()
    s32.forward(to_dev(c32.X, "fp32"))
    with pytest.raises(OooError, match="UNSUPPORTED"):
        s32.plan_regions()
    s32.close()


# ------------------------------------------------------------------ degenerate shapes
@pytest.mark.parametrize("dtype,need_dx", [("bf16", False), ("bf16", True), ("fp32", False), ("fp32", True)])
def test_single_layer_stack_all_schedules(dtype, need_dx):
    """L = 1: the step is the seed, dW_1 (and dO_1 with input grad) and F_1;
    every schedule degenerates to the same op list and must be bit-exact."""
    case = Case([320, 192], ["gelu"], 136, dtype, need_dx=need_dx)
    ref = case.oracle(1)
    stk = case.stack()
    base = None
    for kind, k in [("in_order", 0), ("first_k", 0), ("first_k", 1)]:
        out = case.run(stk, kind, k, graph=(dtype == "bf16" and kind == "first_k" and k == 1))
        _check(max_err(out, ref), BF16_TOL if dtype == "bf16" else FP32_TOL)
        if base is None:
            base = out["raw"]
        assert torch.equal(out["raw"], base), (kind, k)
    stk.close()


def test_bf16_narrowest_and_widest_widths():
    """The 64-wide minimum next to a 4096-wide FFN layer (widths at both ends
    of the tile plans), ragged token tail, with input grad."""
    case = Case([64, 4096, 64, 128], ["gelu", "relu", "id"], 200, "bf16", need_dx=True)
    ref = case.oracle(2)
    stk = case.stack()
    out = case.run(stk, "first_k", 2)
    _check(max_err(out, ref), BF16_TOL)
    inorder = case.run(stk, "in_order", 0)
    assert torch.equal(inorder["raw"], out["raw"])
    stk.close()


# ------------------- the N > 1 data plane on one GPU: a one-rank NCCL communicator
def _nccl_stack(case, monkeypatch, **kw):
    from paper_conf_eurosys_ohlks22_b200.stack import get_unique_id
    # the bit-exact setting SURVEY §8e pins for N > 1 (one rank: NCCL's own path)
    monkeypatch.setenv("NCCL_ALGO", "Ring")
    monkeypatch.setenv("NCCL_PROTO", "Simple")
    return case.stack(unique_id=get_unique_id(), **kw)


@pytest.mark.parametrize("kind,k,tokens", [("first_k", 2, 520), ("in_order", 0, 520), ("first_k", 5, 520),
                                          ("first_k", 2, 16)])
def test_bf16_nccl_one_rank_fused_steps_bit_exact(monkeypatch, kind, k, tokens):
    """A real NCCL communicator (world_size 1, ooo_get_unique_id) drives the
    whole N > 1 data plane through the captured fused step:
    per-bucket cuStreamWaitValue32 on the engine's dW counters ->
    ncclAllReduce -> cuStreamWriteValue32 of the flag F_i(t+1) waits on, with
    the 16-SM reserve.  Over three steps with fresh inputs the gradients and Y
    equal the non-communicating stack bit for bit (the all-reduce of one rank
    is the identity) and the oracle within the bf16 gate; the library's
    launch records show one all-reduce per bucket."""
    dims, acts = [256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"]
    cases = [Case(dims, acts, tokens, "bf16", step=t) for t in range(4)]
    plain = cases[0].stack(bucket_layers=2)
    comm = _nccl_stack(cases[0], monkeypatch, bucket_layers=2)
    Xb = [to_dev(cases[0].X, "bf16") for _ in range(2)]
    dYb = [to_dev(cases[0].dY, "bf16") for _ in range(2)]
    Yb = [torch.empty(cases[0].M, dims[-1], dtype=torch.bfloat16, device="cuda") for _ in range(2)]
    plain.forward(Xb[0], Yb[0])
    comm.forward(Xb[1], Yb[1])
    comm.set_timing(True)                    # launch records captured into the graph
    g = [plain.graph(Xb[0], Yb[0], dYb[0], kind, k), comm.graph(Xb[1], Yb[1], dYb[1], kind, k)]
    for t in range(3):
        for j in range(2):                   # step t's dY, step t+1's X into the captured buffers
            dYb[j].copy_(to_dev(cases[t].dY, "bf16"))
            Xb[j].copy_(to_dev(cases[t + 1].X, "bf16"))
            g[j].launch()
        torch.cuda.synchronize()
        assert torch.equal(comm.grads_buf, plain.grads_buf), t
        assert torch.equal(Yb[0], Yb[1]), t
        ref = cases[t].oracle(k if kind == "first_k" else 0)
        _check(max_err({"Y": ref.Y[0], "dW": [to_np(w) for w in comm.dW], "db": [to_np(v) for v in comm.db],
                        "dX": None}, ref), BF16_TOL)
        assert rel_fro(to_np(Yb[1]), cases[t + 1].oracle().Y[0]) <= BF16_TOL
    recs = comm.timing()
    assert sum(r["kind"] == "allreduce" for r in recs) == 3, recs     # ceil(5 / 2) buckets
    comm.set_timing(False)
    for x in g:
        x.close()
    # the stand-alone all-reduce of every bucket (bench's AR_ms): identity at one rank
    before = comm.grads_buf.clone()
    comm.allreduce_buckets()
    torch.cuda.synchronize()
    assert torch.equal(comm.grads_buf, before)
    plain.close()
    comm.close()


def test_bf16_nccl_one_rank_eager_rules(monkeypatch):
    """Eager use of a communicating stack: backward + join (all-reduces after
    the engine) is bit-exact with the plain stack; an eager fused step
    (forward with a backward pending) is refused with OOO_ERR_UNSUPPORTED
    (ooo.h), and the stack stays usable after the refusal."""
    from paper_conf_eurosys_ohlks22_b200._lib import OooError
    case = Case([256, 512, 256, 256], ["gelu", "id", "id"], 264, "bf16")
    plain = case.stack()
    comm = _nccl_stack(case, monkeypatch)
    a = case.run(plain, "first_k", 1)
    b = case.run(comm, "first_k", 1)
    assert torch.equal(a["raw"], b["raw"])
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    comm.forward(X)
    comm.backward(dY, "first_k", 1)
    with pytest.raises(OooError, match="UNSUPPORTED"):
        comm.forward(X)
    comm.join()
    torch.cuda.synchronize()
    assert torch.equal(comm.grads_buf, plain.grads_buf)
    plain.close()
    comm.close()


def test_bf16_misaligned_activation_rejected():
    """the engine stores 32-byte row vectors, so a 16-byte aligned
    view of Y (or X, dY, dX) is rejected before anything is enqueued."""
    from paper_conf_eurosys_ohlks22_b200._lib import OooError
    case = Case([256, 256], ["id"], 64, "bf16")
    stk = case.stack()
    X = to_dev(case.X, "bf16")
    big = torch.empty(64 * 256 + 8, dtype=torch.bfloat16, device="cuda")
    Ymis = big[8:].view(64, 256)                 # 16-byte offset
    with pytest.raises(OooError, match="aligned"):
        stk.forward(X, Ymis)
    stk.forward(X)
    stk.close()


def test_graph_timing_slots_every_launch():
    """ooo_graph_set_timing_slots: each of the timed launches of a captured
    step keeps its own per-kernel CUDA-event durations (bench.py's roofline
    takes the engine kernel's mean over all timed launches); the slots do
    not change the results."""
    case = Case([256, 512, 256, 256], ["gelu", "id", "id"], 520, "bf16")
    stk = case.stack()
    base = case.run(stk, "first_k", 1, graph=True, launches=1)
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    Y = stk.forward(X)
    stk.set_timing(True)
    g = stk.graph(X, Y, dY, "first_k", 1)
    stk.set_timing(False)
    g.set_timing_slots(6)
    for _ in range(8):
        g.launch()
    torch.cuda.synchronize()
    per = g.timing()
    assert len(per) == 6
    kinds = [r["kind"] for r in per[0]]
    assert "engine_step" in kinds and "seed" in kinds, kinds
    for recs in per:
        assert [r["kind"] for r in recs] == kinds
        assert all(r["ms"] > 0 for r in recs)
    starts = [recs[0]["start_ms"] for recs in per]
    assert starts == sorted(starts) and starts[-1] > starts[0]
    g.close()
    stk.join()
    torch.cuda.synchronize()
    assert torch.equal(stk.grads_buf, base["raw"])
    stk.close()


# ------------------- NEXT-4: prioritised, partitioned all-reduce issue (§5.1)
def _valid_chunk_order(order, nchunks):
    seen = {}
    for b, c in order:
        assert c == seen.get(b, 0), order
        seen[b] = c + 1
    assert seen == nchunks, (seen, nchunks)


@pytest.mark.parametrize("mode", ["nccl", "emulated"])
def test_bf16_prioritised_partitioned_comm_bit_exact(monkeypatch, mode):
    """comm_priority=1 with 64 KiB chunks: the captured fused steps issue
    every bucket's all-reduce as fixed chunks in the prioritised order (a
    valid chunk order: each bucket's chunks in sequence, all present), and
    give gradients / Y bit-identical to the plain stack over three steps,
    for both schedules -- a one-rank NCCL communicator (real ncclAllReduce
    per chunk) and the emulated 8-rank link."""
    dims, acts = [256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"]
    cases = [Case(dims, acts, 520, "bf16", step=t) for t in range(4)]
    kw = dict(bucket_layers=2, comm_priority=1, comm_chunk_bytes=64 * 1024)
    if mode == "nccl":
        comm = _nccl_stack(cases[0], monkeypatch, **kw)
    else:
        monkeypatch.setenv("OOO_EMULATE_AR_N", "8")
        monkeypatch.setenv("OOO_EMULATE_AR_GBPS", "50")
        comm = cases[0].stack(**kw)
        monkeypatch.delenv("OOO_EMULATE_AR_N")
        monkeypatch.delenv("OOO_EMULATE_AR_GBPS")
    plain = cases[0].stack(bucket_layers=2)
    # chunk count per bucket: bucket bytes / 64 KiB (32768 bf16 elements), rounded up
    nel = [dims[i] * dims[i + 1] + dims[i + 1] for i in range(len(acts))]
    buckets = [sum(nel[j] for j in range(b, min(b + 2, len(acts)))) for b in range(0, len(acts), 2)]
    nchunks = {b: -(-e // 32768) for b, e in enumerate(buckets)}
    for kind, k in (("first_k", 5), ("in_order", 0)):
        Xb = [to_dev(cases[0].X, "bf16") for _ in range(2)]
        dYb = [to_dev(cases[0].dY, "bf16") for _ in range(2)]
        Yb = [torch.empty(cases[0].M, dims[-1], dtype=torch.bfloat16, device="cuda") for _ in range(2)]
        plain.forward(Xb[0], Yb[0])
        comm.forward(Xb[1], Yb[1])
        g = [plain.graph(Xb[0], Yb[0], dYb[0], kind, k), comm.graph(Xb[1], Yb[1], dYb[1], kind, k)]
        _valid_chunk_order(comm.comm_issue_order(), nchunks)
        for t in range(3):
            for j in range(2):
                dYb[j].copy_(to_dev(cases[t].dY, "bf16"))
                Xb[j].copy_(to_dev(cases[t + 1].X, "bf16"))
                g[j].launch()
            torch.cuda.synchronize()
            assert torch.equal(comm.grads_buf, plain.grads_buf), (kind, t)
            assert torch.equal(Yb[0], Yb[1]), (kind, t)
        for x in g:
            x.close()
    ref = cases[2].oracle(0)
    _check(max_err({"Y": ref.Y[0], "dW": [to_np(w) for w in comm.dW], "db": [to_np(v) for v in comm.db],
                    "dX": None}, ref), BF16_TOL)
    plain.close()
    comm.close()


# ------------------- NEXT-3: cross-layer model parallelism (§5.2.1)
@pytest.mark.parametrize("n_stages,placement", [(2, "modulo"), (2, "contiguous"), (3, "modulo")])
def test_bf16_pipeline_fast_forward_and_modulo_bit_exact(n_stages, placement):
    """Groups of 6 layers (BERT-shaped blocks at width 256, identity at every
    group boundary) on n SM-partition stages: conventional backprop and
    gradient fast-forwarding give bit-identical gradients and Y, equal to the
    oracle's partitioned step (oracle/pipeline.py) within the bf16 gate, and
    dW bit-identical to the unpartitioned engine stack (reading M2), over two
    captured iterations."""
    from oracle import pipeline as PL
    from paper_conf_eurosys_ohlks22_b200.stack import Pipeline
    h, blocks = 256, 6
    dims, acts = [h], []
    for _ in range(blocks):
        dims += [h, h, h, h, 4 * h, h]
        acts += ["id", "id", "id", "id", "gelu", "id"]
    case = Case(dims, acts, 264, "bf16")
    Wt = [to_dev(w, "bf16") for w in case.W]
    bt = [to_dev(v, "bf16") for v in case.b]
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    outs = {}
    for ff in (False, True):
        pipe = Pipeline(dims, acts, case.M, Wt, bt, group_layers=6, n_stages=n_stages, placement=placement)
        Y = torch.empty(case.M, dims[-1], dtype=torch.bfloat16, device="cuda")
        g = pipe.graph(X, dY, Y, fast_forward=ff)
        for _ in range(2):
            g.launch()
        torch.cuda.synchronize()
        outs[ff] = (Y.clone(), pipe.grads_buf.clone(), [to_np(w) for w in pipe.dW], [to_np(v) for v in pipe.db])
        g.close()
        pipe.close()
    assert torch.equal(outs[False][0], outs[True][0]) and torch.equal(outs[False][1], outs[True][1])
    Yo, gW, gb = PL.mp_step(case.X, case.dY, case.W, case.b, acts, 6, "bf16")
    # 36 bf16 layers end to end: the G3 gate max(1e-2, 2 x the rounding random-walk floor)
    _check({"Y": rel_fro(to_np(outs[True][0]), Yo),
            "dW": max(rel_fro(a, r) for a, r in zip(outs[True][2], gW)),
            "db": max(rel_fro(a, r) for a, r in zip(outs[True][3], gb))}, max(BF16_TOL, 2 * bf16_floor(len(acts))))
    stk = case.stack()
    whole = case.run(stk, "first_k", 0)
    stk.close()
    assert all(np.array_equal(a, r) for a, r in zip(outs[True][2], whole["dW"]))
    # db of a group's top layer comes from the seed kernel's column sums (another fp32
    # summation order than the engine epilogue's): equal up to the final bf16 rounding
    assert max(rel_fro(a, r) for a, r in zip(outs[True][3], whole["db"])) < 4e-3


def test_graph_host_buffer_steps():
    """ooo_graph_upload / ooo_graph_launch_host (the e2e path bench.py times):
    two graphs over two buffer sets used alternately with pinned host
    buffers give, step for step, the Y (read back to host) and gradients of
    the device-buffer path."""
    cases = [Case([256, 512, 256, 256], ["gelu", "id", "id"], 264, "bf16", step=t) for t in range(4)]
    ref = cases[0].stack()
    stk = cases[0].stack()
    bufs = []
    for p in range(2):
        X = to_dev(cases[0].X, "bf16")
        dY = to_dev(cases[0].dY, "bf16")
        Y = stk.forward(X)
        torch.cuda.synchronize()
        bufs.append({"g": stk.graph(X, Y, dY, "first_k", 1),
                     "hX": torch.empty(X.shape, dtype=X.dtype, pin_memory=True),
                     "hdY": torch.empty(dY.shape, dtype=dY.dtype, pin_memory=True),
                     "hY": torch.empty(Y.shape, dtype=Y.dtype, pin_memory=True)})
    # both graphs' buffers hold forward(cases[0].X) state; the stack's stores hold the last forward
    cs = torch.cuda.Stream()
    Xr = to_dev(cases[0].X, "bf16")
    ref.forward(Xr)
    for t in range(3):
        b = bufs[t % 2]
        b["hX"].copy_(torch.from_numpy(cases[t + 1].X).to(torch.bfloat16))
        b["hdY"].copy_(torch.from_numpy(cases[t].dY).to(torch.bfloat16))
        b["g"].upload(b["hX"], b["hdY"], cs)
        b["g"].launch_host(b["hY"], torch.cuda.current_stream(), cs)
        torch.cuda.synchronize()
        ref.backward(to_dev(cases[t].dY, "bf16"), "first_k", 1)
        ref.join()
        Yr = ref.forward(to_dev(cases[t + 1].X, "bf16"))
        torch.cuda.synchronize()
        assert torch.equal(b["hY"], Yr.cpu()), t
        assert torch.equal(stk.grads_buf, ref.grads_buf), t
    for b in bufs:
        b["g"].close()
    stk.close()
    ref.close()


def test_bf16_pipeline_nccl_loopback(monkeypatch):
    """The multi-rank pipeline data plane on one GPU: a one-rank communicator
    in loopback (every group boundary is an ncclSend / ncclRecv to itself on
    the comm stream, dX sent after ooo_input_grad_wait mid-kernel or after the
    whole backward) gives Y and gradients bit-identical to the SM-partition
    pipeline, fast-forwarded and conventional."""
    from paper_conf_eurosys_ohlks22_b200.stack import Pipeline, get_unique_id
    monkeypatch.setenv("NCCL_ALGO", "Ring")
    monkeypatch.setenv("NCCL_PROTO", "Simple")
    h = 256
    dims, acts = [h], []
    for _ in range(4):
        dims += [h, h, 4 * h, h]
        acts += ["id", "id", "gelu", "id"]
    case = Case(dims, acts, 264, "bf16")
    Wt = [to_dev(w, "bf16") for w in case.W]
    bt = [to_dev(v, "bf16") for v in case.b]
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    for ff in (True, False):
        res = []
        for mode in ("partition", "loopback"):
            kw = dict(n_stages=2) if mode == "partition" else dict(n_stages=1, unique_id=get_unique_id())
            pipe = Pipeline(dims, acts, case.M, Wt, bt, group_layers=4, placement="modulo", **kw)
            Y = torch.empty(case.M, dims[-1], dtype=torch.bfloat16, device="cuda")
            g = pipe.graph(X, dY, Y, fast_forward=ff)
            for _ in range(2):
                g.launch()
            torch.cuda.synchronize()
            res.append((Y.clone(), torch.cat([w.reshape(-1) for w in pipe.dW] + list(pipe.db))))
            g.close()
            pipe.close()
        assert torch.equal(res[0][0], res[1][0]), ff
        assert torch.equal(res[0][1], res[1][1]), ff


@pytest.mark.parametrize("dtype,n", [("bf16", 4), ("bf16", 8), ("fp32", 2)])
def test_pack_scale_average_over(dtype, n):
    """The pack/scale step (reading Q9) with a divisor != 1 on
    the GPU: average_over = n scales every dW_i / db_i by 1/n before the
    all-reduce; a power of two, so the result is the unscaled gradient / n
    exactly (bf16 and fp32), for the engine (bf16) and the per-layer path
    (fp32), and the oracle's N-rank mean of n identical shards."""
    case = Case([256, 512, 256, 128], ["gelu", "id", "id"], 264 if dtype == "bf16" else 64, dtype)
    plain = case.stack()
    scaled = case.stack(average_over=n)
    a = case.run(plain, "first_k", 1)
    b = case.run(scaled, "first_k", 1, graph=dtype == "bf16")
    for x, y in zip(a["dW"] + a["db"], b["dW"] + b["db"]):
        assert np.array_equal(x / n, y)
    from oracle import layers as O
    from oracle import schedule as S
    ref = O.dp_step([case.X] * n, [case.dY] * n, case.W, case.b, case.acts, S.reverse_first_k(case.L, 1),
                    "bf16" if dtype == "bf16" else "fp64")
    # the oracle's mean over n identical shards is the local gradient; ours is it / n
    _check({"dW": max(rel_fro(g * n, r) for g, r in zip(b["dW"], ref.gW)),
            "db": max(rel_fro(g * n, r) for g, r in zip(b["db"], ref.gb))}, BF16_TOL if dtype == "bf16" else FP32_TOL)
    plain.close()
    scaled.close()


def test_wait_bound_traps_instead_of_hanging():
    """Hang protection: with a bucket's all-reduce flag never
    written, F_i(t+1) can never start; the engine's waits are bounded by the
    stack's wait_timeout_ms (1.5 s here) and the step fails with a CUDA error
    instead of hanging the GPU.  Run in child processes (a trap ends the CUDA
    context); the control run with the flag written completes."""
    import subprocess
    import sys
    import time
    child = __file__.rsplit("/", 1)[0] + "/helpers/trap_child.py"
    r = subprocess.run([sys.executable, child], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, (r.returncode, r.stdout[-500:], r.stderr[-500:])
    t0 = time.time()
    r = subprocess.run([sys.executable, child, "drop"], capture_output=True, text=True, timeout=300)
    assert r.returncode == 3, (r.returncode, r.stdout[-500:], r.stderr[-500:])
    assert time.time() - t0 < 120
