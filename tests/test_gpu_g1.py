"""G1 teacher-forced parity (SURVEY §8c, table "G1"): every step of the GPU
path -- F_i, the loss-gradient seed, dO_i, dW_i / db_i -- recomputed by the
oracle in float64 from the GPU's OWN stored inputs of that step, for every
layer of every bf16 config at full size (C2 BERT-base 72 layers, C3
BERT-large 144, C4 GPT-2-medium 144 at 512 tokens, C5 MLP96 at 16 tokens),
in the launch configuration bench.py times (captured fused step).

Unlike the end-to-end gate (G3), no rounding random walk accumulates over
the depth, so the bar is 1e-2 per step (expected ~2e-3: one bf16 rounding of
the output, 2^-9 relative).  Each step's error is the relative Frobenius
norm over a seeded sample of its output: 64 token rows of F_i / dO_i (all
columns), 64 rows (input features) of dW_i (full K = M reduction), all of
db_i.  The inputs read back through ooo_tensor (X_i, the Z_i store -- which
holds gelu'(Z_i) for GELU layers of the bf16 engine, readings --
and dZ_i) are the GPU's; the expected values are the oracle's step functions
(oracle/layers.py step_F / step_dO / step_dW / act_fwd / act_grad).

OOO_PARITY_OUT=<file.json>: the measured per-config maxima are appended
there (profiles/r02_parity.md is written from it).
"""
import numpy as np
import pytest
import torch

from oracle import layers as O
from paper_conf_eurosys_ohlks22_b200 import configs
from tests.gpu_helpers import Case, record_parity, to_dev, to_np

pytestmark = pytest.mark.gpu

TOL = 1e-2
SAMPLE = 64


def _rows(n, k, rng):
    return np.sort(rng.choice(n, size=min(k, n), replace=False))


def teacher_forced(case, stk, Y, rng):
    """Per-step errors of the GPU stores left by forward(X); backward(dY);
    join -- each step recomputed from its own GPU inputs."""
    L, M = case.L, case.M
    W = case.W                                     # host copies of the bf16 weights (exact)
    b = case.b
    errs = {"F": [], "F_zstore": [], "seed": [], "dO": [], "dW": [], "db": []}
    g = lambda t, idx=None: to_np(t if idx is None else t[idx])  # noqa: E731
    rows_t = torch.from_numpy(_rows(M, SAMPLE, rng)).cuda()
    rows = rows_t.cpu().numpy()
    for i in range(1, L + 1):
        act = case.acts[i - 1]
        Xi = g(stk.tensor("X", i), rows_t)
        Xn = g(Y if i == L else stk.tensor("X", i + 1), rows_t)
        Zref = O.step_F(Xi, W[i - 1], b[i - 1])
        errs["F"].append(O.rel_fro(Xn, O.act_fwd(act, Zref)))
        zs = stk.tensor("Z", i)
        if act == "gelu":
            errs["F_zstore"].append(O.rel_fro(g(zs, rows_t), O.act_grad("gelu", Zref)))
        elif act == "relu":
            errs["F_zstore"].append(O.rel_fro(g(zs, rows_t), Zref))
    # seed: dZ_L = dY * act_L'(Z_L)
    zL = stk.tensor("Z", L)
    dYs = case.dY[rows]
    if case.acts[-1] == "id":
        fac = np.ones_like(dYs)
    elif case.acts[-1] == "gelu":
        fac = g(zL, rows_t)                         # stored gelu'(Z_L)
    else:
        fac = (g(zL, rows_t) > 0).astype(np.float64)
    errs["seed"].append(O.rel_fro(g(stk.tensor("dZ", L), rows_t), dYs * fac))
    for i in range(L, 1, -1):
        Gi = g(stk.tensor("dZ", i), rows_t)
        prev = case.acts[i - 2]
        if prev == "id":
            fac = None
        elif prev == "gelu":
            fac = g(stk.tensor("Z", i - 1), rows_t)             # the GPU's stored gelu'(Z_{i-1})
        else:
            fac = O.act_grad("relu", g(stk.tensor("Z", i - 1), rows_t))
        errs["dO"].append(O.rel_fro(g(stk.tensor("dZ", i - 1), rows_t), O.step_dO(Gi, W[i - 1], fac)))
    for i in range(1, L + 1):
        din = case.dims[i - 1]
        feat = torch.from_numpy(_rows(din, SAMPLE, rng)).cuda()
        Xc = to_np(stk.tensor("X", i)[:, feat])                  # M x |feat|
        G = to_np(stk.tensor("dZ", i))                           # M x d_i
        dWs, dbs = O.step_dW(Xc, G)
        errs["dW"].append(O.rel_fro(to_np(stk.dW[i - 1][feat]), dWs))
        errs["db"].append(O.rel_fro(to_np(stk.db[i - 1]), dbs))
    return {k: (max(v) if v else None) for k, v in errs.items()}, {k: len(v) for k, v in errs.items()}


@pytest.mark.parametrize("cfg", [configs.C2, configs.C3, configs.C4, configs.C5],
                         ids=["bert_base", "bert_large", "gpt2_medium", "mlp96"])
def test_g1_teacher_forced_every_layer_full_size(cfg):
    case = Case(cfg.dims, cfg.acts, cfg.tokens, "bf16")
    stk = case.stack(bucket_layers=6 if cfg.L % 6 == 0 else 1)
    X, dY = to_dev(case.X, "bf16"), to_dev(case.dY, "bf16")
    Y = stk.forward(X)
    k = cfg.L // 6
    # bench.py's launch configuration: the captured fused step [backward; forward]
    # -- replayed once with the same X, so the stores afterwards hold forward(X)
    # and the backward of the forward(X) before it; the gradients of that
    # backward sit in `grads`.  dZ_i stays from the backward.
    g = stk.graph(X, Y, dY, "first_k", k)
    g.launch()
    torch.cuda.synchronize()
    g.close()
    rng = np.random.default_rng(20220405)
    worst, counts = teacher_forced(case, stk, Y, rng)
    print(cfg.name, "G1 per-step max errors", worst, counts)
    record_parity(f"g1_{cfg.name}", {"config": cfg.name, "layers": cfg.L, "tokens": cfg.tokens, "max_err": worst,
                              "steps_checked": counts, "tol": TOL})
    for kind, v in worst.items():
        if v is not None:
            assert v <= TOL, (kind, v, worst)
    stk.close()
