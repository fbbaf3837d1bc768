"""Oracle: forward/backward of a dense-layer stack, executed op by op.

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``): the product path never
imports this module.

What is computed (the plain definition; the method only *reorders* it, P:260
"our optimizations do not change the semantics", §8):

  Layer i (1-based, i = 1..L), paper §2 P:84-89 / §3 P:99:
      F_i      :  Z_i = X_i W_i + 1 b_i^T ;   X_{i+1} = act_i(Z_i)
  Backward, seeded by the loss gradient dO_{L+1} ("T(dO_{L+1}) = 0",
  P:93), here the upstream gradient dY = dL/dX_{L+1}:
      seed     :  G_L = dY * act_L'(Z_L)
      dO_i     :  G_{i-1} = (G_i W_i^T) * act_{i-1}'(Z_{i-1})   (i >= 2)
                  dX      =  G_1 W_1^T                          (i == 1, only
                  when the input gradient is requested; reading Q1)
      dW_i     :  dW_i = X_i^T G_i ,  db_i = 1^T G_i
  The output gradient dO_i feeds the next (lower) layer; the weight gradient
  dW_i "is not used to compute any other gradients; it is only used to update
  the layer's weight parameters" (§3), so any order of the dW ops that
  respects "dW_i after G_i exists" gives identical results (pinned in tests).

  Data parallelism (§5.1): every rank r holds the same W, b and its
  own token shard; the synchronised gradient S[dW_i] is the rank average
  gbar_i = (1/N) sum_r dW_i^(r)  (reading Q9: mean, pre-scaled by 1/N).

bf16 storage mode (reading Q10/Q11 of DESIGN.md): the GPU stores tensors in
bf16 and accumulates in fp32.  The oracle mirrors each *storage* point by
rounding to bf16 (round-to-nearest-even via fp32) and computes every product
and sum in float64: inputs, W, b, Z_i, X_{i+1}, G_i, each rank's scaled
dW/db, and the final average.

Activations (reading of DESIGN.md): identity, ReLU (relu'(0) = 0), GELU with
the exact erf form gelu(z) = z Phi(z), gelu'(z) = Phi(z) + z phi(z).
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np
from scipy.special import erf

ACTS = ("id", "relu", "gelu")


# ---------------------------------------------------------------- rounding
def round_bf16(x: np.ndarray) -> np.ndarray:
    """Round to bfloat16 with round-to-nearest-even, via float32 (Q11).

    Returns float64 values that are exactly representable in bf16.  NaN stays
    NaN, +-inf stays inf.  Pinned against ``torch.Tensor.to(torch.bfloat16)``.
    """
    x32 = np.asarray(x, dtype=np.float64).astype(np.float32)
    u = x32.view(np.uint32).astype(np.uint64)
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    r = ((u + np.uint64(0x7FFF) + lsb) & np.uint64(0xFFFF0000)).astype(np.uint32)
    nan = np.isnan(x32)
    r = np.where(nan, np.uint32(0x7FC00000), r)
    return r.view(np.float32).astype(np.float64)


def round_fp32(x: np.ndarray) -> np.ndarray:
    return np.asarray(x, dtype=np.float64).astype(np.float32).astype(np.float64)


def storage_round(x: np.ndarray, dtype: str) -> np.ndarray:
    if dtype == "bf16":
        return round_bf16(x)
    if dtype == "fp32":
        return round_fp32(x)
    if dtype == "fp64":
        return np.asarray(x, dtype=np.float64)
    raise ValueError(dtype)


# ------------------------------------------------------------- activations
def act_fwd(name: str, z: np.ndarray) -> np.ndarray:
    if name == "id":
        return z.copy()
    if name == "relu":
        return np.where(z > 0.0, z, 0.0)
    if name == "gelu":
        return z * 0.5 * (1.0 + erf(z / math.sqrt(2.0)))
    raise ValueError(name)


def act_grad(name: str, z: np.ndarray) -> np.ndarray:
    """d act / dz evaluated at z (closed forms; pinned against finite differences)."""
    if name == "id":
        return np.ones_like(z)
    if name == "relu":
        return np.where(z > 0.0, 1.0, 0.0)
    if name == "gelu":
        cdf = 0.5 * (1.0 + erf(z / math.sqrt(2.0)))
        pdf = np.exp(-0.5 * z * z) / math.sqrt(2.0 * math.pi)
        return cdf + z * pdf
    raise ValueError(name)


# ------------------------------------------------- single steps (per op)
# The arithmetic of one op from given inputs, in float64 without storage
# rounding.  forward / op_dO / op_dW below are built from these, so every pin
# of the full stack (finite differences, fp64 autograd, P:99 invariance) also
# pins them; the teacher-forced GPU tests call them on the
# GPU's own stored inputs of each step.
def step_F(X: np.ndarray, W: np.ndarray, b: np.ndarray) -> np.ndarray:
    """F_i (§2): Z_i = X_i W_i + 1 b_i^T."""
    return X @ W + b[None, :]


def step_dO(G: np.ndarray, W: np.ndarray, factor: np.ndarray | None) -> np.ndarray:
    """dO_i: (G_i W_i^T) * act_{i-1}'(Z_{i-1}); factor None = dX (i == 1)."""
    P = G @ W.T
    return P if factor is None else P * factor


def step_dW(X: np.ndarray, G: np.ndarray) -> tuple:
    """dW_i: (X_i^T G_i, 1^T G_i)."""
    return X.T @ G, G.sum(axis=0)


# ------------------------------------------------------------------ forward
@dataclass
class ForwardState:
    """Stored activations of one forward pass F_1..F_L ("the computed
    outputs are stored for backpropagation").  Index 0 is layer 1."""
    X: list            # X[i-1] = X_i (input of layer i); X[L] = X_{L+1} = Y
    Z: list            # Z[i-1] = Z_i


def forward(X1: np.ndarray, W: list, b: list, acts: list, dtype: str = "fp64") -> ForwardState:
    """F_1 .. F_L in layer order (P:84 constraint T(F_{i+1}) >= T(F_i) + F_i)."""
    L = len(W)
    assert len(b) == L and len(acts) == L
    Xs = [storage_round(X1, dtype)]
    Zs = []
    for i in range(L):
        Z = storage_round(step_F(Xs[i], W[i], b[i]), dtype)
        Zs.append(Z)
        Xs.append(storage_round(act_fwd(acts[i], Z), dtype))
    return ForwardState(X=Xs, Z=Zs)


# ----------------------------------------------------------------- backward
@dataclass
class BackwardState:
    """Gradients produced while executing a schedule D (one rank)."""
    G: dict = field(default_factory=dict)     # G[i] = dZ_i
    dW: dict = field(default_factory=dict)    # dW[i]
    db: dict = field(default_factory=dict)    # db[i]
    dX: np.ndarray | None = None
    order: list = field(default_factory=list)


def seed(state: ForwardState, dY: np.ndarray, acts: list, dtype: str) -> np.ndarray:
    """dO_{L+1}: G_L = dY * act_L'(Z_L)."""
    L = len(acts)
    return storage_round(storage_round(dY, dtype) * act_grad(acts[L - 1], state.Z[L - 1]), dtype)


def op_dO(i: int, bs: BackwardState, state: ForwardState, W: list, acts: list, dtype: str) -> None:
    """Output-gradient op dO_i: consumes G_i, produces G_{i-1}
    (or dX for i == 1)."""
    if i not in bs.G:
        raise RuntimeError(f"dO_{i} scheduled before G_{i} exists (violates P:84 dependency)")
    if i == 1:
        bs.dX = storage_round(step_dO(bs.G[i], W[i - 1], None), dtype)
    else:
        bs.G[i - 1] = storage_round(step_dO(bs.G[i], W[i - 1], act_grad(acts[i - 2], state.Z[i - 2])), dtype)
    bs.order.append(+i)


def op_dW(i: int, bs: BackwardState, state: ForwardState) -> None:
    """Weight-gradient op dW_i: dW_i = X_i^T G_i, db_i = 1^T G_i.
    Unscaled and unrounded; rank averaging + storage rounding happen in
    ``dp_average`` (S[dW_i], §5.1)."""
    if i not in bs.G:
        raise RuntimeError(f"dW_{i} scheduled before G_{i} exists (violates P:84 dependency)")
    bs.dW[i], bs.db[i] = step_dW(state.X[i - 1], bs.G[i])
    bs.order.append(-i)


def run_backward(D: list, state: ForwardState, dY: np.ndarray, W: list, acts: list,
                 dtype: str = "fp64") -> BackwardState:
    """Execute a backward schedule D (list of +i = dO_i, -i = dW_i) op by op.

    Raises if D violates a dependency.  The result must not depend on D
    (P:99); the tests check bit equality over every D(L, k) and over random
    topological orders.
    """
    L = len(W)
    bs = BackwardState()
    bs.G[L] = seed(state, dY, acts, dtype)
    for op in D:
        if op > 0:
            op_dO(op, bs, state, W, acts, dtype)
        elif op < 0:
            op_dW(-op, bs, state)
        else:
            raise ValueError("op 0")
    missing = [i for i in range(1, L + 1) if i not in bs.dW]
    if missing:
        raise RuntimeError(f"schedule did not compute dW for layers {missing}")
    return bs


# ------------------------------------------------------- data parallelism
def dp_average(per_rank: list, L: int, dtype: str) -> tuple[list, list]:
    """S[dW_i] for all i: gbar_i = (1/N) sum_r dW_i^(r) (§5.1 P:176-180,
    reading Q9).  In bf16 mode each rank's scaled gradient is stored in bf16
    before the sum (the GPU's bucket) and the result is rounded once."""
    N = len(per_rank)
    gW, gb = [], []
    for i in range(1, L + 1):
        sW = np.zeros_like(per_rank[0].dW[i])
        sb = np.zeros_like(per_rank[0].db[i])
        for bs in per_rank:
            sW = sW + storage_round(bs.dW[i] * (1.0 / N), dtype)
            sb = sb + storage_round(bs.db[i] * (1.0 / N), dtype)
        gW.append(storage_round(sW, dtype))
        gb.append(storage_round(sb, dtype))
    return gW, gb


@dataclass
class StepResult:
    gW: list                 # averaged dW_i, i = 1..L (index 0 = layer 1)
    gb: list
    Y: list                  # per-rank X_{L+1}
    dX: list                 # per-rank input gradient (None unless requested)
    fwd: list                # per-rank ForwardState
    bwd: list                # per-rank BackwardState


def dp_step(X_shards: list, dY_shards: list, W: list, b: list, acts: list, D: list,
            dtype: str = "fp64") -> StepResult:
    """One data-parallel iteration on N simulated ranks: forward, backward in
    schedule D, then the averaged gradient sync.  W, b must already be
    storage-rounded by the caller (they are shared)."""
    L = len(W)
    fwds, bwds = [], []
    for X, dY in zip(X_shards, dY_shards):
        st = forward(X, W, b, acts, dtype)
        fwds.append(st)
        bwds.append(run_backward(D, st, dY, W, acts, dtype))
    gW, gb = dp_average(bwds, L, dtype)
    return StepResult(gW=gW, gb=gb, Y=[f.X[L] for f in fwds], dX=[b_.dX for b_ in bwds],
                      fwd=fwds, bwd=bwds)


def loss_surrogate(Y: np.ndarray, dY: np.ndarray) -> float:
    """Reading Q8: the boundary takes dY directly; the finite-difference test
    uses l = sum(dY * Y) so that dl/dY = dY exactly."""
    return float(np.sum(dY * Y))


def rel_fro(a: np.ndarray, ref: np.ndarray) -> float:
    """max-relative Frobenius error used by the parity gates (north star)."""
    a = np.asarray(a, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    den = np.linalg.norm(ref)
    num = np.linalg.norm(a - ref)
    if den == 0.0:
        return float(num)
    return float(num / den)
