"""Oracle: cross-layer model parallelism with gradient fast-forwarding and
modulo layer allocation (§5.2.1).

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).

What the method computes: the same gradients as the unpartitioned stack --
model parallelism only places layers on GPUs, and fast-forwarding / modulo
allocation only reorder ("prioritizes the executions of the output
gradient computations over those of the weight gradient computations";
P:234 "we allocate l'th layer ... to GPU_{l mod n}").  What changes is where
the stages hand tensors over: a group's output is the next group's input
(forward), and a group's input gradient dX is the previous group's dY
(backward, "the output gradient ... to the next GPU").  Readings
(M1-M3):

M1  the unit of allocation is a group of consecutive layers (the paper
    allocates transformer blocks);
M2  the hand-off tensors are stored in the storage dtype: group j's seed is
    dZ_L = st(st(dX_{j+1}) * act'(Z_L)) -- one extra rounding of dX versus the
    unpartitioned stack, none when the boundary layer's activation is the
    identity (the BERT/GPT blocks of the configs);
M3  the timing of fast-forwarding and modulo allocation is the unit-time
    model of Fig. 5 (oracle/unit_sim.mp_iteration: 23 / 19 / 16).

The schedule inside a group does not matter for the values; this
oracle runs each group's backward in reverse first-k(all) order (every dW
after the dO chain: fast-forwarding).
"""
from __future__ import annotations

import numpy as np

from . import layers as O
from . import schedule as S


def mp_step(X: np.ndarray, dY: np.ndarray, W: list, b: list, acts: list, group_layers: int,
            dtype: str = "fp64") -> tuple:
    """One iteration of the partitioned stack.  Returns (Y, gW, gb): the
    output and every layer's weight / bias gradient (one data-parallel rank:
    storage-rounded like the unpartitioned oracle's S[dW])."""
    L = len(W)
    if L % group_layers:
        raise ValueError("group_layers must divide L")
    G = L // group_layers
    grp = [list(range(j * group_layers, (j + 1) * group_layers)) for j in range(G)]
    states = []
    x = O.storage_round(X, dtype)
    for j in range(G):                                     # forward: group j's output -> group j+1's input
        st = O.forward(x, [W[i] for i in grp[j]], [b[i] for i in grp[j]], [acts[i] for i in grp[j]], dtype)
        states.append(st)
        x = st.X[-1]
    Y = x
    gW, gb = [None] * L, [None] * L
    dy = O.storage_round(dY, dtype)
    for j in range(G - 1, -1, -1):                         # backward: dX of group j -> dY of group j-1
        need_dx = j > 0
        D = S.reverse_first_k(group_layers, group_layers, need_dx)
        bs = O.run_backward(D, states[j], dy, [W[i] for i in grp[j]], [acts[i] for i in grp[j]], dtype)
        for li, i in enumerate(grp[j]):
            gW[i] = O.storage_round(bs.dW[li + 1], dtype)
            gb[i] = O.storage_round(bs.db[li + 1], dtype)
        if need_dx:
            dy = bs.dX
    return Y, gW, gb
