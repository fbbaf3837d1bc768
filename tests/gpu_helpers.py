"""Shared helpers for the ``-m gpu`` parity tests: seeded inputs -> both the
oracle (NumPy fp64) and the CUDA path (through the C ABI via the ctypes
binding).  No expected value is ever derived from the CUDA path."""
from __future__ import annotations

import math

import numpy as np
import torch

from oracle import layers as O
from oracle import schedule as S
from paper_conf_eurosys_ohlks22_b200 import synth
from paper_conf_eurosys_ohlks22_b200.stack import OooStack

TDT = {"bf16": torch.bfloat16, "fp32": torch.float32}


def to_dev(a: np.ndarray, dtype: str) -> torch.Tensor:
    # values are already representable in the storage dtype -> exact cast
    return torch.from_numpy(np.ascontiguousarray(a)).to(TDT[dtype]).cuda().contiguous()


def to_np(t: torch.Tensor) -> np.ndarray:
    return t.detach().float().cpu().numpy().astype(np.float64)


class Case:
    """Seeded inputs of one stack shape (reading Q13)."""

    def __init__(self, dims, acts, tokens, dtype, need_dx=False, seed=synth.SEED, rank=0, step=0):
        self.dims, self.acts, self.M, self.dtype, self.need_dx = list(dims), list(acts), tokens, dtype, need_dx
        self.L = len(acts)
        self.W, self.b = synth.weights(dims, acts, dtype, seed)
        self.X = synth.x_shard(tokens, dims[0], rank, dtype, seed, step)
        self.dY = synth.dy_shard(tokens, dims[-1], rank, dtype, seed, step)

    def oracle(self, k=0):
        D = S.reverse_first_k(self.L, k, self.need_dx)
        return O.dp_step([self.X], [self.dY], self.W, self.b, self.acts, D,
                         "bf16" if self.dtype == "bf16" else "fp64")

    def stack(self, **kw) -> OooStack:
        Wt = [to_dev(w, self.dtype) for w in self.W]
        bt = [to_dev(v, self.dtype) for v in self.b]
        return OooStack(self.dims, self.acts, self.M, Wt, bt, dtype=self.dtype,
                        need_input_grad=self.need_dx, **kw)

    def run(self, stk: OooStack, kind="first_k", k=0, graph=False, launches=1):
        Xt = to_dev(self.X, self.dtype)
        dYt = to_dev(self.dY, self.dtype)
        dX = torch.empty(self.M, self.dims[0], dtype=TDT[self.dtype], device="cuda") if self.need_dx else None
        Y = stk.forward(Xt)
        Y0 = Y.clone()
        if graph:
            g = stk.graph(Xt, Y, dYt, kind, k, dX)
            for _ in range(launches):
                g.launch()
            torch.cuda.synchronize()
            g.close()
        else:
            stk.backward(dYt, kind, k, dX)
            stk.join()
        torch.cuda.synchronize()
        return {
            "Y": to_np(Y0),
            "dW": [to_np(w) for w in stk.dW],
            "db": [to_np(v) for v in stk.db],
            "dX": to_np(dX) if dX is not None else None,
            "raw": stk.grads_buf.clone(),
        }


def max_err(gpu, ref) -> dict:
    errs = {"Y": O.rel_fro(gpu["Y"], ref.Y[0])}
    errs["dW"] = max(O.rel_fro(g, r) for g, r in zip(gpu["dW"], ref.gW))
    errs["db"] = max(O.rel_fro(g, r) for g, r in zip(gpu["db"], ref.gb))
    if gpu["dX"] is not None:
        errs["dX"] = O.rel_fro(gpu["dX"], ref.dX[0])
    return errs


def record_parity(name: str, data: dict) -> None:
    """Append measured errors to $OOO_PARITY_OUT (JSON lines) when set, so a
    GPU run can commit the table of measured errors (profiles/r02_parity.md)."""
    import json
    import os
    path = os.environ.get("OOO_PARITY_OUT")
    if path:
        with open(path, "a") as f:
            f.write(json.dumps({"test": name, **data}) + "\n")


def bf16_floor(L: int) -> float:
    """Random-walk floor of two independently rounded bf16 pipelines
    (SURVEY §8c G3): sqrt(2L) * 2^-9 / sqrt(3)."""
    return math.sqrt(2 * L) * 2.0 ** -9 / math.sqrt(3)
