"""Seeded synthetic inputs (reading Q13 of DESIGN.md).

This module holds input *generators only* -- no arithmetic of the method.  It
is the one module both the oracle-side tests and the CUDA-side tests/bench
draw inputs from, so the two sides consume identical bits.

Recipe (the paper trains real BERT/GPT/ResNet and publishes no tensors, so the
workloads are matched in shape, not in values):
  * W_i (d_{i-1} x d_i): (semi-)orthogonal, from the QR of a Gaussian matrix,
    gain 1 (identity / GELU) or sqrt(2) (ReLU), times sqrt(d_i / d_{i-1}) when
    the layer expands.  Orthogonal init keeps deep bf16 stacks well
    conditioned (SURVEY §8c evidence).
  * b_i ~ N(0, 0.1^2).
  * X (M x d_0) and dY (M x d_L) ~ N(0, 1).
  * numpy ``default_rng([seed, tag, ...])``: tag 0 = X (per rank), 1 = dY
    (per rank), 2 = W_i / b_i (shared by every rank, per layer).
  * Everything generated in float64 and rounded to the storage dtype by the
    caller-visible helper ``to_storage`` (bf16 RNE via fp32, or fp32).
"""
from __future__ import annotations

import math

import numpy as np

SEED = 20220405


def _rng(*key) -> np.random.Generator:
    return np.random.default_rng([int(k) for k in key])


def _bits_bf16(x: np.ndarray) -> np.ndarray:
    """float64 -> bf16 bit pattern (uint16), RNE via fp32."""
    x32 = np.ascontiguousarray(x, dtype=np.float64).astype(np.float32)
    u = x32.view(np.uint32).astype(np.uint64)
    lsb = (u >> np.uint64(16)) & np.uint64(1)
    r = ((u + np.uint64(0x7FFF) + lsb) >> np.uint64(16)).astype(np.uint16)
    r = np.where(np.isnan(x32), np.uint16(0x7FC0), r)
    return r


def to_storage(x: np.ndarray, dtype: str) -> np.ndarray:
    """Round float64 data to the storage dtype; returns float64 values."""
    if dtype == "bf16":
        b = _bits_bf16(x).astype(np.uint32) << np.uint32(16)
        return b.view(np.float32).astype(np.float64)
    if dtype == "fp32":
        return np.asarray(x, dtype=np.float64).astype(np.float32).astype(np.float64)
    raise ValueError(dtype)


def storage_bytes(x: np.ndarray, dtype: str) -> np.ndarray:
    """Pack float64 values (already representable) into the storage format:
    uint16 bf16 bit patterns or float32."""
    if dtype == "bf16":
        return _bits_bf16(x)
    if dtype == "fp32":
        return np.asarray(x, dtype=np.float32)
    raise ValueError(dtype)


def gain(act: str) -> float:
    return math.sqrt(2.0) if act == "relu" else 1.0


def weight(d_in: int, d_out: int, act: str, layer: int, seed: int = SEED) -> np.ndarray:
    rng = _rng(seed, 2, layer, 0)
    n, m = max(d_in, d_out), min(d_in, d_out)
    g = rng.standard_normal((n, m))
    q, r = np.linalg.qr(g)
    q = q * np.sign(np.diag(r))[None, :]
    W = q if d_in >= d_out else q.T           # d_in x d_out
    scale = gain(act) * (math.sqrt(d_out / d_in) if d_out > d_in else 1.0)
    return W * scale


def bias(d_out: int, layer: int, seed: int = SEED) -> np.ndarray:
    return 0.1 * _rng(seed, 2, layer, 1).standard_normal(d_out)


def weights(dims, acts, dtype: str, seed: int = SEED):
    """Shared W_i, b_i (already rounded to the storage dtype)."""
    W, b = [], []
    for i in range(len(acts)):
        W.append(to_storage(weight(dims[i], dims[i + 1], acts[i], i + 1, seed), dtype))
        b.append(to_storage(bias(dims[i + 1], i + 1, seed), dtype))
    return W, b


def x_shard(M: int, d0: int, rank: int, dtype: str, seed: int = SEED, step: int = 0) -> np.ndarray:
    return to_storage(_rng(seed, 0, rank, step).standard_normal((M, d0)), dtype)


def dy_shard(M: int, dL: int, rank: int, dtype: str, seed: int = SEED, step: int = 0) -> np.ndarray:
    return to_storage(_rng(seed, 1, rank, step).standard_normal((M, dL)), dtype)


def weights_torch(dims, acts, dtype: str, device, seed: int = SEED):
    """Same recipe as ``weights`` (orthogonal W with gain, b ~ N(0, 0.1^2)),
    generated on the GPU with torch for the full-size bench configs (not
    bit-identical to the NumPy stream; used only where no oracle compares)."""
    import torch
    tdt = {"bf16": torch.bfloat16, "fp32": torch.float32}[dtype]
    g = torch.Generator(device=device)
    W, b = [], []
    for i in range(len(acts)):
        g.manual_seed(seed * 1000 + i)
        d_in, d_out = dims[i], dims[i + 1]
        n, m = max(d_in, d_out), min(d_in, d_out)
        q, r = torch.linalg.qr(torch.randn(n, m, generator=g, device=device, dtype=torch.float32))
        q = q * torch.sign(torch.diagonal(r))[None, :]
        w = q if d_in >= d_out else q.T
        scale = gain(acts[i]) * (math.sqrt(d_out / d_in) if d_out > d_in else 1.0)
        W.append((w * scale).to(tdt).contiguous())
        b.append((0.1 * torch.randn(d_out, generator=g, device=device)).to(tdt).contiguous())
    return W, b


def activations_torch(M: int, d: int, dtype: str, device, seed: int, rank: int, tag: int):
    import torch
    tdt = {"bf16": torch.bfloat16, "fp32": torch.float32}[dtype]
    g = torch.Generator(device=device)
    g.manual_seed(seed * 7919 + rank * 31 + tag)
    return torch.randn(M, d, generator=g, device=device).to(tdt).contiguous()
