"""Workload shapes of BASELINE.json's configs (readings Q6/Q7/Q16).

Pure data: layer widths, activations, tokens per GPU and storage dtype.  No
arithmetic of the method lives here, so both the product path (bench) and the
oracle-side tests may import it.

Reading Q6: a BERT/GPT-shaped block is 6 chained Linear layers
Q, K, V, O (h->h, identity), FFN1 (h->4h, GELU-erf), FFN2 (4h->h, identity);
this matches a transformer block's weight/bias count (12h^2 + 9h) and leaves
out attention maths, LayerNorm and embeddings.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class StackConfig:
    name: str
    dims: tuple          # L+1 widths d_0..d_L
    acts: tuple          # L activations ("id" | "relu" | "gelu")
    tokens: int          # M, rows per GPU per iteration
    dtype: str           # "bf16" | "fp32"
    note: str = ""

    @property
    def L(self) -> int:
        return len(self.acts)

    def params(self) -> int:
        return sum(self.dims[i] * self.dims[i + 1] + self.dims[i + 1] for i in range(self.L))

    def hbm_min_bytes(self, need_input_grad: bool = False) -> int:
        """Compulsory HBM bytes of one step if every op streams its operands
        once (no reuse across ops through L2): F_i reads X_i, W_i and writes
        Z_i (+ X_{i+1} when act_i != id); dO_i reads dZ_i, W_i (+ Z_{i-1} for
        act') and writes dZ_{i-1}; dW_i reads X_i, dZ_i and writes dW_i, db_i."""
        e = 2 if self.dtype == "bf16" else 4
        M, d, a = self.tokens, self.dims, self.acts
        t = 0
        for i in range(self.L):
            din, dout = d[i], d[i + 1]
            t += M * din + din * dout + M * dout * (2 if a[i] != "id" else 1)
            if i > 0 or need_input_grad:
                t += M * dout + din * dout + M * din * (2 if i > 0 and a[i - 1] != "id" else 1)
            t += M * din + M * dout + din * dout + dout
        return t * e

    def gemm_flops(self, need_input_grad: bool = False) -> int:
        """fwd + dX (layers 2..L, plus 1 if requested) + dW, 2*M*din*dout each."""
        M = self.tokens
        f = 0
        for i in range(self.L):
            mnk = 2 * M * self.dims[i] * self.dims[i + 1]
            f += mnk                      # forward
            f += mnk                      # dW
            if i > 0 or need_input_grad:
                f += mnk                  # dX
        return f


def transformer_stack(name: str, blocks: int, h: int, tokens: int, dtype: str = "bf16",
                      note: str = "") -> StackConfig:
    dims = [h]
    acts = []
    for _ in range(blocks):
        for _q in range(4):               # Q, K, V, O
            dims.append(h)
            acts.append("id")
        dims.append(4 * h)                # FFN1
        acts.append("gelu")
        dims.append(h)                    # FFN2
        acts.append("id")
    return StackConfig(name, tuple(dims), tuple(acts), tokens, dtype, note)


def mlp(name: str, layers: int, width: int, tokens: int, hidden_act: str, top_act: str,
        dtype: str, note: str = "") -> StackConfig:
    dims = tuple([width] * (layers + 1))
    acts = tuple([hidden_act] * (layers - 1) + [top_act])
    return StackConfig(name, dims, acts, tokens, dtype, note)


# BASELINE.json "configs", in order.
C1 = mlp("mlp4_w256_b32_fp32", 4, 256, 32, "relu", "id", "fp32",
         "configs[0]: 4-layer MLP width 256, batch 32, fp32, 1 GPU")
C2 = transformer_stack("bert_base_stack", 12, 768, 32 * 128, "bf16",
                       "configs[1]: BERT-base-shaped 12-block linear stack, 32x128 tokens/GPU")
C3 = transformer_stack("bert_large_stack", 24, 1024, 32 * 128, "bf16",
                       "configs[2]: BERT-large-shaped 24-block stack, 32x128 tokens/GPU (Q7)")
C4 = transformer_stack("gpt2_medium_stack", 24, 1024, 1 * 512, "bf16",
                       "configs[3]: GPT-2-medium-shaped 24-block stack, 1x512 tokens/GPU (Q7)")
C5 = mlp("mlp96_w1024_b16", 96, 1024, 16, "gelu", "id", "bf16",
         "configs[4]: 96-layer MLP width 1024, batch 16 (Q16: GELU hidden, identity top)")

CONFIGS = {c.name: c for c in (C1, C2, C3, C4, C5)}
ALIASES = {"C1": C1.name, "C2": C2.name, "C3": C3.name, "C4": C4.name, "C5": C5.name}


def get(name: str) -> StackConfig:
    name = ALIASES.get(name, name)
    return CONFIGS[name]


def scaled(cfg: StackConfig, tokens: int | None = None, blocks_or_layers: int | None = None,
           width_div: int = 1) -> StackConfig:
    """A smaller stack with the same structure (for oracle-sized parity tests)."""
    dims = list(cfg.dims)
    acts = list(cfg.acts)
    if blocks_or_layers is not None:
        acts = acts[:blocks_or_layers]
        dims = dims[:blocks_or_layers + 1]
    dims = [d // width_div for d in dims]
    return StackConfig(cfg.name + "_scaled", tuple(dims), tuple(acts),
                       tokens if tokens is not None else cfg.tokens, cfg.dtype)
