"""Library baseline for context: the same training step (backward(t) +
forward(t+1) of a config's layer stack) as a plain sequence of torch/cuBLAS
ops, in-order, captured in one CUDA graph.  Not part of the product path.

    python tools/torch_baseline.py [C2] [reps]
"""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402

cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 30
dev = torch.device("cuda")
dt = torch.bfloat16 if cfg.dtype == "bf16" else torch.float32
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
L = len(W)
acts = cfg.acts


def act(a, z):
    if a == "gelu":
        return torch.nn.functional.gelu(z)
    if a == "relu":
        return torch.relu(z)
    return z


def act_grad(a, z, g):
    if a == "gelu":
        zf = z.float()
        cdf = 0.5 * (1 + torch.erf(zf * 0.7071067811865476))
        pdf = torch.exp(-0.5 * zf * zf) * 0.3989422804014327
        return (g.float() * (cdf + zf * pdf)).to(z.dtype)
    if a == "relu":
        return g * (z > 0)
    return g


Xs, Zs = [None] * (L + 1), [None] * L
dW = [torch.empty_like(w) for w in W]
db = [torch.empty_like(x) for x in b]


def forward():
    x = X
    for i in range(L):
        Xs[i] = x
        z = torch.addmm(b[i], x, W[i])
        Zs[i] = z
        x = act(acts[i], z)
    return x


def backward():
    g = act_grad(acts[L - 1], Zs[L - 1], dY)
    for i in range(L - 1, -1, -1):
        torch.mm(Xs[i].t(), g, out=dW[i])
        db[i].copy_(g.float().sum(0))
        if i > 0:
            g = act_grad(acts[i - 1], Zs[i - 1], g @ W[i].t())


def step():
    backward()
    forward()


forward()
s = torch.cuda.Stream()
s.wait_stream(torch.cuda.current_stream())
with torch.cuda.stream(s):
    for _ in range(3):
        step()
torch.cuda.current_stream().wait_stream(s)
g = torch.cuda.CUDAGraph()
with torch.cuda.graph(g):
    step()
for _ in range(5):
    g.replay()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
for _ in range(reps):
    g.replay()
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
print(json.dumps({"config": cfg.name, "impl": "torch/cuBLAS in-order, CUDA graph", "ms_per_step": ms,
                  "iters_per_s": 1e3 / ms}))
