"""Run a few eager forward/backward passes of a config (for ncu captures of
the engine kernels): python tools/engine_once.py [C2] [reps] [k | regions]
With k = "regions" the Algorithm 1 plan is made first; the CUDA profiler is
started only after planning (use ncu --profile-from-start off)."""
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
karg = sys.argv[3] if len(sys.argv) > 3 else str(cfg.L // 6)
kind, k = ("regions", 0) if karg == "regions" else ("first_k", int(karg))
dev = torch.device("cuda")
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
Y = stk.forward(X)
if kind == "regions":
    stk.plan_regions(region_layers=6)
    Y = stk.forward(X)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
for _ in range(reps):
    stk.backward(dY, kind, k)
    stk.forward(X, Y)
torch.cuda.synchronize()
print("ok")
