"""Run a few eager forward/backward passes of a config (for ncu captures of
the engine kernels): python tools/engine_once.py [C2] [reps] [k]"""
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
k = int(sys.argv[3]) if len(sys.argv) > 3 else cfg.L // 6
dev = torch.device("cuda")
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
Y = stk.forward(X)
for _ in range(reps):
    stk.backward(dY, "first_k", k)
    stk.forward(X, Y)
torch.cuda.synchronize()
print("ok")
