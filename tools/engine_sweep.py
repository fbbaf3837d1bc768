"""Time one captured training step under different library knobs (env vars
read at ooo_create_stack): OOO_EBN, OOO_ENGINE_CTAS, OOO_SPLITK, OOO_CG, ...

    python tools/engine_sweep.py C2 "" "OOO_EBN=128" "OOO_ENGINE_CTAS=132"
A tuning aid, not part of the product path.
"""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
variants = sys.argv[2:] or [""]
dev = torch.device("cuda")
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
base_env = dict(os.environ)
for v in variants:
    os.environ.clear()
    os.environ.update(base_env)
    for kv in v.split(","):
        if "=" in kv:
            k_, val = kv.split("=", 1)
            os.environ[k_] = val
    res = {"variant": v}
    stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
    Y = stk.forward(X)
    for kind, k in (("first_k", cfg.L // 6), ("in_order", 0)):
        g = stk.graph(X, Y, dY, kind, k)
        for _ in range(5):
            g.launch()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        e0.record()
        for _ in range(30):
            g.launch()
        e1.record()
        torch.cuda.synchronize()
        res[kind] = e0.elapsed_time(e1) / 30
        g.close()
    stk.close()
    print(json.dumps(res), flush=True)
