"""Device time of forward-only launches and of forward + backward-alone
(unfused: each joined) launch pairs of a config,
for the variants given as environment settings (A/B of library knobs):
    python tools/fwd_time.py C5 "" "OOO_SKINNY=0"
A tuning aid, not part of the product path."""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402


def main():
    cfg = configs.get(sys.argv[1])
    dev = torch.device("cuda")
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    base = dict(os.environ)
    res = {}
    for v in sys.argv[2:] or [""]:
        os.environ.clear()
        os.environ.update(base)
        for kv in v.split(","):
            if "=" in kv:
                k, val = kv.split("=", 1)
                os.environ[k] = val
        stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
        Y = stk.forward(X)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        out = {}
        for name, fn in (("forward", lambda: stk.forward(X, Y)),
                         ("backward", lambda: (stk.forward(X, Y), stk.join(), stk.backward(dY, "first_k", 0),
                                               stk.join()))):
            for _ in range(3):
                fn()
            torch.cuda.synchronize()
            e0.record()
            for _ in range(20):
                fn()
            e1.record()
            torch.cuda.synchronize()
            out[name] = round(e0.elapsed_time(e1) / 20, 4)
        res[v or "default"] = out
        stk.close()
    print(json.dumps({"config": cfg.name, "ms": res}))


if __name__ == "__main__":
    main()
