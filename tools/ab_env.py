"""A/B of library knobs (environment variables read at stack creation /
graph capture) on one box, all graphs timed in interleaved runs:
    python tools/ab_env.py C4 "" "OOO_SPLITK_LONGK=0" "OOO_EBN=128" [...]
Prints ms per step of first_k(0) and in_order for each variant.  A tuning
aid, not part of the product path."""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402


def main():
    cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
    variants = sys.argv[2:] or [""]
    dev = torch.device("cuda")
    stream = torch.cuda.current_stream()
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    base = dict(os.environ)
    graphs, keys, stacks = [], [], []
    for v in variants:
        for kv in v.split(","):
            if "=" in kv:
                k, val = kv.split("=", 1)
                os.environ[k] = val
        stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype, bucket_layers=6)
        stacks.append(stk)
        Y = stk.forward(X)
        for kind, k in (("first_k", 0), ("in_order", 0)):
            graphs.append(stk.graph(X, Y, dY, kind, k))
            keys.append((v, kind))
        os.environ.clear()
        os.environ.update(base)
    for g in graphs:
        for _ in range(3):
            g.launch(stream)
    ev = [[] for _ in graphs]
    torch.cuda.synchronize()
    for _ in range(4):
        for j, g in enumerate(graphs):
            a, e = torch.cuda.Event(True), torch.cuda.Event(True)
            a.record(stream)
            for _ in range(20):
                g.launch(stream)
            e.record(stream)
            ev[j].append((a, e))
    torch.cuda.synchronize()
    res = {}
    for (v, kind), e in zip(keys, ev):
        res.setdefault(v or "default", {})[kind] = round(sum(a.elapsed_time(b) for a, b in e) / (20 * len(e)), 4)
    print(json.dumps({"config": cfg.name, "ms": res}), flush=True)


if __name__ == "__main__":
    main()
