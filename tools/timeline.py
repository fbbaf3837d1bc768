"""Per-launch timeline of one captured training step (library CUDA events).

    python tools/timeline.py [config] [k] [schedule]
Prints each launch (stream, kind, layer, start, duration) of the last replay
and per-stream busy time; a tuning aid, not part of the product path.
"""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
k = int(sys.argv[2]) if len(sys.argv) > 2 else 12
kind = sys.argv[3] if len(sys.argv) > 3 else "first_k"
dev = torch.device("cuda")
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
Y = stk.forward(X)
stk.set_timing(True)
g = stk.graph(X, Y, dY, kind, k)
for _ in range(5):
    g.launch()
torch.cuda.synchronize()
recs = stk.timing()
busy = {}
end = 0.0
for r in recs:
    busy[r["stream"]] = busy.get(r["stream"], 0.0) + r["ms"]
    end = max(end, r["start_ms"] + r["ms"])
    print(f"s{r['stream']} {r['kind']:9s} L{r['layer']:3d} start {r['start_ms']*1e3:9.1f}us dur {r['ms']*1e3:7.1f}us grid {r['grid']}")
print(json.dumps({"span_ms": end, "busy_ms": busy}))
