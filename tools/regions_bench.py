"""Single-GPU multi-stream ooo with Algorithm 1 regions (§4.1) vs reverse
first-k and in-order, one captured step each (tuning / evidence tool).

    python tools/regions_bench.py C2 [region_layers ...] [--reps=N]
Prints one JSON line per config: profiling (planning) time, plan summary and
ms/step of regions / first_k(k) / in_order.
"""
import json
import sys
import time

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402


def timed(g, stream, steps=30, reps=3):
    for _ in range(3):
        g.launch(stream)
    best = 1e9
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(steps):
            g.launch(stream)
        e1.record(stream)
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) / steps)
    return best


cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
rls = [int(a) for a in sys.argv[2:] if not a.startswith("--")] or [6]
REPS = next((int(a[7:]) for a in sys.argv[2:] if a.startswith("--reps=")), 1)
dev = torch.device("cuda")
stream = torch.cuda.current_stream()
W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
Y = stk.forward(X)
res = {"config": cfg.name}
for kind, k in (("in_order", 0), ("first_k", 0), ("first_k", cfg.L // 6)):
    g = stk.graph(X, Y, dY, kind, k)
    res[f"{kind}({k})_ms"] = timed(g, stream)
    g.close()
for rl in rls:
    t0 = time.time()
    plan = stk.plan_regions(region_layers=rl, reps=REPS)
    t_plan = time.time() - t0
    stk.forward(X, Y)
    g = stk.graph(X, Y, dY, "regions", 0)
    res[f"regions(rl={rl})"] = {"ms": timed(g, stream), "plan_s": t_plan, "n_regions": plan["n_regions"],
                                 "k_pre": plan["k_pre"], "region_of": plan["region_of"],
                                 "t_main_ms": [round(t, 4) for t in plan["t_main_ms"]]}
    g.close()
print(json.dumps(res), flush=True)
