"""k sweep of ooo_first_k(k) against in_order on one GPU (SURVEY §8d asks for
the C3 k curve).  Times one captured training step per k (seed + one fused
engine launch) with CUDA events and prints a markdown table.

    python tools/ksweep.py C3 0,1,2,3,4,6,8,12,18,24,36,48,72,96,120,144 [steps]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402


def main():
    cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C3")
    ks = [int(k) for k in (sys.argv[2] if len(sys.argv) > 2 else "0,1,2,4,8,16").split(",")]
    steps = int(sys.argv[3]) if len(sys.argv) > 3 else 30
    dev = torch.device("cuda")
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
    stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
    Y = stk.forward(X)
    st = torch.cuda.current_stream()

    def time_graph(kind, k):
        g = stk.graph(X, Y, dY, kind, k)
        for _ in range(5):
            g.launch(st)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        best = float("inf")
        for _ in range(3):
            e0.record(st)
            for _ in range(steps):
                g.launch(st)
            e1.record(st)
            torch.cuda.synchronize()
            best = min(best, e0.elapsed_time(e1) / steps)
        g.close()
        return best

    ms_in = time_graph("in_order", 0)
    print(f"# k sweep, {cfg.name} (L = {cfg.L}, M = {cfg.tokens}), 1 B200, best of 3 x {steps} steps\n")
    print(f"in_order: {ms_in:.3f} ms/step ({1e3 / ms_in:.1f} it/s)\n")
    print("| k | ms/step | it/s | speedup vs in_order |\n|---|---|---|---|")
    for k in ks:
        if k > cfg.L:
            continue
        ms = time_graph("first_k", k)
        print(f"| {k} | {ms:.3f} | {1e3 / ms:.1f} | {ms_in / ms:.3f} |")
    stk.close()


if __name__ == "__main__":
    main()
