"""Data-parallel exposed communication on ONE GPU with an emulated all-reduce
(measurement aid; no NCCL): each bucket's S[dW_i] holds the comm stream for
the ring all-reduce time 2(n-1)/n x bytes / BW + latency (OOO_EMULATE_AR_*),
the engine keeps the 16-SM NCCL reserve, and F_i waits for its bucket's flag
exactly as at N = n.  Exposed = T(step) - T(same step, zero-time comm);
hidden = 1 - exposed / sum of the bucket times.

    python tools/emulated_dp.py C3 [n ...] [--k 0,6,24,144]
"""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

GBPS, LAT_US = 900.0, 8.0


def timed(g, stream, steps=20, reps=3):
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


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    cfg = configs.get(args[0] if args else "C3")
    ns = [int(a) for a in args[1:]] or [8]
    ks = [0, cfg.L // 24, cfg.L // 6, cfg.L // 2, cfg.L]
    for a in sys.argv[1:]:
        if a.startswith("--k="):
            ks = [int(x) for x in a[4:].split(",")]
    dev = torch.device("cuda")
    stream = torch.cuda.current_stream()
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    elt = 2
    for n in ns:
        res = {"config": cfg.name, "emulated_n": n, "link_GBps": GBPS, "latency_us": LAT_US}
        buckets = []
        for i in range(cfg.L):
            nb = (cfg.dims[i] * cfg.dims[i + 1] + cfg.dims[i + 1]) * elt
            buckets.append(2.0 * (n - 1) / n * nb / (GBPS * 1e9) * 1e3 + LAT_US * 1e-3)
        res["allreduce_total_ms"] = sum(buckets)
        times = {}
        for label, gbps, lat in (("on", GBPS, LAT_US), ("off", 1e9, 0.0)):
            os.environ.update({"OOO_EMULATE_AR_N": str(n), "OOO_EMULATE_AR_GBPS": str(gbps),
                               "OOO_EMULATE_AR_LAT_US": str(lat)})
            stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
            Y = stk.forward(X)
            for kind, k in [("in_order", 0)] + [("first_k", k) for k in ks]:
                g = stk.graph(X, Y, dY, kind, k)
                times[(label, kind, k)] = timed(g, stream)
                g.close()
            stk.close()
        for key in ("OOO_EMULATE_AR_N", "OOO_EMULATE_AR_GBPS", "OOO_EMULATE_AR_LAT_US"):
            os.environ.pop(key, None)
        rows = {}
        for kind, k in [("in_order", 0)] + [("first_k", k) for k in ks]:
            on, off = times[("on", kind, k)], times[("off", kind, k)]
            exp = max(0.0, on - off)
            rows[f"{kind}({k})"] = {"ms": round(on, 4), "ms_comm_off": round(off, 4), "exposed_ms": round(exp, 4),
                                    "hidden_fraction": round(1.0 - exp / res["allreduce_total_ms"], 4)}
        res["schedules"] = rows
        best = min((v["ms"], s) for s, v in rows.items() if s.startswith("first_k"))
        res["best_ooo"] = best[1]
        res["ooo_speedup_vs_in_order"] = round(rows["in_order(0)"]["ms"] / best[0], 4)
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
