"""Data-parallel exposed communication on ONE GPU with an emulated all-reduce
(measurement aid; no NCCL): each bucket's S[dW_i] holds the comm stream for
the ring all-reduce time 2(n-1)/n x bytes / BW + latency (OOO_EMULATE_AR_*),
the engine keeps the 16-SM NCCL reserve, and F_i waits for its bucket's flag
exactly as at N = n.  Exposed = T(step) - T(same step, zero-time comm);
hidden = 1 - exposed / sum of the bucket times.

    python tools/emulated_dp.py C3 [n ...] [--k=0,6,24,144] [--bucket-layers=1] [--chunk-mb=4]

Each schedule is timed with the FIFO issue order and with the prioritised,
partitioned order (NEXT-4, Fig. 4(b): chunks of --chunk-mb MB, lowest
layer first); every graph is timed in interleaved runs (drift hits all alike).
"""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

GBPS, LAT_US = 900.0, 8.0


def interleaved(graphs, stream, steps=20, reps=3):
    for g in graphs:
        for _ in range(3):
            g.launch(stream)
    out = [[] for _ in graphs]
    torch.cuda.synchronize()
    for _ in range(reps):
        for j, g in enumerate(graphs):
            e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
            e0.record(stream)
            for _ in range(steps):
                g.launch(stream)
            e1.record(stream)
            out[j].append((e0, e1))
    torch.cuda.synchronize()
    return [sum(a.elapsed_time(b) for a, b in ev) / (steps * len(ev)) for ev in out]


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    cfg = configs.get(args[0] if args else "C3")
    ns = [int(a) for a in args[1:]] or [8]
    ks = [0, cfg.L // 24, cfg.L // 6, cfg.L // 2, cfg.L]
    bl, chunk_mb = 1, 4.0
    for a in sys.argv[1:]:
        if a.startswith("--k="):
            ks = [int(x) for x in a[4:].split(",")]
        if a.startswith("--bucket-layers="):
            bl = int(a.split("=", 1)[1])
        if a.startswith("--chunk-mb="):
            chunk_mb = float(a.split("=", 1)[1])
    dev = torch.device("cuda")
    stream = torch.cuda.current_stream()
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, synth.SEED, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, synth.SEED, 0, 1)
    elt = 2
    for n in ns:
        res = {"config": cfg.name, "emulated_n": n, "link_GBps": GBPS, "latency_us": LAT_US, "bucket_layers": bl,
               "chunk_mb": chunk_mb}
        nbk = (cfg.L + bl - 1) // bl
        res["allreduce_total_ms"] = sum(2.0 * (n - 1) / n * (cfg.dims[i] * cfg.dims[i + 1] + cfg.dims[i + 1]) * elt
                                        / (GBPS * 1e9) * 1e3 for i in range(cfg.L)) + nbk * LAT_US * 1e-3
        scheds = [("in_order", 0)] + [("first_k", k) for k in ks]
        graphs, keys, stacks = [], [], []
        for label, gbps, lat, pr in (("fifo", GBPS, LAT_US, 0), ("prio", GBPS, LAT_US, 1), ("off", 1e9, 0.0, 0)):
            os.environ.update({"OOO_EMULATE_AR_N": str(n), "OOO_EMULATE_AR_GBPS": str(gbps),
                               "OOO_EMULATE_AR_LAT_US": str(lat)})
            stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype, bucket_layers=bl,
                           comm_priority=pr, comm_chunk_bytes=int(chunk_mb * 2 ** 20) if pr else 0)
            stacks.append(stk)
            Y = stk.forward(X)
            for kind, k in scheds:
                graphs.append(stk.graph(X, Y, dY, kind, k))
                keys.append((label, kind, k))
        for key in ("OOO_EMULATE_AR_N", "OOO_EMULATE_AR_GBPS", "OOO_EMULATE_AR_LAT_US"):
            os.environ.pop(key, None)
        times = dict(zip(keys, interleaved(graphs, stream)))
        for g in graphs:
            g.close()
        for stk in stacks:
            stk.close()
        rows = {}
        for kind, k in scheds:
            off = times[("off", kind, k)]
            for label in ("fifo", "prio"):
                on = times[(label, kind, k)]
                exp = max(0.0, on - off)
                rows[f"{kind}({k}){'' if label == 'fifo' else '+prio'}"] = {
                    "ms": round(on, 4), "ms_comm_off": round(off, 4), "exposed_ms": round(exp, 4),
                    "hidden_fraction": round(1.0 - exp / res["allreduce_total_ms"], 4)}
        res["schedules"] = rows
        best = min((v["ms"], s) for s, v in rows.items() if s.startswith("first_k") and "+prio" not in s)
        bestp = min((v["ms"], s) for s, v in rows.items() if "+prio" in s)
        res["best_ooo"] = best[1]
        res["best_prioritised"] = bestp[1]
        res["ooo_speedup_vs_in_order"] = round(rows["in_order(0)"]["ms"] / best[0], 4)
        res["prioritised_speedup_vs_fifo_best"] = round(best[0] / bestp[0], 4)
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
