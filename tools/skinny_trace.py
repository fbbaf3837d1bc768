"""Per-op latency breakdown of the skinny-stack kernel (debug build
lib/libooo_trace.so, python -m paper_conf_eurosys_ohlks22_b200.build --trace):
    python tools/skinny_trace.py [C5]
For each chain op of one fused step (dO chain, then F chain): mean over its
tiles of hand-off (previous op's last publish -> this tile's A loads
issued), mainloop (A issued -> the leader's accumulator ready), reduction
wait (-> the 7 peers' partials in), epilogue + publish.  A tuning aid."""
import os
import sys

ROOT = __file__.rsplit("/tools/", 1)[0]
os.environ.setdefault("OOO_LIB", os.path.join(ROOT, "paper_conf_eurosys_ohlks22_b200", "lib", "libooo_trace.so"))
sys.path.insert(0, ROOT)

import ctypes  # noqa: E402

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_ohlks22_b200 import _lib, configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402


def main():
    cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C5")
    lib = _lib.load()
    lib.ooo_debug_set_trace.restype = ctypes.c_int32
    lib.ooo_debug_set_trace.argtypes = [ctypes.c_void_p]
    dev = torch.device("cuda")
    W, b = synth.weights_torch(cfg.dims, cfg.acts, cfg.dtype, dev)
    stk = OooStack(cfg.dims, cfg.acts, cfg.tokens, W, b, dtype=cfg.dtype)
    X = synth.activations_torch(cfg.tokens, cfg.dims[0], cfg.dtype, dev, 1, 0, 0)
    dY = synth.activations_torch(cfg.tokens, cfg.dims[-1], cfg.dtype, dev, 1, 0, 1)
    Y = stk.forward(X)
    for _ in range(3):
        stk.backward(dY, "first_k", 0)
        stk.forward(X, Y)
    torch.cuda.synchronize()
    base = 3 * 200000 * 8
    buf = torch.zeros(base + 800 * 32 * 8, dtype=torch.int64, device=dev)
    _lib.check(lib.ooo_debug_set_trace(buf.data_ptr()))
    stk.backward(dY, "first_k", 0)
    stk.forward(X, Y)
    torch.cuda.synchronize()
    _lib.check(lib.ooo_debug_set_trace(None))
    t = buf[base:].cpu().numpy().view(np.uint64).reshape(800, 32, 8).astype(np.float64)
    L = cfg.L
    ops = [("dO", i) for i in range(L, 1, -1)] + [("F", i) for i in range(1, L + 1)]
    t0 = t[t > 0].min()
    t = np.where(t > 0, (t - t0) / 1e3, np.nan)
    prev_pub = 0.0
    rows = []
    for j, (k, i) in enumerate(ops):
        s = t[j]
        ok = ~np.isnan(s[:, 3])
        if not ok.any():
            continue
        s = s[ok]
        a = s[:, 5]
        rows.append((k, i, np.nanmean(a) - prev_pub, np.nanmean(s[:, 1] - a), np.nanmean(s[:, 2] - s[:, 1]),
                     np.nanmean(s[:, 3] - s[:, 2]), np.nanmax(s[:, 3]), np.nanmean(a - s[:, 4]),
                     np.nanmean(s[:, 6] - s[:, 2]), np.nanmean(s[:, 7] - s[:, 6]), np.nanmean(s[:, 3] - s[:, 7])))
        prev_pub = np.nanmax(s[:, 3])
    print(f"{'op':>8} {'handoff':>8} {'main':>7} {'redwait':>8} {'epi+pub':>8} {'done':>9} {'gate->A':>8}"
          f" {'epi':>6} {'dbp+f':>6} {'pub':>6} (us)")
    for r in rows[:8] + rows[L - 4: L + 4] + rows[-4:]:
        print(f"{r[0]:>4}{r[1]:>4} {r[2]:8.2f} {r[3]:7.2f} {r[4]:8.2f} {r[5]:8.2f} {r[6]:9.1f} {r[7]:8.2f}"
              f" {r[8]:6.2f} {r[9]:6.2f} {r[10]:6.2f}")
    arr = np.array([r[2:6] + r[8:11] for r in rows])
    print("mean over ops: handoff %.2f main %.2f redwait %.2f epi+pub %.2f (epi %.2f, dbpart+fence %.2f, reds %.2f) us;"
          " last publish %.1f us" % (*arr.mean(0), rows[-1][6]))


if __name__ == "__main__":
    main()
