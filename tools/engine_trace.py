"""Per-task timeline of the persistent engine (debug build libooo_trace.so).

    python -m paper_conf_eurosys_ohlks22_b200.build --trace
    python tools/engine_trace.py [C2] [k]

For each op of the backward-alone, forward-alone and fused-step queues: number of tiles, time from
the pass start to its first dispense / first input-ready / last completion,
mean per-tile durations (dispense->ready = dependency wait, ready->acc =
mainloop, acc->done = epilogue) and the number of distinct CTAs.  A tuning
aid, not part of the product path.
"""
import os
import sys

ROOT = __file__.rsplit("/tools/", 1)[0]
os.environ.setdefault("OOO_LIB", os.path.join(ROOT, "paper_conf_eurosys_ohlks22_b200", "lib", "libooo_trace.so"))
sys.path.insert(0, ROOT)

import ctypes  # noqa: E402

import torch  # noqa: E402

from paper_conf_eurosys_ohlks22_b200 import _lib, configs, synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack, schedule_order  # noqa: E402


KIND = {0: "F", 1: "dX", 2: "dW", 3: "cp"}


def last_queue(lib, stk):
    """(kind, layer, ntiles) of the most recent engine launch (debug export)."""
    lib.ooo_debug_last_queue.restype = ctypes.c_int32
    lib.ooo_debug_last_queue.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32]
    buf = (ctypes.c_int32 * (5 * 1024))()
    n = lib.ooo_debug_last_queue(stk._h, buf, 1024)
    return [(KIND[buf[5 * j]], buf[5 * j + 1], buf[5 * j + 3] * buf[5 * j + 4], buf[5 * j + 2], buf[5 * j + 4])
            for j in range(n)]


def report(name, ops, buf):
    import numpy as np
    allb = buf.cpu().numpy().view(np.uint64)
    out = os.path.join(ROOT, "gpurun_out", "trace_" + name.split()[0] + "_" + name.split()[1] + ".npz")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    np.savez_compressed(out, raw=allb[: 3 * 200000 * 8], ops=np.array([list(o) for o in ops], dtype=object))
    raw8 = allb[: 200000 * 8].reshape(-1, 8)
    epi = allb[200000 * 8: 2 * 200000 * 8].reshape(-1, 8).astype(np.float64)   # epilogue phase clocks
    raw = raw8[:, :4]
    clk = raw8[:, 4:].astype(np.float64)
    cta = (raw >> np.uint64(48)).astype(np.int64)
    t = (raw & np.uint64((1 << 48) - 1)).astype(np.float64)
    valid = t[:, 3] > 0
    t0 = t[t[:, 0] > 0, 0].min()
    t = (t - t0) / 1e3
    # SM clock: cycles between "ready" and "acc ready" over the same interval in ns
    dc = clk[valid, 2] - clk[valid, 1]
    dt = (t[valid, 2] - t[valid, 1])
    ok = dt > 1.0
    mhz = np.median(dc[ok] / (dt[ok] * 1e3) * 1e3) if ok.any() else float("nan")
    print(f"== {name}: {int(valid.sum())} tasks, span {t[valid, 3].max():.1f} us, SM clock ~{mhz:.0f} MHz")
    first = 0
    for kind, layer, n, *_ in ops:
        s = slice(first, first + n)
        first += n
        tt = t[s]
        dn = raw[s, 3] > 0                       # split-K: only the last split of a tile publishes
        td = tt[dn] if dn.any() else tt
        print(f"{kind} L{layer:3d} tiles {n:4d} disp {tt[:,0].min():8.1f} ready {tt[:,1].min():8.1f}"
              f"..{tt[:,1].max():8.1f} done {td[:,3].min():8.1f}..{td[:,3].max():8.1f}"
              f" wait {np.mean(tt[:,1]-tt[:,0]):6.1f} main {np.mean(tt[:,2]-tt[:,1]):6.1f}"
              f" epi {np.mean(td[:,3]-td[:,2]):5.1f} published {int(dn.sum())} ctas {len(set(cta[s, 3]))}")
        g = allb[2 * 200000 * 8:].reshape(-1, 8)[s]
        if g[:, 7].max() > 0:
            m48 = np.uint64((1 << 48) - 1)
            f6 = ((g[:, 6] & m48).astype(np.float64) - t0) / 1e3
            f7 = ((g[:, 7] & m48).astype(np.float64) - t0) / 1e3
            ok = g[:, 7] > 0
            print(f"     loads: first {np.mean(f6[ok] - tt[ok, 1]):6.1f} after ready, last {np.mean(f7[ok] - tt[ok, 1]):6.1f};"
                  f" acc {np.mean(tt[ok, 2] - f7[ok]):6.1f} after last; last-load range {f7[ok].min():8.1f}..{f7[ok].max():8.1f}")
        e = epi[s]
        sk = dn & (e[:, 7] > 0)                  # split-K last arrivals: phase A, arrival, reduction + epilogue
        if sk.any():
            es = e[sk]
            print(f"     split-K cycles: partial store {np.median(es[:, 6] - es[:, 0]):6.0f} arrival"
                  f" {np.median(es[:, 7] - es[:, 6]):6.0f} reduce+epilogue {np.median(es[:, 3] - es[:, 7]):6.0f}"
                  f" publish {np.median(es[:, 5] - es[:, 3]):6.0f}")
        elif e[:, 5].max() > 0:
            d = lambda a, b: np.median(e[:, b] - e[:, a])  # noqa: E731
            print(f"     epi cycles: tmem_ld {d(0, 1):6.0f} chunk0 {d(1, 2):6.0f} loop {d(0, 3):6.0f}"
                  f" tail {d(3, 4):6.0f} bar {d(4, 5):6.0f}")


def main():
    cfg = configs.get(sys.argv[1] if len(sys.argv) > 1 else "C2")
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 12
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
        stk.backward(dY, "first_k", k)
        stk.forward(X, Y)
    torch.cuda.synchronize()
    buf = torch.zeros(3 * 200000 * 8, dtype=torch.int64, device=dev)
    _lib.check(lib.ooo_debug_set_trace(buf.data_ptr()))
    stk.backward(dY, "first_k", k)
    stk.join()
    torch.cuda.synchronize()
    report(f"backward first_k({k}) alone", last_queue(lib, stk), buf)
    buf.zero_()
    stk.forward(X, Y)
    torch.cuda.synchronize()
    report("forward alone", last_queue(lib, stk), buf)
    buf.zero_()
    stk.backward(dY, "first_k", k)
    stk.forward(X, Y)
    torch.cuda.synchronize()
    report(f"fused step first_k({k})", last_queue(lib, stk), buf)
    _lib.check(lib.ooo_debug_set_trace(None))


if __name__ == "__main__":
    main()
