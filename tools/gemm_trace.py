"""Per-tile pipeline stamps of one isolated engine GEMM (debug build):
    python tools/gemm_trace.py MxNxK"""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
os.environ.setdefault("OOO_LIB", os.path.join(ROOT, "paper_conf_eurosys_ohlks22_b200", "lib", "libooo_trace.so"))
os.environ["OOO_DBG"] = str(int(os.environ.get("OOO_DBG", "0")) | 8)
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_ohlks22_b200 import _lib  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

M, N, K = (int(x) for x in sys.argv[1].split("x"))
dev = torch.device("cuda")
W = [(torch.randn(K, N, device=dev) / K ** 0.5).to(torch.bfloat16)]
b = [torch.zeros(N, device=dev, dtype=torch.bfloat16)]
X = torch.randn(M, K, device=dev).to(torch.bfloat16)
stk = OooStack([K, N], ["id"], M, W, b, dtype="bf16")
Y = stk.forward(X)
for _ in range(3):
    stk.forward(X, Y)
torch.cuda.synchronize()
lib = _lib.load()
lib.ooo_debug_set_trace.restype = ctypes.c_int32
lib.ooo_debug_set_trace.argtypes = [ctypes.c_void_p]
buf = torch.zeros(3 * 200000 * 8, dtype=torch.int64, device=dev)
_lib.check(lib.ooo_debug_set_trace(buf.data_ptr()))
e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
e0.record()
stk.forward(X, Y)
e1.record()
torch.cuda.synchronize()
_lib.check(lib.ooo_debug_set_trace(None))
a = buf.cpu().numpy().view(np.uint64)
m48 = np.uint64((1 << 48) - 1)
r8 = a[: 200000 * 8].reshape(-1, 8)
e3 = a[2 * 200000 * 8:].reshape(-1, 8)
t = (r8[:, :4] & m48).astype(np.float64)
v = t[:, 3] > 0
n = int(v.sum())
t0 = t[v, 0].min()
t = (t[:n] - t0) / 1e3
g = ((e3[:n] & m48).astype(np.float64) - t0) / 1e3
nkb = (K + 63) // 64
print(f"{M}x{N}x{K}: {n} tiles, launch (events) {e0.elapsed_time(e1) * 1e3:.1f} us, tiles span {t[:, 3].max():.1f} us")
for name, x in [("dispatch", t[:, 0]), ("ready", t[:, 1]), ("accfree", g[:, 4]), ("first load", g[:, 6]),
                ("last load", g[:, 7]), ("mma end", g[:, 5]), ("acc ready", t[:, 2]), ("done", t[:, 3])]:
    print(f"  {name:10s} min {x.min():8.1f} med {np.median(x):8.1f} max {x.max():8.1f}")
print(f"  per k-block (first->last load)/(nkb-1): {np.median((g[:, 7] - g[:, 6]) / max(1, nkb - 1)):.3f} us;"
      f" mma end - first load: {np.median(g[:, 5] - g[:, 6]):.1f} us for {nkb} k-blocks")
k = e3.reshape(-1, 8) if False else a[2 * 200000 * 8:].reshape(-1, 8)[150000:150000 + nkb].astype(np.float64)
if k[:, 0].max() > 0:
    base = k[0, 0]
    print("  kb  prod-after-empty  mma-wait-start  mma-data-ready   (cycles rel. to kb0 issue; CTA 0)")
    for i in list(range(0, min(nkb, 12))) + list(range(max(12, nkb - 6), nkb)):
        print(f"  {i:3d} {k[i, 0] - base:10.0f} {k[i, 2] - base:10.0f} {k[i, 3] - base:10.0f}")
    d = np.diff(k[:, 3])
    print(f"  median cycles between MMA data-ready of consecutive k-blocks: {np.median(d):.0f}")
    lat = k[6:, 3] - k[6:, 0]
    print(f"  median cycles producer issue -> data ready (same kb): {np.median(k[:, 3] - k[:, 0]):.0f}")
stk.close()
