"""Mainloop rate per operand-layout kind on equal-size GEMMs (trace build):
a [D, D, D] stack with M tokens -> F (A K-major, B MN-major), dX (K, K),
dW (MN, MN).  Prints us per 64-deep k-block (ready -> accumulator ready)."""
import os
import sys

ROOT = __file__.rsplit("/tools/", 1)[0]
os.environ.setdefault("OOO_LIB", os.path.join(ROOT, "paper_conf_eurosys_ohlks22_b200", "lib", "libooo_trace.so"))
sys.path.insert(0, ROOT)
import ctypes  # noqa: E402

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_eurosys_ohlks22_b200 import _lib  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

D = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
M = int(sys.argv[2]) if len(sys.argv) > 2 else 8192
lib = _lib.load()
lib.ooo_debug_set_trace.argtypes = [ctypes.c_void_p]
dev = torch.device("cuda")
W = [(torch.randn(D, D, device=dev) / D ** 0.5).to(torch.bfloat16) for _ in range(2)]
b = [torch.zeros(D, device=dev, dtype=torch.bfloat16) for _ in range(2)]
X = torch.randn(M, D, device=dev).to(torch.bfloat16)
dY = torch.randn(M, D, device=dev).to(torch.bfloat16)
stk = OooStack([D, D, D], ["id", "id"], M, W, b)
Y = stk.forward(X)
stk.backward(dY, "in_order", 0)
stk.forward(X, Y)
torch.cuda.synchronize()
buf = torch.zeros(100000 * 8, dtype=torch.int64, device=dev)


def stats(name, sl, nkb):
    raw = buf.cpu().numpy().view(np.uint64).reshape(-1, 8)[sl]
    t = (raw[:, :4] & np.uint64((1 << 48) - 1)).astype(np.float64) / 1e3
    c = raw[:, 4:].astype(np.float64)
    main = t[:, 2] - t[:, 1]
    mhz = np.median((c[:, 2] - c[:, 1]) / np.maximum(main, 1e-3))
    print(f"{name:4s} tiles {len(main):5d}  main/kb {np.median(main) / nkb:.3f} us  clock {mhz:.0f} MHz")


CG = int(os.environ.get("OOO_CG", "2"))
pairs_m = ((M + 127) // 128 + CG - 1) // CG
nt = D // 256
nkb = D // 64
lib.ooo_debug_set_trace(buf.data_ptr())
stk.backward(dY, "in_order", 0)        # queue: dO_2, dW_2, dW_1
torch.cuda.synchronize()
n_dx = pairs_m * nt
n_dw = (((D + 127) // 128 + CG - 1) // CG) * nt
stats("dX", slice(0, n_dx), nkb)
stats("dW", slice(n_dx, n_dx + n_dw), M // 64)
buf.zero_()
stk.forward(X, Y)
torch.cuda.synchronize()
stats("F", slice(0, pairs_m * nt), nkb)
lib.ooo_debug_set_trace(None)
