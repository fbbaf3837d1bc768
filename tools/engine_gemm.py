"""Throughput of the engine's forward pass on single-layer stacks (one GEMM
per pass) vs torch.matmul (cuBLAS) -- isolates the engine mainloop/epilogue
from the layer-chain dependencies.  python tools/engine_gemm.py [MxNxK ...]
The first forward runs normally and fills the X_1 store with the real X; the
timed forwards then run with OOO_DBG=8 (the engine skips its X -> X_1 copy
task, which would otherwise add an M x K copy to the GEMM time) on that same,
real X_1, and Y of the last timed pass is checked against an fp32 matmul
(rel_err): a number with rel_err > 1e-2 is not a measurement."""
import json
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

shapes = [(8192, 8192, 8192), (4096, 3072, 768), (4096, 768, 3072), (4096, 768, 768), (16384, 4096, 4096)]
if len(sys.argv) > 1:
    shapes = [tuple(int(x) for x in s.split("x")) for s in sys.argv[1:]]
dev = torch.device("cuda")
for (M, N, K) in shapes:
    W = [(torch.randn(K, N, device=dev) / K ** 0.5).to(torch.bfloat16)]
    b = [torch.zeros(N, device=dev, dtype=torch.bfloat16)]
    X = torch.randn(M, K, device=dev).to(torch.bfloat16)
    stk = OooStack([K, N], ["id"], M, W, b, dtype="bf16")
    Y = stk.forward(X)                 # real copy: X_1 = X
    torch.cuda.synchronize()
    os.environ["OOO_DBG"] = str(int(os.environ.get("OOO_DBG", "0")) | 8)
    for _ in range(3):
        stk.forward(X, Y)
    reps = 10
    stk.set_timing(True)
    ms = []
    for _ in range(reps):
        stk.set_timing(True)
        stk.forward(X, Y)
        torch.cuda.synchronize()
        ms += [r["ms"] for r in stk.timing() if r["kind"] in ("engine_fwd", "fwd_gemm")]
    ms = sorted(ms)[len(ms) // 2]
    del os.environ["OOO_DBG"]
    ref = (X.float() @ W[0].float())
    err = ((Y.float() - ref).norm() / ref.norm()).item()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    for _ in range(3):
        torch.matmul(X, W[0])
    e0.record()
    for _ in range(reps):
        torch.matmul(X, W[0])
    e1.record()
    torch.cuda.synchronize()
    cub = e0.elapsed_time(e1) / reps
    fl = 2.0 * M * N * K
    print(json.dumps({"M": M, "N": N, "K": K, "ours_us": ms * 1e3, "ours_tflops": fl / ms / 1e9,
                      "cublas_us": cub * 1e3, "cublas_tflops": fl / cub / 1e9, "rel_err": err}), flush=True)
    stk.close()
