"""Microbenchmark of the library's forward GEMM kernel in isolation.

A 1-layer identity stack [K -> N] with M tokens: ooo_forward = one copy of X
(M x K) + one tcgen05 GEMM (+bias).  Timed with the library's per-launch
events (the GEMM alone) and compared with torch.matmul (cuBLAS) on the same
shape.  Not part of the product path; a tuning aid.
"""
import json
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200.stack import OooStack  # noqa: E402

shapes = [(8192, 8192, 8192), (4096, 3072, 768), (4096, 768, 768), (4096, 768, 3072),
          (4096, 4096, 1024), (4096, 1024, 1024), (4096, 1024, 4096)]
if len(sys.argv) > 1:
    shapes = [tuple(int(x) for x in s.split("x")) for s in sys.argv[1:]]
dev = torch.device("cuda")
out = []
for (M, N, K) in shapes:
    W = [(torch.randn(K, N, device=dev) / K ** 0.5).to(torch.bfloat16)]
    b = [torch.zeros(N, device=dev, dtype=torch.bfloat16)]
    X = torch.randn(M, K, device=dev).to(torch.bfloat16)
    stk = OooStack([K, N], ["id"], M, W, b, dtype="bf16")
    Y = stk.forward(X)
    stk.set_timing(True)
    reps = 20
    ms = []
    for _ in range(reps):
        stk.set_timing(True)
        stk.forward(X, Y)
        torch.cuda.synchronize()
        recs = [r for r in stk.timing() if r["kind"] == "fwd_gemm"]
        ms.append(recs[0]["ms"])
    ms = sorted(ms)[reps // 2]
    ref = (X.float() @ W[0].float()).to(torch.bfloat16)
    err = ((Y.float() - ref.float()).norm() / ref.float().norm()).item()
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
    r = {"M": M, "N": N, "K": K, "ours_us": ms * 1e3, "ours_tflops": fl / ms / 1e9,
         "cublas_us": cub * 1e3, "cublas_tflops": fl / cub / 1e9, "rel_err": err}
    print(json.dumps(r), flush=True)
    stk.close()
