import os, sys, time
sys.path.insert(0, os.getcwd())
os.environ["OOO_EMULATE_AR_N"] = sys.argv[1] if len(sys.argv) > 1 else "8"
os.environ["OOO_EMULATE_AR_GBPS"] = "50"
import torch
from tests.gpu_helpers import Case, to_dev
dims, acts = [256, 512, 256, 256, 512, 256], ["gelu", "id", "id", "gelu", "id"]
M = int(sys.argv[2]) if len(sys.argv) > 2 else 520
bl = int(sys.argv[3]) if len(sys.argv) > 3 else 2
cases = [Case(dims, acts, M, "bf16", step=t) for t in range(3)]
stk = cases[0].stack(bucket_layers=bl)
Xs = [to_dev(c.X, "bf16") for c in cases]
dYs = [to_dev(c.dY, "bf16") for c in cases]
def step(msg):
    t0 = time.time(); torch.cuda.synchronize(); print(msg, "ok", round(time.time() - t0, 3), flush=True)
Y = stk.forward(Xs[0]); step("fwd0")
for t in range(3):
    stk.backward(dYs[t], "first_k", 2); print("bwd enq", t, flush=True)
    if t < 2:
        Y = stk.forward(Xs[t + 1]); step(f"fused {t}")
    else:
        stk.join(); step("join")
print("done")
