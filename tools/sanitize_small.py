"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): the bf16 engine (CTA pairs; 1-CTA tiles with split-K; pairs with
a long-K split) and the skinny cluster kernel, eager (forward, backward +
join) and the captured fused step, the comm-gated step (OOO_TEST_COMM_GATE) and the one-rank NCCL
data plane, plus the fp32 per-layer path.  Engine waits are bounded at
10 min (the sanitizer slows the spin-waiting CTAs by orders of magnitude).

    compute-sanitizer --tool memcheck python tools/sanitize_small.py
"""
import os
import sys

import torch

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
from paper_conf_eurosys_ohlks22_b200 import synth  # noqa: E402
from paper_conf_eurosys_ohlks22_b200.stack import OooStack, get_unique_id  # noqa: E402

TMO = 600000


def tens(a, dt):
    return torch.from_numpy(a).to(dt).cuda().contiguous()


def run(dims, acts, M, dtype, label, **kw):
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    Wn, bn = synth.weights(dims, acts, dtype)
    W, b = [tens(w, tdt) for w in Wn], [tens(x, tdt) for x in bn]
    X = tens(synth.x_shard(M, dims[0], 0, dtype), tdt)
    dY = tens(synth.dy_shard(M, dims[-1], 0, dtype), tdt)
    stk = OooStack(dims, acts, M, W, b, dtype=dtype, bucket_layers=2, wait_timeout_ms=TMO, **kw)
    Y = stk.forward(X)
    stk.backward(dY, "first_k", 2)
    stk.join()
    torch.cuda.synchronize()
    g1 = stk.grads_buf.clone()
    if dtype == "bf16":
        stk.forward(X, Y)
        g = stk.graph(X, Y, dY, "first_k", 2)
        g.launch()
        g.launch()
        torch.cuda.synchronize()
        g.close()
        assert torch.equal(stk.grads_buf, g1), label
    stk.close()
    print("ok", label, flush=True)


dims, acts = [256, 512, 256, 256, 512], ["gelu", "id", "relu", "id"]
run(dims, acts, 264, "bf16", "engine pairs (M=264)")
run(dims, acts, 16, "bf16", "skinny cluster kernel (M=16)")
os.environ["OOO_SKINNY"] = "0"
run(dims, acts, 16, "bf16", "engine 1-CTA tiles, split-K (M=16)")
del os.environ["OOO_SKINNY"]
run([256, 4096, 256], ["gelu", "id"], 264, "bf16", "engine pairs, long-K split (M=264)")
os.environ["OOO_TEST_COMM_GATE"] = "1"
run(dims, acts, 264, "bf16", "comm-gated fused step")
del os.environ["OOO_TEST_COMM_GATE"]
run(dims, acts, 264, "bf16", "one-rank NCCL", unique_id=get_unique_id())
run([256, 256, 256], ["relu", "id"], 32, "fp32", "fp32 SIMT path")
print("sanitize workload done", flush=True)
