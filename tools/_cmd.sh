for cg in 1 2; do OOO_CG=$cg timeout 120 python tools/engine_gemm.py 8192x8192x8192 4096x768x3072 2>&1 | tail -2; done
