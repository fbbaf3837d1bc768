for v in ""; do
  OOO_LIB=$PWD/paper_conf_eurosys_ohlks22_b200/lib/libooo$v.so timeout 120 python tools/engine_gemm.py 2304x2048x8192 2304x2048x2048 8192x8192x8192 4096x768x768 2>&1 | grep -v Warn | python3 -c "
import sys,json
r=[json.loads(l) for l in sys.stdin if l.startswith('{')]
print('lib$v', [(x['M'],x['N'],x['K'],round(x['ours_us'],1),round(x['ours_tflops']),round(x['cublas_tflops'])) for x in r], 'per-kb us', round((r[0]['ours_us']-r[1]['ours_us'])/96,3))"
done
