for v in _s0 _s64 _s256; do
  OOO_LIB=$PWD/paper_conf_eurosys_ohlks22_b200/lib/libooo$v.so timeout 120 python tools/engine_gemm.py 2304x2048x8192 2304x2048x2048 2>&1 | grep -v Warn | python3 -c "
import sys,json
r=[json.loads(l) for l in sys.stdin if l.startswith('{')]
print('lib$v', [round(x['ours_us'],1) for x in r], 'per-kb us', round((r[0]['ours_us']-r[1]['ours_us'])/96,3))"
  OOO_LIB=$PWD/paper_conf_eurosys_ohlks22_b200/lib/libooo$v.so timeout 300 python tools/engine_sweep.py C2 "" 2>&1 | tail -1
done
