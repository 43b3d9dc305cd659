# A/B of complex64 fused/compiled passes between two library builds (run under gpurun):
#   VARIANTS="c64mb2 c64new" bash tools/ab_c64.sh   (ab/liblfqs_<variant>.so)
for v in ${VARIANTS:-c64mb2 c64new c64mb2 c64new}; do
  echo "== $v"
  LFQS_LIBRARY=$PWD/ab/liblfqs_$v.so timeout 400 python tools/bench_circuits.py --n 31 --c64 \
    --modes ${MODES:-fused,jit,jit+phase} --circuits qft,grover,random,sycamore,ghz 2>&1 | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l); print(d['circuit'], d['mode'], round(d['ms'],1), d.get('max_abs_err', d.get('norm2')))
  except Exception: print(l.strip()[:200])"
done
