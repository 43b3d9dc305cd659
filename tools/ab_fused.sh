for v in ${VARIANTS:-list flat list flat}; do echo "== $v"; LFQS_LIBRARY=$PWD/ab/liblfqs_$v.so python tools/bench_circuits.py --n 30 --modes fused --circuits qft,grover,random,sycamore,ghz 2>&1 | python -c "
import sys,json
for l in sys.stdin:
  try: d=json.loads(l); print(d['circuit'], round(d['ms'],1))
  except Exception: print(l.strip()[:200])"; done
