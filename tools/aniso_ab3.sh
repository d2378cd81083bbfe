#!/bin/bash
# k_aniso A/B: current tree vs _ab_old (C2a bench lines, 3 reps each) + aniso tests
cd "$(dirname "$0")/.."
O=gpurun_out
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; r=k.get('replay') or {}; print('$2', round(d['value']), 'A', round(1e3*k['A_ms'],1), 'Lpar', round(1e3*(k.get('Lpar_ms') or 0),2), 'replay Lpar', round(1e3*(r.get('Lpar_ms') or 0),2))" 2>&1 | tail -1; }
[ -n "$TESTS" ] && MAS_TEST_TRANSPORTS=1 timeout 900 python -m pytest $TESTS -q -x 2>&1 | tail -2
for rep in 1 2 3; do
  for v in new old; do
    d=.; [ $v = old ] && d=_ab_old
    (cd $d && python bench.py --config C2a --no-cpu-baseline --no-e2e > /root/repo/$O/a3_${v}_$rep.log 2>&1); summ $O/a3_${v}_$rep.log "$v"
  done
done
