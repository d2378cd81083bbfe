#!/bin/bash
# scalar kernel A at 3 blocks per SM (current tree) vs 2 (_ab_old), C2 chunk sweep, C1
cd "$(dirname "$0")/.."
O=gpurun_out
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; r=k.get('replay') or {}; print('$2', round(d['value']), round(1e3*k['A_ms'],1), round(1e3*(k['B_ms'] or 0),1), 'replay', round(1e3*(r.get('A_ms') or 0),1), round(1e3*(r.get('B_ms') or 0),1), d['clocks']['sm_mhz'])" 2>&1 | tail -1; }
for v in new old; do
  d=.; [ $v = old ] && d=_ab_old
  for ch in 32 26 22 19 16; do
    (cd $d && MAS_CHUNK=$ch python bench.py --config C2 --no-cpu-baseline --no-e2e > /root/repo/$O/mb_${v}_$ch.log 2>&1); summ $O/mb_${v}_$ch.log "$v C2 chunk $ch"
  done
  for ch in default 8 11 16; do
    if [ $ch = default ]; then unset MAS_CHUNK; else export MAS_CHUNK=$ch; fi
    (cd $d && python bench.py --config C1 --no-cpu-baseline --no-e2e > /root/repo/$O/mb1_${v}_$ch.log 2>&1); summ $O/mb1_${v}_$ch.log "$v C1 chunk $ch"
  done
  unset MAS_CHUNK
done
