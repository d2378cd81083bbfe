#!/bin/bash
# C2 kernel A/B vs the r-chunk length (MAS_CHUNK experiment hook) and tile shape
cd "$(dirname "$0")/.."
O=gpurun_out
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; r=k.get('replay') or {}; print('$2', round(d['value']), round(1e3*k['A_ms'],1), round(1e3*(k['B_ms'] or 0),1), 'replay', round(1e3*(r.get('A_ms') or 0),1), round(1e3*(r.get('B_ms') or 0),1), d['clocks']['sm_mhz'])"; }
for ch in ${CHUNKS:-default 8 11 13 16 22 26 32 43 64}; do
  if [ $ch = default ]; then unset MAS_CHUNK; else export MAS_CHUNK=$ch; fi
  python bench.py --config ${CFG:-C2} $EXTRA --no-cpu-baseline --no-e2e > $O/c2sweep_$ch.log 2>&1; summ $O/c2sweep_$ch.log "chunk $ch"
done
