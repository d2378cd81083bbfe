#!/bin/bash
# Interleaved A/B of environment settings on bench configs:
#   CFGS="C2 C2a" tools/r6_envab.sh rounds "ENV1=.. ENV2=.." "ENV=.." ...
cd "$(dirname "$0")/.."
R="$1"; shift
for r in $(seq 1 $R); do
  for cfg in ${CFGS:-C2}; do
    for ev in "$@"; do
      env $ev python bench.py --config $cfg --solver ${SOLVER:-pcg} --steps ${STEPS:-5} --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | \
        python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$cfg [$ev]', 'round $r', 'iters/s %.1f'%d['value'], ' '.join('%s %.4f'%(n,k[n]) for n in ('A_ms','B_ms','Lpar_ms') if k.get(n)), 'clk', d['clocks']['sm_mhz'])"
    done
  done
done
