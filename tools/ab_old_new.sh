#!/bin/bash
# A/B: bench lines of the current tree against an older worktree in _ab_old/
# (git worktree add _ab_old <commit>; build both here); plus the test files in $TESTS
cd "$(dirname "$0")/.."
O=gpurun_out
summ() { tail -1 $1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$2', round(d['value']), round(1e3*k['A_ms'],1), round(1e3*(k['B_ms'] or 0),1), d['clocks']['sm_mhz'], d['clocks']['reasons'])"; }
[ -n "$TESTS" ] && MAS_TEST_TRANSPORTS=1 timeout 900 python -m pytest $TESTS -q -x 2>&1 | tail -2
for rep in 1 2; do
 for v in old new; do
  d=.; [ $v = old ] && d=_ab_old
  [ -d $d ] || continue
  for c in ${CONFIGS:-C3 C3s8}; do (cd $d && python bench.py --config $c --no-cpu-baseline --no-e2e > /root/repo/$O/ab_${v}_${c}_$rep.log 2>&1); summ $O/ab_${v}_${c}_$rep.log "$v $c"; done
 done
done
