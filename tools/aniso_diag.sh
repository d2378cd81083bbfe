#!/bin/bash
# k_aniso diagnostics / A/B by replay time: default build, _ab_old and _ab_2
# (built with experiment flags; labels in $L1 / $L2)
cd "$(dirname "$0")/.."
[ -n "$TESTS2" ] && (cd _ab_2 && MAS_TEST_TRANSPORTS=1 timeout 900 python -m pytest $TESTS2 -q -x 2>&1 | tail -2)
for rep in 1 2; do
  python tools/aniso_kbench.py default
  (cd _ab_old && python ../tools/aniso_kbench.py ${L1:-ab_old})
  (cd _ab_2 && python ../tools/aniso_kbench.py ${L2:-ab_2})
done
