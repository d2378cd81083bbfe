#!/bin/bash
# A/B comparison of build variants, interleaved to average out clock drift:
#   tools/abtest.sh "<flags A>" "<flags B>" [rounds]   (CFGS selects configs)
A="$1"; B="$2"; R="${3:-3}"
for r in $(seq 1 $R); do
  for v in A B; do
    fl=$([ $v = A ] && echo "$A" || echo "$B")
    MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1 || { echo "build failed $v"; continue; }
    for cfg in ${CFGS:-C3}; do
      python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$v', '$cfg', 'round $r', 'iters/s %.1f'%d['value'], 'A %.4f ms'%k['A_ms'], 'B %.4f ms'%k['B_ms'], 'clk', d['clocks']['sm_mhz'])"
    done
  done
done
