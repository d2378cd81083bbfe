#!/bin/bash
# quick GPU check: parity tests + short bench summary
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
for cfg in ${CFGS:-C3}; do
timeout 600 python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$cfg', 'iters/s %.1f'%d['value'], 'A %.3f ms %.0f GB/s'%(k['A_ms'],k['A_GBs']), 'B %.3f ms %.0f GB/s'%(k['B_ms'],k['B_GBs']), 'iter %.0f GB/s frac %.3f'%(k['iter_alg_GBs'],k['iter_frac']), 'it/solve', d['config']['iters_per_solve'], 'clk', d['clocks']['sm_mhz'])"
done
