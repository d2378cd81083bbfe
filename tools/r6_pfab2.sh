#!/bin/bash
# CG1 prefetch distance A/B (C3 cg1, C3 pcg unchanged check) + CG1 GPU tests
cd "$(dirname "$0")/.."
python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_single_reduction.py tests/test_gpu_fullsize.py -m gpu -q -x 2>&1 | tail -1
for r in 1 2; do for fl in "" "-DMAS_PF_DIST_CG1=1"; do
  MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
  for c in "C3 cg1" "C3 pcg" "C2 cg1"; do set -- $c
    python bench.py --config $1 --solver $2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('[$fl] $1 $2 round $r', 'iters/s %.1f'%d['value'], 'A_ms %.4f'%k['A_ms'], 'clk', d['clocks']['sm_mhz'])"
  done
done; done
python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
