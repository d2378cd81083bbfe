#!/bin/bash
# Interleaved A/B/... of build-flag variants on one config, printing the
# per-kernel times of bench.py (kernels dict):
#   CFG=C2a tools/abflags.sh rounds "<flags 1>" "<flags 2>" ...
R="$1"; shift
for r in $(seq 1 $R); do
  for fl in "$@"; do
    MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1 || { echo "build failed [$fl]"; continue; }
    python bench.py --config ${CFG:-C2a} --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('[$fl]', 'round $r', 'iters/s %.1f'%d['value'], ' '.join('%s %.4f'%(n,k[n]) for n in ('A_ms','B_ms','Lpar_ms') if n in k), 'clk', d['clocks']['sm_mhz'])"
  done
done
python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
