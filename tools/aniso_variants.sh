#!/bin/bash
# k_aniso geometry A/B: tile height WJ, blocks per SM, ring slots (compile-time)
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r2k}
for v in "16 1 4" "8 2 4" "8 3 3"; do
  set -- $v
  export MAS_NVCC_FLAGS="-DMAS_ANISO_WJ=$1 -DMAS_ANISO_BPS=$2 -DMAS_ANISO_SLOTS=$3"
  python paper_conf_ipps_caplansl23_b200/build.py --force > $O/${TAG}_build_$1_$2_$3.log 2>&1 || { echo "build $v failed"; continue; }
  timeout 600 python -m pytest tests/test_gpu_aniso.py -m gpu -q -x > $O/${TAG}_tests_$1_$2_$3.log 2>&1
  t="$(tail -1 $O/${TAG}_tests_$1_$2_$3.log)"
  for p in 64; do
    MAS_TMA_PROMO=$p python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_c2a_$1_$2_$3_p$p.log 2>&1
    echo "WJ=$1 BPS=$2 SLOTS=$3 promo $p [$t]: $(tail -1 $O/${TAG}_c2a_$1_$2_$3_p$p.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('%.0f iters/s, Lpar %.2f us' % (d['value'], 1e3*k['Lpar_ms']))")"
  done
done
