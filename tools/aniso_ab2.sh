#!/bin/bash
# k_aniso A/B on one box: variants built with MAS_NVCC_FLAGS, C2a bench twice each, interleaved
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r2n}
mkdir -p /tmp/libs
for v in "base:" "qnow:-DMAS_ANISO_QNOW" "qtma:-DMAS_ANISO_QTMA" "zero:-DMAS_ANISO_ZERO"; do
  name=${v%%:*}; flags=${v#*:}
  MAS_NVCC_FLAGS="$flags" python paper_conf_ipps_caplansl23_b200/build.py --force > /dev/null 2>&1 || echo "build $name failed"
  cp paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so /tmp/libs/$name.so
done
for rep in 1 2; do
  for name in base qnow qtma zero; do
    cp /tmp/libs/$name.so paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so
    python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_${name}_$rep.log 2>&1
    echo "$name rep $rep: $(tail -1 $O/${TAG}_${name}_$rep.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('%.0f iters/s, Lpar %.2f us' % (d['value'], 1e3*k['Lpar_ms']))")"
  done
done
cp /tmp/libs/base.so paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so
