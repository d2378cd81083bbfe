#!/bin/bash
# k_aniso consumer V2 (per-warp corners, no barrier) vs V1, one box
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r3d}
mkdir -p /tmp/libs
for v in "v2:" "v1:-DMAS_ANISO_V1"; do
  name=${v%%:*}; flags=${v#*:}
  MAS_NVCC_FLAGS="$flags" python paper_conf_ipps_caplansl23_b200/build.py --force > $O/${TAG}_build_$name.log 2>&1 || echo "build $name failed"
  cp paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so /tmp/libs/$name.so
done
cp /tmp/libs/v2.so paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so
timeout 900 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py -m gpu -q -x > $O/${TAG}_tests_v2.log 2>&1
echo "v2 tests rc=$?: $(tail -1 $O/${TAG}_tests_v2.log)"
grep -E "FAILED|assert " $O/${TAG}_tests_v2.log | head -5
for rep in 1 2; do
  for name in v2 v1; do
    cp /tmp/libs/$name.so paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so
    python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_${name}_$rep.log 2>&1
    echo "$name rep $rep: $(tail -1 $O/${TAG}_${name}_$rep.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('%.0f iters/s, Lpar %.2f us' % (d['value'], 1e3*k['Lpar_ms']))")"
  done
done
cp /tmp/libs/v2.so paper_conf_ipps_caplansl23_b200/lib/libmaspcg.so
