#!/bin/bash
# k_aniso A/B: parity tests, then C2a bench lines per TMA L2-promotion setting
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r2j}
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py tests/test_gpu_fullsize.py -m gpu -q -x > $O/${TAG}_tests.log 2>&1
echo "tests rc=$?: $(tail -1 $O/${TAG}_tests.log)"
for p in 256 128 64 0; do
  MAS_TMA_PROMO=$p python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_c2a_p$p.log 2>&1
  echo "promo $p: $(tail -1 $O/${TAG}_c2a_p$p.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('%.0f iters/s, Lpar %.2f us, A %.2f, B %.2f' % (d['value'], 1e3*k['Lpar_ms'], 1e3*k['A_ms'], 1e3*k['B_ms']))")"
done
for p in 256 0; do
  MAS_NO_GRAPH=1 MAS_TMA_PROMO=$p /usr/local/cuda/bin/ncu --set full --clock-control none -k regex:k_aniso --launch-skip 2 --launch-count 1 \
    -f -o $O/${TAG}_kaniso_p$p python tools/prof_driver.py --config C2a > /dev/null 2>&1
done
