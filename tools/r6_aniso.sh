#!/bin/bash
# k_aniso consumer rework: aniso parity suites, then C2a bench lines
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r6b}
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
timeout 900 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py tests/test_gpu_fullsize.py tests/test_gpu_multiprocess_p2p.py -m gpu -q -x > $O/${TAG}_tests.log 2>&1
echo "tests rc=$?: $(tail -1 $O/${TAG}_tests.log)"
for r in 1 2; do
  python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_c2a_$r.log 2>&1
  echo "C2a $r: $(tail -1 $O/${TAG}_c2a_$r.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('%.0f iters/s, Lpar %.2f us, A %.2f, B %.2f, replay Lpar %.2f clk %s' % (d['value'], 1e3*k['Lpar_ms'], 1e3*k['A_ms'], 1e3*k['B_ms'], 1e3*k['replay']['Lpar_ms'], d['clocks']['sm_mhz']))")"
done
MAS_NO_GRAPH=1 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_aniso --launch-skip 3 --launch-count 1 \
  -f -o $O/${TAG}_C2a_kaniso python tools/prof_driver.py --config C2a > /dev/null 2>&1
grep -E "FAILED|Error" $O/${TAG}_tests.log | head
