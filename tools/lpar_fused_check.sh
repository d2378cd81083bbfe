#!/bin/bash
# fused L_par in kernel A: aniso parity suites (fused default and separate), C2a benches
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r3l}
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || { tail -5 $O/${TAG}_build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py tests/test_gpu_multiprocess_p2p.py tests/test_gpu_nccl_one_rank.py tests/test_gpu_fullsize.py -m gpu -q > $O/${TAG}_tests_fused.log 2>&1
echo "default tests rc=$?: $(tail -1 $O/${TAG}_tests_fused.log)"; grep -E "^FAILED" $O/${TAG}_tests_fused.log | head
MAS_LPAR_FUSED=1 timeout 900 python -m pytest tests/test_gpu_aniso.py -m gpu -q > $O/${TAG}_tests_sep.log 2>&1
echo "fused-env tests rc=$?: $(tail -1 $O/${TAG}_tests_sep.log)"
for v in "separate:" "fused:MAS_LPAR_FUSED=1"; do
  name=${v%%:*}; envs=${v#*:}
  env $envs python bench.py --config C2a --no-cpu-baseline --no-e2e > $O/${TAG}_c2a_$name.log 2>&1
  echo "$name: $(tail -1 $O/${TAG}_c2a_$name.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; r=k.get('replay',{}); print('%.0f iters/s, A %.2f us, Lpar %s, frac %.3f, replay A %.2f us' % (d['value'], 1e3*k['A_ms'], k.get('Lpar_ms'), d['roofline']['frac'], 1e3*r.get('A_ms',0)))")"
done
