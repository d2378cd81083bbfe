#!/bin/bash
# k_aniso A/B of build variants (C2a kernel times), plus the aniso parity suite
# on the first non-default variant
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r6e}
MAS_NVCC_FLAGS="$1" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1 && \
  timeout 600 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py -m gpu -q -x > $O/${TAG}_tests.log 2>&1
echo "tests [$1] rc=$?: $(tail -1 $O/${TAG}_tests.log)"
CFG=C2a bash tools/abflags.sh 2 "" "$@"
