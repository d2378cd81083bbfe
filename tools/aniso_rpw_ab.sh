#!/bin/bash
# k_aniso RPW A/B: current tree (RPW 1) vs _ab_old built with -DMAS_ANISO_RPW=2;
# the aniso GPU tests on the RPW=2 build first
cd "$(dirname "$0")/.."
O=gpurun_out
(cd _ab_old && MAS_TEST_TRANSPORTS=1 timeout 900 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py -q -x 2>&1 | tail -2)
CONFIGS="${CONFIGS:-C2a}" bash tools/aniso_ab3.sh
