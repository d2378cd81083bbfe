#!/bin/bash
# k_aniso V3 A/B: current tree (V1) vs _ab_old built with -DMAS_ANISO_V3; the
# aniso GPU tests on the V3 build first (graph == host loop, vranks, P2P, full size)
cd "$(dirname "$0")/.."
(cd _ab_old && MAS_TEST_TRANSPORTS=1 timeout 900 python -m pytest tests/test_gpu_aniso.py tests/test_gpu_aniso_vranks.py tests/test_gpu_multiprocess_p2p.py -q -x 2>&1 | tail -4)
(cd _ab_old && timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x -k c2a 2>&1 | tail -2)
bash tools/aniso_ab3.sh
