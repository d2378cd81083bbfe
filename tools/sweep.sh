#!/bin/bash
# build variants on the GPU box and print the quick bench line for each
for fl in "$@"; do
  MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1 || { echo "build failed: $fl"; continue; }
  echo "== $fl"
  CFGS="${CFGS:-C3}" tools/quick.sh 2>&1 | grep -v passed
done
