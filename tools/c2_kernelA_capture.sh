#!/bin/bash
# C2 kernel A under the two-iteration x update: one even (A(2): no x) and one
# odd (A(3): x and p_{k-2}) launch, ncu --set full each
cd "$(dirname "$0")/.."
O=gpurun_out; NCU=/usr/local/cuda/bin/ncu; TAG=${TAG:-r5c}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for skip in 2 3; do
  MAS_NO_GRAPH=1 $NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip $skip --launch-count 1 \
    -f -o $O/${TAG}_C2_kernelA_s$skip python tools/prof_driver.py --config C2 > /dev/null 2>&1
  echo "skip $skip rc=$?"
done
ls -la $O/${TAG}_C2_kernelA_s*.ncu-rep
