#!/bin/bash
# Kernel A of the scalar configs under the two-iteration x update: one even
# (A(2): no x) and one odd (A(3): x and p_{k-2}) launch, ncu --set full each
#   CFGS="C2a C2t" tools/r6_kernelA_capture.sh
cd "$(dirname "$0")/.."
O=gpurun_out; NCU=/usr/local/cuda/bin/ncu; TAG=${TAG:-r6c}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in ${CFGS:-C2a C2t}; do
  for skip in 2 3; do
    MAS_NO_GRAPH=1 $NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip $skip --launch-count 1 \
      -f -o $O/${TAG}_${cfg}_kernelA_s$skip python tools/prof_driver.py --config $cfg > /dev/null 2>&1
    echo "$cfg skip $skip rc=$?"
  done
done
ls -la $O/${TAG}_*_kernelA_s*.ncu-rep
