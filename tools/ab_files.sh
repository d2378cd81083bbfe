#!/bin/bash
# A/B of the committed kernels.cu (A) vs the working copy (B): both are
# compiled from include stubs selected by -DMAS_AB_OLD.
set -e
cd "$(dirname "$0")/.."
K=paper_conf_ipps_caplansl23_b200/csrc/kernels.cu
cp $K /tmp/ab_new.cu
git show HEAD:$K > paper_conf_ipps_caplansl23_b200/csrc/kernels_old.inc
cp /tmp/ab_new.cu paper_conf_ipps_caplansl23_b200/csrc/kernels_new.inc
printf '#ifdef MAS_AB_OLD\n#include "kernels_old.inc"\n#else\n#include "kernels_new.inc"\n#endif\n' > $K
echo "stubs ready"
