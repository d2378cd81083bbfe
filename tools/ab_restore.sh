#!/bin/bash
cd "$(dirname "$0")/.."
cp /tmp/ab_new.cu paper_conf_ipps_caplansl23_b200/csrc/kernels.cu
rm -f paper_conf_ipps_caplansl23_b200/csrc/kernels_old.inc paper_conf_ipps_caplansl23_b200/csrc/kernels_new.inc
