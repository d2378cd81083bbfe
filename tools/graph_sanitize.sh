#!/bin/bash
# compute-sanitizer on the CUDA-graph solve loop: the round-2 one-graph form
# (default) and the round-1 form (MAS_GRAPH_PRE=1: iteration 1 launched as
# plain kernels ahead of the graph).  Output: gpurun_out/san_*.txt
cd "$(dirname "$0")/.."
out=gpurun_out
mkdir -p $out
CS=/usr/local/cuda/bin/compute-sanitizer
python -c "import __graft_entry__ as g; g.build()" || exit 1
for tool in memcheck initcheck synccheck racecheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python tools/graph_san_min.py > $out/san_${tool}.txt 2>&1
  echo "$tool rc=$?: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Program hit' $out/san_${tool}.txt | head -3)"
done
MAS_GRAPH_PRE=1 timeout 600 $CS --tool memcheck --print-limit 20 python tools/graph_san_min.py > $out/san_memcheck_pre.txt 2>&1
echo "memcheck MAS_GRAPH_PRE=1 rc=$?: $(grep -E 'ERROR SUMMARY|Program hit' $out/san_memcheck_pre.txt | head -3)"
timeout 1200 $CS --tool memcheck --print-limit 20 python tools/graph_san_min.py --c3full > $out/san_memcheck_c3.txt 2>&1
echo "memcheck with full C3 rc=$?: $(grep -E 'ERROR SUMMARY|Program hit' $out/san_memcheck_c3.txt | head -3)"
