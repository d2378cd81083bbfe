#!/bin/bash
# compute-sanitizer on the separable-corner-sum k_aniso (host loop: every mode;
# shapes with a single phi tile, a ragged phi tile, ragged theta tiles and
# multi-segment blocks) and memcheck/initcheck on the graph loop
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r6s}; CS=/usr/local/cuda/bin/compute-sanitizer
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
for shape in "16 24 64" "24 20 70" "40 32 128"; do
  for tool in racecheck synccheck memcheck initcheck; do
    MAS_NO_GRAPH=1 timeout 900 $CS --tool $tool --print-limit 20 python tools/aniso_stages.py $shape > $O/${TAG}_${tool}_${shape// /x}.txt 2>&1
    echo "host loop $shape $tool rc=$?: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Program hit' $O/${TAG}_${tool}_${shape// /x}.txt | head -2 | tr '\n' ' ')"
  done
done
for tool in memcheck initcheck; do
  timeout 900 $CS --tool $tool --print-limit 20 python tools/aniso_stages.py 24 20 70 > $O/${TAG}_graph_${tool}.txt 2>&1
  echo "graph loop 24x20x70 $tool rc=$?: $(grep -E 'ERROR SUMMARY|Program hit' $O/${TAG}_graph_${tool}.txt | head -2 | tr '\n' ' ')"
done
