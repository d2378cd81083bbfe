#!/bin/bash
# ncu launch lists of the bench's timed steps (no kernel replay): C3, C2a, C2
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r4l}; NCU=/usr/local/cuda/bin/ncu
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in C3 C2a C2; do
  $NCU --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file $O/${TAG}_launches_$c.csv \
    python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-replay > /dev/null 2>&1
done
ls -la $O/${TAG}_launches_*.csv
