#!/bin/bash
# the scalar-operator bench lines again (after the byte-accounting fix)
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r5y}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in C2 C2a C2t C1; do python bench.py --config $cfg > $O/${TAG}_bench_$cfg.log 2>&1; done
for f in $O/${TAG}_bench_*.log; do echo "$f: $(tail -1 $f | cut -c1-120)"; done
