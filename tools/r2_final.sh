#!/bin/bash
# Round-2 closing session: full GPU suite, smoke, bench lines of every config
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r2z}
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_gputest.log 2>&1
echo "gpu suite rc=$?: $(tail -1 $O/${TAG}_gputest.log)"
python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
python bench.py > $O/${TAG}_bench_C3.log 2>&1
python bench.py --impl reference > $O/${TAG}_bench_C3_reference.log 2>&1
for cfg in C2 C2a C2t C1; do python bench.py --config $cfg > $O/${TAG}_bench_$cfg.log 2>&1; done
python bench.py --config C2 --solver cg1 --no-cpu-baseline > $O/${TAG}_bench_C2_cg1.log 2>&1
python bench.py --config C1 --solver cg1 --no-cpu-baseline > $O/${TAG}_bench_C1_cg1.log 2>&1
python bench.py --solver cg1 --no-cpu-baseline --no-e2e > $O/${TAG}_bench_C3_cg1.log 2>&1
python bench.py --config C3s8 --no-cpu-baseline --no-e2e > $O/${TAG}_bench_C3s8.log 2>&1
for f in $O/${TAG}_bench_*.log; do echo "$f: $(tail -1 $f | cut -c1-200)"; done
grep -E "FAILED" $O/${TAG}_gputest.log | head
