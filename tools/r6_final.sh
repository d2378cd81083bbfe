#!/bin/bash
# Closing evidence of the round-2 final session: full GPU suite, smoke, every
# bench line, the staggered stack bench, launch lists, ncu --set full captures.
# Outputs gpurun_out/${TAG}_*.
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r6z}; NCU=/usr/local/cuda/bin/ncu
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
if [ -z "$SKIP_TESTS" ]; then
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_gputest.log 2>&1
echo "gpu suite rc=$?: $(tail -1 $O/${TAG}_gputest.log)"
python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
fi
python bench.py > $O/${TAG}_bench_C3.log 2>&1
python bench.py --impl reference > $O/${TAG}_bench_C3_reference.log 2>&1
for cfg in C2 C2a C2t C1; do python bench.py --config $cfg > $O/${TAG}_bench_$cfg.log 2>&1; done
python bench.py --config C2 --solver cg1 --no-cpu-baseline > $O/${TAG}_bench_C2_cg1.log 2>&1
python bench.py --config C1 --solver cg1 --no-cpu-baseline > $O/${TAG}_bench_C1_cg1.log 2>&1
python bench.py --solver cg1 --no-cpu-baseline --no-e2e > $O/${TAG}_bench_C3_cg1.log 2>&1
python bench.py --config C3s8 --no-cpu-baseline --no-e2e > $O/${TAG}_bench_C3s8.log 2>&1
python tools/stack_bench.py > $O/${TAG}_stack_bench.json 2> $O/${TAG}_stack_bench.err
for f in $O/${TAG}_bench_*.log; do echo "$f: $(tail -1 $f | cut -c1-100)"; done
[ -n "$SKIP_NCU" ] && exit 0
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_C3.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-replay > /dev/null 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none -c 900 --csv --log-file $O/${TAG}_launches_C2a.csv \
  python bench.py --config C2a --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-replay > /dev/null 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none -c 900 --csv --log-file $O/${TAG}_launches_C2.csv \
  python bench.py --config C2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-replay > /dev/null 2>&1
export MAS_NO_GRAPH=1
cap() {  # name regex skip args...
  local name=$1 rx=$2 skip=$3; shift 3
  $NCU --set full --clock-control none --import-source on -k regex:$rx --launch-skip $skip --launch-count 1 \
    -f -o $O/${TAG}_$name python tools/prof_driver.py "$@" > $O/${TAG}_$name.log 2>&1
  echo "$name rc=$?"
}
cap C3_kernelA k_stencil 2 --config C3
cap C3_kernelB k_pcg_b 1 --config C3
cap C2a_kaniso k_aniso 3 --config C2a  # launches: coef, diag, RESID, PCGA
cap C2_kernelB k_pcg_b 1 --config C2
ls -la $O/${TAG}_*.ncu-rep
grep -E "FAILED" $O/${TAG}_gputest.log | head
