#!/bin/bash
# ncu captures of round 2.  ncu cannot profile kernel nodes of a graph that
# has conditional nodes, so the driver runs the host-driven loop
# (MAS_NO_GRAPH=1: the same kernels launched one by one).  Launch lists: the
# bench command (its profiled second pass launches every kernel plainly).
cd "$(dirname "$0")/.."
TAG=${TAG:-r2i}
O=gpurun_out; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
export MAS_NO_GRAPH=1
cap() {  # name regex skip args...
  local name=$1 rx=$2 skip=$3; shift 3
  $NCU --set full --clock-control none --import-source on -k regex:$rx --launch-skip $skip --launch-count 1 \
    -f -o $O/${TAG}_$name python tools/prof_driver.py "$@" > $O/${TAG}_$name.log 2>&1
  echo "$name rc=$?: $(grep -c '==PROF==' $O/${TAG}_$name.log) prof lines"
}
cap C3_kernelA k_stencil 2 --config C3
cap C3_kernelB k_pcg_b 1 --config C3
cap C2a_kaniso k_aniso 3 --config C2a  # launches: coef, diag, RESID, PCGA
cap C2_kernelA k_stencil 2 --config C2
cap C2_kernelB k_pcg_b 1 --config C2
cap C2_cg1 k_stencil 3 --config C2 --solver cg1
cap C3_cg1 k_stencil 3 --config C3 --solver cg1
cap C2t_pole k_pole_avg 4 --config C2t
unset MAS_NO_GRAPH
$NCU --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $O/${TAG}_launches_C3.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none -c 900 --csv --log-file $O/${TAG}_launches_C2a.csv \
  python bench.py --config C2a --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none -c 900 --csv --log-file $O/${TAG}_launches_C2.csv \
  python bench.py --config C2 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
python bench.py > $O/${TAG}_bench_C3.log 2>&1
tail -1 $O/${TAG}_bench_C3.log | cut -c1-400
ls $O/${TAG}_*
