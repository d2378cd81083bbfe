#!/bin/bash
# Round-2 measurement session: bench lines, ncu launch lists and --set full
# captures of the dominant kernels.  Outputs gpurun_out/${TAG}_*.
cd "$(dirname "$0")/.."
TAG=${TAG:-r2h}
O=gpurun_out; mkdir -p $O
NCU=/usr/local/cuda/bin/ncu
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
# bench lines (the default C3 line first: e2e and cpu_baseline included)
python bench.py > $O/${TAG}_bench_C3.log 2>&1
for cfg in C2 C2a C2t C1; do python bench.py --config $cfg --no-cpu-baseline > $O/${TAG}_bench_$cfg.log 2>&1; done
python bench.py --config C2 --solver cg1 --no-cpu-baseline > $O/${TAG}_bench_C2_cg1.log 2>&1
python bench.py --solver cg1 --no-cpu-baseline --no-e2e > $O/${TAG}_bench_C3_cg1.log 2>&1
# launch lists (the bench command itself, 2 steps)
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/${TAG}_launches_C3.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
$NCU --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file $O/${TAG}_launches_C2a.csv \
  python bench.py --config C2a --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
# full captures: kernel A (3rd k_stencil launch: RESID, A(1), A(2)), kernel B, k_aniso, CG1
$NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip 2 --launch-count 1 \
  -f -o $O/${TAG}_C3_kernelA python tools/prof_driver.py --config C3 > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_pcg_b --launch-skip 1 --launch-count 1 \
  -f -o $O/${TAG}_C3_kernelB python tools/prof_driver.py --config C3 > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_aniso --launch-skip 2 --launch-count 1 \
  -f -o $O/${TAG}_C2a_kaniso python tools/prof_driver.py --config C2a > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip 2 --launch-count 1 \
  -f -o $O/${TAG}_C2_kernelA python tools/prof_driver.py --config C2 > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_pcg_b --launch-skip 1 --launch-count 1 \
  -f -o $O/${TAG}_C2_kernelB python tools/prof_driver.py --config C2 > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip 3 --launch-count 1 \
  -f -o $O/${TAG}_C2_cg1 python tools/prof_driver.py --config C2 --solver cg1 > /dev/null 2>&1
$NCU --set full --clock-control none --import-source on -k regex:k_stencil --launch-skip 3 --launch-count 1 \
  -f -o $O/${TAG}_C3_cg1 python tools/prof_driver.py --config C3 --solver cg1 > /dev/null 2>&1
ls -la $O/${TAG}_* | awk '{print $5, $9}'
for f in $O/${TAG}_bench_*.log; do echo "$f: $(tail -1 $f | cut -c1-160)"; done
