cd $GRAFT_REPO_ROOT
O=gpurun_out; TAG=r6a
python -c "import __graft_entry__ as g; g.build()" > $O/${TAG}_build.log 2>&1 || exit 1
timeout 1500 python -m pytest tests -m gpu -q > $O/${TAG}_gputest.log 2>&1
echo "gpu suite rc=$?: $(tail -1 $O/${TAG}_gputest.log)"
python -c "import __graft_entry__ as g; g.smoke()" > $O/${TAG}_smoke.log 2>&1; echo "smoke rc=$?"
python bench.py > $O/${TAG}_bench_C3.log 2>&1
for cfg in C2 C2a; do python bench.py --config $cfg --no-cpu-baseline > $O/${TAG}_bench_$cfg.log 2>&1; done
for f in $O/${TAG}_bench_*.log; do echo "$f: $(tail -1 $f | cut -c1-400)"; done
