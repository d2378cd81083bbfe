cd $GRAFT_REPO_ROOT
for r in 1 2; do for fl in "" "-DMAS_PF_DIST=2" "-DMAS_PF_DIST=4"; do
  MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
  for sv in pcg cg1; do
    python bench.py --config C3 --solver $sv --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('[$fl] $sv round $r', 'iters/s %.1f'%d['value'], 'A_ms %.4f'%k['A_ms'], 'clk', d['clocks']['sm_mhz'])"
  done
done; done
