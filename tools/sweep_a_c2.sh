# kernel A (scalar) occupancy x r-chunk sweep on C2
for fl in "" "-DMAS_MINB1=3"; do
  MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1 || { echo "build failed [$fl]"; continue; }
  for ch in 32 26 22; do
    MAS_CHUNK=$ch python bench.py --config C2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('[$fl] chunk $ch', 'iters/s %.0f'%d['value'], 'A %.4f'%k['A_ms'], 'B %.4f'%k['B_ms'])"
  done
done
python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
