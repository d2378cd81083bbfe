# kernel A (scalar) at 3-4 blocks/SM with shorter r-chunks on C2
for fl in "-DMAS_MINB1=4" "-DMAS_MINB1=3"; do
  MAS_NVCC_FLAGS="$fl" python paper_conf_ipps_caplansl23_b200/build.py --force -v 2>&1 | grep -A1 "k_stencilILi2ELi1ELb0" | grep -o "Used [0-9]* registers\|[0-9]* bytes spill stores" | tr "\n" " "; echo
  for ch in 16 11; do
    MAS_CHUNK=$ch python bench.py --config C2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('[$fl] chunk $ch', 'iters/s %.0f'%d['value'], 'A %.4f'%k['A_ms'])"
  done
done
python paper_conf_ipps_caplansl23_b200/build.py --force >/dev/null 2>&1
