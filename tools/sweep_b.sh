# kernel-B grid size sweep (MAS_BBLOCKS) on the configs in CFGS
for cfg in ${CFGS:-C2 C3}; do for bb in ${BBS:-1184 888 740 592 444}; do
MAS_BBLOCKS=$bb python bench.py --config $cfg --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('$cfg bblocks $bb', 'iters/s %.1f'%d['value'], 'A %.4f'%k['A_ms'], 'B %.4f'%k['B_ms'], 'clk', d['clocks']['sm_mhz'])"
done; done
