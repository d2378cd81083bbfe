for ch in 32 16 11; do for bb in 1184 592 296; do
MAS_CHUNK=$ch MAS_BBLOCKS=$bb python bench.py --config C2 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); k=d['kernels']; print('chunk $ch bblocks $bb', 'iters/s %.0f'%d['value'], 'A %.4f'%k['A_ms'], 'B %.4f'%k['B_ms'])"
done; done
