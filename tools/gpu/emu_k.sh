# per-kernel device time at the G-rank per-GPU slices (rank 0's share, no NCCL)
for g in 1 2 4 8; do
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/$g 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']
print('G=$g per-GPU', round(d['value'],1), 'ms/step', round(d['ms_per_step'],1), {k:(v['ms'],v['launches']) for k,v in r['kernels'].items()}, 'k_mean', r.get('k_mean'))"
done
