# fc1_head pair mode (2-SM MMAs, PSIM_FC1_PAIR) A/B at G = 1 / 8 / 4
for g in 1 8 4; do for r in 1 2; do for v in 0 1; do
  emu=""; [ $g -gt 1 ] && emu="--emulate-rank 0/$g"
  PSIM_FC1_PAIR=$v timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e $emu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('G=$g pair=$v run $r VALUE', round(d['value'],1), 'cycles', d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done; done; done
