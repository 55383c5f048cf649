# A/B of the fc1_head N-split (PSIM_FC1_SPLIT=0 disables) at the G = 8 and G = 4 slices and G = 1
for g in 8 4; do for r in 1 2; do for v in 0 1; do
  PSIM_FC1_SPLIT=$v timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --emulate-rank 0/$g 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('G=$g split=$v run $r VALUE', round(d['value'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
done; done; done
PSIM_FC1_SPLIT=1 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('G=1 VALUE', round(d['value'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
