# A/B of two builds on the same box: tools/gpu/ab/A.so vs tools/gpu/ab/B.so, alternating, config 3,
# device-resident value and per-kernel times; then the G=8 slice
for r in 1 2; do for v in A B; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 300 python bench.py --steps 5 --warmup 2 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v run $r VALUE', round(d['value'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
done; done
for v in A B; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --emulate-rank 0/8 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v G=8 VALUE', round(d['value'],1), {k:v['ms'] for k,v in r['kernels'].items()})"
done
