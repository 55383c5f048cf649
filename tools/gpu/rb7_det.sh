# determinism of the RB7 path: the config-5 G = 8 slice three times per build
for v in $1; do for r in 1 2 3; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 900 python bench.py --config c5 --steps 1 --warmup 1 --no-cpu --no-e2e --emulate-rank 0/8 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v c5/8 run $r', round(d['value'],2), d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done; done
