for v in A B; do
  PSIM_LIB=tools/gpu/ab/$v.so timeout 600 python bench.py --config c5s --steps 1 --warmup 1 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v c5s VALUE', round(d['value'],2), 'cycles', d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
  PSIM_LIB=tools/gpu/ab/$v.so timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e --layerwise 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v c3 layerwise VALUE', round(d['value'],2), 'cycles', d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done
