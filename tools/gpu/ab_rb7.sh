# RB7: fused residual blocks (resblock.cu) vs layer-wise k3 convs, config-5 per-GPU slice
for v in 0 1; do
  PSIM_RB7_FUSED=$v timeout 600 python bench.py --config c5s --steps 1 --warmup 1 --no-cpu --no-e2e 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('rb7_fused=$v VALUE', round(d['value'],2), 'ms', round(d['ms_per_step'],1), 'cycles', d['total_cycles'], {k:v['ms'] for k,v in r['kernels'].items()})"
done
