# bench variants (no tests)
B=paper_conf_sc_pandeylfhl22_b200
for v in "$@"; do
cp tools/gpu/lib$v.so $B/libpsim.so
timeout 600 python bench.py --config c3 --steps 2 --warmup 1 --no-cpu --no-e2e 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), r['frac'], {k: v['ms'] for k, v in r['kernels'].items()})"
done
cp tools/gpu/libA.so $B/libpsim.so
