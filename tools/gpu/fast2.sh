bash tools/gpu/fastcheck.sh
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --emulate-rank 0/8 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('G=8 per-GPU VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1), 'x8 =', round(8*d['value'],1))"
