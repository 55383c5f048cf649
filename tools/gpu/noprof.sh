mkdir -p gpurun_out
PSIM_NOPROF=1 timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('NOPROF VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1))" || true
timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('PROF VALUE', round(d['value'],1), 'ms', round(d['ms_per_step'],1))"
