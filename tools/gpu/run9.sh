timeout 900 python -m pytest tests -x -q -m "gpu" -k "residency or s3_c3_small or fused_full or s1_device" 2>&1 | tail -3
timeout 900 python bench.py --config c3 --steps 2 --warmup 1 --no-cpu 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('VALUE', d['value'], 'E2E', d['e2e'], 'ms', d['ms_per_step'], r['kernels'])"
