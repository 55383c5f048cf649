timeout 600 python -m pytest tests -x -q -m "gpu" -k "s3_c3_small or fused_full or s1_hand or config2" 2>&1 | tail -5
timeout 300 python __graft_entry__.py smoke 2>&1 | tail -1
timeout 600 python bench.py --config c3 --steps 2 --warmup 1 --cpu-budget 3 --no-e2e 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('VALUE', d['value'], 'ms', d['ms_per_step'], r['kernel'], r['frac'], r['kernels'])"
