for c in 16 64 256; do
PSIM_CHUNK=$c timeout 900 python bench.py --config c3 --steps 2 --warmup 1 --no-cpu 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('CHUNK $c VALUE', round(d['value'],1), 'E2E', round(d['e2e']['value'],1))"
done
