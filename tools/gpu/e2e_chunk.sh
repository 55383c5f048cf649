# e2e (pinned host trace, streaming loader) vs the loader chunk length in lockstep steps (PSIM_CHUNK)
for r in 1 2; do for c in 32 64 128 256; do
  PSIM_CHUNK=$c timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('chunk $c run $r value', round(d['value'],1), 'e2e', round(d['e2e']['value'],1))"
done; done
